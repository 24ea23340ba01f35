// internal.h -- library-private types of libsplitcnn (not part of the C ABI).
#pragma once
#include <cstdint>
#include <string>
#include <vector>

#include "../../include/splitcnn.h"

namespace splitcnn {

constexpr int kMaxSplits = SPLITCNN_MAX_SPLITS;

inline int round_up(int x, int m) { return (x + m - 1) / m * m; }

// Geometry of one activation level (host side).
struct Level {
    int N, C, Cpad, H, W;
    std::vector<int32_t> bh, bw;  // n + 1 boundaries
    int nh() const { return (int)bh.size() - 1; }
    int nw() const { return (int)bw.size() - 1; }
    int npatch() const { return nh() * nw(); }
    int ph(int i) const { return bh[i + 1] - bh[i]; }
    int pw(int j) const { return bw[j + 1] - bw[j]; }
    // element offset of patch (i, j): N*Cpad*(bh[i]*W + h_i*bw[j])   (splitcnn.h "Levels")
    int64_t offset(int i, int j) const {
        return (int64_t)N * Cpad * ((int64_t)bh[i] * W + (int64_t)ph(i) * bw[j]);
    }
    int64_t patch_elems(int i, int j) const { return (int64_t)N * ph(i) * pw(j) * Cpad; }
    int64_t total() const { return (int64_t)N * H * W * Cpad; }
};

struct LayerGeom {
    splitcnn_layer_t L;
    std::vector<int32_t> pad_h, pad_w;  // 2 per patch row / column: (begin, end)
};

}  // namespace splitcnn

struct splitcnn_plan_s {
    int N = 0;
    std::vector<splitcnn::Level> levels;     // nlayers + 1
    std::vector<splitcnn::LayerGeom> layers; // nlayers
};

namespace splitcnn {

// ---------------------------------------------------------------- kernel-side descriptors
// Passed by value as kernel parameters (<= ~600 B).
struct LevelDesc {
    int N, C, Cpad, H, W, nh, nw;
    int bh[kMaxSplits + 1];
    int bw[kMaxSplits + 1];
};

struct LayerDesc {
    int kh, kw, sh, sw;
    int pad_h[2 * kMaxSplits];
    int pad_w[2 * kMaxSplits];
};

LevelDesc make_level_desc(const Level &l);
LayerDesc make_layer_desc(const LayerGeom &g);

// error plumbing
void set_error(const std::string &msg);
splitcnn_status_t fail(splitcnn_status_t s, const std::string &msg);
splitcnn_status_t check_launch(const char *what);

}  // namespace splitcnn

namespace splitcnn {
void count_launch(int n = 1);  // every kernel launch of the library (splitcnn_kernel_launches)
}
