// plan.cpp -- host-side Split-CNN planning, the library's own
// implementation (it shares nothing with oracle/plan.py).
//
//   I_i = s * O_i                          SURVEY R2 (inside [lb, ub] of Eq. 1-2)
//   p_{i,b} = p_b (i = 0) | I_i + p_b - O_i s                 P:139 with the R1 correction
//   p_{i,e} = p_e (i = N-1) | (O_{i+1} - 1) s + k - (I_{i+1} + p_b)
//   O^{m-1} = I^m  (chaining); O given at the last layer's output (R4)
//   boundaries: even floor(iL/n) (R3), stochastic P:167-171 with the R5 SplitMix64 stream.
#include <cmath>
#include <cstdio>
#include <cstring>
#include <new>

#include "internal.h"

using namespace splitcnn;

namespace splitcnn {

LevelDesc make_level_desc(const Level &l) {
    LevelDesc d;
    std::memset(&d, 0, sizeof(d));
    d.N = l.N; d.C = l.C; d.Cpad = l.Cpad; d.H = l.H; d.W = l.W;
    d.nh = l.nh(); d.nw = l.nw();
    for (int i = 0; i <= d.nh; ++i) d.bh[i] = l.bh[i];
    for (int j = 0; j <= d.nw; ++j) d.bw[j] = l.bw[j];
    return d;
}

LayerDesc make_layer_desc(const LayerGeom &g) {
    LayerDesc d;
    std::memset(&d, 0, sizeof(d));
    d.kh = g.L.kh; d.kw = g.L.kw; d.sh = g.L.sh; d.sw = g.L.sw;
    for (size_t i = 0; i < g.pad_h.size(); ++i) d.pad_h[i] = g.pad_h[i];
    for (size_t j = 0; j < g.pad_w.size(); ++j) d.pad_w[j] = g.pad_w[j];
    return d;
}

}  // namespace splitcnn

static int out_len(int L, int k, int s, int pb, int pe) {
    int num = L + pb + pe - k;
    if (num < 0) return 0;
    return num / s + 1;
}

extern "C" splitcnn_status_t splitcnn_boundaries_even(int32_t L, int32_t n, int32_t *O) {
    if (!O || n < 1 || n > L) return fail(SPLITCNN_ERR_INVALID_VALUE, "boundaries_even: need 1 <= n <= L");
    for (int i = 0; i <= n; ++i) O[i] = (int32_t)(((int64_t)i * L) / n);
    return SPLITCNN_OK;
}

namespace {
struct SplitMix64 {
    uint64_t s;
    uint64_t next() {
        s += 0x9E3779B97F4A7C15ull;
        uint64_t z = s;
        z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
        z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
        return z ^ (z >> 31);
    }
};

void draw_dim(SplitMix64 &g, int L, int n, double omega, int32_t *O) {
    O[0] = 0;
    for (int i = 1; i < n; ++i) {
        // DiscreteUniform(ceil((i - w) L / N), floor((i + w) L / N)), inclusive
        long lo = (long)std::ceil((i - omega) * L / n);
        long hi = (long)std::floor((i + omega) * L / n);
        if (lo > hi) O[i] = (int32_t)(((int64_t)i * L) / n);   // R5: empty range, no draw
        else O[i] = (int32_t)(lo + (long)(g.next() % (uint64_t)(hi - lo + 1)));
    }
    O[n] = L;
}
}  // namespace

extern "C" splitcnn_status_t splitcnn_boundaries_random(int32_t Lh, int32_t nh, int32_t Lw, int32_t nw,
                                                        double omega, uint64_t seed, uint64_t step,
                                                        int32_t *O_h, int32_t *O_w) {
    if (!O_h || !O_w) return fail(SPLITCNN_ERR_INVALID_VALUE, "boundaries_random: null output");
    if (!(omega >= 0.0 && omega < 0.5)) return fail(SPLITCNN_ERR_INVALID_VALUE, "omega must be in [0, 0.5) (P:171)");
    if (nh < 1 || nh > Lh || nw < 1 || nw > Lw) return fail(SPLITCNN_ERR_INVALID_VALUE, "need 1 <= n <= L");
    SplitMix64 g{seed ^ (step * 0x9E3779B97F4A7C15ull)};
    draw_dim(g, Lh, nh, omega, O_h);
    draw_dim(g, Lw, nw, omega, O_w);
    return SPLITCNN_OK;
}

static bool strictly_increasing(const std::vector<int32_t> &v) {
    for (size_t i = 0; i + 1 < v.size(); ++i)
        if (v[i + 1] <= v[i]) return false;
    return true;
}

extern "C" splitcnn_status_t splitcnn_plan_create(const splitcnn_layer_t *layers, int32_t nlayers, int32_t N,
                                                  int32_t C, int32_t H, int32_t W, const int32_t *O_h,
                                                  int32_t n_h, const int32_t *O_w, int32_t n_w,
                                                  splitcnn_plan_t *out) {
    if (!out || !layers || !O_h || !O_w || nlayers < 1 || N < 1 || C < 1 || H < 1 || W < 1)
        return fail(SPLITCNN_ERR_INVALID_VALUE, "plan_create: bad argument");
    if (n_h < 1 || n_w < 1 || n_h > kMaxSplits || n_w > kMaxSplits)
        return fail(SPLITCNN_ERR_INVALID_VALUE, "plan_create: patch grid must be 1..32 per dimension");
    *out = nullptr;
    // forward pass over sizes
    std::vector<int> Hs{H}, Ws{W}, Cs{C};
    for (int m = 0; m < nlayers; ++m) {
        const splitcnn_layer_t &l = layers[m];
        if (l.op != SPLITCNN_OP_CONV && l.op != SPLITCNN_OP_MAXPOOL)
            return fail(SPLITCNN_ERR_INVALID_VALUE, "plan_create: unknown op");
        if (l.kh < 1 || l.kw < 1 || l.sh < 1 || l.sw < 1 || l.ph_b < 0 || l.pw_b < 0 || l.ph_e < 0 || l.pw_e < 0)
            return fail(SPLITCNN_ERR_INVALID_VALUE, "plan_create: bad window / stride / padding");
        if (l.cin != Cs.back()) return fail(SPLITCNN_ERR_INVALID_VALUE, "plan_create: channel chain mismatch");
        if (l.op == SPLITCNN_OP_MAXPOOL && l.cout != l.cin)
            return fail(SPLITCNN_ERR_INVALID_VALUE, "plan_create: maxpool needs cout == cin");
        if (l.op == SPLITCNN_OP_MAXPOOL && l.kh * l.kw > 127)
            return fail(SPLITCNN_ERR_UNSUPPORTED, "plan_create: pool window > 127 elements");
        int ho = out_len(Hs.back(), l.kh, l.sh, l.ph_b, l.ph_e);
        int wo = out_len(Ws.back(), l.kw, l.sw, l.pw_b, l.pw_e);
        if (ho <= 0 || wo <= 0) return fail(SPLITCNN_ERR_INVALID_VALUE, "plan_create: output size <= 0");
        Hs.push_back(ho); Ws.push_back(wo); Cs.push_back(l.cout);
    }
    std::vector<int32_t> Oh(O_h, O_h + n_h + 1), Ow(O_w, O_w + n_w + 1);
    if (Oh[0] != 0 || Oh[n_h] != Hs.back() || Ow[0] != 0 || Ow[n_w] != Ws.back())
        return fail(SPLITCNN_ERR_INVALID_VALUE, "plan_create: O must run from 0 to the last layer's output length");
    if (!strictly_increasing(Oh) || !strictly_increasing(Ow))
        return fail(SPLITCNN_ERR_INVALID_VALUE, "plan_create: O must be strictly increasing (empty patch)");

    auto *p = new (std::nothrow) splitcnn_plan_s;
    if (!p) return fail(SPLITCNN_ERR_OOM, "plan_create: out of host memory");
    p->N = N;
    p->levels.resize(nlayers + 1);
    p->layers.resize(nlayers);
    for (int m = 0; m <= nlayers; ++m) {
        Level &lv = p->levels[m];
        lv.N = N; lv.C = Cs[m]; lv.Cpad = round_up(Cs[m], 8); lv.H = Hs[m]; lv.W = Ws[m];
    }
    p->levels[nlayers].bh = Oh;
    p->levels[nlayers].bw = Ow;
    for (int m = nlayers - 1; m >= 0; --m) {
        const splitcnn_layer_t &l = layers[m];
        const Level &outl = p->levels[m + 1];
        Level &inl = p->levels[m];
        LayerGeom &g = p->layers[m];
        g.L = l;
        for (int dim = 0; dim < 2; ++dim) {
            const std::vector<int32_t> &O = dim == 0 ? outl.bh : outl.bw;
            std::vector<int32_t> &I = dim == 0 ? inl.bh : inl.bw;
            std::vector<int32_t> &pads = dim == 0 ? g.pad_h : g.pad_w;
            int k = dim == 0 ? l.kh : l.kw, s = dim == 0 ? l.sh : l.sw;
            int pb = dim == 0 ? l.ph_b : l.pw_b, pe = dim == 0 ? l.ph_e : l.pw_e;
            int Lin = dim == 0 ? inl.H : inl.W;
            int n = (int)O.size() - 1;
            I.assign(n + 1, 0);
            for (int i = 0; i < n; ++i) I[i] = s * O[i];   // R2
            I[n] = Lin;
            if (!strictly_increasing(I)) {
                delete p;
                return fail(SPLITCNN_ERR_INVALID_VALUE, "plan_create: empty input patch at some level");
            }
            pads.assign(2 * n, 0);
            for (int i = 0; i < n; ++i) {
                pads[2 * i] = (i == 0) ? pb : I[i] + pb - O[i] * s;                         // P:139 (R1)
                pads[2 * i + 1] = (i == n - 1) ? pe : (O[i + 1] - 1) * s + k - (I[i + 1] + pb);
            }
        }
    }
    // kernels index one patch's 8-channel units (N * h * w * Cpad / 8) in 32 bits
    for (const auto &lv : p->levels)
        for (int i = 0; i < lv.nh(); ++i)
            for (int j = 0; j < lv.nw(); ++j)
                if (lv.patch_elems(i, j) / 8 >= (int64_t)1 << 31) {
                    delete p;
                    return fail(SPLITCNN_ERR_UNSUPPORTED, "plan_create: a patch holds >= 2^34 elements");
                }
    *out = p;
    return SPLITCNN_OK;
}

extern "C" splitcnn_status_t splitcnn_plan_destroy(splitcnn_plan_t plan) {
    delete plan;
    return SPLITCNN_OK;
}

extern "C" splitcnn_status_t splitcnn_plan_num_layers(splitcnn_plan_t plan, int32_t *n) {
    if (!plan || !n) return fail(SPLITCNN_ERR_INVALID_VALUE, "null argument");
    *n = (int32_t)plan->layers.size();
    return SPLITCNN_OK;
}

extern "C" splitcnn_status_t splitcnn_plan_level(splitcnn_plan_t plan, int32_t level, splitcnn_level_t *out) {
    if (!plan || !out || level < 0 || level >= (int)plan->levels.size())
        return fail(SPLITCNN_ERR_INVALID_VALUE, "plan_level: bad level");
    const Level &l = plan->levels[level];
    out->N = l.N; out->C = l.C; out->Cpad = l.Cpad; out->H = l.H; out->W = l.W;
    out->n_h = l.nh(); out->n_w = l.nw();
    out->bh = l.bh.data(); out->bw = l.bw.data();
    out->total_elems = l.total();
    return SPLITCNN_OK;
}

extern "C" splitcnn_status_t splitcnn_plan_layer(splitcnn_plan_t plan, int32_t layer, splitcnn_layer_geom_t *out) {
    if (!plan || !out || layer < 0 || layer >= (int)plan->layers.size())
        return fail(SPLITCNN_ERR_INVALID_VALUE, "plan_layer: bad layer");
    const LayerGeom &g = plan->layers[layer];
    out->layer = g.L;
    out->n_h = (int32_t)g.pad_h.size() / 2;
    out->n_w = (int32_t)g.pad_w.size() / 2;
    out->pad_h = g.pad_h.data();
    out->pad_w = g.pad_w.data();
    return SPLITCNN_OK;
}
