// k_memops.cu -- HBM-bound kernels of the split region:
//   split  (Eq. 4)  full tensor  -> patch-major NHWC buffers (+ transpose, + channel pad)
//   merge  (Eq. 7)  patch buffers -> full tensor
//   max-pool forward / backward per patch (Eq. 6 with Op = max-pool)
// One thread moves 8 channels (16 B in bf16) of one pixel; grid.y enumerates patches.
#include <map>
#include <algorithm>
#include <type_traits>
#include <cstdlib>

#include "common.cuh"
#include "kernels.h"

namespace splitcnn {

// ============================================================ split / merge
// Unit index u (< 2^31 per patch, checked on the host) -> coordinates by fast division; the
// divisors are fixed per patch, so each thread builds its multipliers once.
struct Dec3 {
    FastDiv a, b, c;
};
__device__ __forceinline__ Dec3 make_dec3(uint32_t a, uint32_t b, uint32_t c) {
    return {make_fastdiv(a), make_fastdiv(b), make_fastdiv(c)};
}
// u -> (x0 = u % a, x1 = (u / a) % b, x2 = (u / ab) % c, x3 = u / abc)
__device__ __forceinline__ void dec3(uint32_t u, const Dec3 &d, int &x0, int &x1, int &x2, int &x3) {
    uint32_t r;
    u = fdivmod(u, d.a, r); x0 = (int)r;
    u = fdivmod(u, d.b, r); x1 = (int)r;
    u = fdivmod(u, d.c, r); x2 = (int)r;
    x3 = (int)u;
}
template <typename T, bool NCHW, bool S2D = false>
__global__ void __launch_bounds__(256) split_kernel(LevelDesc L, const T *__restrict__ x, T *__restrict__ P, int p0,
                                                    int xc = 0, int row0 = 0, int xH = 0) {
    // x holds rows [row0, row0 + xH) of the logical tensor (a rank's own rows); xH == 0: all L.H rows
    if (xH == 0) xH = L.H;
    const PatchGeo g = patch_geo(L, p0 + blockIdx.y);
    const int G = L.Cpad / 8;
    const uint32_t units = (uint32_t)L.N * g.hp * g.wp * G;
    // NCHW: pixel-fastest (coalesced reads of each channel plane).  NHWC, and the space-to-depth split
    // (whose level may be much wider than its input, e.g. 12 real of 64 channels): channel-fastest, so a
    // warp writes whole 16-byte-group rows of consecutive pixels (coalesced stores)
    constexpr bool PIXEL_FAST = NCHW && !S2D;
    const Dec3 d = PIXEL_FAST ? make_dec3(g.wp, g.hp, G) : make_dec3(G, g.wp, g.hp);
    for (uint32_t u = blockIdx.x * blockDim.x + threadIdx.x; u < units; u += gridDim.x * blockDim.x) {
        int n, h, w, cg;
        if (PIXEL_FAST) dec3(u, d, w, h, cg, n);
        else dec3(u, d, cg, w, h, n);
        const int hg = g.h0 + h, wg = g.w0 + w, c0 = cg * 8;
        float v[8];
        if (S2D && std::is_same<T, __nv_bfloat16>::value) {   // raw 16-bit gathers; all-zero groups skip loads
            const int H2 = 2 * L.H, W2 = 2 * L.W, cmax = min(L.C, 4 * xc);
            uint32_t w4[4] = {0u, 0u, 0u, 0u};
            if (c0 < cmax) {
                const uint16_t *xb = reinterpret_cast<const uint16_t *>(x);
#pragma unroll
                for (int k = 0; k < 8; ++k) {
                    const int cc = c0 + k;
                    if (cc < cmax)
                        w4[k >> 1] |= (uint32_t)__ldg(xb + (((int64_t)n * xc + (cc >> 2)) * H2 + 2 * hg + ((cc >> 1) & 1)) * W2 +
                                                      2 * wg + (cc & 1)) << (16 * (k & 1));
                }
            }
            *reinterpret_cast<uint4 *>(P + g.off + (((int64_t)n * g.hp + h) * g.wp + w) * L.Cpad + c0) =
                make_uint4(w4[0], w4[1], w4[2], w4[3]);
            continue;
        } else if (S2D) {   // level channel 4c + 2ph + pw of (hg, wg) = x[n, c, 2hg + ph, 2wg + pw]  (c < xc; else 0)
            const int C4 = xc, H2 = 2 * L.H, W2 = 2 * L.W, cmax = min(L.C, 4 * xc);
#pragma unroll
            for (int k = 0; k < 8; ++k) {
                const int cc = c0 + k;
                v[k] = (cc < cmax) ? to_f(x[(((int64_t)n * C4 + (cc >> 2)) * H2 + 2 * hg + ((cc >> 1) & 1)) * W2 + 2 * wg + (cc & 1)])
                                   : 0.f;
            }
        } else if (NCHW && std::is_same<T, __nv_bfloat16>::value) {
            // bf16 NCHW: raw 16-bit gathers from up to 8 channel planes packed into one 16-byte store
            const uint16_t *src = reinterpret_cast<const uint16_t *>(x) + (((int64_t)n * L.C + c0) * xH + hg - row0) * L.W + wg;
            const int64_t cs = (int64_t)xH * L.W;
            const int nc = min(8, L.C - c0);
            uint32_t w4[4] = {0u, 0u, 0u, 0u};
#pragma unroll
            for (int k = 0; k < 8; ++k)
                if (k < nc) w4[k >> 1] |= (uint32_t)__ldg(src + k * cs) << (16 * (k & 1));
            *reinterpret_cast<uint4 *>(P + g.off + (((int64_t)n * g.hp + h) * g.wp + w) * L.Cpad + c0) =
                make_uint4(w4[0], w4[1], w4[2], w4[3]);
            continue;
        } else if (NCHW) {
#pragma unroll
            for (int k = 0; k < 8; ++k)
                v[k] = (c0 + k < L.C) ? to_f(x[(((int64_t)n * L.C + c0 + k) * xH + hg - row0) * L.W + wg]) : 0.f;
        } else {
            const T *src = x + (((int64_t)n * xH + hg - row0) * L.W + wg) * L.C + c0;
            if ((L.C & 7) == 0) {
                load8(src, v);
            } else {
#pragma unroll
                for (int k = 0; k < 8; ++k) v[k] = (c0 + k < L.C) ? to_f(src[k]) : 0.f;
            }
        }
        store8(P + g.off + (((int64_t)n * g.hp + h) * g.wp + w) * L.Cpad + c0, v);
    }
}

template <typename T, bool NCHW>
__global__ void __launch_bounds__(256) merge_kernel(LevelDesc L, const T *__restrict__ P, T *__restrict__ y, int p0) {
    const PatchGeo g = patch_geo(L, p0 + blockIdx.y);
    const int G = L.Cpad / 8;
    const uint32_t units = (uint32_t)L.N * g.hp * g.wp * G;
    const Dec3 d = NCHW ? make_dec3(g.wp, g.hp, G) : make_dec3(G, g.wp, g.hp);
    for (uint32_t u = blockIdx.x * blockDim.x + threadIdx.x; u < units; u += gridDim.x * blockDim.x) {
        int n, h, w, cg;
        if (NCHW) dec3(u, d, w, h, cg, n);   
        else dec3(u, d, cg, w, h, n);        
        const int hg = g.h0 + h, wg = g.w0 + w, c0 = cg * 8;
        float v[8];
        load8(P + g.off + (((int64_t)n * g.hp + h) * g.wp + w) * L.Cpad + c0, v);
        if (NCHW) {
#pragma unroll
            for (int k = 0; k < 8; ++k)
                if (c0 + k < L.C) y[(((int64_t)n * L.C + c0 + k) * L.H + hg) * L.W + wg] = from_f<T>(v[k]);
        } else {
            T *dst = y + (((int64_t)n * L.H + hg) * L.W + wg) * L.C + c0;
            if ((L.C & 7) == 0) {
                store8(dst, v);
            } else {
#pragma unroll
                for (int k = 0; k < 8; ++k)
                    if (c0 + k < L.C) dst[k] = from_f<T>(v[k]);
            }
        }
    }
}

// HBM-bound kernels: about 16 resident 256-thread blocks per SM over the whole launch (grid.y =
// patches), each thread striding over several 8-channel units -- not one short-lived block per 256 units
static int npatch_launch = 1;
static int grid_x_for(int64_t units) {
    int64_t b = (units + 255) / 256;
    const int64_t cap = std::max<int64_t>(1, (148 * 16 + npatch_launch - 1) / npatch_launch);
    return (int)std::max<int64_t>(1, std::min(b, cap));
}

// Register-heavy kernels (the 3x3 / stride-2 pool backward: a few resident blocks per SM, long per-thread
// loops): exactly one wave of resident blocks over all patches -- its old grid left 1.3 waves, a tail with
// a third of the SMs busy (ncu, C3 max-pool: 248 -> 200 us)
template <typename K>
static dim3 resident_grid(K kernel, int64_t units, int npatch) {
    static std::map<const void *, int> bps_cache;
    int &bps = bps_cache[(const void *)kernel];
    if (!bps) {
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&bps, kernel, 256, 0);
        if (bps <= 0) bps = 1;
    }
    int dev = 0, sms = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    const int64_t per_patch = std::max<int64_t>(1, (int64_t)std::max(1, sms) * bps / std::max(1, npatch));
    return dim3((unsigned)std::max<int64_t>(1, std::min(per_patch, (units + 255) / 256)), (unsigned)npatch);
}

static int64_t max_patch_units(const Level &L, int p0, int p1, int per_pixel) {
    int64_t m = 0;
    for (int q = p0; q < p1; ++q) {
        int i = q / L.nw(), j = q % L.nw();
        int64_t u = (int64_t)L.N * L.ph(i) * L.pw(j) * per_pixel;
        if (u > m) m = u;
    }
    return m;
}

template <typename T>
void launch_split_t(const Level &L, const void *x, int layout, void *P, int p0, int p1, cudaStream_t st, int xc,
                    int row0, int xH) {
    npatch_launch = p1 - p0;
    dim3 grid(grid_x_for(max_patch_units(L, p0, p1, L.Cpad / 8)), p1 - p0);
    LevelDesc d = make_level_desc(L);
    if (layout == SPLITCNN_NCHW_S2D)
        { split_kernel<T, true, true><<<grid, 256, 0, st>>>(d, (const T *)x, (T *)P, p0, xc > 0 ? xc : L.C / 4); count_launch(); }
    else if (layout == SPLITCNN_NCHW)
        { split_kernel<T, true><<<grid, 256, 0, st>>>(d, (const T *)x, (T *)P, p0, 0, row0, xH); count_launch(); }
    else
        { split_kernel<T, false><<<grid, 256, 0, st>>>(d, (const T *)x, (T *)P, p0, 0, row0, xH); count_launch(); }
}

template <typename T>
void launch_merge_t(const Level &L, const void *P, void *y, int layout, int p0, int p1, cudaStream_t st) {
    npatch_launch = p1 - p0;
    dim3 grid(grid_x_for(max_patch_units(L, p0, p1, L.Cpad / 8)), p1 - p0);
    LevelDesc d = make_level_desc(L);
    if (layout == SPLITCNN_NCHW)
        { merge_kernel<T, true><<<grid, 256, 0, st>>>(d, (const T *)P, (T *)y, p0); count_launch(); }
    else
        { merge_kernel<T, false><<<grid, 256, 0, st>>>(d, (const T *)P, (T *)y, p0); count_launch(); }
}

void launch_split(splitcnn_dtype_t dt, const Level &L, const void *x, int layout, void *P, int p0, int p1, cudaStream_t st,
                  int xc, int row0, int xH) {
    if (dt == SPLITCNN_BF16) launch_split_t<__nv_bfloat16>(L, x, layout, P, p0, p1, st, xc, row0, xH);
    else launch_split_t<float>(L, x, layout, P, p0, p1, st, xc, row0, xH);
}
void launch_merge(splitcnn_dtype_t dt, const Level &L, const void *P, void *y, int layout, int p0, int p1, cudaStream_t st) {
    if (dt == SPLITCNN_BF16) launch_merge_t<__nv_bfloat16>(L, P, y, layout, p0, p1, st);
    else launch_merge_t<float>(L, P, y, layout, p0, p1, st);
}

// ============================================================ max-pool
// Forward: one thread = one output pixel x 8 channels.  The window max uses strict '>'
// in row-major window order, so the argmax is the FIRST maximum (R9).  Padding is skipped (R7).
template <typename T>
__global__ void __launch_bounds__(256) pool_fwd_kernel(LevelDesc Li, LevelDesc Lo, LayerDesc ly, const T *__restrict__ X,
                                                       T *__restrict__ Y, uint8_t *__restrict__ A, int p0, int relu_bit) {
    const int q = p0 + blockIdx.y;
    const PatchGeo gi = patch_geo(Li, q), go = patch_geo(Lo, q);
    const int pt = ly.pad_h[2 * gi.i], pl = ly.pad_w[2 * gi.j];
    const int G = Li.Cpad / 8;
    const uint32_t units = (uint32_t)Lo.N * go.hp * go.wp * G;
    const Dec3 d = make_dec3(G, go.wp, go.hp);
    for (uint32_t u = blockIdx.x * blockDim.x + threadIdx.x; u < units; u += gridDim.x * blockDim.x) {
        int cg, ow, oh, n;
        dec3(u, d, cg, ow, oh, n);
        float best[8];
        int arg[8];
#pragma unroll
        for (int k = 0; k < 8; ++k) { best[k] = -INFINITY; arg[k] = -1; }
        for (int r = 0; r < ly.kh; ++r) {
            const int h = oh * ly.sh - pt + r;
            if (h < 0 || h >= gi.hp) continue;
            for (int c = 0; c < ly.kw; ++c) {
                const int w = ow * ly.sw - pl + c;
                if (w < 0 || w >= gi.wp) continue;
                float v[8];
                load8(X + gi.off + (((int64_t)n * gi.hp + h) * gi.wp + w) * Li.Cpad + cg * 8, v);
                const int idx = r * ly.kw + c;
#pragma unroll
                for (int k = 0; k < 8; ++k)
                    if (arg[k] < 0 || v[k] > best[k]) { best[k] = v[k]; arg[k] = idx; }
            }
        }
        const int64_t o = go.off + (((int64_t)n * go.hp + oh) * go.wp + ow) * Lo.Cpad + cg * 8;
        store8(Y + o, best);
        uint32_t lo = 0, hi = 0;
#pragma unroll
        for (int k = 0; k < 8; ++k) {
            uint32_t b = (uint32_t)(arg[k] & 0x7f) | ((relu_bit && best[k] > 0.f) ? 0x80u : 0u);
            if (k < 4) lo |= b << (8 * k); else hi |= b << (8 * (k - 4));
        }
        *reinterpret_cast<uint2 *>(A + o) = make_uint2(lo, hi);
    }
}

__device__ __forceinline__ int floordiv(int a, int b) { return (a >= 0) ? a / b : -((-a + b - 1) / b); }

// Backward: gather form -- one thread = one INPUT pixel x 8 channels; it visits every window
// that covers the pixel in (oh, ow) ascending order and adds dY where the argmax points at it.
// Every dX element is written once (no memset, no atomics, deterministic order).
template <typename T>
__global__ void __launch_bounds__(256) pool_bwd_kernel(LevelDesc Li, LevelDesc Lo, LayerDesc ly, const T *__restrict__ dY,
                                                       const uint8_t *__restrict__ A, T *__restrict__ dX, int p0, int relu_bit) {
    const int q = p0 + blockIdx.y;
    const PatchGeo gi = patch_geo(Li, q), go = patch_geo(Lo, q);
    const int pt = ly.pad_h[2 * gi.i], pl = ly.pad_w[2 * gi.j];
    const int G = Li.Cpad / 8;
    const uint32_t units = (uint32_t)Li.N * gi.hp * gi.wp * G;
    const Dec3 d = make_dec3(G, gi.wp, gi.hp);
    for (uint32_t u = blockIdx.x * blockDim.x + threadIdx.x; u < units; u += gridDim.x * blockDim.x) {
        int cg, w, h, n;
        dec3(u, d, cg, w, h, n);
        int oh_lo = floordiv(h + pt - ly.kh, ly.sh) + 1, oh_hi = floordiv(h + pt, ly.sh);
        int ow_lo = floordiv(w + pl - ly.kw, ly.sw) + 1, ow_hi = floordiv(w + pl, ly.sw);
        if (oh_lo < 0) oh_lo = 0;
        if (ow_lo < 0) ow_lo = 0;
        if (oh_hi > go.hp - 1) oh_hi = go.hp - 1;
        if (ow_hi > go.wp - 1) ow_hi = go.wp - 1;
        float acc[8];
#pragma unroll
        for (int k = 0; k < 8; ++k) acc[k] = 0.f;
        for (int oh = oh_lo; oh <= oh_hi; ++oh)
            for (int ow = ow_lo; ow <= ow_hi; ++ow) {
                const int idx = (h - (oh * ly.sh - pt)) * ly.kw + (w - (ow * ly.sw - pl));
                const int64_t o = go.off + (((int64_t)n * go.hp + oh) * go.wp + ow) * Lo.Cpad + cg * 8;
                const uint2 a2 = __ldg(reinterpret_cast<const uint2 *>(A + o));
                float g[8];
                load8(dY + o, g);
#pragma unroll
                for (int k = 0; k < 8; ++k) {
                    const uint32_t b = ((k < 4 ? a2.x : a2.y) >> (8 * (k & 3))) & 0xffu;
                    const bool hit = (int)(b & 0x7fu) == idx && (!relu_bit || (b & 0x80u));
                    acc[k] += hit ? g[k] : 0.f;
                }
            }
        store8(dX + gi.off + (((int64_t)n * gi.hp + h) * gi.wp + w) * Li.Cpad + cg * 8, acc);
    }
}

// Backward for non-overlapping windows that tile the patch exactly (k = s, p = 0, hp = ho*s, wp = wo*s,
// the VGG case): one thread per OUTPUT pixel x 8 channels reads dY + argmax once and writes the whole
// k x k window (dY at the argmax, 0 elsewhere) -- every dX element written exactly once, coalesced.
template <typename T>
__global__ void __launch_bounds__(256) pool_bwd_scatter_kernel(LevelDesc Li, LevelDesc Lo, LayerDesc ly,
                                                               const T *__restrict__ dY, const uint8_t *__restrict__ A,
                                                               T *__restrict__ dX, int p0, int relu_bit) {
    const int q = p0 + blockIdx.y;
    const PatchGeo gi = patch_geo(Li, q), go = patch_geo(Lo, q);
    const int G = Li.Cpad / 8;
    const uint32_t units = (uint32_t)Lo.N * go.hp * go.wp * G;
    const Dec3 d = make_dec3(G, go.wp, go.hp);
    const uint32_t stride = gridDim.x * blockDim.x;
    // two units per iteration: both units' dY + argmax loads are in flight before the first store
    for (uint32_t u0 = blockIdx.x * blockDim.x + threadIdx.x; u0 < units; u0 += 2 * stride) {
        int64_t o[2];
        uint2 a2[2];
        float g[2][8];
        int oh[2], ow[2], n[2], cg[2];
        bool ok[2];
#pragma unroll
        for (int k = 0; k < 2; ++k) {
            const uint32_t u = u0 + k * stride;
            ok[k] = u < units;
            dec3(ok[k] ? u : u0, d, cg[k], ow[k], oh[k], n[k]);
            o[k] = go.off + (((int64_t)n[k] * go.hp + oh[k]) * go.wp + ow[k]) * Lo.Cpad + cg[k] * 8;
            if (ok[k]) {
                a2[k] = __ldg(reinterpret_cast<const uint2 *>(A + o[k]));
                load8(dY + o[k], g[k]);
            }
        }
#pragma unroll
        for (int k = 0; k < 2; ++k) {
            if (!ok[k]) continue;
            for (int r = 0; r < ly.kh; ++r)
                for (int c = 0; c < ly.kw; ++c) {
                    const int idx = r * ly.kw + c;
                    float v[8];
#pragma unroll
                    for (int e = 0; e < 8; ++e) {
                        const uint32_t b = ((e < 4 ? a2[k].x : a2[k].y) >> (8 * (e & 3))) & 0xffu;
                        v[e] = ((int)(b & 0x7fu) == idx && (!relu_bit || (b & 0x80u))) ? g[k][e] : 0.f;
                    }
                    const int h = oh[k] * ly.sh + r, w = ow[k] * ly.sw + c;
                    store8(dX + gi.off + (((int64_t)n[k] * gi.hp + h) * gi.wp + w) * Li.Cpad + cg[k] * 8, v);
                }
        }
    }
}

// Backward for 3x3 / stride-2 windows (ResNet's max-pool, any pads): one thread = a 2x2 block of
// input pixels (padded rows 2a+1, 2a+2 and columns 2b+1, 2b+2) x 8 channels.  Those four pixels are
// covered exactly by the windows (a|a+1, b|b+1); the thread loads each of them once (instead of once
// per covered pixel, 9 loads for 4 pixels in the gather form) and sums in the gather kernel's order
// (oh ascending, then ow) -> bitwise the same dX.
// 8 channels kept packed until used (bf16: 4 registers instead of 8) -- the 3x3 backward holds four of them
template <typename T> struct Raw8;
template <> struct Raw8<__nv_bfloat16> {
    uint4 w;
    __device__ __forceinline__ void load(const __nv_bfloat16 *p) { w = __ldg(reinterpret_cast<const uint4 *>(p)); }
    __device__ __forceinline__ float get(int k) const {
        const uint32_t x = k < 2 ? w.x : k < 4 ? w.y : k < 6 ? w.z : w.w;
        return __uint_as_float((k & 1) ? (x & 0xFFFF0000u) : (x << 16));
    }
};
template <> struct Raw8<float> {
    float4 a, b;
    __device__ __forceinline__ void load(const float *p) {
        a = __ldg(reinterpret_cast<const float4 *>(p));
        b = __ldg(reinterpret_cast<const float4 *>(p) + 1);
    }
    __device__ __forceinline__ float get(int k) const {
        return k == 0 ? a.x : k == 1 ? a.y : k == 2 ? a.z : k == 3 ? a.w : k == 4 ? b.x : k == 5 ? b.y : k == 6 ? b.z : b.w;
    }
};

template <typename T>
__global__ void __launch_bounds__(256, 4) pool_bwd_k3s2_kernel(LevelDesc Li, LevelDesc Lo, LayerDesc ly,
                                                            const T *__restrict__ dY, const uint8_t *__restrict__ A,
                                                            T *__restrict__ dX, int p0, int relu_bit) {
    const int q = p0 + blockIdx.y;
    const PatchGeo gi = patch_geo(Li, q), go = patch_geo(Lo, q);
    const int pt = ly.pad_h[2 * gi.i], pl = ly.pad_w[2 * gi.j];
    const int a_lo = floordiv(pt - 1, 2), a_hi = floordiv(gi.hp + pt - 2, 2);
    const int b_lo = floordiv(pl - 1, 2), b_hi = floordiv(gi.wp + pl - 2, 2);
    const int na = a_hi - a_lo + 1, nb = b_hi - b_lo + 1;
    const int G = Li.Cpad / 8;
    if (na <= 0 || nb <= 0) return;
    const uint32_t units = (uint32_t)Li.N * na * nb * G;
    const Dec3 d = make_dec3(G, nb, na);
    for (uint32_t u = blockIdx.x * blockDim.x + threadIdx.x; u < units; u += gridDim.x * blockDim.x) {
        int cg, bi, ai, n;
        dec3(u, d, cg, bi, ai, n);
        const int a = a_lo + ai, b = b_lo + bi;
        uint2 am[4];
        Raw8<T> g[4];
        bool in[4];
#pragma unroll
        for (int t = 0; t < 4; ++t) {            // t = 2*(oh - a) + (ow - b)
            const int oh = a + (t >> 1), ow = b + (t & 1);
            in[t] = oh >= 0 && oh < go.hp && ow >= 0 && ow < go.wp;
            if (in[t]) {
                const int64_t o = go.off + (((int64_t)n * go.hp + oh) * go.wp + ow) * Lo.Cpad + cg * 8;
                am[t] = __ldg(reinterpret_cast<const uint2 *>(A + o));
                g[t].load(dY + o);
            }
        }
        const uint32_t keep = relu_bit ? 0xFFFFFFFFu : 0x7F7F7F7Fu;
#pragma unroll
        for (int py = 0; py < 2; ++py)
#pragma unroll
            for (int px = 0; px < 2; ++px) {
                const int h = 2 * a + 1 + py - pt, w = 2 * b + 1 + px - pl;
                if (h < 0 || h >= gi.hp || w < 0 || w >= gi.wp) continue;
                float acc[8];
#pragma unroll
                for (int k = 0; k < 8; ++k) acc[k] = 0.f;
#pragma unroll
                for (int t = 0; t < 4; ++t) {
                    const int dh = t >> 1, dw = t & 1;
                    if (!in[t] || (dh && !py) || (dw && !px)) continue;   // window (a+dh, b+dw) covers the pixel?
                    const int idx = (1 + py - 2 * dh) * 3 + (1 + px - 2 * dw);
                    // hit bytes by one packed compare per 4 argmax bytes (| 0x80 when the ReLU bit gates)
                    const uint32_t tgt = (uint32_t)(idx | (relu_bit ? 0x80 : 0)) * 0x01010101u;
                    const uint32_t e_lo = __vcmpeq4(am[t].x & keep, tgt), e_hi = __vcmpeq4(am[t].y & keep, tgt);
#pragma unroll
                    for (int k = 0; k < 8; ++k) {
                        const bool hit = ((k < 4 ? e_lo : e_hi) >> (8 * (k & 3))) & 1u;
                        acc[k] += hit ? g[t].get(k) : 0.f;
                    }
                }
                store8(dX + gi.off + (((int64_t)n * gi.hp + h) * gi.wp + w) * Li.Cpad + cg * 8, acc);
            }
    }
}

// ------------------------------------------------------------ 2x2 / stride-2 bf16 fast paths (VGG pools)
// Windows tile the patch exactly (k = s = 2, no padding, hp = 2 ho): no bounds checks, and the 8 channels
// of a unit are handled as 4 bf16x2 words with packed compares / selects -- the generic kernels spend
// ~440 instructions per unit (ncu), these a fraction of it.  Same results bit for bit: strict '>' in
// row-major window order (first maximum), ReLU bit = [max > 0] exactly as the float compare.
__device__ __forceinline__ uint32_t bf2_gt(uint32_t a, uint32_t b) {
    return __hgt2_mask(*reinterpret_cast<const __nv_bfloat162 *>(&a), *reinterpret_cast<const __nv_bfloat162 *>(&b));
}

__global__ void __launch_bounds__(256) pool2x2_fwd_bf16_kernel(LevelDesc Li, LevelDesc Lo, const __nv_bfloat16 *__restrict__ X,
                                                               __nv_bfloat16 *__restrict__ Y, uint8_t *__restrict__ A,
                                                               int p0, int relu_bit) {
    const int q = p0 + blockIdx.y;
    const PatchGeo gi = patch_geo(Li, q), go = patch_geo(Lo, q);
    const int G = Li.Cpad / 8;
    const uint32_t units = (uint32_t)Lo.N * go.hp * go.wp * G;
    const Dec3 d = make_dec3(G, go.wp, go.hp);
    for (uint32_t u = blockIdx.x * blockDim.x + threadIdx.x; u < units; u += gridDim.x * blockDim.x) {
        int cg, ow, oh, n;
        dec3(u, d, cg, ow, oh, n);
        const __nv_bfloat16 *x0 = X + gi.off + (((int64_t)n * gi.hp + 2 * oh) * gi.wp + 2 * ow) * Li.Cpad + cg * 8;
        const int64_t rs = (int64_t)gi.wp * Li.Cpad;
        uint4 v[4];
        v[0] = __ldg(reinterpret_cast<const uint4 *>(x0));
        v[1] = __ldg(reinterpret_cast<const uint4 *>(x0 + Li.Cpad));
        v[2] = __ldg(reinterpret_cast<const uint4 *>(x0 + rs));
        v[3] = __ldg(reinterpret_cast<const uint4 *>(x0 + rs + Li.Cpad));
        uint32_t best[4], arg[4];
#pragma unroll
        for (int j = 0; j < 4; ++j) {
            const uint32_t *w0 = reinterpret_cast<const uint32_t *>(&v[0]);
            best[j] = w0[j];
            arg[j] = 0;
#pragma unroll
            for (int t = 1; t < 4; ++t) {
                const uint32_t w = reinterpret_cast<const uint32_t *>(&v[t])[j];
                const uint32_t m = bf2_gt(w, best[j]);
                best[j] = (w & m) | (best[j] & ~m);
                arg[j] = ((uint32_t)(t * 0x00010001u) & m) | (arg[j] & ~m);
            }
        }
        const int64_t o = go.off + (((int64_t)n * go.hp + oh) * go.wp + ow) * Lo.Cpad + cg * 8;
        *reinterpret_cast<uint4 *>(Y + o) = make_uint4(best[0], best[1], best[2], best[3]);
        // argmax bytes as in the 3x3 kernel: window index in bytes 0 / 2 of each arg word | [max > 0] << 7, one PRMT
        uint32_t bw[4];
#pragma unroll
        for (int j = 0; j < 4; ++j) bw[j] = arg[j] | (relu_bit ? (bf2_gt(best[j], 0u) & 0x00800080u) : 0u);
        *reinterpret_cast<uint2 *>(A + o) = make_uint2(__byte_perm(bw[0], bw[1], 0x6420), __byte_perm(bw[2], bw[3], 0x6420));
    }
}

// 3x3 / stride-2 bf16 forward (ResNet's max-pool, pads per patch): 9 window positions in row-major
// order with per-position bounds (skipped = -inf), packed bf16x2 compares; bit-identical to the generic
// kernel (first maximum, strict '>'; the first in-bounds position initialises the maximum).
__global__ void __launch_bounds__(256, 4) pool3x3s2_fwd_bf16_kernel(LevelDesc Li, LevelDesc Lo, LayerDesc ly,
                                                                 const __nv_bfloat16 *__restrict__ X,
                                                                 __nv_bfloat16 *__restrict__ Y, uint8_t *__restrict__ A,
                                                                 int p0, int relu_bit) {
    const int q = p0 + blockIdx.y;
    const PatchGeo gi = patch_geo(Li, q), go = patch_geo(Lo, q);
    const int pt = ly.pad_h[2 * gi.i], pl = ly.pad_w[2 * gi.j];
    const int G = Li.Cpad / 8;
    const uint32_t units = (uint32_t)Lo.N * go.hp * go.wp * G;
    const Dec3 d = make_dec3(G, go.wp, go.hp);
    for (uint32_t u = blockIdx.x * blockDim.x + threadIdx.x; u < units; u += gridDim.x * blockDim.x) {
        int cg, ow, oh, n;
        dec3(u, d, cg, ow, oh, n);
        const int h0 = 2 * oh - pt, w0 = 2 * ow - pl;
        uint4 v[9];
        uint32_t inb = 0;
#pragma unroll
        for (int t = 0; t < 9; ++t) {
            const int h = h0 + t / 3, w = w0 + t % 3;
            if (h >= 0 && h < gi.hp && w >= 0 && w < gi.wp) {
                inb |= 1u << t;
                v[t] = __ldg(reinterpret_cast<const uint4 *>(X + gi.off + (((int64_t)n * gi.hp + h) * gi.wp + w) * Li.Cpad + cg * 8));
            }
        }
        uint32_t best[4] = {0, 0, 0, 0}, arg[4] = {0, 0, 0, 0};
        bool first = true;
        if (inb == 0x1FFu) {   // the whole window inside the patch (all but the border rows / columns): no checks
            const uint32_t *w0v = reinterpret_cast<const uint32_t *>(&v[0]);
#pragma unroll
            for (int j = 0; j < 4; ++j) best[j] = w0v[j];
#pragma unroll
            for (int t = 1; t < 9; ++t) {
                const uint32_t *w = reinterpret_cast<const uint32_t *>(&v[t]);
#pragma unroll
                for (int j = 0; j < 4; ++j) {
                    const uint32_t m = bf2_gt(w[j], best[j]);
                    best[j] = (w[j] & m) | (best[j] & ~m);
                    arg[j] = ((uint32_t)(t * 0x00010001u) & m) | (arg[j] & ~m);
                }
            }
            first = false;
        } else {
#pragma unroll
            for (int t = 0; t < 9; ++t) {
                if (!(inb & (1u << t))) continue;
                const uint32_t *w = reinterpret_cast<const uint32_t *>(&v[t]);
#pragma unroll
                for (int j = 0; j < 4; ++j) {
                    const uint32_t m = first ? 0xFFFFFFFFu : bf2_gt(w[j], best[j]);
                    best[j] = (w[j] & m) | (best[j] & ~m);
                    arg[j] = ((uint32_t)(t * 0x00010001u) & m) | (arg[j] & ~m);
                }
                first = false;
            }
        }
        const int64_t o = go.off + (((int64_t)n * go.hp + oh) * go.wp + ow) * Lo.Cpad + cg * 8;
        if (first) {   // no in-bounds position: impossible for a valid plan (pads < k); -inf
            const uint32_t ninf = 0xFF80FF80u;
            best[0] = best[1] = best[2] = best[3] = ninf;
        }
        *reinterpret_cast<uint4 *>(Y + o) = make_uint4(best[0], best[1], best[2], best[3]);
        // argmax byte = window index (bits 0-3, already in bytes 0 / 2 of each arg word) | [max > 0] << 7 (the
        // packed bf16 compare with +0: false for NaN, zero and negatives); two words' bytes 0 / 2 by one PRMT
        uint32_t bw[4];
#pragma unroll
        for (int j = 0; j < 4; ++j) bw[j] = arg[j] | (relu_bit ? (bf2_gt(best[j], 0u) & 0x00800080u) : 0u);
        *reinterpret_cast<uint2 *>(A + o) = make_uint2(__byte_perm(bw[0], bw[1], 0x6420), __byte_perm(bw[2], bw[3], 0x6420));
    }
}

__global__ void __launch_bounds__(256) pool2x2_bwd_bf16_kernel(LevelDesc Li, LevelDesc Lo, const __nv_bfloat16 *__restrict__ dY,
                                                               const uint8_t *__restrict__ A, __nv_bfloat16 *__restrict__ dX,
                                                               int p0, int relu_bit) {
    const int q = p0 + blockIdx.y;
    const PatchGeo gi = patch_geo(Li, q), go = patch_geo(Lo, q);
    const int G = Li.Cpad / 8;
    const uint32_t units = (uint32_t)Lo.N * go.hp * go.wp * G;
    const Dec3 d = make_dec3(G, go.wp, go.hp);
    for (uint32_t u = blockIdx.x * blockDim.x + threadIdx.x; u < units; u += gridDim.x * blockDim.x) {
        int cg, ow, oh, n;
        dec3(u, d, cg, ow, oh, n);
        const int64_t o = go.off + (((int64_t)n * go.hp + oh) * go.wp + ow) * Lo.Cpad + cg * 8;
        const uint2 a2 = __ldg(reinterpret_cast<const uint2 *>(A + o));
        const uint4 g = __ldg(reinterpret_cast<const uint4 *>(dY + o));
        __nv_bfloat16 *x0 = dX + gi.off + (((int64_t)n * gi.hp + 2 * oh) * gi.wp + 2 * ow) * Li.Cpad + cg * 8;
        const int64_t rs = (int64_t)gi.wp * Li.Cpad;
        // hit byte k <=> argmax byte == t (| 0x80 when the ReLU bit gates it)
        const uint32_t keep = relu_bit ? 0xFFFFFFFFu : 0x7F7F7F7Fu;
#pragma unroll
        for (int t = 0; t < 4; ++t) {
            const uint32_t tgt = (uint32_t)(t | (relu_bit ? 0x80 : 0)) * 0x01010101u;
            const uint32_t e_lo = __vcmpeq4(a2.x & keep, tgt), e_hi = __vcmpeq4(a2.y & keep, tgt);
            const uint4 r = make_uint4(g.x & __byte_perm(e_lo, 0, 0x1100), g.y & __byte_perm(e_lo, 0, 0x3322),
                                       g.z & __byte_perm(e_hi, 0, 0x1100), g.w & __byte_perm(e_hi, 0, 0x3322));
            *reinterpret_cast<uint4 *>(x0 + (t >> 1) * rs + (t & 1) * Li.Cpad) = r;
        }
    }
}

template <typename T>
void launch_pool_fwd_t(const Level &Li, const Level &Lo, const LayerGeom &g, const void *x, void *y, uint8_t *a,
                       int relu_bit, int p0, int p1, cudaStream_t st) {
    npatch_launch = p1 - p0;
    dim3 grid(grid_x_for(max_patch_units(Lo, p0, p1, Lo.Cpad / 8)), p1 - p0);
    bool exact = std::is_same<T, __nv_bfloat16>::value && g.L.kh == 2 && g.L.kw == 2 && g.L.sh == 2 && g.L.sw == 2;
    for (size_t i = 0; exact && i < g.pad_h.size(); ++i) exact = g.pad_h[i] == 0;
    for (size_t i = 0; exact && i < g.pad_w.size(); ++i) exact = g.pad_w[i] == 0;
    for (int i = 0; exact && i < Li.nh(); ++i) exact = Li.ph(i) == 2 * Lo.ph(i);
    for (int j = 0; exact && j < Li.nw(); ++j) exact = Li.pw(j) == 2 * Lo.pw(j);
    if (std::is_same<T, __nv_bfloat16>::value && g.L.kh == 3 && g.L.kw == 3 && g.L.sh == 2 && g.L.sw == 2) {
        // (the forward keeps the 16-blocks-per-SM grid: 4 resident at <= 64 registers, so 4 whole waves,
        // measured faster than one resident wave: 0.154 vs 0.168 ms for C3's max-pool)
        pool3x3s2_fwd_bf16_kernel<<<grid, 256, 0, st>>>(make_level_desc(Li), make_level_desc(Lo), make_layer_desc(g),
                                                        (const __nv_bfloat16 *)x, (__nv_bfloat16 *)y, a, p0, relu_bit);
        count_launch();
        return;
    }
    if (exact) {
        pool2x2_fwd_bf16_kernel<<<grid, 256, 0, st>>>(make_level_desc(Li), make_level_desc(Lo), (const __nv_bfloat16 *)x,
                                                      (__nv_bfloat16 *)y, a, p0, relu_bit);
        count_launch();
        return;
    }
    { pool_fwd_kernel<T><<<grid, 256, 0, st>>>(make_level_desc(Li), make_level_desc(Lo), make_layer_desc(g),
                                             (const T *)x, (T *)y, a, p0, relu_bit); count_launch(); }
}
template <typename T>
void launch_pool_bwd_t(const Level &Li, const Level &Lo, const LayerGeom &g, const void *dy, const uint8_t *a, void *dx,
                       int relu_bit, int p0, int p1, cudaStream_t st) {
    bool exact = g.L.kh == g.L.sh && g.L.kw == g.L.sw;
    for (size_t i = 0; exact && i < g.pad_h.size(); ++i) exact = g.pad_h[i] == 0;
    for (size_t i = 0; exact && i < g.pad_w.size(); ++i) exact = g.pad_w[i] == 0;
    for (int i = 0; exact && i < Li.nh(); ++i) exact = Li.ph(i) == Lo.ph(i) * g.L.sh;
    for (int j = 0; exact && j < Li.nw(); ++j) exact = Li.pw(j) == Lo.pw(j) * g.L.sw;
    if (exact && std::is_same<T, __nv_bfloat16>::value && g.L.kh == 2 && g.L.kw == 2) {
        npatch_launch = p1 - p0;
        dim3 grid(grid_x_for(max_patch_units(Lo, p0, p1, Lo.Cpad / 8)), p1 - p0);
        pool2x2_bwd_bf16_kernel<<<grid, 256, 0, st>>>(make_level_desc(Li), make_level_desc(Lo), (const __nv_bfloat16 *)dy,
                                                      a, (__nv_bfloat16 *)dx, p0, relu_bit);
        count_launch();
        return;
    }
    if (exact) {
        npatch_launch = p1 - p0;
        dim3 grid(grid_x_for(max_patch_units(Lo, p0, p1, Lo.Cpad / 8)), p1 - p0);
        pool_bwd_scatter_kernel<T><<<grid, 256, 0, st>>>(make_level_desc(Li), make_level_desc(Lo), make_layer_desc(g),
                                                         (const T *)dy, a, (T *)dx, p0, relu_bit);
        count_launch();
        return;
    }
    npatch_launch = p1 - p0;
    dim3 grid(grid_x_for(max_patch_units(Li, p0, p1, Li.Cpad / 8)), p1 - p0);
    if (g.L.kh == 3 && g.L.kw == 3 && g.L.sh == 2 && g.L.sw == 2) {
        const dim3 g4 = resident_grid(pool_bwd_k3s2_kernel<T>, max_patch_units(Li, p0, p1, Li.Cpad / 8) / 4 + 1, p1 - p0);
        pool_bwd_k3s2_kernel<T><<<g4, 256, 0, st>>>(make_level_desc(Li), make_level_desc(Lo), make_layer_desc(g),
                                                    (const T *)dy, a, (T *)dx, p0, relu_bit);
        count_launch();
        return;
    }
    { pool_bwd_kernel<T><<<grid, 256, 0, st>>>(make_level_desc(Li), make_level_desc(Lo), make_layer_desc(g),
                                             (const T *)dy, a, (T *)dx, p0, relu_bit); count_launch(); }
}

// ============================================================ residual add (ResNet blocks)
// Pointwise over the contiguous element range of patches [p0, p1) of one level (patch buffers of
// a level are laid out back to back, so the range is one flat span):
//   forward   y = a + b            (RELU: y = max(a + b, 0))
//   backward  y = (a + b) * [m > 0] (m = the block's ReLU output; sums the two gradient
//                                    contributions of a fork and applies its ReLU mask once)
// One thread = 8 elements (16 B of bf16); y may alias a or b (each element is read, then written,
// by the same thread).  fp32 sum, one rounding to T.
template <typename T, bool RELU, bool MASK, bool HASB = true>
__global__ void __launch_bounds__(256) add_kernel(const T *a, const T *b, T *y, const T *__restrict__ m, int64_t n8) {
    for (int64_t u = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; u < n8; u += (int64_t)gridDim.x * blockDim.x) {
        float va[8], vb[8] = {0, 0, 0, 0, 0, 0, 0, 0}, vm[8];
        load8(a + u * 8, va);
        if (HASB) load8(b + u * 8, vb);
        if (MASK) load8(m + u * 8, vm);
#pragma unroll
        for (int k = 0; k < 8; ++k) {
            float s = va[k] + vb[k];
            if (RELU) s = fmaxf(s, 0.f);
            if (MASK) s = vm[k] > 0.f ? s : 0.f;
            va[k] = s;
        }
        store8(y + u * 8, va);
    }
}

template <typename T>
void launch_add_t(const void *a, const void *b, void *y, const void *m, int relu, int64_t n, cudaStream_t st) {
    const int64_t n8 = n / 8;
    const int grid = (int)std::max<int64_t>(1, std::min<int64_t>((n8 + 255) / 256, 148 * 8));
    if (m && !b)   // ReLU backward alone: y = a * [m > 0]
        add_kernel<T, false, true, false><<<grid, 256, 0, st>>>((const T *)a, nullptr, (T *)y, (const T *)m, n8);
    else if (m)
        add_kernel<T, false, true><<<grid, 256, 0, st>>>((const T *)a, (const T *)b, (T *)y, (const T *)m, n8);
    else if (relu)
        add_kernel<T, true, false><<<grid, 256, 0, st>>>((const T *)a, (const T *)b, (T *)y, nullptr, n8);
    else
        add_kernel<T, false, false><<<grid, 256, 0, st>>>((const T *)a, (const T *)b, (T *)y, nullptr, n8);
    count_launch();
}

void launch_add(splitcnn_dtype_t dt, const void *a, const void *b, void *y, const void *m, int relu, int64_t n,
                cudaStream_t st) {
    if (dt == SPLITCNN_BF16) launch_add_t<__nv_bfloat16>(a, b, y, m, relu, n, st);
    else launch_add_t<float>(a, b, y, m, relu, n, st);
}

// ============================================================ global average pool (ResNet head, f2)
// Forward: y[n][c] = mean over every pixel of image n in every patch of the level (the logical H x W).
// One block per (image, 256-channel slab); thread = 8 channels x a pixel stride; fixed-order reduction.
template <typename T>
__global__ void __launch_bounds__(256) gap_fwd_kernel(LevelDesc L, const T *__restrict__ x, T *__restrict__ y) {
    __shared__ float red[256][8];
    const int n = blockIdx.x, G = L.Cpad / 8;
    const int gs = min(32, G - blockIdx.y * 32);            // channel groups in this slab
    const int cg = blockIdx.y * 32 + (int)(threadIdx.x % gs), lanes = 256 / gs, pl = threadIdx.x / gs;
    float acc[8] = {0, 0, 0, 0, 0, 0, 0, 0};
    if (pl < lanes) {
        for (int q = 0; q < L.nh * L.nw; ++q) {
            const PatchGeo g = patch_geo(L, q);
            const int64_t base = g.off + (int64_t)n * g.hp * g.wp * L.Cpad;
            for (int px = pl; px < g.hp * g.wp; px += lanes) {
                float v[8];
                load8(x + base + (int64_t)px * L.Cpad + cg * 8, v);
#pragma unroll
                for (int e = 0; e < 8; ++e) acc[e] += v[e];
            }
        }
    }
#pragma unroll
    for (int e = 0; e < 8; ++e) red[threadIdx.x][e] = acc[e];
    __syncthreads();
    if ((int)threadIdx.x < gs) {
        float s8[8] = {0, 0, 0, 0, 0, 0, 0, 0};
        for (int l = 0; l < lanes; ++l)
#pragma unroll
            for (int e = 0; e < 8; ++e) s8[e] += red[l * gs + threadIdx.x][e];
        const float inv = 1.f / (float)(L.H * L.W);
#pragma unroll
        for (int e = 0; e < 8; ++e) s8[e] *= inv;
        store8(y + (int64_t)n * L.Cpad + cg * 8, s8);
    }
}

// Backward: dx[n][h][w][c] = dy[n][c] / (H W) at every pixel of every patch.
template <typename T>
__global__ void __launch_bounds__(256) gap_bwd_kernel(LevelDesc L, const T *__restrict__ dy, T *__restrict__ dx, int p0) {
    const PatchGeo g = patch_geo(L, p0 + blockIdx.y);
    const int G = L.Cpad / 8;
    const uint32_t units = (uint32_t)L.N * g.hp * g.wp * G;
    const float inv = 1.f / (float)(L.H * L.W);
    const FastDiv fg = make_fastdiv((uint32_t)G), fp = make_fastdiv((uint32_t)(g.hp * g.wp));
    for (uint32_t u = blockIdx.x * blockDim.x + threadIdx.x; u < units; u += gridDim.x * blockDim.x) {
        uint32_t cg, px;
        const uint32_t r = fdivmod(u, fg, cg);
        const uint32_t n = fdivmod(r, fp, px);
        float v[8];
        load8(dy + (int64_t)n * L.Cpad + cg * 8, v);
#pragma unroll
        for (int e = 0; e < 8; ++e) v[e] *= inv;
        store8(dx + g.off + (int64_t)r * L.Cpad + cg * 8, v);
    }
}

void launch_gap(splitcnn_dtype_t dt, bool fwd, const Level &L, const void *a, void *b, cudaStream_t st) {
    const LevelDesc d = make_level_desc(L);
    if (fwd) {
        dim3 grid((unsigned)L.N, (unsigned)((L.Cpad / 8 + 31) / 32));
        if (dt == SPLITCNN_BF16) gap_fwd_kernel<__nv_bfloat16><<<grid, 256, 0, st>>>(d, (const __nv_bfloat16 *)a, (__nv_bfloat16 *)b);
        else gap_fwd_kernel<float><<<grid, 256, 0, st>>>(d, (const float *)a, (float *)b);
    } else {
        npatch_launch = L.npatch();
        dim3 grid(grid_x_for(max_patch_units(L, 0, L.npatch(), L.Cpad / 8)), L.npatch());
        if (dt == SPLITCNN_BF16) gap_bwd_kernel<__nv_bfloat16><<<grid, 256, 0, st>>>(d, (const __nv_bfloat16 *)a, (__nv_bfloat16 *)b, 0);
        else gap_bwd_kernel<float><<<grid, 256, 0, st>>>(d, (const float *)a, (float *)b, 0);
    }
    count_launch();
}

void launch_pool_fwd(splitcnn_dtype_t dt, const Level &Li, const Level &Lo, const LayerGeom &g, const void *x, void *y,
                     uint8_t *a, int relu_bit, int p0, int p1, cudaStream_t st) {
    if (dt == SPLITCNN_BF16) launch_pool_fwd_t<__nv_bfloat16>(Li, Lo, g, x, y, a, relu_bit, p0, p1, st);
    else launch_pool_fwd_t<float>(Li, Lo, g, x, y, a, relu_bit, p0, p1, st);
}
void launch_pool_bwd(splitcnn_dtype_t dt, const Level &Li, const Level &Lo, const LayerGeom &g, const void *dy,
                     const uint8_t *a, void *dx, int relu_bit, int p0, int p1, cudaStream_t st) {
    if (dt == SPLITCNN_BF16) launch_pool_bwd_t<__nv_bfloat16>(Li, Lo, g, dy, a, dx, relu_bit, p0, p1, st);
    else launch_pool_bwd_t<float>(Li, Lo, g, dy, a, dx, relu_bit, p0, p1, st);
}

}  // namespace splitcnn
