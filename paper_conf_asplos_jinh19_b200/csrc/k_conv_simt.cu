// k_conv_simt.cu -- CUDA-core (FFMA, fp32 accumulate) split convolution kernels.
//
// These are the fp32-accurate path (SPLITCNN_FP32) and the general fallback for shapes the
// tcgen05 kernel does not take.  Each pass is an implicit GEMM over ONE patch at a time
// (grid.z = patch), reading the patch-major NHWC buffers directly; taps that fall outside the
// patch read zero, which is exactly the patch-local padding of Eq. 6.
//
//   FWD   : M = N*Ho*Wo pixels, N = Cout, K = kh*kw*Cin_pad;  A = X~_p (gather), B = W^T
//   DGRAD : M = N*Hp*Wp pixels, N = Cin_pad, K = kh*kw*Cout_pad; A = dY_p (strided gather), B = W
//   WGRAD : M = Cout, N = kh*kw*Cin_pad, K = pixels of one chunk of one patch (split-K);
//           partials -> workspace -> fixed-order reduction (deterministic)
#include <algorithm>
#include <cstdlib>
#include <type_traits>

#include "common.cuh"
#include "kernels.h"

namespace splitcnn {

enum { MODE_FWD = 0, MODE_DGRAD = 1, MODE_WGRAD = 2 };

struct SimtArgs {
    LevelDesc Li, Lo;
    LayerDesc ly;
    const void *x;        // FWD: X (level m); DGRAD: dY (level m+1); WGRAD: dY
    const void *w;        // weights [Cout][kh][kw][Cin_pad]   (WGRAD: X, level m)
    const float *bias;
    void *y;              // FWD: Y (level m+1); DGRAD: dX (level m); WGRAD: float partials
    const void *relu_src; // DGRAD mask (level m)
    int Cout;             // true output channels of the layer
    int relu;
    int p0;
    int cpp;              // WGRAD: chunks per patch
};

constexpr int BM = 64, BN = 64, BK = 8, NT = 256;

template <typename T, int MODE>
__global__ void __launch_bounds__(NT) conv_simt_kernel(SimtArgs a) {
    __shared__ float As[2][BK][BM + 4];
    __shared__ float Bs[2][BK][BN + 4];

    const int tid = threadIdx.x;
    const int zq = blockIdx.z;
    const int q = a.p0 + (MODE == MODE_WGRAD ? zq / a.cpp : zq);
    const PatchGeo gi = patch_geo(a.Li, q), go = patch_geo(a.Lo, q);
    const int pt = a.ly.pad_h[2 * gi.i], pl = a.ly.pad_w[2 * gi.j];
    const int kh = a.ly.kh, kw = a.ly.kw, sh = a.ly.sh, sw = a.ly.sw;
    const int Cpi = a.Li.Cpad, Cpo = a.Lo.Cpad, N = a.Li.N;

    int M, Ncols, Ktot, kbeg = 0;
    if (MODE == MODE_FWD) { M = N * go.hp * go.wp; Ncols = Cpo; Ktot = kh * kw * Cpi; }
    else if (MODE == MODE_DGRAD) { M = N * gi.hp * gi.wp; Ncols = Cpi; Ktot = kh * kw * Cpo; }
    else {
        M = a.Cout; Ncols = kh * kw * Cpi;
        const int P = N * go.hp * go.wp;
        const int chunk = (P + a.cpp - 1) / a.cpp;
        kbeg = (zq % a.cpp) * chunk;
        Ktot = min(P, kbeg + chunk);
    }
    const int m0 = blockIdx.x * BM, n0 = blockIdx.y * BN;
    if (m0 >= M || n0 >= Ncols) {
        if (MODE != MODE_WGRAD) return;
    }

    const T *X = (const T *)a.x;
    const T *Wt = (const T *)a.w;

    // element (row, k) of A and (k, col) of B
    auto loadA = [&](int m, int k) -> float {
        if (m >= M || k >= Ktot) return 0.f;
        if (MODE == MODE_FWD) {
            const int ci = k % Cpi, rc = k / Cpi, r = rc / kw, c = rc % kw;
            const int ow = m % go.wp, t = m / go.wp, oh = t % go.hp, n = t / go.hp;
            const int h = oh * sh - pt + r, w = ow * sw - pl + c;
            if (h < 0 || h >= gi.hp || w < 0 || w >= gi.wp) return 0.f;
            return to_f(X[gi.off + (((int64_t)n * gi.hp + h) * gi.wp + w) * Cpi + ci]);
        } else if (MODE == MODE_DGRAD) {
            const int co = k % Cpo, rc = k / Cpo, r = rc / kw, c = rc % kw;
            const int w = m % gi.wp, t = m / gi.wp, h = t % gi.hp, n = t / gi.hp;
            const int th = h + pt - r, tw = w + pl - c;
            if (th < 0 || tw < 0 || th % sh || tw % sw) return 0.f;
            const int oh = th / sh, ow = tw / sw;
            if (oh >= go.hp || ow >= go.wp) return 0.f;
            return to_f(X[go.off + (((int64_t)n * go.hp + oh) * go.wp + ow) * Cpo + co]);
        } else {  // A(co, pixel) = dY
            if (k < kbeg) return 0.f;
            return to_f(X[go.off + (int64_t)k * Cpo + m]);
        }
    };
    auto loadB = [&](int k, int col) -> float {
        if (k >= Ktot || col >= Ncols) return 0.f;
        if (MODE == MODE_FWD) {
            if (col >= a.Cout) return 0.f;
            return to_f(Wt[(int64_t)col * Ktot + k]);
        } else if (MODE == MODE_DGRAD) {
            const int co = k % Cpo, rc = k / Cpo;
            if (co >= a.Cout) return 0.f;
            return to_f(Wt[((int64_t)co * kh * kw + rc) * Cpi + col]);
        } else {  // B(pixel, (r,c,ci)) = X~
            if (k < kbeg) return 0.f;
            const int ci = col % Cpi, rc = col / Cpi, r = rc / kw, c = rc % kw;
            const int ow = k % go.wp, t = k / go.wp, oh = t % go.hp, n = t / go.hp;
            const int h = oh * sh - pt + r, w = ow * sw - pl + c;
            if (h < 0 || h >= gi.hp || w < 0 || w >= gi.wp) return 0.f;
            return to_f(Wt[gi.off + (((int64_t)n * gi.hp + h) * gi.wp + w) * Cpi + ci]);
        }
    };
    // lane mapping: make the memory-contiguous index lane-fastest
    //   FWD:   A k-fast (ci contiguous), B k-fast (weights rows)
    //   DGRAD: A k-fast (co contiguous), B col-fast (ci contiguous)
    //   WGRAD: A row-fast (co contiguous), B col-fast (ci contiguous)
    constexpr bool A_KFAST = (MODE != MODE_WGRAD);
    constexpr bool B_KFAST = (MODE == MODE_FWD);

    float ra[2], rb[2];
    auto fetch = [&](int kt) {
#pragma unroll
        for (int s = 0; s < 2; ++s) {
            const int e = tid + s * NT;
            int mi, ki;
            if (A_KFAST) { ki = e % BK; mi = e / BK; } else { mi = e % BM; ki = e / BM; }
            ra[s] = loadA(m0 + mi, kt + ki);
            int ni, kj;
            if (B_KFAST) { kj = e % BK; ni = e / BK; } else { ni = e % BN; kj = e / BN; }
            rb[s] = loadB(kt + kj, n0 + ni);
        }
    };
    auto stash = [&](int buf) {
#pragma unroll
        for (int s = 0; s < 2; ++s) {
            const int e = tid + s * NT;
            int mi, ki;
            if (A_KFAST) { ki = e % BK; mi = e / BK; } else { mi = e % BM; ki = e / BM; }
            As[buf][ki][mi] = ra[s];
            int ni, kj;
            if (B_KFAST) { kj = e % BK; ni = e / BK; } else { ni = e % BN; kj = e / BN; }
            Bs[buf][kj][ni] = rb[s];
        }
    };

    float acc[4][4];
#pragma unroll
    for (int i = 0; i < 4; ++i)
#pragma unroll
        for (int j = 0; j < 4; ++j) acc[i][j] = 0.f;
    const int tx = tid % 16, ty = tid / 16;

    const int kstart = (MODE == MODE_WGRAD) ? (kbeg / BK) * BK : 0;
    int buf = 0;
    if (m0 < M && n0 < Ncols && kstart < Ktot) {
        fetch(kstart);
        stash(0);
        __syncthreads();
        for (int kt = kstart; kt < Ktot; kt += BK) {
            const bool more = kt + BK < Ktot;
            if (more) fetch(kt + BK);
#pragma unroll
            for (int kk = 0; kk < BK; ++kk) {
                float av[4], bv[4];
#pragma unroll
                for (int i = 0; i < 4; ++i) av[i] = As[buf][kk][ty * 4 + i];
#pragma unroll
                for (int j = 0; j < 4; ++j) bv[j] = Bs[buf][kk][tx * 4 + j];
#pragma unroll
                for (int i = 0; i < 4; ++i)
#pragma unroll
                    for (int j = 0; j < 4; ++j) acc[i][j] = fmaf(av[i], bv[j], acc[i][j]);
            }
            if (more) {
                stash(buf ^ 1);
                __syncthreads();
                buf ^= 1;
            }
        }
    }

    // epilogue
#pragma unroll
    for (int i = 0; i < 4; ++i) {
        const int m = m0 + ty * 4 + i;
        if (m >= M) continue;
#pragma unroll
        for (int j = 0; j < 4; ++j) {
            const int col = n0 + tx * 4 + j;
            if (col >= Ncols) continue;
            float v = acc[i][j];
            if (MODE == MODE_FWD) {
                if (col < a.Cout) {
                    if (a.bias) v += a.bias[col];
                    if (a.relu) v = fmaxf(v, 0.f);
                } else {
                    v = 0.f;
                }
                ((T *)a.y)[go.off + (int64_t)m * Cpo + col] = from_f<T>(v);
            } else if (MODE == MODE_DGRAD) {
                const int64_t o = gi.off + (int64_t)m * Cpi + col;
                if (a.relu_src && !(to_f(((const T *)a.relu_src)[o]) > 0.f)) v = 0.f;
                ((T *)a.y)[o] = from_f<T>(v);
            } else {
                ((float *)a.y)[((int64_t)zq * M + m) * Ncols + col] = v;
            }
        }
    }
}

// out[i] = beta * out[i] + sum_z part[z][i] for two segments (blockIdx.y: 0 = dW, 1 = db).  A block is
// 32 column lanes x 8 z-slices: slice k sums z = k, k+8, ... in ascending order, then slice 0 adds the
// 8 slice sums in ascending slice order -- a fixed summation tree independent of scheduling, so the
// result is bitwise reproducible.  VEC = 4: each column lane owns 4 consecutive floats (n % 4 == 0).
template <int VEC>
__global__ void __launch_bounds__(256) reduce_partials_kernel(const float *__restrict__ part0, int64_t n0,
                                                              float *__restrict__ out0, int Z0,
                                                              const float *__restrict__ part1, int64_t n1,
                                                              float *__restrict__ out1, int Z1, float beta) {
    using V = typename std::conditional<VEC == 4, float4, float>::type;
    const int Z = blockIdx.y ? Z1 : Z0;
    const float *part = blockIdx.y ? part1 : part0;
    float *out = blockIdx.y ? out1 : out0;
    const int64_t nv = (blockIdx.y ? n1 : n0) / VEC;
    const int64_t col = (int64_t)blockIdx.x * 32 + (threadIdx.x & 31);
    const int zs = threadIdx.x >> 5;
    __shared__ V red[8][32];
    if ((int64_t)blockIdx.x * 32 >= nv) return;   // whole block idle (the shorter segment)
    V s;
    float *sf = reinterpret_cast<float *>(&s);
#pragma unroll
    for (int e = 0; e < VEC; ++e) sf[e] = 0.f;
    if (col < nv) {
        const V *pv = reinterpret_cast<const V *>(part) + col;
        int z = zs;
        for (; z + 24 < Z; z += 32) {   // 4 independent loads in flight, added in z order
            const V a = __ldg(pv + (int64_t)z * nv), b = __ldg(pv + (int64_t)(z + 8) * nv);
            const V c = __ldg(pv + (int64_t)(z + 16) * nv), d = __ldg(pv + (int64_t)(z + 24) * nv);
            const float *af = reinterpret_cast<const float *>(&a), *bf = reinterpret_cast<const float *>(&b);
            const float *cf = reinterpret_cast<const float *>(&c), *df = reinterpret_cast<const float *>(&d);
#pragma unroll
            for (int e = 0; e < VEC; ++e) sf[e] = (((sf[e] + af[e]) + bf[e]) + cf[e]) + df[e];
        }
        for (; z < Z; z += 8) {
            const V a = __ldg(pv + (int64_t)z * nv);
            const float *af = reinterpret_cast<const float *>(&a);
#pragma unroll
            for (int e = 0; e < VEC; ++e) sf[e] += af[e];
        }
    }
    red[zs][threadIdx.x & 31] = s;
    __syncthreads();
    if (zs == 0 && col < nv) {
        V t = red[0][threadIdx.x];
        float *tf = reinterpret_cast<float *>(&t);
#pragma unroll
        for (int k = 1; k < 8; ++k) {
            const V u = red[k][threadIdx.x];
            const float *uf = reinterpret_cast<const float *>(&u);
#pragma unroll
            for (int e = 0; e < VEC; ++e) tf[e] += uf[e];
        }
        V *ov = reinterpret_cast<V *>(out) + col;
        if (beta != 0.f) {
            const V o = *ov;
            const float *of = reinterpret_cast<const float *>(&o);
#pragma unroll
            for (int e = 0; e < VEC; ++e) tf[e] += beta * of[e];
        }
        *ov = t;
    }
}

// Few partials (Z <= 8, e.g. the single-split weight gradients of the small-M CIFAR tails): one thread per
// vector column sums its Z partials in z order, grid-stride -- the 8-warp z split above would leave all but
// Z warps idle and launch one block per 32 columns.  Bitwise equal to it: both compute
// ((0 + p_0) + p_1) + ... + beta * out, and a sum started at +0 is never -0, so its + 0 terms change nothing.
template <int VEC>
__global__ void __launch_bounds__(256) reduce_few_kernel(const float *__restrict__ part0, int64_t n0,
                                                         float *__restrict__ out0, int Z0,
                                                         const float *__restrict__ part1, int64_t n1,
                                                         float *__restrict__ out1, int Z1, float beta) {
    using V = typename std::conditional<VEC == 4, float4, float>::type;
    const int Z = blockIdx.y ? Z1 : Z0;
    const float *part = blockIdx.y ? part1 : part0;
    float *out = blockIdx.y ? out1 : out0;
    const int64_t nv = (blockIdx.y ? n1 : n0) / VEC;
    for (int64_t col = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; col < nv; col += (int64_t)gridDim.x * blockDim.x) {
        const V *pv = reinterpret_cast<const V *>(part) + col;
        V t;
        float *tf = reinterpret_cast<float *>(&t);
#pragma unroll
        for (int e = 0; e < VEC; ++e) tf[e] = 0.f;
        for (int z = 0; z < Z; ++z) {
            const V a = __ldg(pv + (int64_t)z * nv);
            const float *af = reinterpret_cast<const float *>(&a);
#pragma unroll
            for (int e = 0; e < VEC; ++e) tf[e] += af[e];
        }
        V *ov = reinterpret_cast<V *>(out) + col;
        if (beta != 0.f) {
            const V o = *ov;
            const float *of = reinterpret_cast<const float *>(&o);
#pragma unroll
            for (int e = 0; e < VEC; ++e) tf[e] += beta * of[e];
        }
        *ov = t;
    }
}

// Column sums of the patch-buffer range [p0, p1) viewed as a [P pixels][Cpad] matrix (the patches of
// a range are contiguous): block b sums rows [b*R, (b+1)*R) with 16-byte loads, reduces its pixel
// lanes in shared memory in a fixed order and writes part[b][Cout].  Deterministic.
template <typename T>
__global__ void __launch_bounds__(256) colsum_kernel(const T *__restrict__ base, int64_t P, int Cpad, int Cout,
                                                     int64_t R, float *__restrict__ part) {
    __shared__ float red[256][8];
    const int G = Cpad / 8;
    const int lanes = 256 / G;
    const int cg = threadIdx.x % G, pl = threadIdx.x / G;
    float acc[8] = {0, 0, 0, 0, 0, 0, 0, 0};
    const int64_t r0 = blockIdx.x * R, r1 = min(P, r0 + R);
    if (pl < lanes) {
#pragma unroll 4
        for (int64_t r = r0 + pl; r < r1; r += lanes) {
            float v[8];
            load8(base + r * Cpad + cg * 8, v);
#pragma unroll
            for (int e = 0; e < 8; ++e) acc[e] += v[e];
        }
    }
#pragma unroll
    for (int e = 0; e < 8; ++e) red[threadIdx.x][e] = acc[e];
    __syncthreads();
    if (threadIdx.x < G) {
        float s8[8] = {0, 0, 0, 0, 0, 0, 0, 0};
        for (int l = 0; l < lanes; ++l)
#pragma unroll
            for (int e = 0; e < 8; ++e) s8[e] += red[l * G + threadIdx.x][e];
#pragma unroll
        for (int e = 0; e < 8; ++e)
            if (threadIdx.x * 8 + e < Cout) part[(int64_t)blockIdx.x * Cout + threadIdx.x * 8 + e] = s8[e];
    }
}

// Shared-memory-free variant (channel groups G = Cpad/8 with 32 % G == 0 or G % 32 == 0): it runs on
// the side stream concurrently with the wgrad GEMM, whose CTAs leave no shared memory free on their
// SM, so the colsum blocks must need none to co-reside.  Each warp reduces its pixel lanes with
// shuffles (fixed xor order) and writes its own partial row: RB = G >= 32 ? 256/G : 8 rows per block.
template <typename T>
__global__ void __launch_bounds__(256) colsum_warp_kernel(const T *__restrict__ base, int64_t P, int Cpad, int Cout,
                                                          int64_t R, float *__restrict__ part) {
    const int G = Cpad / 8;
    const int lanes = 256 / G;
    const int cg = threadIdx.x % G, pl = threadIdx.x / G;
    float acc[8] = {0, 0, 0, 0, 0, 0, 0, 0};
    const int64_t r0 = blockIdx.x * R, r1 = min(P, r0 + R);
    for (int64_t r = r0 + pl; r < r1; r += lanes) {
        float v[8];
        load8(base + r * Cpad + cg * 8, v);
#pragma unroll
        for (int e = 0; e < 8; ++e) acc[e] += v[e];
    }
    int row;
    if (G < 32) {
        for (int o = G; o < 32; o <<= 1)
#pragma unroll
            for (int e = 0; e < 8; ++e) acc[e] += __shfl_xor_sync(0xffffffffu, acc[e], o);
        if ((threadIdx.x & 31) >= G) return;
        row = blockIdx.x * 8 + (threadIdx.x >> 5);
    } else {
        row = blockIdx.x * lanes + pl;
    }
#pragma unroll
    for (int e = 0; e < 8; ++e)
        if (cg * 8 + e < Cout) part[(int64_t)row * Cout + cg * 8 + e] = acc[e];
}

// part[b][:] = sum of rows [b*chunk, (b+1)*chunk) of rows[Z][n], in row order (deterministic)
__global__ void __launch_bounds__(256) rows_sum_kernel(const float *__restrict__ rows, int Z, int n, int chunk,
                                                       float *__restrict__ part) {
    const int col = blockIdx.x * 256 + threadIdx.x;
    if (col >= n) return;
    const int z0 = blockIdx.y * chunk, z1 = min(Z, z0 + chunk);
    float s = 0.f;
#pragma unroll 8
    for (int z = z0; z < z1; ++z) s += __ldg(rows + (int64_t)z * n + col);
    part[(int64_t)blockIdx.y * n + col] = s;
}

// returns the number of partial rows left in part[0..) (at most 4 * 148); the db workspace region holds
// 9 * 4 * 148 rows: the warp variant writes its (up to 8 per block) rows after the first 4 * 148 and
// folds them into part[0..) in fixed-size chunks, so the final reduction sees at most 4 * 148 rows
int launch_db_partials(splitcnn_dtype_t dt, const Level &Lo, const void *dy, float *part, int cout, int p0, int p1,
                       cudaStream_t st) {
    auto off = [&](int q) -> int64_t {
        if (q >= Lo.npatch()) return Lo.total();
        return Lo.offset(q / Lo.nw(), q % Lo.nw());
    };
    const int64_t e0 = off(p0), e1 = off(p1);
    const int64_t P = (e1 - e0) / Lo.Cpad;
    if (P <= 0) return 0;          // empty patch range: no partials (the reduce then applies beta alone)
    const int Z = 4 * 148;
    const int64_t R = (P + Z - 1) / Z;
    const int Zr = (int)((P + R - 1) / R);
    const int G = Lo.Cpad / 8;
    // when the warp variant pays (same-box A/Bs, profiles/r1_ab_colsum_fold.txt): a dY of >= 32 MB (below
    // that -- C2's 32x32 layers -- the extra fold launch costs more than co-residency saves), except the
    // 64-channel 224x224 layers (>= 1 GB at G = 8), where the shared-memory kernel measured faster
    const int64_t dy_bytes = P * Lo.Cpad * (int64_t)(dt == SPLITCNN_BF16 ? 2 : 4);
    const bool warp_ok = G <= 64 && (32 % G == 0 || G % 32 == 0) && dy_bytes >= (32ll << 20) &&
                         (G >= 16 || dy_bytes < (1ll << 30));
    if (warp_ok) {
        const int RB = G >= 32 ? 256 / G : 8;
        float *rows = part + (int64_t)Z * cout;
        if (dt == SPLITCNN_BF16)
            colsum_warp_kernel<__nv_bfloat16><<<Zr, 256, 0, st>>>((const __nv_bfloat16 *)dy + e0, P, Lo.Cpad, cout, R, rows);
        else
            colsum_warp_kernel<float><<<Zr, 256, 0, st>>>((const float *)dy + e0, P, Lo.Cpad, cout, R, rows);
        count_launch();
        const int nrows = Zr * RB, chunk = 2 * RB;
        const int nch = (nrows + chunk - 1) / chunk;
        rows_sum_kernel<<<dim3((unsigned)((cout + 255) / 256), (unsigned)nch), 256, 0, st>>>(rows, nrows, cout, chunk, part);
        count_launch();
        return nch;
    }
    // small dY (< 32 MB, the CIFAR-sized levels): at most 128 partial rows of >= 64 pixels each -- one row
    // per block of a few pixels would leave the (serial-in-z) reduction of ~600 partials as the long pole
    int64_t Rs = R;
    if (dy_bytes < (32ll << 20)) Rs = std::max<int64_t>({R, 64, (P + 127) / 128});
    const int Zs = (int)((P + Rs - 1) / Rs);
    if (dt == SPLITCNN_BF16)
        colsum_kernel<__nv_bfloat16><<<Zs, 256, 0, st>>>((const __nv_bfloat16 *)dy + e0, P, Lo.Cpad, cout, Rs, part);
    else
        colsum_kernel<float><<<Zs, 256, 0, st>>>((const float *)dy + e0, P, Lo.Cpad, cout, Rs, part);
    count_launch();
    return Zs;
}

void launch_reduce2(const float *part0, int64_t n0, float *out0, int Z0, const float *part1, int64_t n1, float *out1,
                    int Z1, float beta, cudaStream_t st) {
    if (!part1 || !out1) n1 = 0;
    auto al16 = [](const void *q) { return ((uintptr_t)q & 15) == 0; };
    const bool vec = n0 % 4 == 0 && n1 % 4 == 0 && al16(part0) && al16(out0) && (n1 == 0 || (al16(part1) && al16(out1)));
    const int64_t cols = std::max(n0, n1) / (vec ? 4 : 1);
    if (std::max(Z0, n1 > 0 ? Z1 : 0) <= 8) {
        dim3 grid((unsigned)std::max<int64_t>(1, std::min<int64_t>((cols + 255) / 256, 148 * 16)), n1 > 0 ? 2 : 1);
        if (vec) reduce_few_kernel<4><<<grid, 256, 0, st>>>(part0, n0, out0, Z0, part1, n1, out1, Z1, beta);
        else reduce_few_kernel<1><<<grid, 256, 0, st>>>(part0, n0, out0, Z0, part1, n1, out1, Z1, beta);
        count_launch();
        return;
    }
    dim3 grid((unsigned)((cols + 31) / 32), n1 > 0 ? 2 : 1);
    if (vec) reduce_partials_kernel<4><<<grid, 256, 0, st>>>(part0, n0, out0, Z0, part1, n1, out1, Z1, beta);
    else reduce_partials_kernel<1><<<grid, 256, 0, st>>>(part0, n0, out0, Z0, part1, n1, out1, Z1, beta);
    count_launch();
}

void launch_reduce(const float *part, int Z, int64_t n, float *out, float beta, cudaStream_t st) {
    launch_reduce2(part, n, out, Z, nullptr, 0, nullptr, 0, beta, st);
}

static int64_t max_pixels(const Level &L, int p0, int p1) {
    int64_t m = 0;
    for (int q = p0; q < p1; ++q) {
        int i = q / L.nw(), j = q % L.nw();
        m = std::max<int64_t>(m, (int64_t)L.N * L.ph(i) * L.pw(j));
    }
    return m;
}

void launch_conv_fwd_simt(splitcnn_dtype_t dt, const Level &Li, const Level &Lo, const LayerGeom &g, const void *x,
                          const void *w, const float *bias, void *y, int relu, int p0, int p1, cudaStream_t st) {
    SimtArgs a{};
    a.Li = make_level_desc(Li); a.Lo = make_level_desc(Lo); a.ly = make_layer_desc(g);
    a.x = x; a.w = w; a.bias = bias; a.y = y; a.Cout = g.L.cout; a.relu = relu; a.p0 = p0;
    dim3 grid((unsigned)((max_pixels(Lo, p0, p1) + BM - 1) / BM), (Lo.Cpad + BN - 1) / BN, p1 - p0);
    if (dt == SPLITCNN_BF16) conv_simt_kernel<__nv_bfloat16, MODE_FWD><<<grid, NT, 0, st>>>(a);
    else conv_simt_kernel<float, MODE_FWD><<<grid, NT, 0, st>>>(a);
    count_launch();
}

void launch_conv_dgrad_simt(splitcnn_dtype_t dt, const Level &Li, const Level &Lo, const LayerGeom &g, const void *dy,
                            const void *w, void *dx, const void *relu_src, int p0, int p1, cudaStream_t st) {
    SimtArgs a{};
    a.Li = make_level_desc(Li); a.Lo = make_level_desc(Lo); a.ly = make_layer_desc(g);
    a.x = dy; a.w = w; a.y = dx; a.relu_src = relu_src; a.Cout = g.L.cout; a.p0 = p0;
    dim3 grid((unsigned)((max_pixels(Li, p0, p1) + BM - 1) / BM), (Li.Cpad + BN - 1) / BN, p1 - p0);
    if (dt == SPLITCNN_BF16) conv_simt_kernel<__nv_bfloat16, MODE_DGRAD><<<grid, NT, 0, st>>>(a);
    else conv_simt_kernel<float, MODE_DGRAD><<<grid, NT, 0, st>>>(a);
    count_launch();
}

// split-K chunking for the wgrad: a fixed function of the plan, so workspace_size agrees.
int wgrad_simt_chunks_per_patch(const Level &Li, const Level &Lo, const LayerGeom &g, int npatch) {
    const int tiles = ((g.L.cout + BM - 1) / BM) * ((g.L.kh * g.L.kw * Li.Cpad + BN - 1) / BN);
    int cpp = (4 * 148 + tiles * npatch - 1) / (tiles * npatch);
    int64_t minpix = INT64_MAX;
    for (int i = 0; i < Lo.nh(); ++i)
        for (int j = 0; j < Lo.nw(); ++j) minpix = std::min<int64_t>(minpix, (int64_t)Lo.N * Lo.ph(i) * Lo.pw(j));
    cpp = std::max(1, std::min<int>(cpp, (int)std::max<int64_t>(1, minpix / 256)));
    return std::min(cpp, 64);
}

size_t wgrad_simt_ws_bytes(const Level &Li, const Level &Lo, const LayerGeom &g) {
    const int np = Lo.nh() * Lo.nw();
    const int cpp = wgrad_simt_chunks_per_patch(Li, Lo, g, np);
    const int64_t Z = (int64_t)np * cpp;
    const int64_t ncols = (int64_t)g.L.kh * g.L.kw * Li.Cpad;
    return (size_t)(Z * g.L.cout * ncols + 9 * 4 * 148 * g.L.cout) * sizeof(float);   // + db partial rows
}

void launch_conv_wgrad_simt(splitcnn_dtype_t dt, const Level &Li, const Level &Lo, const LayerGeom &g, const void *x,
                            const void *dy, float *dw, float *db, float beta, void *ws, int p0, int p1, cudaStream_t st) {
    const int np_all = Lo.nh() * Lo.nw();
    const int cpp = wgrad_simt_chunks_per_patch(Li, Lo, g, np_all);
    const int Z = (p1 - p0) * cpp;
    const int ncols = g.L.kh * g.L.kw * Li.Cpad;
    float *part = (float *)ws;
    float *part_db = part + (int64_t)Z * g.L.cout * ncols;
    SimtArgs a{};
    a.Li = make_level_desc(Li); a.Lo = make_level_desc(Lo); a.ly = make_layer_desc(g);
    a.x = dy; a.w = x; a.y = part; a.Cout = g.L.cout; a.p0 = p0; a.cpp = cpp;
    dim3 grid((g.L.cout + BM - 1) / BM, (ncols + BN - 1) / BN, Z);
    if (Z > 0) {                   // empty patch range: dW = beta * dW (the reduce below, Z = 0)
        if (dt == SPLITCNN_BF16) conv_simt_kernel<__nv_bfloat16, MODE_WGRAD><<<grid, NT, 0, st>>>(a);
        else conv_simt_kernel<float, MODE_WGRAD><<<grid, NT, 0, st>>>(a);
        count_launch();
    }
    const int64_t n = (int64_t)g.L.cout * ncols;
    launch_reduce(part, Z, n, dw, beta, st);
    if (db) {
        const int Zd = launch_db_partials(dt, Lo, dy, part_db, g.L.cout, p0, p1, st);
        launch_reduce(part_db, Zd, g.L.cout, db, beta, st);
    }
}

}  // namespace splitcnn
