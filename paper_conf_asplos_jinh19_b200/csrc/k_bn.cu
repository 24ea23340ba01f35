// k_bn.cu -- whole-tensor batch normalisation on split levels.
//
// BN is not a window operator: Split-CNN leaves it unsplit, i.e. its statistics are those of
// the LOGICAL tensor (all patches, all images, all pixels), exactly the unsplit BN.  On patch
// buffers that is a per-channel reduction over the contiguous span of patches [p0, p1) (patches of
// a level are stored back to back, each [N][Hp][Wp][Cpad]), so the whole span is one flat
// [P pixels][Cpad] array.  Under patch sharding each rank reduces its span and the caller sums the
// 2*C partial sums across ranks (a 2C-float allreduce) before the apply step.
//
//   stats    s0[c] = sum x,            s1[c] = sum x^2
//   fwd      mean = s0/M, var = s1/M - mean^2 (biased, as training-mode BN), invstd = 1/sqrt(var+eps)
//            y = gamma*(x-mean)*invstd + beta  (+ ReLU)
//   bwd sums g = dy*[y>0] (ReLU fused) ,  t0[c] = sum g,  t1[c] = sum g*xhat
//   bwd      dx = gamma*invstd*(g - t0/M - xhat*t1/M),  dgamma = t1, dbeta = t0
//
// Reductions: per-block fp32 partials over a fixed pixel range, then ONE fixed-order fp64 sum per
// channel -> bitwise reproducible run to run (R14).
#include <algorithm>

#include "common.cuh"
#include "kernels.h"

namespace splitcnn {

constexpr int BN_THREADS = 256;

// MODE 0: (x, x^2).  MODE 1: (g, g*xhat) with g = dy*[y > 0] (y nullable), xhat from mean_invstd.
template <typename T, int MODE>
__global__ void __launch_bounds__(BN_THREADS) bn_reduce_kernel(const T *__restrict__ x, const T *__restrict__ dy,
                                                               const T *__restrict__ y, const float *__restrict__ mi,
                                                               int64_t P, int Cpad, int C, int64_t R,
                                                               float *__restrict__ part) {
    __shared__ float red[BN_THREADS][16];
    const int G = Cpad / 8;
    const int lanes = BN_THREADS / G;
    const int cg = threadIdx.x % G, pl = threadIdx.x / G;
    float a0[8], a1[8], mean[8], inv[8];
#pragma unroll
    for (int e = 0; e < 8; ++e) {
        a0[e] = a1[e] = 0.f;
        const int c = min(cg * 8 + e, C - 1);
        mean[e] = MODE == 1 ? mi[c] : 0.f;
        inv[e] = MODE == 1 ? mi[C + c] : 0.f;
    }
    const int64_t r0 = blockIdx.x * R, r1 = min(P, r0 + R);
    if (pl < lanes) {
        for (int64_t r = r0 + pl; r < r1; r += lanes) {
            float v[8];
            load8(x + r * Cpad + cg * 8, v);
            if (MODE == 0) {
#pragma unroll
                for (int e = 0; e < 8; ++e) { a0[e] += v[e]; a1[e] += v[e] * v[e]; }
            } else {
                float g[8], m[8];
                load8(dy + r * Cpad + cg * 8, g);
                if (y) {
                    load8(y + r * Cpad + cg * 8, m);
#pragma unroll
                    for (int e = 0; e < 8; ++e) g[e] = m[e] > 0.f ? g[e] : 0.f;
                }
#pragma unroll
                for (int e = 0; e < 8; ++e) { a0[e] += g[e]; a1[e] += g[e] * ((v[e] - mean[e]) * inv[e]); }
            }
        }
    }
#pragma unroll
    for (int e = 0; e < 8; ++e) { red[threadIdx.x][e] = a0[e]; red[threadIdx.x][8 + e] = a1[e]; }
    __syncthreads();
    if (threadIdx.x < G) {
        float s0[8] = {0, 0, 0, 0, 0, 0, 0, 0}, s1[8] = {0, 0, 0, 0, 0, 0, 0, 0};
        for (int l = 0; l < lanes; ++l)
#pragma unroll
            for (int e = 0; e < 8; ++e) { s0[e] += red[l * G + threadIdx.x][e]; s1[e] += red[l * G + threadIdx.x][8 + e]; }
#pragma unroll
        for (int e = 0; e < 8; ++e) {
            const int c = threadIdx.x * 8 + e;
            if (c < C) {
                part[((int64_t)blockIdx.x * 2 + 0) * C + c] = s0[e];
                part[((int64_t)blockIdx.x * 2 + 1) * C + c] = s1[e];
            }
        }
    }
}

// out[i] = sum over z of part[z][i] (i < 2C) in fp64: one warp per column, lane l sums z = l, l+32, ...
// in order, then a fixed xor-tree across lanes -- the same order every run (bitwise reproducible)
__global__ void bn_sum_partials_kernel(const float *__restrict__ part, int Z, int C, float *__restrict__ out) {
    const int i = blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5);
    const int lane = threadIdx.x & 31;
    if (i >= 2 * C) return;
    double s = 0.0;
    for (int z = lane; z < Z; z += 32) s += (double)__ldg(part + (int64_t)z * 2 * C + i);
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
    if (lane == 0) out[i] = (float)s;
}

// mean_invstd[0][c] = mean, [1][c] = 1/sqrt(var + eps)  (fp64 arithmetic on the fp32 sums)
__global__ void bn_finalize_kernel(const float *__restrict__ sums, int C, double count, float eps,
                                   float *__restrict__ mi) {
    const int c = blockIdx.x * blockDim.x + threadIdx.x;
    if (c >= C) return;
    const double mean = (double)sums[c] / count;
    double var = (double)sums[C + c] / count - mean * mean;
    if (var < 0.0) var = 0.0;
    mi[c] = (float)mean;
    mi[C + c] = (float)(1.0 / sqrt(var + (double)eps));
}

template <typename T, bool RELU>
__global__ void __launch_bounds__(BN_THREADS) bn_apply_kernel(const T *x, const float *__restrict__ mi,
                                                              const float *__restrict__ gamma,
                                                              const float *__restrict__ beta, T *y,
                                                              int64_t n8, int G, int C) {
    if (blockDim.x % G == 0) {
        // the grid stride is a multiple of G: this thread always sees the same 8 channels -> per-channel
        // scale / shift once, no 64-bit modulo per unit
        const int cg = threadIdx.x % G;
        float sc_[8], sh[8];
#pragma unroll
        for (int e = 0; e < 8; ++e) {
            const int c = cg * 8 + e;
            sc_[e] = c < C ? gamma[c] * mi[C + c] : 0.f;
            sh[e] = c < C ? beta[c] - mi[c] * sc_[e] : 0.f;
        }
        for (int64_t u = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; u < n8; u += (int64_t)gridDim.x * blockDim.x) {
            float v[8];
            load8(x + u * 8, v);
#pragma unroll
            for (int e = 0; e < 8; ++e) {
                float o = fmaf(v[e], sc_[e], sh[e]);
                if (RELU) o = fmaxf(o, 0.f);
                v[e] = o;
            }
            store8(y + u * 8, v);
        }
        return;
    }
    for (int64_t u = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; u < n8; u += (int64_t)gridDim.x * blockDim.x) {
        const int cg = (int)(u % G);
        float v[8];
        load8(x + u * 8, v);
#pragma unroll
        for (int e = 0; e < 8; ++e) {
            const int c = cg * 8 + e;
            if (c < C) {
                const float s = gamma[c] * mi[C + c];
                float o = (v[e] - mi[c]) * s + beta[c];
                if (RELU) o = fmaxf(o, 0.f);
                v[e] = o;
            } else {
                v[e] = 0.f;
            }
        }
        store8(y + u * 8, v);
    }
}

template <typename T>
__global__ void __launch_bounds__(BN_THREADS) bn_bwd_kernel(const T *dy, const T *__restrict__ x,
                                                            const T *__restrict__ y, const float *__restrict__ mi,
                                                            const float *__restrict__ gamma,
                                                            const float *__restrict__ t, float invM, T *dx,
                                                            int64_t n8, int G, int C) {
    if (blockDim.x % G == 0) {      // fixed channels per thread (see bn_apply_kernel)
        const int cg = threadIdx.x % G;
        float k1[8], mean[8], inv[8], t0[8], t1[8];
#pragma unroll
        for (int e = 0; e < 8; ++e) {
            const int c = min(cg * 8 + e, C - 1);
            const bool ok = cg * 8 + e < C;
            inv[e] = mi[C + c];
            mean[e] = mi[c];
            k1[e] = ok ? gamma[c] * inv[e] : 0.f;
            t0[e] = t[c] * invM;
            t1[e] = t[C + c] * invM;
        }
        for (int64_t u = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; u < n8; u += (int64_t)gridDim.x * blockDim.x) {
            float g[8], v[8], m[8];
            load8(dy + u * 8, g);
            load8(x + u * 8, v);
            if (y) load8(y + u * 8, m);
#pragma unroll
            for (int e = 0; e < 8; ++e) {
                const float ge = (!y || m[e] > 0.f) ? g[e] : 0.f;
                const float xh = (v[e] - mean[e]) * inv[e];
                g[e] = k1[e] * (ge - t0[e] - xh * t1[e]);
            }
            store8(dx + u * 8, g);
        }
        return;
    }
    for (int64_t u = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; u < n8; u += (int64_t)gridDim.x * blockDim.x) {
        const int cg = (int)(u % G);
        float g[8], v[8], m[8];
        load8(dy + u * 8, g);
        load8(x + u * 8, v);
        if (y) load8(y + u * 8, m);
#pragma unroll
        for (int e = 0; e < 8; ++e) {
            const int c = cg * 8 + e;
            if (c < C) {
                const float ge = (!y || m[e] > 0.f) ? g[e] : 0.f;
                const float inv = mi[C + c];
                const float xh = (v[e] - mi[c]) * inv;
                g[e] = gamma[c] * inv * (ge - t[c] * invM - xh * t[C + c] * invM);
            } else {
                g[e] = 0.f;
            }
        }
        store8(dx + u * 8, g);
    }
}

static int bn_grid(int64_t n8) { return (int)std::max<int64_t>(1, std::min<int64_t>((n8 + 255) / 256, 148 * 8)); }

size_t bn_ws_bytes(int C) { return (size_t)4 * 148 * 2 * C * sizeof(float) + 256; }

template <typename T>
static void bn_reduce_t(int mode, const void *x, const void *dy, const void *y, const float *mi, int64_t P, int Cpad,
                        int C, float *part, float *sums, cudaStream_t st) {
    const int Zt = 4 * 148;
    const int64_t R = std::max<int64_t>(1, (P + Zt - 1) / Zt);
    const int Z = (int)std::max<int64_t>(1, (P + R - 1) / R);
    if (mode == 0)
        bn_reduce_kernel<T, 0><<<Z, BN_THREADS, 0, st>>>((const T *)x, nullptr, nullptr, nullptr, P, Cpad, C, R, part);
    else
        bn_reduce_kernel<T, 1><<<Z, BN_THREADS, 0, st>>>((const T *)x, (const T *)dy, (const T *)y, mi, P, Cpad, C, R,
                                                         part);
    bn_sum_partials_kernel<<<(2 * C + 7) / 8, 256, 0, st>>>(part, Z, C, sums);
    count_launch(2);
}

void launch_bn_reduce(splitcnn_dtype_t dt, int mode, const void *x, const void *dy, const void *y, const float *mi,
                      int64_t P, int Cpad, int C, float *part, float *sums, cudaStream_t st) {
    if (dt == SPLITCNN_BF16) bn_reduce_t<__nv_bfloat16>(mode, x, dy, y, mi, P, Cpad, C, part, sums, st);
    else bn_reduce_t<float>(mode, x, dy, y, mi, P, Cpad, C, part, sums, st);
}

void launch_bn_fwd(splitcnn_dtype_t dt, const void *x, const float *sums, double count, const float *gamma,
                   const float *beta, float eps, float *mi, void *y, int relu, int64_t n, int Cpad, int C,
                   cudaStream_t st) {
    bn_finalize_kernel<<<(C + 127) / 128, 128, 0, st>>>(sums, C, count, eps, mi);
    const int64_t n8 = n / 8;
    const int G = Cpad / 8, grid = bn_grid(n8);
    if (dt == SPLITCNN_BF16) {
        if (relu) bn_apply_kernel<__nv_bfloat16, true><<<grid, BN_THREADS, 0, st>>>((const __nv_bfloat16 *)x, mi, gamma, beta, (__nv_bfloat16 *)y, n8, G, C);
        else bn_apply_kernel<__nv_bfloat16, false><<<grid, BN_THREADS, 0, st>>>((const __nv_bfloat16 *)x, mi, gamma, beta, (__nv_bfloat16 *)y, n8, G, C);
    } else {
        if (relu) bn_apply_kernel<float, true><<<grid, BN_THREADS, 0, st>>>((const float *)x, mi, gamma, beta, (float *)y, n8, G, C);
        else bn_apply_kernel<float, false><<<grid, BN_THREADS, 0, st>>>((const float *)x, mi, gamma, beta, (float *)y, n8, G, C);
    }
    count_launch(2);
}

void launch_bn_bwd(splitcnn_dtype_t dt, const void *dy, const void *x, const void *y, const float *mi,
                   const float *gamma, const float *t, double count, void *dx, int64_t n, int Cpad, int C,
                   cudaStream_t st) {
    const int64_t n8 = n / 8;
    const int G = Cpad / 8, grid = bn_grid(n8);
    const float invM = (float)(1.0 / count);
    if (dt == SPLITCNN_BF16)
        bn_bwd_kernel<__nv_bfloat16><<<grid, BN_THREADS, 0, st>>>((const __nv_bfloat16 *)dy, (const __nv_bfloat16 *)x,
                                                                  (const __nv_bfloat16 *)y, mi, gamma, t, invM,
                                                                  (__nv_bfloat16 *)dx, n8, G, C);
    else
        bn_bwd_kernel<float><<<grid, BN_THREADS, 0, st>>>((const float *)dy, (const float *)x, (const float *)y, mi, gamma,
                                                          t, invM, (float *)dx, n8, G, C);
    count_launch();
}

}  // namespace splitcnn
