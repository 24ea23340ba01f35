// common.cuh -- device helpers shared by the libsplitcnn kernels.
#pragma once
#include <cuda_bf16.h>
#include <cuda_runtime.h>
#include <cstdint>

#include "internal.h"

namespace splitcnn {

// ---------------------------------------------------------------- patch geometry on device
// n / d and n % d for 0 <= n < 2^31 with a host-precomputed multiplier (round-up method)
struct FastDiv {
    uint32_t d, mul, shr;
};
__device__ __forceinline__ uint32_t fdiv(uint32_t n, const FastDiv &f) { return (__umulhi(n, f.mul) + n) >> f.shr; }
__device__ __forceinline__ uint32_t fdivmod(uint32_t n, const FastDiv &f, uint32_t &rem) {
    const uint32_t q = fdiv(n, f);
    rem = n - q * f.d;
    return q;
}
__host__ __device__ inline FastDiv make_fastdiv(uint32_t d) {
    FastDiv f;
    f.d = d;
    uint32_t l = 0;
    while ((1ull << l) < d) ++l;  // (once per thread / launch)
    f.shr = l;
    f.mul = (uint32_t)(((1ull << 32) * ((1ull << l) - d)) / d + 1);
    return f;
}

struct PatchGeo {
    int i, j;     // patch row / column
    int h0, w0;   // global start
    int hp, wp;   // extents
    int64_t off;  // element offset of the patch buffer
};

__device__ __forceinline__ PatchGeo patch_geo(const LevelDesc &L, int q) {
    PatchGeo g;
    g.i = q / L.nw;
    g.j = q - g.i * L.nw;
    g.h0 = L.bh[g.i];
    g.w0 = L.bw[g.j];
    g.hp = L.bh[g.i + 1] - g.h0;
    g.wp = L.bw[g.j + 1] - g.w0;
    g.off = (int64_t)L.N * L.Cpad * ((int64_t)g.h0 * L.W + (int64_t)g.hp * g.w0);
    return g;
}

// ---------------------------------------------------------------- 8-channel vectors
template <typename T> struct Vec8;
template <> struct Vec8<__nv_bfloat16> {
    using raw = uint4;  // 16 B
};
template <> struct Vec8<float> {
    struct raw { float4 a, b; };  // 32 B
};

template <typename T>
__device__ __forceinline__ void load8(const T *p, float (&v)[8]);
template <>
__device__ __forceinline__ void load8<__nv_bfloat16>(const __nv_bfloat16 *p, float (&v)[8]) {
    uint4 r = __ldg(reinterpret_cast<const uint4 *>(p));
    const __nv_bfloat162 *h = reinterpret_cast<const __nv_bfloat162 *>(&r);
#pragma unroll
    for (int k = 0; k < 4; ++k) {
        float2 f = __bfloat1622float2(h[k]);
        v[2 * k] = f.x;
        v[2 * k + 1] = f.y;
    }
}
template <>
__device__ __forceinline__ void load8<float>(const float *p, float (&v)[8]) {
    float4 a = __ldg(reinterpret_cast<const float4 *>(p));
    float4 b = __ldg(reinterpret_cast<const float4 *>(p) + 1);
    v[0] = a.x; v[1] = a.y; v[2] = a.z; v[3] = a.w;
    v[4] = b.x; v[5] = b.y; v[6] = b.z; v[7] = b.w;
}

template <typename T>
__device__ __forceinline__ void store8(T *p, const float (&v)[8]);
template <>
__device__ __forceinline__ void store8<__nv_bfloat16>(__nv_bfloat16 *p, const float (&v)[8]) {
    uint4 r;
    __nv_bfloat162 *h = reinterpret_cast<__nv_bfloat162 *>(&r);
#pragma unroll
    for (int k = 0; k < 4; ++k) h[k] = __floats2bfloat162_rn(v[2 * k], v[2 * k + 1]);
    *reinterpret_cast<uint4 *>(p) = r;
}
template <>
__device__ __forceinline__ void store8<float>(float *p, const float (&v)[8]) {
    reinterpret_cast<float4 *>(p)[0] = make_float4(v[0], v[1], v[2], v[3]);
    reinterpret_cast<float4 *>(p)[1] = make_float4(v[4], v[5], v[6], v[7]);
}

__device__ __forceinline__ float to_f(float x) { return x; }
__device__ __forceinline__ float to_f(__nv_bfloat16 x) { return __bfloat162float(x); }
template <typename T> __device__ __forceinline__ T from_f(float x);
template <> __device__ __forceinline__ float from_f<float>(float x) { return x; }
template <> __device__ __forceinline__ __nv_bfloat16 from_f<__nv_bfloat16>(float x) { return __float2bfloat16_rn(x); }

}  // namespace splitcnn
