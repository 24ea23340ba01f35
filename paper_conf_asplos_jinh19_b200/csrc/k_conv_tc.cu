// k_conv_tc.cu -- tcgen05 implicit-GEMM split convolution for sm_100a (bf16 in, fp32 accumulate).
//
// One persistent, warp-specialised kernel serves the forward pass (Eq. 6) and the stride-1
// data gradient (the forward mainloop on dY with spatially flipped, transposed weights and the
// complementary per-patch pads k-1-p).  The patch-local zero padding of Split-CNN is folded into
// the tile loads: every patch gets its OWN 4-D TMA tensor map whose extents are the patch
// extents, so TMA's out-of-bounds zero fill IS the patch padding -- no window ever reads across a
// patch boundary and the kernel has no boundary branches.
//
//   GEMM view (per patch):  M = output pixels (n, oh, ow) tiled as BNn x BH x BW boxes (<= 128 rows),
//                           N = output channels (BN <= 256 per tile), K = taps x input channels.
//   warp 0      TMA producer: per K step one 4-D box of the input patch at the tap's offset
//               (element strides = conv stride) + one 2-D box of the weights, 128B/64B/32B swizzle
//   warp 1      MMA issuer (one thread): tcgen05.mma 128 x BN x 16 into a TMEM accumulator;
//               tcgen05.commit frees the smem stage / publishes the accumulator
//   warps 2-5   epilogue: tcgen05.ld -> +bias, ReLU (fwd) or ReLU-mask (dgrad) -> bf16 -> global
//   TMEM accumulators are double-buffered so the epilogue of tile t overlaps the mainloop of t+1.
#include <cuda.h>
#include <cudaTypedefs.h>

#include <algorithm>
#include <cstdlib>
#include <cstring>
#include <mutex>
#include <string>
#include <type_traits>
#include <unordered_map>
#include <vector>

#include "common.cuh"
#include "kernels.h"
#include "tc_ptx.cuh"

namespace splitcnn {

constexpr int TC_MAXP = 64;  // patches per launch (tensor maps live in the kernel parameters)

static bool wgrad_tc_ok(const Level &Li, const Level &Lo, const LayerGeom &g);
size_t wgrad_tc_ws_bytes(const Level &Li, const Level &Lo, const LayerGeom &g);

struct TcConvParams {
    CUtensorMap mapA[TC_MAXP];
    CUtensorMap mapY[TC_MAXP];   // output patch maps (TMA store of the staged tile)
    CUtensorMap mapR[TC_MAXP];   // ReLU-mask source maps (dgrad), same geometry as the output
    CUtensorMap mapB;
    int64_t out_off[TC_MAXP];
    int tile_prefix[TC_MAXP + 1];
    int out_h[TC_MAXP], out_w[TC_MAXP];
    int pt[TC_MAXP], pl[TC_MAXP];
    int nhb[TC_MAXP], nwb[TC_MAXP];
    int npatch;
    int N, BW, BH, BNn, rows_box, nnb, nco;
    int kh, kw, s;
    int cpadc;       // channels per A box (min(Cpad_A, 64))
    int cchunks;     // 64-channel chunks per tap (Cpad_A >= 64)
    int tps;         // taps per K step (Cpad_A < 64)
    int ksteps;      // K steps per tile
    int kchan;       // Cpad of the A side (K = taps * kchan)
    int a3d;         // 8-channel A: 3-D maps with pixels merged into 128-byte-wide rows (coordinate 8*w)
    int halo;        // stride-1 halo mode: one A box per (channel chunk, kernel row) serves the kw column taps
    int tall;        // halo, resident weights, one image per tile: ONE A box of BH + kh - 1 rows per channel chunk
                     // serves every kernel row (view r = r * Wp pixel rows on) -- K step = a channel chunk
    int halo8;       // 8-channel halo mode: ONE merged-row box per tile serves all taps (no-swizzle K-major A)
    int hn;          // narrow-row halo: 16- / 32-channel input (32 / 64 B SW32 / SW64 rows), one MMA per tap and 16
                     // channels; a kernel row's taps are one 64-element K box of the weights
    int b3d;         // halo: the kw taps' weights arrive as one 3-D box
    int Wp;          // halo: input box width = 8 + kw - 1
    uint32_t a_stage;  // bytes per A stage (1024-aligned)
    int bres;          // halo: all weights resident in smem (loaded once per CTA)
    uint32_t bres_off, bres_bytes;
    int BN, Cout, Cpo;
    int stages;
    uint32_t tmem_cols;
    uint32_t a_layout, a_sbo, a_lbo, a_chunk_bytes, a_tx_bytes, b_tx_bytes;
    const float *bias;
    __nv_bfloat16 *y;
    const __nv_bfloat16 *relu_src;
    int relu;
    int accum;        // TF32 direct epilogue: y = acc + y (3xTF32 passes), bias / ReLU / mask after the sum
    int res;          // forward: the relu_src tile is a residual, y = act(acc + bias + residual) (ResNet join)
    int tpp;          // tiles per patch when uniform (O(1) decode), else 0
    int direct;       // 1: per-thread global stores (odd channel pads); 0: smem-staged TMA store
    int ychunk;       // channels per output box (64, 32, 16 or 8)
    uint32_t y_mask;  // swizzle mask of the staging tile (7 / 3 / 1 / 0)
    uint32_t stage_off, bar_off;  // smem layout
    int ybufs;                    // staging buffers (2: the TMA store of tile t overlaps tile t+1)
    int egroups;                  // 2: two independent 4-warp epilogue groups, one per TMEM accumulator
    int yring;                    // egroups == 2: staging tiles per group (a ring: up to yring - 1 TMA stores in flight)
    int nacc_g;                   // TMEM accumulators per epilogue group (2 with dual issue)
    int dual;                     // two MMA-issuing warps (1 and 10) take alternate tiles (short-K tiles)
    int cta2;                     // 2-CTA MMA (cluster of 2, M = 256): each CTA owns one 128-row M box and N/2 of B
    int BNh;                      // rows of B per CTA (BN / 2 in 2-CTA mode, else BN)
    int total_m, total_pairs, m_tpp;
    int m_prefix[TC_MAXP + 1];
    uint32_t ybuf_bytes;
    int uni;                      // every patch has the same tile grid: O(1) decode by fast division
    FastDiv fd_tpp, fd_mtpp, fd_nco, fd_nwb, fd_nhb;
    int ysh;                      // log2(ychunk)
    // fused 2x2 / stride-2 max-pool epilogue (POOL): pooled values + argmax bytes of level layer+2
    __nv_bfloat16 *pool_y;
    uint8_t *pool_a;
    int64_t pool_off[TC_MAXP];
};

static_assert(sizeof(TcConvParams) <= 32700, "kernel parameter space is 32 KB");

// 2-CTA mode: M box index (across patches) -> patch, image block, row block, column block
__device__ __forceinline__ void decode_mbox(const TcConvParams &p, int m, int &ql, int &nb, int &hb, int &wb) {
    if (p.uni) {
        uint32_t idx, r;
        ql = (int)fdivmod((uint32_t)m, p.fd_mtpp, idx);
        idx = fdivmod(idx, p.fd_nwb, r);
        wb = (int)r;
        nb = (int)fdivmod(idx, p.fd_nhb, r);
        hb = (int)r;
        return;
    }
    ql = 0;
    while (m >= p.m_prefix[ql + 1]) ++ql;
    int idx = m - p.m_prefix[ql];
    wb = idx % p.nwb[ql];
    idx /= p.nwb[ql];
    hb = idx % p.nhb[ql];
    nb = idx / p.nhb[ql];
}

__device__ __forceinline__ void decode_tile(const TcConvParams &p, int t, int &ql, int &nb, int &hb, int &wb, int &cb) {
    if (p.uni) {
        uint32_t idx, r;
        ql = (int)fdivmod((uint32_t)t, p.fd_tpp, idx);
        idx = fdivmod(idx, p.fd_nco, r);
        cb = (int)r;
        idx = fdivmod(idx, p.fd_nwb, r);
        wb = (int)r;
        nb = (int)fdivmod(idx, p.fd_nhb, r);
        hb = (int)r;
        return;
    }
    ql = 0;
    while (t >= p.tile_prefix[ql + 1]) ++ql;
    int idx = t - p.tile_prefix[ql];
    cb = idx % p.nco;
    idx /= p.nco;
    wb = idx % p.nwb[ql];
    idx /= p.nwb[ql];
    hb = idx % p.nhb[ql];
    nb = idx / p.nhb[ql];
}

// work item t of this CTA -> (patch, image block, row block, column block, co block); `valid` false for
// the idle second half of an odd last pair
__device__ __forceinline__ void get_tile(const TcConvParams &p, int t, uint32_t rank, int &ql, int &nb, int &hb, int &wb,
                                         int &cb, bool &valid) {
    if (p.cta2) {
        uint32_t r;
        const int mp = (int)fdivmod((uint32_t)t, p.fd_nco, r);
        cb = (int)r;
        int m = 2 * mp + (int)rank;
        valid = m < p.total_m;
        m = min(m, p.total_m - 1);
        decode_mbox(p, m, ql, nb, hb, wb);
    } else {
        decode_tile(p, t, ql, nb, hb, wb, cb);
        valid = true;
    }
}


// producer warp, MMA warp, 8 epilogue warps (2 per TMEM lane quadrant), a second MMA warp (dual issue)
constexpr int CONV_THREADS = 64 + 256 + 32;

// packed epilogue arithmetic (the epilogue warps are issue-latency bound on the narrow-N layers: every
// instruction per column shows): two fp32 adds per FADD2, ReLU fused into the bf16x2 rounding (F2FP.RELU:
// round-to-nearest then clamp at 0 == round(max(x, 0)) for every non-NaN x), the dgrad ReLU mask applied
// to the ROUNDED pair as a bitwise select (bf16(0) = +0, so masking after rounding is bit-identical)
__device__ __forceinline__ void add2(float &a, float &b, float c, float d) {
    uint64_t x = ((uint64_t)__float_as_uint(b) << 32) | __float_as_uint(a);
    const uint64_t y = ((uint64_t)__float_as_uint(d) << 32) | __float_as_uint(c);
    asm("add.rn.f32x2 %0, %0, %1;" : "+l"(x) : "l"(y));
    a = __uint_as_float((uint32_t)x);
    b = __uint_as_float((uint32_t)(x >> 32));
}
template <bool RELU>
__device__ __forceinline__ uint32_t pack_bf16x2(float lo, float hi) {
    uint32_t r;
    if (RELU) asm("cvt.rn.relu.bf16x2.f32 %0, %1, %2;" : "=r"(r) : "f"(hi), "f"(lo));
    else asm("cvt.rn.bf16x2.f32 %0, %1, %2;" : "=r"(r) : "f"(hi), "f"(lo));
    return r;
}
// bf16x2 word m -> 0xFFFF per half where that half is > 0 (NaN / zero / negative: 0)
__device__ __forceinline__ uint32_t pos_mask2(uint32_t m) {
    const uint32_t z = 0u;
    return __hgt2_mask(*reinterpret_cast<const __nv_bfloat162 *>(&m), *reinterpret_cast<const __nv_bfloat162 *>(&z));
}

// 8 accumulator columns (all real channels) -> bf16x8: +bias, ReLU, dgrad ReLU mask
template <bool BIAS, bool RELU, bool MASK>
__device__ __forceinline__ uint4 epi8_full(const uint32_t *r, const float *sb, uint4 m4, bool res = false) {
    float o[8];
#pragma unroll
    for (int e = 0; e < 8; ++e) o[e] = __uint_as_float(r[e]);
    if (BIAS) {
        const float4 b0 = *reinterpret_cast<const float4 *>(sb);
        const float4 b1 = *reinterpret_cast<const float4 *>(sb + 4);
        add2(o[0], o[1], b0.x, b0.y); add2(o[2], o[3], b0.z, b0.w);
        add2(o[4], o[5], b1.x, b1.y); add2(o[6], o[7], b1.z, b1.w);
    }
    if (MASK && res) {   // residual join fused into the forward epilogue: the tile holds the shortcut
        const __nv_bfloat162 *mh = reinterpret_cast<const __nv_bfloat162 *>(&m4);
#pragma unroll
        for (int e = 0; e < 4; ++e) {
            const float2 mf = __bfloat1622float2(mh[e]);
            add2(o[2 * e], o[2 * e + 1], mf.x, mf.y);
        }
    }
    uint32_t w[4];
#pragma unroll
    for (int e = 0; e < 4; ++e) w[e] = pack_bf16x2<RELU>(o[2 * e], o[2 * e + 1]);
    if (MASK && !res) {
        w[0] &= pos_mask2(m4.x); w[1] &= pos_mask2(m4.y);
        w[2] &= pos_mask2(m4.z); w[3] &= pos_mask2(m4.w);
    }
    return make_uint4(w[0], w[1], w[2], w[3]);
}

// 8 accumulator columns -> bf16x8 with the fused epilogue (bias, ReLU, or the dgrad ReLU mask)
template <bool BIAS, bool RELU, bool MASK>
__device__ __forceinline__ uint4 epi8(const uint32_t *r, const float *sb, int co, int Cout, uint4 m4, bool res = false) {
    float o[8];
#pragma unroll
    for (int e = 0; e < 8; ++e) o[e] = __uint_as_float(r[e]);
    if (co + 8 <= Cout) {
        if (BIAS) {
            const float4 b0 = *reinterpret_cast<const float4 *>(sb + co);
            const float4 b1 = *reinterpret_cast<const float4 *>(sb + co + 4);
            add2(o[0], o[1], b0.x, b0.y); add2(o[2], o[3], b0.z, b0.w);
            add2(o[4], o[5], b1.x, b1.y); add2(o[6], o[7], b1.z, b1.w);
        }
    } else {
#pragma unroll
        for (int e = 0; e < 8; ++e) o[e] = (co + e < Cout) ? (BIAS ? o[e] + sb[co + e] : o[e]) : 0.f;
    }
    if (MASK && res) {   // residual join (padding channels of the shortcut are zero)
        const __nv_bfloat162 *mh = reinterpret_cast<const __nv_bfloat162 *>(&m4);
#pragma unroll
        for (int e = 0; e < 4; ++e) {
            const float2 mf = __bfloat1622float2(mh[e]);
            add2(o[2 * e], o[2 * e + 1], mf.x, mf.y);
        }
    }
    uint32_t w[4];
#pragma unroll
    for (int e = 0; e < 4; ++e) w[e] = pack_bf16x2<RELU>(o[2 * e], o[2 * e + 1]);
    if (MASK && !res) {
        w[0] &= pos_mask2(m4.x); w[1] &= pos_mask2(m4.y);
        w[2] &= pos_mask2(m4.z); w[3] &= pos_mask2(m4.w);
    }
    return make_uint4(w[0], w[1], w[2], w[3]);
}

// Fused 2x2 / stride-2 max-pool of 16 accumulator columns (pool semantics of
// pool_fwd_kernel: max over the window of the bf16-ROUNDED conv outputs, argmax = r*2 + c of the FIRST
// maximum in window order, bit 7 = [max > 0]).  Rows are pixels (w fastest, BW a power of two, BH even),
// so the window partners of row m are m^1 (c) and m^BW (r), both in the same warp: two shuffle rounds.
// All lanes take part; `writer` (w and h even, pixel in range) stores 16 pooled values (32 B) and 16
// argmax bytes (16 B).
__device__ __forceinline__ void pool16(const float *v, int bw, bool writer, __nv_bfloat16 *yp, uint8_t *ap) {
    float best[16];
    uint32_t arg = 0;   // 2 bits per column
#pragma unroll
    for (int e = 0; e < 16; ++e) best[e] = __bfloat162float(__float2bfloat16_rn(v[e]));
#pragma unroll
    for (int e = 0; e < 16; ++e) {   // column partner: window index c = 1 (valid for even-w rows)
        const float o = __shfl_xor_sync(0xffffffffu, best[e], 1);
        if (o > best[e]) { best[e] = o; arg |= 1u << (2 * e); }
    }
    const uint32_t oarg = __shfl_xor_sync(0xffffffffu, arg, bw);
#pragma unroll
    for (int e = 0; e < 16; ++e) {   // row partner: window indices 2 + c (valid for even-h rows)
        const float o = __shfl_xor_sync(0xffffffffu, best[e], bw);
        if (o > best[e]) { best[e] = o; arg = (arg & ~(3u << (2 * e))) | ((2u + ((oarg >> (2 * e)) & 1u)) << (2 * e)); }
    }
    if (!writer) return;
    uint4 pk[2];
    __nv_bfloat162 *h2 = reinterpret_cast<__nv_bfloat162 *>(pk);
#pragma unroll
    for (int e = 0; e < 8; ++e) h2[e] = __floats2bfloat162_rn(best[2 * e], best[2 * e + 1]);
    reinterpret_cast<uint4 *>(yp)[0] = pk[0];
    reinterpret_cast<uint4 *>(yp)[1] = pk[1];
    uint32_t ab[4] = {0, 0, 0, 0};
#pragma unroll
    for (int e = 0; e < 16; ++e)
        ab[e >> 2] |= (((arg >> (2 * e)) & 3u) | (best[e] > 0.f ? 0x80u : 0u)) << (8 * (e & 3));
    *reinterpret_cast<uint4 *>(ap) = make_uint4(ab[0], ab[1], ab[2], ab[3]);
}

// The same on 32 columns already packed as bf16x2 words w[16] (the conv epilogue's rounded values):
// bf16x2 compares (__hgt2_mask) and bitwise selects, so a tie keeps the FIRST element bit for bit
// (as pool_fwd_kernel's strict '>') and half the shuffles of the fp32 form.
__device__ __forceinline__ uint32_t bsel(uint32_t m, uint32_t a, uint32_t b) { return (a & m) | (b & ~m); }
__device__ __forceinline__ uint32_t hgt2(uint32_t a, uint32_t b) {
    return __hgt2_mask(*reinterpret_cast<const __nv_bfloat162 *>(&a), *reinterpret_cast<const __nv_bfloat162 *>(&b));
}
__device__ __forceinline__ void pool32(const uint32_t *w, int bw, bool writer, __nv_bfloat16 *yp, uint8_t *ap) {
    uint32_t best[16], cmask[16], amask[16];
#pragma unroll
    for (int e = 0; e < 16; ++e) {   // column partner (window index c = 1)
        const uint32_t o = __shfl_xor_sync(0xffffffffu, w[e], 1);
        cmask[e] = hgt2(o, w[e]);
        best[e] = bsel(cmask[e], o, w[e]);
    }
#pragma unroll
    for (int e = 0; e < 16; ++e) {   // row partner (window indices 2 + c)
        const uint32_t o = __shfl_xor_sync(0xffffffffu, best[e], bw);
        const uint32_t oc = __shfl_xor_sync(0xffffffffu, cmask[e], bw);
        const uint32_t m = hgt2(o, best[e]);
        best[e] = bsel(m, o, best[e]);
        // per half: bit 1 = row index (m), bit 0 = column index of the winning row
        amask[e] = (m & 0x00020002u) | (bsel(m, oc, cmask[e]) & 0x00010001u);
    }
    if (!writer) return;
    uint4 *y4 = reinterpret_cast<uint4 *>(yp);
#pragma unroll
    for (int q = 0; q < 4; ++q) y4[q] = make_uint4(best[4 * q], best[4 * q + 1], best[4 * q + 2], best[4 * q + 3]);
    // argmax byte per element: window index (bits 0-1, already at bits 0-1 / 16-17 of amask) | [max > 0] << 7,
    // two elements per word in bytes 0 and 2, then two words' bytes interleaved into four by one PRMT
    uint32_t ab[8];
#pragma unroll
    for (int q = 0; q < 8; ++q) {
        const uint32_t v0 = amask[2 * q] | (pos_mask2(best[2 * q]) & 0x00800080u);
        const uint32_t v1 = amask[2 * q + 1] | (pos_mask2(best[2 * q + 1]) & 0x00800080u);
        ab[q] = __byte_perm(v0, v1, 0x6420);
    }
    reinterpret_cast<uint4 *>(ap)[0] = make_uint4(ab[0], ab[1], ab[2], ab[3]);
    reinterpret_cast<uint4 *>(ap)[1] = make_uint4(ab[4], ab[5], ab[6], ab[7]);
}

// TF32: fp32 operands (kind::tf32 MMAs on the same byte-addressed tiles: an fp32 channel is two bf16
// "channels" of the byte layout) and fp32 outputs through the direct epilogue (host: P.direct = 1)
template <bool BIAS, bool RELU, bool MASK, bool CTA2, bool POOL = false, bool TF32 = false>
__global__ void __launch_bounds__(CONV_THREADS, 1) conv_tc_kernel(const __grid_constant__ TcConvParams p) {
    extern __shared__ uint8_t smem_raw[];
    uint8_t *smem = smem_raw + ((1024u - (tc::smem_u32(smem_raw) & 1023u)) & 1023u);   // keeps the shared space
    const int S = p.stages;
    const uint32_t b_stage = p.b_tx_bytes;   // BN x 128 B per tap box (kw boxes in halo mode)
    uint8_t *sA = smem;
    uint8_t *sB = smem + (size_t)S * p.a_stage;
    uint8_t *sY = smem + p.stage_off;  // output staging tile (1024-aligned)
    uint64_t *full = (uint64_t *)(smem + p.bar_off);
    uint64_t *empty = full + S;
    uint64_t *tfull = empty + S;
    uint64_t *tempty = tfull + 4;
    uint64_t *ybar = tempty + 4;
    uint64_t *wbar = ybar + 1;
    uint32_t *tmem_slot = (uint32_t *)(wbar + 2);
    uint8_t *sW = smem + p.bres_off;   // resident weights (bres)
    float *sbias = (float *)(smem + p.bar_off + 512);   // [Cout] bias (16-byte aligned)

    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const uint32_t rank = CTA2 ? tc::cluster_ctarank() : 0u;
    const bool leader = rank == 0;
    // launched with programmatic stream serialization (PDL): this grid's CTAs are placed while the previous
    // kernel drains; nothing below touches global memory before the previous grid is complete and visible
    tc::grid_dep_launch();
    tc::grid_dep_wait();
    if (warp == 0 && lane == 0) {
        for (int s = 0; s < S; ++s) {
            tc::mbar_init(&full[s], 1);
            tc::mbar_init(&empty[s], 1);
        }
        for (int a = 0; a < 4; ++a) {
            tc::mbar_init(&tfull[a], 1);
            // the leader's accumulator-empty barrier hears both CTAs' epilogues in 2-CTA mode
            tc::mbar_init(&tempty[a], (p.egroups == 2 ? 4 : 8) * (CTA2 ? 2 : 1));
        }
        tc::mbar_init(ybar, 1);
        tc::mbar_init(wbar, 1);
        tc::mbar_init(wbar + 1, 1);   // group 1's mask barrier
        uint64_t *mbarR = reinterpret_cast<uint64_t *>(smem + p.bar_off + 256);   // mask ring: 4 slots x 2 groups
        for (int r = 0; r < 8; ++r) tc::mbar_init(&mbarR[r], 1);
        tc::fence_barrier_init();
    }
    if (BIAS)
        for (int i = threadIdx.x; i < p.Cout; i += blockDim.x) sbias[i] = __ldg(p.bias + i);
    if (warp == 1) {
        if (CTA2) tc::tmem_alloc2(tmem_slot, p.tmem_cols);
        else tc::tmem_alloc_dyn(tmem_slot, p.tmem_cols);
    }
    tc::tc_fence_before();
    if (CTA2) tc::cluster_sync_all();
    else __syncthreads();
    tc::tc_fence_after();
    const uint32_t tmem_base = *tmem_slot;
    const int total = CTA2 ? p.total_pairs : p.tile_prefix[p.npatch];
    const int tfirst = CTA2 ? (int)tc::cluster_id_x() : (int)blockIdx.x;
    const int tstep = CTA2 ? (int)tc::nclusters_x() : (int)gridDim.x;
    const int KT = p.kh * p.kw;

    if (warp == 0) {
        if (lane == 0) {
            // ================= TMA producer
            for (int q = 0; q < p.npatch; ++q) tc::tma_prefetch_desc(&p.mapA[q]);
            tc::tma_prefetch_desc(&p.mapB);
            const uint32_t wbar_l = CTA2 ? tc::mapa_shared(wbar, 0) : 0u;
            if (p.bres && p.halo8) {   // the K = taps x 8 filter in 64-wide boxes, once per CTA
                tc::mbar_arrive_expect_tx(wbar, p.bres_bytes);
                for (int kb = 0; kb * 64 < KT * 8; ++kb) tc::tma_load_2d(sW + kb * p.BN * 128, &p.mapB, wbar, kb * 64, 0);
            } else if (p.bres && p.hn) {   // one 64-element K box per kernel row (its kw taps x Cpad channels)
                tc::mbar_arrive_expect_tx(wbar, p.bres_bytes);
                for (int r = 0; r < p.kh; ++r) tc::tma_load_2d(sW + (size_t)r * p.BN * 128, &p.mapB, wbar, r * p.kw * p.kchan, 0);
            } else if (p.bres) {  // every (chunk, kernel row) weight box once, for all tiles of this CTA
                const int rowB0 = (int)rank * p.BNh;  // 2-CTA: this CTA holds rows [rank*BN/2, +BN/2) of B
                if (!CTA2) tc::mbar_arrive_expect_tx(wbar, p.bres_bytes);
                else if (leader) tc::mbar_arrive_expect_tx(wbar, 2 * p.bres_bytes);
                const int nchunk = p.kchan / 64;
                for (int cc = 0; cc < nchunk; ++cc)
                    for (int r = 0; r < p.kh; ++r) {
                        uint8_t *dst = sW + (size_t)((cc * p.kh + r) * p.kw) * p.BNh * 128;
                        if (CTA2) {
                            if (p.b3d) {
                                tc::tma2_load_3d(dst, &p.mapB, wbar_l, cc * 64, rowB0, r * p.kw);
                            } else {
                                for (int c = 0; c < p.kw; ++c)
                                    tc::tma2_load_2d(dst + c * p.BNh * 128, &p.mapB, wbar_l, (r * p.kw + c) * p.kchan + cc * 64, rowB0);
                            }
                        } else if (p.b3d) {
                            tc::tma_load_3d(dst, &p.mapB, wbar, cc * 64, 0, r * p.kw);
                        } else {
                            for (int c = 0; c < p.kw; ++c)
                                tc::tma_load_2d(dst + c * p.BN * 128, &p.mapB, wbar, (r * p.kw + c) * p.kchan + cc * 64, 0);
                        }
                    }
            }
            int stage = 0, it = 0;
            uint32_t ph = 0;
            // dual issue: two stage rings (even / odd stages), iteration it fills ring it & 1, so each MMA
            // warp waits on its own stages in order (a parity wait must never be two phases ahead)
            const int S2 = S & ~1;
            int rs0 = 0, rs1 = 1;            // next stage / phase of ring 0 and ring 1 (registers, no stack)
            uint32_t rph0 = 0u, rph1 = 0u;
            // loop-invariant step / ring length: the per-K-step advance costs what `++stage == S` did (the
            // MMA warp's K-step loop is issue-latency bound for narrow N, every instruction in it shows)
            const int sstep = p.dual ? 2 : 1, Sx = p.dual ? S2 : S;
            auto adv = [&]() {
                stage += sstep;
                if (stage >= Sx) { stage -= Sx; ph ^= 1; }
            };
            for (int t = tfirst; t < total; t += tstep, ++it) {
                int ql, nb, hb, wb, cb;
                bool valid;
                get_tile(p, t, rank, ql, nb, hb, wb, cb, valid);
                if (p.dual) { stage = (it & 1) ? rs1 : rs0; ph = (it & 1) ? rph1 : rph0; }
                const int wbase = wb * p.BW * p.s - p.pl[ql];
                const int hbase = hb * p.BH * p.s - p.pt[ql];
                const int n0 = nb * p.BNn, co0 = cb * p.BN;
                for (int ks = 0; ks < p.ksteps; ++ks) {
                    tc::mbar_wait(&empty[stage], ph ^ 1);
                    uint8_t *a = sA + (size_t)stage * p.a_stage;
                    uint8_t *b = sB + (size_t)stage * b_stage;
                    if (CTA2) {
                        // both CTAs load their own A box and their half of B; bytes land on the leader's barrier
                        const uint32_t fb = tc::mapa_shared(&full[stage], 0);
                        if (leader) tc::mbar_arrive_expect_tx(&full[stage], 2 * (p.a_tx_bytes + p.b_tx_bytes));
                        const int cor = co0 + (int)rank * p.BNh;
                        if (p.halo) {
                            const int cc = p.tall ? ks : ks / p.kh, r = p.tall ? 0 : ks - cc * p.kh;
                            tc::tma2_load_4d(a, &p.mapA[ql], fb, cc * 64, wbase, hbase + r, n0);
                            if (!p.bres) {
                                if (p.b3d) {
                                    tc::tma2_load_3d(b, &p.mapB, fb, cc * 64, cor, r * p.kw);
                                } else {
                                    for (int c = 0; c < p.kw; ++c)
                                        tc::tma2_load_2d(b + c * p.BNh * 128, &p.mapB, fb, (r * p.kw + c) * p.kchan + cc * 64, cor);
                                }
                            }
                        } else {
                            const int tap = ks / p.cchunks, cc = ks - tap * p.cchunks;
                            const int r = tap / p.kw, c = tap - r * p.kw;
                            tc::tma2_load_4d(a, &p.mapA[ql], fb, cc * 64, wbase + c, hbase + r, n0);
                            tc::tma2_load_2d(b, &p.mapB, fb, tap * p.kchan + cc * 64, cor);
                        }
                        adv();
                        continue;
                    }
                    tc::mbar_arrive_expect_tx(&full[stage], p.a_tx_bytes + p.b_tx_bytes);
                    if (p.halo8) {
                        // rows (h) x (8 + kw - 1) pixels x 8 channels; the weights' K = taps*8 in 64-wide boxes
                        tc::tma_load_3d(a, &p.mapA[ql], &full[stage], 8 * wbase, hbase, n0);
                        if (!p.bres)
                            for (int kb = 0; kb * 64 < KT * 8; ++kb)
                                tc::tma_load_2d(b + kb * p.BN * 128, &p.mapB, &full[stage], kb * 64, co0);
                    } else if (p.halo) {
                        const int cc = p.tall ? ks : ks / p.kh, r = p.tall ? 0 : ks - cc * p.kh;
                        tc::tma_load_4d(a, &p.mapA[ql], &full[stage], cc * 64, wbase, hbase + r, n0);
                        if (p.bres) {
                        } else if (p.hn) {
                            tc::tma_load_2d(b, &p.mapB, &full[stage], r * p.kw * p.kchan, co0);
                        } else if (p.b3d) {
                            tc::tma_load_3d(b, &p.mapB, &full[stage], cc * 64, co0, r * p.kw);
                        } else {
                            for (int c = 0; c < p.kw; ++c)
                                tc::tma_load_2d(b + c * p.BN * 128, &p.mapB, &full[stage], (r * p.kw + c) * p.kchan + cc * 64, co0);
                        }
                    } else if (p.tps > 1) {
                        for (int j = 0; j < p.tps; ++j) {
                            const int tap = min(ks * p.tps + j, KT - 1);  // past the last tap: weights are OOB zero
                            const int r = tap / p.kw, c = tap - r * p.kw;
                            if (p.a3d)
                                tc::tma_load_3d(a + j * p.a_chunk_bytes, &p.mapA[ql], &full[stage], 8 * (wbase + c), hbase + r, n0);
                            else
                                tc::tma_load_4d(a + j * p.a_chunk_bytes, &p.mapA[ql], &full[stage], 0, wbase + c, hbase + r, n0);
                        }
                        tc::tma_load_2d(b, &p.mapB, &full[stage], ks * 64, co0);
                    } else {
                        const int tap = ks / p.cchunks, cc = ks - tap * p.cchunks;
                        const int r = tap / p.kw, c = tap - r * p.kw;
                        tc::tma_load_4d(a, &p.mapA[ql], &full[stage], cc * 64, wbase + c, hbase + r, n0);
                        tc::tma_load_2d(b, &p.mapB, &full[stage], tap * p.kchan + cc * 64, co0);
                    }
                    adv();
                }
                if (p.dual) {
                    if (it & 1) { rs1 = stage; rph1 = ph; }
                    else { rs0 = stage; rph0 = ph; }
                }
            }
        }
    } else if (warp == 1 || (warp == 10 && p.dual)) {
        // q (which issuer) is a compile-time constant of each copy of the loop: derived from the warp index
        // it would make the stage index look thread-varying to the compiler, and every descriptor would take
        // a broadcast register move per MMA (the issue path of narrow-N tiles is latency-bound)
        auto mma_run = [&](auto QC) {
            // ================= MMA issuer: the whole warp runs the loop converged; elect.sync issues.
            // In 2-CTA mode only the leader issues (M = 256 over the pair); the peer's warp 1 idles.
            // Dual issue (p.dual): warps 1 and 10 take alternate tiles, so one warp's per-tile handshake
            // (accumulator wait, stage wait, commits) overlaps the other's MMAs -- a tcgen05.mma issue does
            // not run ahead of the tensor pipe by much, so a single issuer leaves it idle for those cycles.
            constexpr int q = decltype(QC)::value;
            const uint32_t idesc = tc::idesc_k<TF32>(CTA2 ? 256 : 128, p.BN);
            // halo8: per tap pair, the descriptor relative to the stage base (start address field 0)
            uint64_t h8_adesc[8], h8_bdesc[8];
            const int h8_npairs = p.halo8 ? (KT + 1) / 2 : 0;
#pragma unroll
            for (int pr = 0; pr < 8; ++pr) {
                h8_adesc[pr] = h8_bdesc[pr] = 0;
                if (pr < h8_npairs) {
                    const int t0 = 2 * pr, t1 = 2 * pr + 1;
                    const int o0 = (t0 / p.kw) * p.Wp + (t0 % p.kw);
                    // a missing second tap (odd KT) re-reads tap t0's pixels (LBO = 0) against zero weights:
                    // a view one pixel on would leave the loaded box for the tile's last row and multiply
                    // stale shared memory (possibly NaN / Inf) by zero
                    const int o1 = t1 < KT ? (t1 / p.kw) * p.Wp + (t1 % p.kw) : o0;
                    h8_adesc[pr] = tc::smem_desc(0, 16u * (uint32_t)(o1 - o0), (uint32_t)p.Wp * 16u, 0) + (uint64_t)o0;
                    h8_bdesc[pr] = tc::smem_desc(0, 16, 1024, 2) + (uint64_t)((((pr >> 2) * p.BN) * 128 + 32 * (pr & 3)) >> 4);
                }
            }
            // generic path: start-address offset (>> 4) of the 4 K=16 slices of a K step
            uint32_t g_aoff[4];
#pragma unroll
            for (int j = 0; j < 4; ++j) {
                const int k0 = 16 * j;
                const int chunk = k0 / p.cpadc;
                g_aoff[j] = (chunk * p.a_chunk_bytes + (uint32_t)((k0 - chunk * p.cpadc) * 2)) >> 4;
            }
            const int istep = p.dual ? 2 : 1;
            int stage = p.dual ? q : 0;   // dual: this warp's stage ring (see the producer)
            uint32_t ph = 0;
            const int S2 = S & ~1;
            // loop-invariant step / ring length: the per-K-step advance costs what `++stage == S` did (the
            // MMA warp's K-step loop is issue-latency bound for narrow N, every instruction in it shows)
            const int sstep = p.dual ? 2 : 1, Sx = p.dual ? S2 : S;
            auto adv = [&]() {
                stage += sstep;
                if (stage >= Sx) { stage -= Sx; ph ^= 1; }
            };
            if (p.bres && leader) tc::mbar_wait(wbar, 0);
            // this warp cycles through two accumulator slots: 0, 1 (one issuer: tile it -> epilogue group
            // it & 1) or 2q, 2q + 1 (dual: warp q's tiles all go to group q, which alternates its two)
            // tile ordinal it of this CTA -> epilogue group it & 1, that group's k = it >> 1-th tile -> slot
            // g * nacc_g + (k & 1) with nacc_g accumulators per group (2: the MMA runs two tiles of a group
            // ahead of its epilogue; also with one issuer)
            int it = q;
            for (int t = leader ? tfirst + q * tstep : total; t < total; t += istep * tstep, it += istep) {
                const int kg = it >> 1;
                const int slot = (it & 1) * p.nacc_g + (p.nacc_g == 2 ? (kg & 1) : 0);
                const uint32_t aph = (uint32_t)((p.nacc_g == 2 ? (kg >> 1) : kg) & 1);
                tc::mbar_wait(&tempty[slot], aph ^ 1);
                tc::tc_fence_after();
                const uint32_t d = tmem_base + (uint32_t)(slot * p.BN);
                for (int ks = 0; ks < p.ksteps; ++ks) {
                    tc::mbar_wait(&full[stage], ph);
                    tc::tc_fence_after();
                    const uint32_t a_base = tc::smem_u32(sA + (size_t)stage * p.a_stage);
                    const uint32_t b_base = tc::smem_u32(sB + (size_t)stage * b_stage);
                    if (p.halo8) {
                        // no-swizzle K-major A: a core matrix is 8 consecutive pixels x 16 B (8 channels);
                        // M groups (output rows) are Wp pixels apart (SBO = Wp*16 B); each MMA covers the
                        // K = 16 of two taps whose views differ by LBO = (pixel offset difference)*16 B.
                        // Descriptors are linear in the start address: tile-invariant parts precomputed.
                        const uint64_t abase = (uint64_t)((a_base >> 4) & 0x3FFF);
                        const uint64_t bbase = (uint64_t)(((p.bres ? tc::smem_u32(sW) : b_base) >> 4) & 0x3FFF);
#pragma unroll
                        for (int pr = 0; pr < 8; ++pr) {
                            if (pr < h8_npairs)
                                tc::mma_k_ws<TF32>(d, h8_adesc[pr] + abase, h8_bdesc[pr] + bbase, idesc, (ks | pr) != 0);
                        }
                        tc::mma_commit_ws(&empty[stage]);
                        adv();
                        continue;
                    }
                    if (p.halo && CTA2 && p.tall) {   // every kernel row from one box: views r * Wp rows on
                        const uint32_t bstep = (uint32_t)p.BNh * 8u;
                        for (int r = 0; r < p.kh; ++r) {
                            const uint64_t a0 = tc::smem_desc(a_base + (uint32_t)(r * p.Wp) * 128u, 16, (uint32_t)p.Wp * 128u, 2);
                            const uint64_t b0 = tc::smem_desc(tc::smem_u32(sW) + (uint32_t)((ks * p.kh + r) * p.kw * p.BNh) * 128u,
                                                              16, 1024, 2);
                            for (int c = 0; c < p.kw; ++c)
                                tc::mma2_bf16_x4_ws(d, a0 + (uint64_t)(8 * c), b0 + (uint64_t)(bstep * c), idesc, (ks | r | c) != 0);
                        }
                        tc::mma2_commit_mc_ws(&empty[stage]);
                        adv();
                        continue;
                    }
                    if (p.halo && CTA2) {
                        const uint64_t a0 = tc::smem_desc(a_base, 16, (uint32_t)p.Wp * 128u, 2);
                        const uint64_t b0 = p.bres ? tc::smem_desc(tc::smem_u32(sW) + (uint32_t)(ks * p.kw * p.BNh) * 128u, 16, 1024, 2)
                                                   : tc::smem_desc(b_base, 16, 1024, 2);
                        const uint32_t bstep = (uint32_t)p.BNh * 8u;
                        for (int c = 0; c < p.kw; ++c)
                            tc::mma2_bf16_x4_ws(d, a0 + (uint64_t)(8 * c), b0 + (uint64_t)(bstep * c), idesc, (ks | c) != 0);
                        tc::mma2_commit_mc_ws(&empty[stage]);
                        adv();
                        continue;
                    }
                    if (CTA2) {
                        const uint64_t a0 = tc::smem_desc(a_base, 16, 1024, 2);
                        const uint64_t b0 = tc::smem_desc(b_base, 16, 1024, 2);
                        tc::mma2_bf16_x4_ws(d, a0, b0, idesc, ks != 0);
                        tc::mma2_commit_mc_ws(&empty[stage]);
                        adv();
                        continue;
                    }
                    if (p.hn) {
                        // narrow rows: tap c of kernel row r is the A box viewed (r * Wp + c) pixel rows on
                        // (SW32 / SW64, address-based), its K = 16 slices 32 B apart; the weights' slice of tap c
                        // is 2 * c * Cpad bytes into the kernel row's 128 B K box
                        const uint32_t rb = 2u * (uint32_t)p.kchan;
                        const int nrow = p.tall ? p.kh : 1;
                        for (int rr = 0; rr < nrow; ++rr) {
                            const int r = p.tall ? rr : ks;
                            const uint64_t a0 = tc::smem_desc(a_base + (uint32_t)(rr * p.Wp) * rb, 16, (uint32_t)p.Wp * rb, p.a_layout);
                            const uint64_t b0 = tc::smem_desc(p.bres ? tc::smem_u32(sW) + (uint32_t)(r * p.BN) * 128u : b_base, 16, 1024, 2);
                            // slice (c, j) sits (c * Cpad / 8 + 2 j) 16-byte units on in BOTH operands: a kernel row
                            // with kw * Cpad = 64 is exactly the four 32-byte steps of one x4 issue
                            if (p.kw * p.kchan == 64) {
                                tc::mma_k_x4_ws<TF32>(d, a0, b0, idesc, (ks | rr) != 0);
                                continue;
                            }
                            for (int c = 0; c < p.kw; ++c)
                                for (int j = 0; j < p.kchan / 16; ++j)
                                    tc::mma_k_ws<TF32>(d, a0 + (uint64_t)((c * rb + 32u * j) >> 4),
                                                       b0 + (uint64_t)((2u * c * p.kchan + 32u * j) >> 4), idesc,
                                                       (ks | rr | c | j) != 0);
                        }
                        tc::mma_commit_ws(&empty[stage]);
                        adv();
                        continue;
                    }
                    if (p.halo && p.tall) {   // every kernel row from one box: views r * Wp rows on
                        const uint32_t bstep = (uint32_t)p.BN * 8u;
                        for (int r = 0; r < p.kh; ++r) {
                            const uint64_t a0 = tc::smem_desc(a_base + (uint32_t)(r * p.Wp) * 128u, 16, (uint32_t)p.Wp * 128u, 2);
                            const uint64_t b0 = tc::smem_desc(tc::smem_u32(sW) + (uint32_t)((ks * p.kh + r) * p.kw * p.BN) * 128u,
                                                              16, 1024, 2);
                            for (int c = 0; c < p.kw; ++c)
                                tc::mma_k_x4_ws<TF32>(d, a0 + (uint64_t)(8 * c), b0 + (uint64_t)(bstep * c), idesc,
                                                      (ks | r | c) != 0);
                        }
                        tc::mma_commit_ws(&empty[stage]);
                        adv();
                        continue;
                    }
                    if (p.halo) {
                        // tap c of this kernel row = the A tile viewed c pixel-rows further on (SW128 is
                        // address-based, probed); 8-pixel M groups are Wp rows apart (SBO = Wp * 128 B).
                        // Descriptors are linear in the start address: per-MMA descriptors are base + constant.
                        const uint64_t a0 = tc::smem_desc(a_base, 16, (uint32_t)p.Wp * 128u, 2);
                        const uint64_t b0 = p.bres ? tc::smem_desc(tc::smem_u32(sW) + (uint32_t)(ks * p.kw * p.BN) * 128u, 16, 1024, 2)
                                                   : tc::smem_desc(b_base, 16, 1024, 2);
                        const uint32_t bstep = (uint32_t)p.BN * 8u;   // BN*128 B >> 4
                        for (int c = 0; c < p.kw; ++c)
                            tc::mma_k_x4_ws<TF32>(d, a0 + (uint64_t)(8 * c), b0 + (uint64_t)(bstep * c), idesc, (ks | c) != 0);
                        tc::mma_commit_ws(&empty[stage]);
                        adv();
                        continue;
                    }
                    const uint64_t a0 = tc::smem_desc(a_base, p.a_lbo, p.a_sbo, p.a_layout);
                    const uint64_t b0 = tc::smem_desc(b_base, 16, 1024, 2);
#pragma unroll
                    for (int j = 0; j < 4; ++j)
                        tc::mma_k_ws<TF32>(d, a0 + (uint64_t)g_aoff[j], b0 + (uint64_t)(2 * j), idesc, (ks | j) != 0);
                    tc::mma_commit_ws(&empty[stage]);
                    adv();
                }
                if (CTA2) tc::mma2_commit_mc_ws(&tfull[slot]);
                else tc::mma_commit_ws(&tfull[slot]);
            }
        };
        if (warp == 1) mma_run(std::integral_constant<int, 0>{});
        else mma_run(std::integral_constant<int, 1>{});
    } else if (warp == 10) {
        // second MMA warp without dual issue: idle
    } else if (!p.direct && p.egroups == 2) {
        // ================= epilogue, two groups: warps 2..5 take even tiles (accumulator 0, staging 0),
        // warps 6..9 odd tiles (accumulator 1, staging 1), so consecutive tiles' epilogues overlap
        const int quad = warp & 3;
        const int g = (warp - 2) >> 2;
        const int row = quad * 32 + lane;
        const int gtid = threadIdx.x - 64 - 128 * g;   // 0..127 within the group
        const uint32_t rowB = (uint32_t)p.ychunk * 2u;
        const uint32_t chunk_bytes = 128u * rowB;
        // ReLU-mask / residual tiles (dgrad mask, fused join) through the staging ring: ring slot s has its own
        // barrier, and the tile that will use slot s is loaded as soon as the TMA store that last read slot s
        // is done -- yring - 1 group tiles ahead, so the load latency hides behind that many tiles' MMAs
        // (one tile ahead left the short-K 64-channel layers waiting on every mask: conv1_2 dgrad)
        uint64_t *mbarR = reinterpret_cast<uint64_t *>(smem + p.bar_off + 256) + 4 * g;
        uint32_t mph = 0;   // phase bit per ring slot
        const bool mpre = MASK && p.yring >= 2;
        auto mask_load = [&](int tt, int slot) {   // gtid 0
            int ql, nb, hb, wb, cb;
            bool valid;
            get_tile(p, tt, rank, ql, nb, hb, wb, cb, valid);
            if (!valid) return;
            const int co0 = cb * p.BN, nch = min(p.BN, p.Cpo - co0) >> p.ysh;
            uint8_t *buf = sY + (size_t)(g * p.yring + slot) * p.ybuf_bytes;
            tc::mbar_arrive_expect_tx(&mbarR[slot], (uint32_t)nch * p.rows_box * rowB);
            for (int c = 0; c < nch; ++c)
                tc::tma_load_4d(buf + c * chunk_bytes, &p.mapR[ql], &mbarR[slot], co0 + c * p.ychunk, wb * p.BW, hb * p.BH,
                                nb * p.BNn);
        };
        if (mpre && gtid == 0)
            for (int j = 0; j < p.yring - 1; ++j) {
                const int tt = tfirst + (g + 2 * j) * tstep;
                if (tt < total) mask_load(tt, j);
            }
        uint64_t *mbar = g ? wbar + 1 : ybar;   // mask without the ring (yring == 1): loaded per tile
        uint32_t yph = 0;
        int it = g, k = 0, ys = 0;   // ys = k % yring (no runtime modulo per tile)
        for (int t = tfirst + g * tstep; t < total; t += 2 * tstep, it += 2, ++k, ys = (ys + 1 == p.yring) ? 0 : ys + 1) {
            const int slot = g * p.nacc_g + (p.nacc_g == 2 ? (k & 1) : 0);
            const uint32_t aph = (uint32_t)((p.nacc_g == 2 ? (k >> 1) : k) & 1);
            const uint32_t tempty_l = tc::mapa_shared(&tempty[slot], 0);   // the leader's (own in 1-CTA mode)
            // staging ring: tile k of this group fills buffer k % yring
            uint8_t *sYb = sY + (size_t)(g * p.yring + ys) * p.ybuf_bytes;
            int ql, nb, hb, wb, cb;
            bool valid;
            get_tile(p, t, rank, ql, nb, hb, wb, cb, valid);
            const int co0 = cb * p.BN;
            const int ow0 = wb * p.BW, oh0 = hb * p.BH, n0 = nb * p.BNn;
            const int ncols = min(p.BN, p.Cpo - co0);
            const int nchunks = ncols >> p.ysh;
            if (POOL) {
                // pooled outputs straight from registers: no staging tile, no store of the conv output
                tc::mbar_wait(&tfull[slot], aph);
                tc::tc_fence_after();
                const uint32_t tacc = tmem_base + (uint32_t)(slot * p.BN) + ((uint32_t)(quad * 32) << 16);
                const int wi = row & (p.BW - 1), hi = (row / p.BW) % p.BH, ni = row / (p.BW * p.BH);
                const int n = n0 + ni, ph = (oh0 + hi) >> 1, pw = (ow0 + wi) >> 1;
                const int poh = p.out_h[ql] >> 1, pow_ = p.out_w[ql] >> 1;
                const bool writer = valid && !(wi & 1) && !(hi & 1) && row < p.rows_box && n < p.N && ph < poh && pw < pow_;
                const int64_t pix = p.pool_off[ql] + (((int64_t)n * poh + ph) * pow_ + pw) * p.Cpo + co0;
                for (int cc = 0; cc < ncols; cc += 32) {   // ncols % 16 == 0; two loads in flight
                    uint32_t r2[2][16];
                    tc::tmem_ld16_nw(tacc + cc, r2[0]);
                    if (cc + 16 < ncols) tc::tmem_ld16_nw(tacc + cc + 16, r2[1]);
                    tc::tmem_wait_ld();
                    if (cc + 32 <= ncols) {   // 32 columns: bias/ReLU/round as the stored-conv epilogue, pool packed
                        uint4 pk[4];
#pragma unroll
                        for (int u = 0; u < 4; ++u)
                            pk[u] = epi8_full<BIAS, RELU, false>(r2[u >> 1] + 8 * (u & 1), sbias + co0 + cc + 8 * u,
                                                                 make_uint4(0, 0, 0, 0));
                        pool32(reinterpret_cast<const uint32_t *>(pk), p.BW, writer, p.pool_y + pix + cc, p.pool_a + pix + cc);
                        continue;
                    }
#pragma unroll
                    for (int hh = 0; hh < 2; ++hh) {
                        if (cc + 16 * hh >= ncols) break;
                        float v[16];
#pragma unroll
                        for (int e = 0; e < 16; ++e) {
                            float o = __uint_as_float(r2[hh][e]);
                            if (BIAS) o += sbias[co0 + cc + 16 * hh + e];
                            if (RELU) o = fmaxf(o, 0.f);
                            v[e] = o;
                        }
                        pool16(v, p.BW, writer, p.pool_y + pix + cc + 16 * hh, p.pool_a + pix + cc + 16 * hh);
                    }
                }
                tc::tc_fence_before();
                __syncwarp();
                if (lane == 0) {
                    if (CTA2) tc::mbar_arrive_remote(tempty_l);
                    else tc::mbar_arrive(&tempty[slot]);
                }
                continue;
            }
            if (gtid == 0) {   // the store that last used this staging buffer (yring - 1 stores back) has read it
                if (p.yring == 1) tc::bulk_wait_read0();
                else if (p.yring == 2) tc::bulk_wait_read1();
                else if (p.yring == 3) tc::bulk_wait_read2();
                else tc::bulk_wait_read3();
            }
            tc::named_bar_sync(1 + g, 128);
            if (mpre && valid) {
                tc::mbar_wait(&mbarR[ys], (mph >> ys) & 1u);
                mph ^= 1u << ys;
            } else if (MASK && valid) {
                if (gtid == 0) {
                    tc::mbar_arrive_expect_tx(mbar, (uint32_t)nchunks * p.rows_box * rowB);
                    for (int c = 0; c < nchunks; ++c)
                        tc::tma_load_4d(sYb + c * chunk_bytes, &p.mapR[ql], mbar, co0 + c * p.ychunk, ow0, oh0, n0);
                }
                tc::mbar_wait(mbar, yph);
                yph ^= 1;
            }
            tc::mbar_wait(&tfull[slot], aph);
            tc::tc_fence_after();
            const uint32_t tacc = tmem_base + (uint32_t)(slot * p.BN) + ((uint32_t)(quad * 32) << 16);
            // fast path: whole 32-column groups of real channels inside one staging chunk (ychunk >= 32)
            const bool fast = (ncols & 31) == 0 && co0 + ncols <= p.Cout && p.ychunk >= 32;
            if (fast) {
                const uint32_t rbase = (uint32_t)row * rowB;
                const uint32_t rsw = ((rbase >> 7) & p.y_mask) << 4;
                for (int cc = 0; cc < ncols; cc += 32) {
                    uint32_t r2[2][16];
                    tc::tmem_ld16_nw(tacc + cc, r2[0]);
                    tc::tmem_ld16_nw(tacc + cc + 16, r2[1]);
                    tc::tmem_wait_ld();
                    uint8_t *cbase = sYb + (cc >> p.ysh) * chunk_bytes + rbase;
                    const uint32_t cb0 = (uint32_t)(cc & (p.ychunk - 1)) * 2u;
#pragma unroll
                    for (int u = 0; u < 4; ++u) {
                        uint4 *dst = reinterpret_cast<uint4 *>(cbase + ((cb0 + 16u * u) ^ rsw));
                        const uint4 m4 = MASK ? *dst : make_uint4(0, 0, 0, 0);
                        *dst = epi8_full<BIAS, RELU, MASK>(r2[u >> 1] + 8 * (u & 1), sbias + co0 + cc + 8 * u, m4, p.res);
                    }
                }
            }
            for (int cc = 0; cc < (fast ? 0 : ncols); cc += 32) {
                uint32_t r[2][16];
                tc::tmem_ld16_nw(tacc + cc, r[0]);
                if (cc + 16 < ncols) tc::tmem_ld16_nw(tacc + cc + 16, r[1]);
                tc::tmem_wait_ld();
#pragma unroll
                for (int u = 0; u < 4; ++u) {
                    const int c8 = cc + 8 * u;
                    if (c8 >= ncols) break;
                    const int k = c8 >> p.ysh;
                    const uint32_t off = tc::swz((uint32_t)row * rowB + (uint32_t)(c8 & (p.ychunk - 1)) * 2u, p.y_mask);
                    uint4 *dst = reinterpret_cast<uint4 *>(sYb + k * chunk_bytes + off);
                    const uint4 m4 = MASK ? *dst : make_uint4(0, 0, 0, 0);
                    *dst = epi8<BIAS, RELU, MASK>(r[u >> 1] + 8 * (u & 1), sbias, co0 + c8, p.Cout, m4, p.res);
                }
            }
            tc::tc_fence_before();
            __syncwarp();
            if (lane == 0) {
                if (CTA2) tc::mbar_arrive_remote(tempty_l);
                else tc::mbar_arrive(&tempty[slot]);
            }
            tc::fence_proxy_async_smem();
            tc::named_bar_sync(1 + g, 128);
            if (gtid == 0) {   // an empty group keeps the ring's wait counts aligned
                if (valid)
                    for (int c = 0; c < nchunks; ++c)
                        tc::tma_store_4d(&p.mapY[ql], sYb + c * chunk_bytes, co0 + c * p.ychunk, ow0, oh0, n0);
                tc::bulk_commit();
                if (mpre) {
                    // tile k + yring - 1 of this group takes the slot of tile k - 1, whose store has read it once
                    // at most the latest bulk group (this tile's store) is still reading
                    const int tt = t + 2 * tstep * (p.yring - 1);
                    if (tt < total) {
                        tc::bulk_wait_read1();
                        mask_load(tt, ys == 0 ? p.yring - 1 : ys - 1);
                    }
                }
            }
        }
        if (gtid == 0) tc::bulk_wait0();
    } else if (!p.direct) {
        // ================= epilogue: warps 2..9, TMEM lane quadrant = warp % 4, column half = (warp-2)/4;
        // accumulator -> fused bias/ReLU/mask -> bf16 -> swizzled smem staging tile -> TMA store
        const int quad = warp & 3;
        const int half = (warp - 2) >> 2;
        const int row = quad * 32 + lane;      // TMEM lane = tile row = staging row
        const int etid = threadIdx.x - 64;     // 0..255
        const uint32_t rowB = (uint32_t)p.ychunk * 2u;
        const uint32_t chunk_bytes = 128u * rowB;
        int acc = 0, yb = 0;
        uint32_t aph = 0, yph = 0;
        for (int t = tfirst; t < total; t += tstep) {
            int ql, nb, hb, wb, cb;
            bool valid;
            get_tile(p, t, rank, ql, nb, hb, wb, cb, valid);
            const int co0 = cb * p.BN;
            const int ow0 = wb * p.BW, oh0 = hb * p.BH, n0 = nb * p.BNn;
            const int ncols = min(p.BN, p.Cpo - co0);       // channels this tile stores (multiple of ychunk)
            const int nchunks = ncols / p.ychunk;
            uint8_t *sYb = sY + (size_t)yb * p.ybuf_bytes;
            if (POOL) {   // fused max-pool: 16-column groups interleaved between the two column halves
                tc::mbar_wait(&tfull[acc], aph);
                tc::tc_fence_after();
                const uint32_t tacc = tmem_base + (uint32_t)(acc * p.BN) + ((uint32_t)(quad * 32) << 16);
                const int wi = row & (p.BW - 1), hi = (row / p.BW) % p.BH, ni = row / (p.BW * p.BH);
                const int n = n0 + ni, ph = (oh0 + hi) >> 1, pw = (ow0 + wi) >> 1;
                const int poh = p.out_h[ql] >> 1, pow_ = p.out_w[ql] >> 1;
                const bool writer = valid && !(wi & 1) && !(hi & 1) && row < p.rows_box && n < p.N && ph < poh && pw < pow_;
                const int64_t pix = p.pool_off[ql] + (((int64_t)n * poh + ph) * pow_ + pw) * p.Cpo + co0;
                for (int cc = 16 * half; cc < ncols; cc += 32) {
                    float v[16];
                    tc::tmem_ld16(tacc + cc, v);
#pragma unroll
                    for (int e = 0; e < 16; ++e) {
                        float o = v[e];
                        if (BIAS) o += sbias[co0 + cc + e];
                        if (RELU) o = fmaxf(o, 0.f);
                        v[e] = o;
                    }
                    pool16(v, p.BW, writer, p.pool_y + pix + cc, p.pool_a + pix + cc);
                }
                tc::tc_fence_before();
                __syncwarp();
                if (lane == 0) {
                    if (CTA2) tc::mbar_arrive_remote(tc::mapa_shared(&tempty[acc], 0));
                    else tc::mbar_arrive(&tempty[acc]);
                }
                acc ^= 1;
                if (acc == 0) aph ^= 1;
                continue;
            }
            // this staging buffer is free once the TMA store that last used it has read it
            if (etid == 0) {
                if (p.ybufs == 2) tc::bulk_wait_read1();
                else tc::bulk_wait_read0();
            }
            tc::named_bar_sync(1, 256);
            if (MASK && valid) {  // ReLU-mask tile (same box as the output) into the staging tile
                if (etid == 0) {
                    tc::mbar_arrive_expect_tx(ybar, (uint32_t)nchunks * p.rows_box * rowB);
                    for (int k = 0; k < nchunks; ++k)
                        tc::tma_load_4d(sYb + k * chunk_bytes, &p.mapR[ql], ybar, co0 + k * p.ychunk, ow0, oh0, n0);
                }
                tc::mbar_wait(ybar, yph);
                yph ^= 1;
            }
            tc::mbar_wait(&tfull[acc], aph);
            tc::tc_fence_after();
            const uint32_t tacc = tmem_base + (uint32_t)(acc * p.BN) + ((uint32_t)(quad * 32) << 16);
            // 16-column groups interleaved between the two column halves
            for (int cc = 16 * half; cc < ncols; cc += 32) {
                uint32_t r[16];
                tc::tmem_ld16_nw(tacc + cc, r);
                tc::tmem_wait_ld();
#pragma unroll
                for (int u = 0; u < 2; ++u) {
                    const int c8 = cc + 8 * u;
                    if (c8 >= ncols) break;
                    const int k = c8 >> p.ysh;
                    const uint32_t off = tc::swz((uint32_t)row * rowB + (uint32_t)(c8 & (p.ychunk - 1)) * 2u, p.y_mask);
                    uint4 *dst = reinterpret_cast<uint4 *>(sYb + k * chunk_bytes + off);
                    const uint4 m4 = MASK ? *dst : make_uint4(0, 0, 0, 0);
                    *dst = epi8<BIAS, RELU, MASK>(r + 8 * u, sbias, co0 + c8, p.Cout, m4, p.res);
                }
            }
            tc::tc_fence_before();
            __syncwarp();
            if (lane == 0) {   // accumulator free: the MMA may proceed (the leader's barrier in 2-CTA mode)
                if (CTA2) tc::mbar_arrive_remote(tc::mapa_shared(&tempty[acc], 0));
                else tc::mbar_arrive(&tempty[acc]);
            }
            tc::fence_proxy_async_smem();
            tc::named_bar_sync(1, 256);
            if (etid == 0 && valid) {
                for (int k = 0; k < nchunks; ++k)
                    tc::tma_store_4d(&p.mapY[ql], sYb + k * chunk_bytes, co0 + k * p.ychunk, ow0, oh0, n0);
                tc::bulk_commit();
            }
            acc ^= 1;
            if (acc == 0) aph ^= 1;
            if (p.ybufs == 2) yb ^= 1;
        }
        if (etid == 0) tc::bulk_wait0();
    } else {
        // ================= epilogue, direct per-thread stores (channel pads without a TMA box fit);
        // warps 6..9 only keep the tempty arrival count
        const int quad = warp & 3;
        const int row = quad * 32 + lane;
        if (warp >= 6) {
            int acc = 0;
            uint32_t aph = 0;
            for (int t = blockIdx.x; t < total; t += gridDim.x) {
                tc::mbar_wait(&tfull[acc], aph);
                __syncwarp();
                if (lane == 0) tc::mbar_arrive(&tempty[acc]);
                acc ^= 1;
                if (acc == 0) aph ^= 1;
            }
        } else {
        const int wi = row % p.BW, hi = (row / p.BW) % p.BH, ni = row / (p.BW * p.BH);
        int acc = 0;
        uint32_t aph = 0;
        for (int t = blockIdx.x; t < total; t += gridDim.x) {
            int ql, nb, hb, wb, cb;
            decode_tile(p, t, ql, nb, hb, wb, cb);
            const int n = nb * p.BNn + ni, oh = hb * p.BH + hi, ow = wb * p.BW + wi;
            const bool valid = row < p.rows_box && n < p.N && oh < p.out_h[ql] && ow < p.out_w[ql];
            const int64_t base = p.out_off[ql] + (((int64_t)n * p.out_h[ql] + oh) * p.out_w[ql] + ow) * p.Cpo;
            const int co0 = cb * p.BN;
            tc::mbar_wait(&tfull[acc], aph);
            tc::tc_fence_after();
            const uint32_t tacc = tmem_base + (uint32_t)(acc * p.BN) + ((uint32_t)(quad * 32) << 16);
            using OT = typename std::conditional<TF32, float, __nv_bfloat16>::type;
            OT *yo = reinterpret_cast<OT *>(p.y);
            const OT *ro = reinterpret_cast<const OT *>(p.relu_src);
            for (int cc = 0; cc < p.BN; cc += 16) {
                float v[16];
                tc::tmem_ld16(tacc + cc, v);
                if (!valid) continue;
#pragma unroll
                for (int g = 0; g < 2; ++g) {
                    const int co = co0 + cc + 8 * g;
                    if (co >= p.Cpo) break;
                    float o[8], yold[8] = {0, 0, 0, 0, 0, 0, 0, 0};
                    if (TF32 && p.accum) {
                        const float *yf = reinterpret_cast<const float *>(yo) + base + co;
                        const float4 a = *reinterpret_cast<const float4 *>(yf);
                        yold[0] = a.x; yold[1] = a.y; yold[2] = a.z; yold[3] = a.w;
                        if (co + 8 <= p.Cpo) {
                            const float4 b = *reinterpret_cast<const float4 *>(yf + 4);
                            yold[4] = b.x; yold[5] = b.y; yold[6] = b.z; yold[7] = b.w;
                        }
                    }
#pragma unroll
                    for (int e = 0; e < 8; ++e) {
                        float x = v[8 * g + e] + yold[e];
                        if (co + e < p.Cout) {
                            if (p.bias) x += __ldg(p.bias + co + e);
                            if (p.relu) x = fmaxf(x, 0.f);
                        } else {
                            x = 0.f;
                        }
                        o[e] = x;
                    }
                    if (TF32 && co + 8 > p.Cpo) {   // fp32 levels pad channels to 4: a 4-channel tail group
                        float *yf = reinterpret_cast<float *>(yo) + base + co;
                        float4 r = make_float4(o[0], o[1], o[2], o[3]);
                        if (ro) {
                            const float4 m = *reinterpret_cast<const float4 *>(reinterpret_cast<const float *>(ro) + base + co);
                            r.x = m.x > 0.f ? r.x : 0.f; r.y = m.y > 0.f ? r.y : 0.f;
                            r.z = m.z > 0.f ? r.z : 0.f; r.w = m.w > 0.f ? r.w : 0.f;
                        }
                        *reinterpret_cast<float4 *>(yf) = r;
                        continue;
                    }
                    if (ro) {
                        float m[8];
                        load8(ro + base + co, m);
#pragma unroll
                        for (int e = 0; e < 8; ++e) o[e] = (m[e] > 0.f) ? o[e] : 0.f;
                    }
                    store8(yo + base + co, o);
                }
            }
            tc::tc_fence_before();
            __syncwarp();
            if (lane == 0) tc::mbar_arrive(&tempty[acc]);
            acc ^= 1;
            if (acc == 0) aph ^= 1;
        }
        }
    }
    tc::tc_fence_before();
    if (CTA2) tc::cluster_sync_all();   // the peer's MMAs write this CTA's TMEM until the leader is done
    else __syncthreads();
    tc::tc_fence_after();
    if (warp == 1) {
        if (CTA2) tc::tmem_dealloc2(tmem_base, p.tmem_cols);
        else tc::tmem_dealloc(tmem_base, p.tmem_cols);
    }
}

// dgrad weights: W'[ci][r'][c'][co] = W[co][kh-1-r'][kw-1-c'][ci], zero for co >= Cout
template <typename T>
__global__ void flip_weights_kernel(const T *__restrict__ W, T *__restrict__ Wt, int Cout,
                                    int Cpad_in, int Cin, int kh, int kw, int Cpad_out, int r0h, int r0w, int step,
                                    int nth, int ntw) {
    // Wt[ci][j][l][co] = W[co][r0h + step*(nth-1-j)][r0w + step*(ntw-1-l)][ci]   (stride-1 dgrad: r0 = 0,
    // step = 1, nt = k -- the 180-degree flip; stride-s phase (rho_h, rho_w): the taps r = r0 (mod s)).
    // One thread per (8-channel ci group, tap, co), co fastest across lanes: it reads the 8 contiguous ci of
    // W[co][rr][cc][ci0..+8) (one 16 / 32-byte load) and writes them down 8 Wt rows, each store coalesced
    // across the warp's consecutive co.  No shared memory: the kernel overlaps whatever else runs.
    const int ntap = nth * ntw, ng = (Cin + 7) / 8;
    const int64_t n = (int64_t)ng * ntap * Cpad_out;
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        const int co = (int)(i % Cpad_out);
        const int64_t t = i / Cpad_out;
        const int tap = (int)(t % ntap), cg = (int)(t / ntap);
        const int j = tap / ntw, l = tap - j * ntw;
        const int rr = r0h + step * (nth - 1 - j), cc = r0w + step * (ntw - 1 - l);
        const int ci0 = cg * 8;
        T v[8];
#pragma unroll
        for (int e = 0; e < 8; ++e) v[e] = from_f<T>(0.f);
        if (co < Cout) {
            const T *src = W + (((int64_t)co * kh + rr) * kw + cc) * Cpad_in + ci0;
            if (ci0 + 8 <= Cpad_in) {   // Cpad_in % 8 == 0 and 16-byte aligned rows: vector loads
                if (sizeof(T) == 2) {
                    *reinterpret_cast<uint4 *>(v) = __ldg(reinterpret_cast<const uint4 *>(src));
                } else {
                    reinterpret_cast<float4 *>(v)[0] = __ldg(reinterpret_cast<const float4 *>(src));
                    reinterpret_cast<float4 *>(v)[1] = __ldg(reinterpret_cast<const float4 *>(src) + 1);
                }
            } else {
#pragma unroll
                for (int e = 0; e < 8; ++e)
                    if (ci0 + e < Cpad_in) v[e] = src[e];
            }
        }
        T *dst = Wt + (((int64_t)ci0 * nth + j) * ntw + l) * Cpad_out + co;
        const int64_t rs = (int64_t)nth * ntw * Cpad_out;   // Wt row stride (one ci)
#pragma unroll
        for (int e = 0; e < 8; ++e)
            if (ci0 + e < Cin) dst[e * rs] = v[e];
    }
}

// Stride-s dgrad, zero phases: dX elements of phase (rh, rw) that no tap reaches (k < s) are zero.
__global__ void zero_phase_kernel(__nv_bfloat16 *__restrict__ dx, LevelDesc L, int S, int rh, int rw, int p0) {
    const PatchGeo g = patch_geo(L, p0 + blockIdx.y);
    const int hq = (g.hp - rh + S - 1) / S, wq = (g.wp - rw + S - 1) / S, G = L.Cpad / 8;
    const int64_t units = (int64_t)L.N * hq * wq * G;
    for (int64_t u = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; u < units; u += (int64_t)gridDim.x * blockDim.x) {
        const int cg = (int)(u % G);
        int64_t t = u / G;
        const int w = (int)(t % wq);
        t /= wq;
        const int h = (int)(t % hq);
        const int n = (int)(t / hq);
        *reinterpret_cast<uint4 *>(dx + g.off + (((int64_t)n * g.hp + h * S + rh) * g.wp + w * S + rw) * L.Cpad + cg * 8) =
            make_uint4(0, 0, 0, 0);
    }
}

// ============================================================ host side
namespace {

PFN_cuTensorMapEncodeTiled_v12000 get_encode() {
    static PFN_cuTensorMapEncodeTiled_v12000 fn = nullptr;
    static std::once_flag once;
    std::call_once(once, [] {
        cudaDriverEntryPointQueryResult q;
        void *p = nullptr;
        if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) == cudaSuccess &&
            q == cudaDriverEntryPointSuccess)
            fn = (PFN_cuTensorMapEncodeTiled_v12000)p;
    });
    return fn;
}

// Tensor-map cache: every conv call builds one map per patch (A, output, mask) plus the weights' map -- ~9k
// cuTensorMapEncodeTiled calls per C5 step, all repeating from step to step (same buffers, same plan).  A
// map is a pure function of its encode arguments, so they are the key (per host thread; cleared when large).
CUresult encode_cached(CUtensorMap *m, CUtensorMapDataType dt, cuuint32_t rank, void *addr, const cuuint64_t *dims,
                       const cuuint64_t *strides, const cuuint32_t *box, const cuuint32_t *es, CUtensorMapInterleave il,
                       CUtensorMapSwizzle sw, CUtensorMapL2promotion l2, CUtensorMapFloatOOBfill oob) {
    static thread_local std::unordered_map<std::string, CUtensorMap> cache;
    uint64_t k[32];
    int n = 0;
    k[n++] = ((uint64_t)dt << 32) | rank;
    k[n++] = (uint64_t)(uintptr_t)addr;
    k[n++] = ((uint64_t)il << 48) | ((uint64_t)sw << 32) | ((uint64_t)l2 << 16) | (uint64_t)oob;
    for (cuuint32_t i = 0; i < rank; ++i) k[n++] = dims[i];
    for (cuuint32_t i = 0; i + 1 < rank; ++i) k[n++] = strides[i];
    for (cuuint32_t i = 0; i < rank; ++i) k[n++] = ((uint64_t)box[i] << 32) | es[i];
    std::string key(reinterpret_cast<const char *>(k), n * sizeof(uint64_t));
    auto it = cache.find(key);
    if (it != cache.end()) {
        *m = it->second;
        return CUDA_SUCCESS;
    }
    const CUresult r = get_encode()(m, dt, rank, addr, dims, strides, box, es, il, sw, l2, oob);
    if (r == CUDA_SUCCESS) {
        if (cache.size() >= 8192) cache.clear();
        cache.emplace(std::move(key), *m);
    }
    return r;
}

int num_sms() {
    static int n = 0;
    if (!n) {
        int dev = 0;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev);
        if (n <= 0) n = 148;
    }
    return n;
}

CUtensorMapSwizzle swz_for(int row_bytes) {
    switch (row_bytes) {
        case 128: return CU_TENSOR_MAP_SWIZZLE_128B;
        case 64: return CU_TENSOR_MAP_SWIZZLE_64B;
        case 32: return CU_TENSOR_MAP_SWIZZLE_32B;
        default: return CU_TENSOR_MAP_SWIZZLE_NONE;
    }
}
uint32_t layout_for(int row_bytes) {  // tcgen05 descriptor layout code
    switch (row_bytes) {
        case 128: return 2;
        case 64: return 4;
        case 32: return 6;
        default: return 0;
    }
}

struct TileShape {
    int BW, BH, BNn;
};

// choose the pixel box (BW x BH x BNn <= 128 rows) minimising the number of tiles over the patches
TileShape choose_tile(const std::vector<std::pair<int, int>> &ext, int N, int s, int bw_max = 128) {
    int maxh = 1, maxw = 1;
    for (auto &e : ext) { maxh = std::max(maxh, e.first); maxw = std::max(maxw, e.second); }
    TileShape best{1, 1, 1};
    long best_tiles = -1;
    const int wlim = std::min(std::min(std::min(maxw, 128), 256 / s), bw_max), hlim = std::min(std::min(maxh, 128), 256 / s);
    for (int bw = 1; bw <= wlim; ++bw) {
        for (int bh = 1; bh <= hlim && bw * bh <= 128; ++bh) {
            const int bn = std::min(std::min(128 / (bw * bh), N), 256);
            long tiles = 0;
            for (auto &e : ext)
                tiles += (long)((N + bn - 1) / bn) * ((e.first + bh - 1) / bh) * ((e.second + bw - 1) / bw);
            if (best_tiles < 0 || tiles < best_tiles || (tiles == best_tiles && bw > best.BW)) {
                best_tiles = tiles;
                best = {bw, bh, bn};
            }
        }
    }
    return best;
}

// tile shape for the fused-pool forward: BW a power of two <= 16 (window partners m^1, m^BW inside a
// warp) and BH even (tiles start at even rows: no 2x2 window straddles a tile)
TileShape choose_tile_pool(const std::vector<std::pair<int, int>> &ext, int N) {
    TileShape best{2, 2, 1};
    long best_tiles = -1;
    for (int bw = 2; bw <= 16; bw *= 2)
        for (int bh = 2; bw * bh <= 128; bh += 2) {
            const int bn = std::min(128 / (bw * bh), N);
            long tiles = 0;
            for (auto &e : ext) tiles += (long)((N + bn - 1) / bn) * ((e.first + bh - 1) / bh) * ((e.second + bw - 1) / bw);
            if (best_tiles < 0 || tiles < best_tiles || (tiles == best_tiles && bw > best.BW)) {
                best_tiles = tiles;
                best = {bw, bh, bn};
            }
        }
    return best;
}

int round_up16(int x) { return (x + 15) / 16 * 16; }

// stages + resident weights + staging ring of the conv kernel (of the 227 KB opt-in shared memory; 220 KB
// -- a 3-deep mask ring for the 64-channel dgrad -- measured no faster there and 5 % slower on the fused
// conv1_2 + pool forward, profiles/r2i/ab_epilogue.txt)
constexpr uint32_t CONV_SMEM_BUDGET = 210u * 1024u;



bool a_channels_ok(int cpad) { return cpad == 8 || cpad == 16 || cpad == 32 || cpad % 64 == 0; }

// mode 0: forward (A = X at level m, out = level m+1); mode 1: dgrad (A = dY at level m+1, out = level m)
// fused max-pool target of the forward pass (level layer+2 values + argmax bytes), or none
// Stride-S data gradient by output phase: dX[S*t + rho] = sum over the taps r = r0 (mod S) -- a
// stride-1 correlation of dY with the (kh' x kw') sub-filter, written through a tensor map that
// views the dX patch at element stride S from (rho_h, rho_w).
struct Phase {
    int S, rh, rw, kh, kw, pt, pl;
};

struct PoolFuse {
    void *y = nullptr;
    uint8_t *a = nullptr;
    const Level *Lp = nullptr;
};

// prec 0: bf16 operands and outputs; 1: TF32 -- fp32 operands through kind::tf32 (the byte layout of an fp32
// level is that of a bf16 level with twice the channels), fp32 outputs by the direct epilogue; accum: add
// into y (TF32 only)
splitcnn_status_t launch_tc(int mode, const Level &La, const Level &Lout, const LayerGeom &g, const void *a_ptr,
                            const void *w_ptr, int w_rows, const float *bias, void *y, const void *relu_src, int relu,
                            int p0, int p1, cudaStream_t st, const PoolFuse *pool = nullptr, const Phase *ph = nullptr,
                            int prec = 0, int accum = 0, int res = 0) {
    const bool tf32 = prec == 1;
    const int es = tf32 ? 4 : 2;          // bytes per element of the operand / output levels
    if (!get_encode()) return fail(SPLITCNN_ERR_CUDA, "cuTensorMapEncodeTiled unavailable");
    auto encode = encode_cached;
    const int kh = ph ? ph->kh : g.L.kh, kw = ph ? ph->kw : g.L.kw, s = mode == 0 ? g.L.sh : 1;
    const int PS = ph ? ph->S : 1, prh = ph ? ph->rh : 0, prw = ph ? ph->rw : 0;
    auto out_ext_h = [&](int i) { return (Lout.ph(i) - prh + PS - 1) / PS; };
    auto out_ext_w = [&](int j) { return (Lout.pw(j) - prw + PS - 1) / PS; };
    const int cpad = La.Cpad * es / 2;    // channels of the byte layout in 2-byte units
    const int cpadc = std::min(cpad, 64);
    const int ncols_out = mode == 0 ? g.L.cout : g.L.cin;
    // N tile: up to 256 output channels; small layers (few 128-pixel M tiles, e.g. 2x2 / 4x4 CIFAR tails)
    // take narrower N tiles so that M tiles x N tiles still covers the SMs
    int BN0 = std::min(256, round_up16(ncols_out));
    {
        long mt = 0;
        for (int q = p0; q < p1; ++q) {
            const int i = q / Lout.nw(), j = q % Lout.nw();
            mt += ((long)La.N * out_ext_h(i) * out_ext_w(j) + 127) / 128;
        }
        while (BN0 > 64 && BN0 % 32 == 0 && mt * ((ncols_out + BN0 - 1) / BN0) < num_sms())
            BN0 /= 2;
    }
    const int nco0 = (ncols_out + BN0 - 1) / BN0;
    const int N = La.N;
    for (int g0 = p0; g0 < p1; g0 += TC_MAXP) {
        const int g1 = std::min(p1, g0 + TC_MAXP);
        int BN = BN0, nco = nco0;   // this launch's N tile (see the wave rule below)
        std::vector<std::pair<int, int>> ext;
        for (int q = g0; q < g1; ++q) {
            const int i = q / Lout.nw(), j = q % Lout.nw();
            ext.push_back({out_ext_h(i), out_ext_w(j)});
        }
        const int a3d = (cpad == 8 && s == 1) ? 1 : 0;  // TMA rows of 16 B are slow: merge 8 pixels per row
        // halo mode for narrow outputs (per-tap TMA boxes cannot keep the MMA fed there)
        // (BN = 256 too: the A box of a kernel row then serves kw taps, -29% of the L2->SM traffic that
        // bounds these layers; same-process A/B: conv3_2 fwd 0.94 -> 0.73 ms, conv4_2 0.88 -> 0.70 ms)
        // (also for 4- and 2-wide patches, whose 8-pixel M groups are half / a quarter full: the per-tap
        // boxes pack whole images but move 3x the operand bytes, and these small layers are bound by the
        // L2 -> SM operand traffic -- C2 1.18 -> 1.30 ms with per-tap boxes there, scripts/ab_halo_narrow.sh)
        const int hn = (s == 1 && !tf32 && (cpad == 16 || cpad == 32) && kw >= 2 && kw * cpad <= 64 && mode != 2) ? 1 : 0;
        const int halo = ((s == 1 && cpad % 64 == 0 && BN <= 256 && kw >= 2 && kw <= 4) || hn) ? 1 : 0;
        const uint32_t rowb = (uint32_t)std::min(cpad, 64) * 2u;                 // bytes per A pixel row
        const uint32_t wboxes = hn ? (uint32_t)kh : (uint32_t)(cpad / 64) * kh * kw;   // BN x 128 B weight boxes
        const int halo8 = (mode == 0 && cpad == 8 && s == 1 && kw <= 8 && kh * kw <= 16) ? 1 : 0;
        TileShape ts = pool ? choose_tile_pool(ext, N) : choose_tile(ext, N, s, a3d ? 32 : 128);
        if (halo8) {  // 8 output columns x BH output rows, one image per tile
            long best = -1;
            for (int bh = 1; bh <= 16; ++bh) {
                long t = 0;
                for (auto &e : ext) t += (long)N * ((e.first + bh - 1) / bh) * ((e.second + 7) / 8);
                if (best < 0 || t < best) { best = t; ts = {8, bh, 1}; }
            }
        } else if (halo) {  // 8 output columns per M group; BH x BNn groups (<= 16)
            long best = -1;
            TileShape hs = ts;
            // tall boxes (one A box for all kernel rows, P.tall) hold one image per tile: with resident weights
            // (one N tile), i.e. the narrow-N layers whose shared-memory traffic the per-row boxes dominate
            // (predicted here as the weights-resident condition below with the largest tall box, BH = 16)
            const uint32_t wres = wboxes * (uint32_t)(BN % 32 == 0 && !hn ? BN / 2 : BN) * 128u;
            const uint32_t tall_max = ((uint32_t)(8 + kw - 1) * (16 + kh - 1) * rowb + 1023u) & ~1023u;
            const bool tall_pre = nco == 1 && wres + (uint32_t)((BN + 63) / 64) * 16384u + 2u * tall_max <= 206u * 1024u;
            auto search = [&](int bnmax, TileShape &out) {
                long best = -1;
                for (int bh = pool ? 2 : 1; bh <= 16; bh += pool ? 2 : 1)   // fused pool: whole 2x2 windows per tile
                    for (int bn = 1; bh * bn <= 16 && bn <= std::min(N, bnmax); ++bn) {
                        long t = 0;
                        for (auto &e : ext) t += (long)((N + bn - 1) / bn) * ((e.first + bh - 1) / bh) * ((e.second + 7) / 8);
                        if (best < 0 || t < best || (t == best && bh * bn > out.BH * out.BNn)) { best = t; out = {8, bh, bn}; }
                    }
                return best;
            };
            const long t_any = search(N, hs);
            TileShape h1 = ts;
            // one image per tile only where it costs at most 1/4 more tiles (28x28 patches: +14 %; a 4x4 CIFAR
            // patch would fill a quarter of the rows)
            if (tall_pre && search(1, h1) * 4 <= t_any * 5) hs = h1;
            (void)best;
            ts = hs;
        }
        // Wave quantisation of the 2-CTA pairs (>= 512 output channels, where the tile shape does not depend
        // on BN): the pair count / 74 clusters leaves a last partial wave -- e.g. C5's unsplit 14x14 conv5
        // layers: 448 pairs at BN = 256 = 6.05 waves -> 7.  Half-width N tiles (BN = 128, 896 pairs -> 13
        // waves of half the work) when that finishes >= 5 % earlier.
        if (halo && !hn && !tf32 && !pool && cpad % 64 == 0 && BN == 256 && ncols_out % 256 == 0 && ncols_out >= 512) {
            long mb = 0;
            for (auto &e : ext)
                mb += (long)((N + ts.BNn - 1) / ts.BNn) * ((e.first + ts.BH - 1) / ts.BH) * ((e.second + ts.BW - 1) / ts.BW);
            const long ncl = std::max(1, num_sms() / 2);
            auto cost = [&](int bn) {
                const long units = ((mb + 1) / 2) * (long)(ncols_out / bn);
                return ((units + ncl - 1) / ncl) * (long)bn;
            };
            if (cost(128) * 100 <= cost(256) * 95) {
                BN = 128;
                nco = ncols_out / 128;
            }
        }
        static thread_local TcConvParams P;  // large; avoid the stack
        std::memset(&P, 0, sizeof(P));
        P.npatch = g1 - g0;
        P.N = N; P.BW = ts.BW; P.BH = ts.BH; P.BNn = ts.BNn; P.rows_box = ts.BW * ts.BH * ts.BNn;
        P.nnb = (N + ts.BNn - 1) / ts.BNn;
        P.nco = nco;
        P.kh = kh; P.kw = kw; P.s = s;
        P.cpadc = cpadc;
        P.kchan = cpad;
        P.a3d = a3d;
        P.halo = halo;
        P.halo8 = halo8;
        P.hn = hn;
        P.egroups = 1;
        P.Wp = 8 + kw - 1;
        if (cpad >= 64) {
            P.cchunks = cpad / 64; P.tps = 1; P.ksteps = kh * kw * P.cchunks;
        } else {
            P.cchunks = 1; P.tps = 64 / cpad; P.ksteps = (kh * kw + P.tps - 1) / P.tps;
        }
        P.BN = BN; P.Cout = ncols_out; P.Cpo = Lout.Cpad;
        const int row_bytes = cpadc * 2;
        P.a_layout = layout_for(row_bytes);
        P.a_sbo = 8u * row_bytes;
        P.a_chunk_bytes = 128u * row_bytes;
        P.a_lbo = row_bytes == 16 ? P.a_chunk_bytes : 16u;
        P.a_tx_bytes = (uint32_t)P.tps * P.rows_box * row_bytes;
        P.b_tx_bytes = (uint32_t)BN * 128u;
        P.a_stage = 16384u;
        P.bres = 0;
        P.bres_bytes = 0;
        // 2-CTA pairs (M = 256): halves each CTA's shared-memory operand traffic per MMA (the 1-CTA
        // kernel is bound by it at N <= 256); needs 64-channel SW128 A boxes and >= 32 output columns
        {
            const int ych0 = std::min(64, Lout.Cpad);
            const bool tma_out = (ych0 == 8 || ych0 == 16 || ych0 == 32 || ych0 == 64) && Lout.Cpad % ych0 == 0;
            long mb = 0;
            for (auto &e : ext) mb += (long)P.nnb * ((e.first + ts.BH - 1) / ts.BH) * ((e.second + ts.BW - 1) / ts.BW);
            P.cta2 = (!tf32 && cpad % 64 == 0 && !halo8 && !a3d && BN % 32 == 0 && tma_out && mb >= 2) ? 1 : 0;
        }
        P.BNh = P.cta2 ? BN / 2 : BN;
        if (P.cta2) P.b_tx_bytes = (uint32_t)P.BNh * 128u;
        if (halo8) {
            P.ksteps = 1;
            P.a_tx_bytes = (uint32_t)P.Wp * (ts.BH + kh - 1) * 16u;
            P.a_stage = (P.a_tx_bytes + 1023u) & ~1023u;
            P.b_tx_bytes = (uint32_t)((kh * kw * 8 + 63) / 64) * BN * 128u;
            if (nco == 1) {   // the whole filter stays in smem (one load per CTA)
                P.bres = 1;
                P.bres_bytes = P.b_tx_bytes;
                P.b_tx_bytes = 0;
            }
        } else if (halo) {
            P.ksteps = hn ? kh : (cpad / 64) * kh;
            P.a_tx_bytes = (uint32_t)P.Wp * ts.BH * ts.BNn * rowb;
            P.a_stage = (P.a_tx_bytes + 1023u) & ~1023u;
            P.b_tx_bytes = (hn ? 1u : (uint32_t)kw) * P.BNh * 128u;
            // weights resident when they fit next to the staging tile and >= 2 A stages
            const uint32_t wbytes = wboxes * P.BNh * 128u;
            const uint32_t stg = (uint32_t)((BN + 63) / 64) * 128u * 128u;   // one staging buffer
            const uint32_t tall_stage = ((uint32_t)P.Wp * (ts.BH + kh - 1) * rowb + 1023u) & ~1023u;
            if (nco == 1 && wbytes + stg + 2u * P.a_stage <= 206u * 1024u) {
                P.bres = 1;
                P.bres_bytes = wbytes;
                P.b_tx_bytes = 0;
                // one (BH + kh - 1)-row box per channel chunk instead of kh BH-row boxes: (BH + kh - 1) / (kh BH)
                // of the TMA shared-memory writes, and the kh*kw*4 MMAs of a chunk in one stage
                if (ts.BNn == 1 && wbytes + stg + 2u * tall_stage <= 206u * 1024u) {
                    P.tall = 1;
                    P.ksteps = hn ? 1 : cpad / 64;
                    P.a_tx_bytes = (uint32_t)P.Wp * (ts.BH + kh - 1) * rowb;
                    P.a_stage = tall_stage;
                }
            }
        }
        const uint32_t stage_bytes = P.a_stage + P.b_tx_bytes;
        // output staging for the TMA-store epilogue: channel box of min(64, Cpo), swizzle to match
        const int ych = std::min(64, Lout.Cpad);
        P.direct = tf32 || !((ych == 8 || ych == 16 || ych == 32 || ych == 64) && Lout.Cpad % ych == 0);
        P.ychunk = ych;
        P.y_mask = ych == 64 ? 7u : ych == 32 ? 3u : ych == 16 ? 1u : 0u;
        const uint32_t ybuf = P.direct ? 0u : (uint32_t)((BN + ych - 1) / ych) * 128u * (uint32_t)ych * 2u;
        P.ybuf_bytes = (ybuf + 1023u) & ~1023u;
        P.ybufs = (!P.direct && P.ybuf_bytes <= 32u * 1024u) ? 2 : 1;
        if (P.bres && P.bres_bytes + 2u * P.ybuf_bytes + 2u * P.a_stage > 206u * 1024u) P.ybufs = 1;
        P.egroups = (P.ybufs == 2) ? 2 : 1;
        if (ph && P.direct) return fail(SPLITCNN_ERR_UNSUPPORTED, "phase dgrad needs a TMA-store output");
        // two groups: a ring of up to 4 staging tiles each, so that a group refills a tile while the TMA
        // stores of its last yring - 1 tiles are still reading theirs (one tile per group serialises the
        // epilogue on the store's shared-memory read, which runs at the HBM write rate: hs_probe.cu)
        P.yring = 1;
        if (P.egroups == 2) {
            const uint32_t min_st = 4;
            for (int r = 4; r >= 2; --r)
                if (P.bres_bytes + 2u * (uint32_t)r * P.ybuf_bytes + min_st * stage_bytes <= CONV_SMEM_BUDGET) { P.yring = r; break; }
        }
        // dual MMA issue for accumulators of <= 128 columns (4 of them in TMEM): short-K tiles (not the
        // 8-channel halo forward, whose 5-MMA tiles are store-bound: in the C5 step dual issue costs it 9 %)
        P.dual = (P.egroups == 2 && BN <= 128 && !tf32 && !halo8) ? 1 : 0;
        P.nacc_g = P.dual ? 2 : 1;
        // the fused pool epilogue stores from registers: no staging tiles
        const uint32_t staging = pool ? 0u : (P.egroups == 2 ? 2u * (uint32_t)P.yring : (uint32_t)P.ybufs) * P.ybuf_bytes;
        P.stages = std::min<int>(8, (int)((CONV_SMEM_BUDGET - staging - P.bres_bytes) / stage_bytes));
        // dual issue splits the stages into two rings: only with >= 2 stages per ring
        if (P.stages < 4) { P.dual = 0; P.nacc_g = 1; }
        P.bres_off = (uint32_t)P.stages * stage_bytes;
        P.stage_off = P.bres_off + ((P.bres_bytes + 1023u) & ~1023u);
        P.bar_off = P.stage_off + ((staging + 1023u) & ~1023u);
        uint32_t cols = 32;
        while (cols < 2u * (uint32_t)P.nacc_g * BN) cols <<= 1;
        P.tmem_cols = cols;
        P.bias = bias;
        P.y = (__nv_bfloat16 *)y;
        P.relu_src = (const __nv_bfloat16 *)relu_src;
        P.relu = relu;
        P.accum = accum;
        P.res = res;
        if (res && (P.direct || pool || mode != 0)) return fail(SPLITCNN_ERR_UNSUPPORTED, "fused residual: TMA-store forward only");
        if (pool && tf32) return fail(SPLITCNN_ERR_UNSUPPORTED, "conv_pool_fwd: bf16 only");
        if (pool) {
            if (halo8 || P.direct || P.Cout != P.Cpo || P.Cout % 16 || (ts.BW & (ts.BW - 1)) || ts.BW > 16 || ts.BH % 2)
                return fail(SPLITCNN_ERR_UNSUPPORTED, "conv_pool_fwd: geometry not fusable");
            P.pool_y = (__nv_bfloat16 *)pool->y;
            P.pool_a = pool->a;
        }
        int tiles = 0, mboxes = 0;
        for (int q = g0; q < g1; ++q) {
            const int ql = q - g0;
            const int i = q / Lout.nw(), j = q % Lout.nw();
            const int oh = out_ext_h(i), ow = out_ext_w(j);
            P.out_h[ql] = oh; P.out_w[ql] = ow;
            P.out_off[ql] = Lout.offset(i, j);
            if (pool) P.pool_off[ql] = pool->Lp->offset(i, j);
            const int pt = g.pad_h[2 * i], pl = g.pad_w[2 * j];
            P.pt[ql] = ph ? ph->pt : mode == 0 ? pt : kh - 1 - pt;
            P.pl[ql] = ph ? ph->pl : mode == 0 ? pl : kw - 1 - pl;
            P.nhb[ql] = (oh + ts.BH - 1) / ts.BH;
            P.nwb[ql] = (ow + ts.BW - 1) / ts.BW;
            P.tile_prefix[ql] = tiles;
            tiles += P.nnb * P.nhb[ql] * P.nwb[ql] * nco;
            P.m_prefix[ql] = mboxes;
            mboxes += P.nnb * P.nhb[ql] * P.nwb[ql];
            // A map over the patch buffer: dims (C, W, H, N), TMA zero fill = patch padding
            const int hp = La.ph(i), wp = La.pw(j);
            void *base = (char *)a_ptr + La.offset(i, j) * es;
            cuuint64_t dims[4] = {(cuuint64_t)cpad, (cuuint64_t)wp, (cuuint64_t)hp, (cuuint64_t)N};
            cuuint64_t strides[3] = {(cuuint64_t)cpad * 2, (cuuint64_t)wp * cpad * 2, (cuuint64_t)hp * wp * cpad * 2};
            cuuint32_t box[4] = {(cuuint32_t)cpadc, (cuuint32_t)(ts.BW * s), (cuuint32_t)(ts.BH * s), (cuuint32_t)ts.BNn};
            cuuint32_t es[4] = {1, (cuuint32_t)s, (cuuint32_t)s, 1};
            if (halo) box[1] = (cuuint32_t)P.Wp;
            if (P.tall) box[2] = (cuuint32_t)(ts.BH + kh - 1);
            CUresult r;
            if (a3d) {
                cuuint64_t d3[3] = {(cuuint64_t)wp * 8, (cuuint64_t)hp, (cuuint64_t)N};
                cuuint64_t s3[2] = {(cuuint64_t)wp * 16, (cuuint64_t)hp * wp * 16};
                cuuint32_t b3[3] = {(cuuint32_t)(ts.BW * 8), (cuuint32_t)ts.BH, (cuuint32_t)ts.BNn};
                if (halo8) { b3[0] = (cuuint32_t)(8 * P.Wp); b3[1] = (cuuint32_t)(ts.BH + kh - 1); b3[2] = 1; }
                cuuint32_t e3[3] = {1, 1, 1};
                r = encode(&P.mapA[ql], CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 3, base, d3, s3, b3, e3,
                           CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                           CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
            } else {
                r = encode(&P.mapA[ql], CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 4, base, dims, strides, box, es,
                           CU_TENSOR_MAP_INTERLEAVE_NONE, swz_for(row_bytes), CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                           CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
            }
            if (r != CUDA_SUCCESS) return fail(SPLITCNN_ERR_CUDA, "cuTensorMapEncodeTiled(A) failed");
            if (!P.direct && !pool) {  // output (and ReLU-mask) maps over the output patch buffer
                const int yc = Lout.Cpad;
                // phase view (S > 1): pixel (h, w) of the view is pixel (S*h + rho_h, S*w + rho_w) of the patch
                const int fh = Lout.ph(i), fw = Lout.pw(j);
                cuuint64_t ydims[4] = {(cuuint64_t)yc, (cuuint64_t)ow, (cuuint64_t)oh, (cuuint64_t)N};
                cuuint64_t ystr[3] = {(cuuint64_t)yc * 2 * PS, (cuuint64_t)fw * yc * 2 * PS, (cuuint64_t)fh * fw * yc * 2};
                cuuint32_t ybox[4] = {(cuuint32_t)P.ychunk, (cuuint32_t)ts.BW, (cuuint32_t)ts.BH, (cuuint32_t)ts.BNn};
                cuuint32_t yes[4] = {1, 1, 1, 1};
                const int64_t yoff = Lout.offset(i, j) + ((int64_t)prh * fw + prw) * yc;
                void *ybase = (char *)y + yoff * 2;
                if (encode(&P.mapY[ql], CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 4, ybase, ydims, ystr, ybox, yes,
                           CU_TENSOR_MAP_INTERLEAVE_NONE, swz_for(P.ychunk * 2), CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                           CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS)
                    return fail(SPLITCNN_ERR_CUDA, "cuTensorMapEncodeTiled(Y) failed");
                if (relu_src) {
                    void *rbase = (char *)relu_src + yoff * 2;
                    if (encode(&P.mapR[ql], CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 4, rbase, ydims, ystr, ybox, yes,
                               CU_TENSOR_MAP_INTERLEAVE_NONE, swz_for(P.ychunk * 2), CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                               CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS)
                        return fail(SPLITCNN_ERR_CUDA, "cuTensorMapEncodeTiled(R) failed");
                }
            }
        }
        P.tile_prefix[P.npatch] = tiles;
        P.m_prefix[P.npatch] = mboxes;
        P.total_m = mboxes;
        P.total_pairs = ((mboxes + 1) / 2) * nco;
        P.m_tpp = P.m_prefix[1];
        for (int ql = 1; ql < P.npatch; ++ql)
            if (P.m_prefix[ql + 1] - P.m_prefix[ql] != P.m_tpp) P.m_tpp = 0;
        P.uni = 1;
        for (int ql = 1; ql < P.npatch; ++ql)
            if (P.nhb[ql] != P.nhb[0] || P.nwb[ql] != P.nwb[0]) P.uni = 0;
        P.fd_tpp = make_fastdiv((uint32_t)std::max(1, P.tile_prefix[1]));
        P.fd_mtpp = make_fastdiv((uint32_t)std::max(1, P.m_prefix[1]));
        P.fd_nco = make_fastdiv((uint32_t)nco);
        P.fd_nwb = make_fastdiv((uint32_t)std::max(1, P.nwb[0]));
        P.fd_nhb = make_fastdiv((uint32_t)std::max(1, P.nhb[0]));
        P.ysh = P.ychunk == 64 ? 6 : P.ychunk == 32 ? 5 : P.ychunk == 16 ? 4 : 3;
        P.tpp = P.tile_prefix[1];
        for (int ql = 1; ql < P.npatch; ++ql)
            if (P.tile_prefix[ql + 1] - P.tile_prefix[ql] != P.tpp) P.tpp = 0;
        {
            const int K = kh * kw * cpad;
            cuuint64_t dims[2] = {(cuuint64_t)K, (cuuint64_t)w_rows};
            cuuint64_t strides[1] = {(cuuint64_t)K * 2};
            cuuint32_t box[2] = {64, (cuuint32_t)P.BNh};
            cuuint32_t es[2] = {1, 1};
            CUresult r = CUDA_ERROR_INVALID_VALUE;
            P.b3d = 0;
            if (halo && !hn) {  // (ci, co, tap) view of [Cout][taps][Cpad]: one box = the kw taps of a kernel row
                cuuint64_t d3[3] = {(cuuint64_t)cpad, (cuuint64_t)w_rows, (cuuint64_t)(kh * kw)};
                cuuint64_t s3[2] = {(cuuint64_t)K * 2, (cuuint64_t)cpad * 2};
                cuuint32_t b3[3] = {64, (cuuint32_t)P.BNh, (cuuint32_t)kw};
                cuuint32_t e3[3] = {1, 1, 1};
                r = encode(&P.mapB, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 3, const_cast<void *>(w_ptr), d3, s3, b3, e3,
                           CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                           CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
                P.b3d = r == CUDA_SUCCESS;
            }
            if (r != CUDA_SUCCESS)
                r = encode(&P.mapB, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, const_cast<void *>(w_ptr), dims, strides, box, es,
                           CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                           CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
            if (r != CUDA_SUCCESS) return fail(SPLITCNN_ERR_CUDA, "cuTensorMapEncodeTiled(B) failed");
        }
        if (tiles == 0) continue;
        const size_t smem = 1024 + (size_t)P.bar_off + 512 + (bias ? 4 * (size_t)g.L.cout : 0) + 64;
        if (smem > 227u * 1024u) return fail(SPLITCNN_ERR_UNSUPPORTED, "conv: shared-memory plan exceeds 227 KB");
        const int grid = P.cta2 ? 2 * std::min(P.total_pairs, num_sms() / 2) : std::min(tiles, num_sms());
        // dual issue halves the stage ring a tile sees: only where a CTA has many tiles to overlap
        const long per_cta = P.cta2 ? ((long)P.total_pairs + grid / 2 - 1) / (grid / 2) : ((long)tiles + grid - 1) / grid;
        if (P.dual && (per_cta < 8 || P.ksteps > 2)) {
            P.dual = 0;
            P.nacc_g = 1;
            uint32_t c2 = 32;
            while (c2 < 2u * BN) c2 <<= 1;
            P.tmem_cols = c2;
        }
        const int mode_bits = (bias ? 4 : 0) | (relu ? 2 : 0) | (relu_src ? 1 : 0);
        auto launch = [&](auto kern) {
            // the smem opt-in per kernel POINTER (every instantiation has the same function type, so this
            // generic lambda is one function: a per-mode key would miss kernels that share a mode)
            static std::vector<const void *> set;
            static std::mutex mu;
            {
                std::lock_guard<std::mutex> lk(mu);
                if (std::find(set.begin(), set.end(), (const void *)kern) == set.end()) {
                    cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024);
                    set.push_back((const void *)kern);
                }
            }
            // programmatic dependent launch (the kernel waits for its predecessor with griddepcontrol.wait
            // before any global access): the CTAs are placed and set up while the previous kernel drains
            cudaLaunchConfig_t cfg = {};
            cfg.gridDim = dim3((unsigned)grid);
            cfg.blockDim = dim3(P.dual ? CONV_THREADS : CONV_THREADS - 32);
            cfg.dynamicSmemBytes = smem;
            cfg.stream = st;
            cudaLaunchAttribute at[2];
            int na = 0;
            if (P.cta2) {
                at[na].id = cudaLaunchAttributeClusterDimension;
                at[na].val.clusterDim.x = 2;
                at[na].val.clusterDim.y = 1;
                at[na].val.clusterDim.z = 1;
                ++na;
            }
            at[na].id = cudaLaunchAttributeProgrammaticStreamSerialization;
            at[na].val.programmaticStreamSerializationAllowed = 1;
            ++na;
            cfg.attrs = at;
            cfg.numAttrs = na;
            cudaLaunchKernelEx(&cfg, kern, P);
        };
        // kernels holding cta_group::2 instructions must be launched as clusters: separate instantiations
        if (pool) {
            const int key = 16 + (bias ? 1 : 0) + (P.cta2 ? 2 : 0);
            auto launch_pool = [&](auto kern) {
                static std::vector<const void *> set;
                static std::mutex mu;
                std::lock_guard<std::mutex> lk(mu);
                if (std::find(set.begin(), set.end(), (const void *)kern) == set.end()) {
                    cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024);
                    set.push_back((const void *)kern);
                }
                if (P.cta2) {
                    cudaLaunchConfig_t cfg = {};
                    cfg.gridDim = dim3((unsigned)grid);
                    cfg.blockDim = dim3(P.dual ? CONV_THREADS : CONV_THREADS - 32);
                    cfg.dynamicSmemBytes = smem;
                    cfg.stream = st;
                    cudaLaunchAttribute at[1];
                    at[0].id = cudaLaunchAttributeClusterDimension;
                    at[0].val.clusterDim.x = 2;
                    at[0].val.clusterDim.y = 1;
                    at[0].val.clusterDim.z = 1;
                    cfg.attrs = at;
                    cfg.numAttrs = 1;
                    cudaLaunchKernelEx(&cfg, kern, P);
                } else {
                    kern<<<grid, P.dual ? CONV_THREADS : CONV_THREADS - 32, smem, st>>>(P);
                }
            };
            switch (key) {
                case 16: launch_pool(conv_tc_kernel<false, true, false, false, true>); break;
                case 17: launch_pool(conv_tc_kernel<true, true, false, false, true>); break;
                case 18: launch_pool(conv_tc_kernel<false, true, false, true, true>); break;
                default: launch_pool(conv_tc_kernel<true, true, false, true, true>); break;
            }
        } else if (tf32) {
            switch (mode_bits) {
                case 0: launch(conv_tc_kernel<false, false, false, false, false, true>); break;
                case 1: launch(conv_tc_kernel<false, false, true, false, false, true>); break;
                case 2: launch(conv_tc_kernel<false, true, false, false, false, true>); break;
                case 3: launch(conv_tc_kernel<false, true, true, false, false, true>); break;
                case 4: launch(conv_tc_kernel<true, false, false, false, false, true>); break;
                case 5: launch(conv_tc_kernel<true, false, true, false, false, true>); break;
                case 6: launch(conv_tc_kernel<true, true, false, false, false, true>); break;
                default: launch(conv_tc_kernel<true, true, true, false, false, true>); break;
            }
        } else if (P.cta2) {
            switch (mode_bits) {
                case 0: launch(conv_tc_kernel<false, false, false, true>); break;
                case 1: launch(conv_tc_kernel<false, false, true, true>); break;
                case 2: launch(conv_tc_kernel<false, true, false, true>); break;
                case 3: launch(conv_tc_kernel<false, true, true, true>); break;
                case 4: launch(conv_tc_kernel<true, false, false, true>); break;
                case 5: launch(conv_tc_kernel<true, false, true, true>); break;
                case 6: launch(conv_tc_kernel<true, true, false, true>); break;
                default: launch(conv_tc_kernel<true, true, true, true>); break;
            }
        } else {
            switch (mode_bits) {
                case 0: launch(conv_tc_kernel<false, false, false, false>); break;
                case 1: launch(conv_tc_kernel<false, false, true, false>); break;
                case 2: launch(conv_tc_kernel<false, true, false, false>); break;
                case 3: launch(conv_tc_kernel<false, true, true, false>); break;
                case 4: launch(conv_tc_kernel<true, false, false, false>); break;
                case 5: launch(conv_tc_kernel<true, false, true, false>); break;
                case 6: launch(conv_tc_kernel<true, true, false, false>); break;
                default: launch(conv_tc_kernel<true, true, true, false>); break;
            }
        }
        count_launch();
        {
            cudaError_t e = cudaGetLastError();
            if (e != cudaSuccess) return fail(SPLITCNN_ERR_CUDA, std::string("conv_tc_kernel: ") + cudaGetErrorString(e));
        }
    }
    return SPLITCNN_OK;
}

}  // namespace

bool conv_tc_supported(int mode, splitcnn_dtype_t dt, const Level &Li, const Level &Lo, const LayerGeom &g) {
    if (dt == SPLITCNN_TF32 || dt == SPLITCNN_FP32) {
        // fp32 storage on kind::tf32 (SPLITCNN_FP32: three passes hi*hi + hi*lo + lo*hi, api.cu): forward and
        // stride-1 data gradient; the byte layout has 2 Cpad two-byte channels
        if (g.L.sh != g.L.sw || Li.npatch() > 1024) return false;
        if (mode == 0) return a_channels_ok(2 * Li.Cpad) && g.L.sh <= 2;
        if (mode == 1) return a_channels_ok(2 * Lo.Cpad) && g.L.sh == 1;
        return false;   // weight gradient: operand splitting onto the bf16 kernels (api.cu)
    }
    if (dt != SPLITCNN_BF16) return false;
    if (g.L.sh != g.L.sw) return false;
    if (Li.npatch() > 1024) return false;
    if (mode == 0) {
        if (!a_channels_ok(Li.Cpad)) return false;
        if (g.L.sh > 2) return false;
        return true;
    }
    if (mode == 1) {
        if (!a_channels_ok(Lo.Cpad)) return false;
        if (g.L.sh == 1) return true;
        // stride S > 1: phase decomposition -- one begin pad per dimension, every patch at least S
        // pixels wide (no empty phase view), TMA-store output channels
        if (g.L.sh > 2 || !(Li.Cpad == 8 || Li.Cpad == 16 || Li.Cpad == 32 || Li.Cpad % 64 == 0)) return false;
        for (int i = 0; i < Li.nh(); ++i)
            if (g.pad_h[2 * i] != g.pad_h[0] || Li.ph(i) < g.L.sh) return false;
        for (int j = 0; j < Li.nw(); ++j)
            if (g.pad_w[2 * j] != g.pad_w[0] || Li.pw(j) < g.L.sw) return false;
        return true;
    }
    if (mode == 2) return wgrad_tc_ok(Li, Lo, g);
    return false;
}

size_t conv_tc_ws_bytes(int mode, const Level &Li, const Level &Lo, const LayerGeom &g, splitcnn_dtype_t dt) {
    if (mode == 2) return wgrad_tc_ws_bytes(Li, Lo, g);
    const size_t es = dt == SPLITCNN_BF16 ? 2 : 4;
    if (mode == 1) return (size_t)g.L.cin * g.L.kh * g.L.kw * Lo.Cpad * es + 256 + (size_t)g.L.sh * g.L.sw * 1024;
    return 0;
}

splitcnn_status_t launch_conv_fwd_tc(const Level &Li, const Level &Lo, const LayerGeom &g, const void *x, const void *w,
                                     const float *bias, void *y, int relu, int p0, int p1, cudaStream_t st,
                                     splitcnn_dtype_t dt, int accum) {
    return launch_tc(0, Li, Lo, g, x, w, g.L.cout, bias, y, nullptr, relu, p0, p1, st, nullptr, nullptr,
                     dt == SPLITCNN_BF16 ? 0 : 1, accum);
}

splitcnn_status_t launch_conv_fwd_res_tc(const Level &Li, const Level &Lo, const LayerGeom &g, const void *x, const void *w,
                                         const float *bias, const void *residual, void *y, int relu, int p0, int p1,
                                         cudaStream_t st) {
    return launch_tc(0, Li, Lo, g, x, w, g.L.cout, bias, y, residual, relu, p0, p1, st, nullptr, nullptr, 0, 0, 1);
}

splitcnn_status_t launch_conv_pool_fwd_tc(const Level &Li, const Level &Lo, const Level &Lp, const LayerGeom &g,
                                          const void *x, const void *w, const float *bias, void *y_pool, uint8_t *argmax,
                                          int p0, int p1, cudaStream_t st) {
    PoolFuse pf;
    pf.y = y_pool;
    pf.a = argmax;
    pf.Lp = &Lp;
    return launch_tc(0, Li, Lo, g, x, w, g.L.cout, bias, nullptr, nullptr, 1, p0, p1, st, &pf, nullptr, 0, 0);
}

template <typename T>
static void flip_weights(const void *w, void *wt, const LayerGeom &g, int cpad_in, int cpad_out, int r0h, int r0w,
                         int step, int nth, int ntw, cudaStream_t st, int max_blocks = 148 * 16) {
    const int64_t n = (int64_t)((g.L.cin + 7) / 8) * nth * ntw * cpad_out;
    flip_weights_kernel<T><<<(unsigned)std::max<int64_t>(1, std::min<int64_t>((n + 255) / 256, max_blocks)), 256, 0, st>>>(
        (const T *)w, (T *)wt, g.L.cout, cpad_in, g.L.cin, g.L.kh, g.L.kw, cpad_out, r0h, r0w, step, nth, ntw);
    count_launch();
}

// Stride-S dgrad phase (rh, rw): first tap (r0h, r0w) and tap counts of its sub-filter (0: no tap reaches it)
struct DgradPhase {
    int r0h, r0w, nth, ntw;
};
static DgradPhase dgrad_phase(const LayerGeom &g, int rh, int rw) {
    const int S = g.L.sh, pbh = g.pad_h[0], pbw = g.pad_w[0];
    DgradPhase d;
    d.r0h = ((rh + pbh) % S + S) % S;
    d.r0w = ((rw + pbw) % S + S) % S;
    d.nth = d.r0h < g.L.kh ? (g.L.kh - d.r0h + S - 1) / S : 0;
    d.ntw = d.r0w < g.L.kw ? (g.L.kw - d.r0w + S - 1) / S : 0;
    return d;
}

// The weights the data gradient multiplies with: stride 1 the 180-degree flip, stride S one sub-filter per
// phase that some tap reaches, 1 KB-aligned one after another (the layout of the dgrad workspace prefix).
// max_blocks: the in-call flip (on the critical path) takes many blocks; a prepared copy built next to the
// forward pass takes one per SM, so the persistent conv CTAs still fit beside it (threads, no shared memory)
void prep_dgrad_weights_tc(const Level &Li, const Level &Lo, const LayerGeom &g, const void *w, void *wt, cudaStream_t st,
                           int max_blocks) {
    const int S = g.L.sh;
    if (max_blocks <= 0) max_blocks = num_sms();
    if (S == 1) {
        flip_weights<__nv_bfloat16>(w, wt, g, Li.Cpad, Lo.Cpad, 0, 0, 1, g.L.kh, g.L.kw, st, max_blocks);
        return;
    }
    char *wsp = (char *)wt;
    for (int rh = 0; rh < S; ++rh)
        for (int rw = 0; rw < S; ++rw) {
            const DgradPhase d = dgrad_phase(g, rh, rw);
            if (d.nth == 0 || d.ntw == 0) continue;
            flip_weights<__nv_bfloat16>(w, wsp, g, Li.Cpad, Lo.Cpad, d.r0h, d.r0w, S, d.nth, d.ntw, st, max_blocks);
            wsp += (((int64_t)g.L.cin * d.nth * d.ntw * Lo.Cpad * 2 + 1023) / 1024) * 1024;
        }
}

// prepared: w already holds prep_dgrad_weights_tc's output (BF16) -- no flip in this call
splitcnn_status_t launch_conv_dgrad_tc(const Level &Li, const Level &Lo, const LayerGeom &g, const void *dy, const void *w,
                                       void *dx, const void *relu_src, void *ws, int p0, int p1, cudaStream_t st,
                                       splitcnn_dtype_t dt, int accum, bool prepared) {
    const int S = g.L.sh;
    if (prepared && dt != SPLITCNN_BF16) return fail(SPLITCNN_ERR_UNSUPPORTED, "prepared dgrad weights: bf16 only");
    if (S == 1) {
        if (!prepared) {
            if (dt == SPLITCNN_BF16) flip_weights<__nv_bfloat16>(w, ws, g, Li.Cpad, Lo.Cpad, 0, 0, 1, g.L.kh, g.L.kw, st);
            else flip_weights<float>(w, ws, g, Li.Cpad, Lo.Cpad, 0, 0, 1, g.L.kh, g.L.kw, st);
        }
        return launch_tc(1, Lo, Li, g, dy, prepared ? w : ws, g.L.cin, nullptr, dx, relu_src, 0, p0, p1, st, nullptr, nullptr,
                         dt == SPLITCNN_BF16 ? 0 : 1, accum);
    }
    if (dt != SPLITCNN_BF16) return fail(SPLITCNN_ERR_UNSUPPORTED, "tf32 strided data gradient");
    // stride S: S*S output phases, each a stride-1 correlation with the taps r = (rho + p_b) (mod S)
    // (every patch of a plan shares its begin pad under R2, checked in conv_tc_supported)
    const int pbh = g.pad_h[0], pbw = g.pad_w[0];
    if (!prepared) prep_dgrad_weights_tc(Li, Lo, g, w, ws, st, 148 * 16);
    const char *wsp = (const char *)(prepared ? w : ws);
    // phases no tap reaches (k < s, e.g. the 1x1 / stride-2 downsample: 3 of 4) are zero: ONE contiguous
    // memset of the patch range (the reached phases overwrite their pixels) instead of one strided zero
    // kernel per phase -- 3 x 11.7 us -> ~17 us for C3's downsample data gradient
    int nzero = 0;
    for (int rh = 0; rh < S; ++rh)
        for (int rw = 0; rw < S; ++rw) {
            const DgradPhase d = dgrad_phase(g, rh, rw);
            nzero += (d.nth == 0 || d.ntw == 0) ? 1 : 0;
        }
    if (nzero > 1) {
        const int64_t e0 = Li.offset(p0 / Li.nw(), p0 % Li.nw());
        const int64_t e1 = p1 >= Li.npatch() ? Li.total() : Li.offset(p1 / Li.nw(), p1 % Li.nw());
        cudaMemsetAsync((__nv_bfloat16 *)dx + e0, 0, (size_t)(e1 - e0) * 2, st);
    }
    for (int rh = 0; rh < S; ++rh)
        for (int rw = 0; rw < S; ++rw) {
            const DgradPhase d = dgrad_phase(g, rh, rw);
            if (d.nth == 0 || d.ntw == 0) {
                if (nzero > 1) continue;   // covered by the memset
                LevelDesc ld = make_level_desc(Li);
                dim3 grid((unsigned)std::max(1, std::min(2048, 148 * 8 / std::max(1, p1 - p0))), (unsigned)(p1 - p0));
                zero_phase_kernel<<<grid, 256, 0, st>>>((__nv_bfloat16 *)dx, ld, S, rh, rw, p0);
                count_launch();
                continue;
            }
            const int ch = (rh + pbh - d.r0h) / S, cw = (rw + pbw - d.r0w) / S;
            Phase ph{S, rh, rw, d.nth, d.ntw, d.nth - 1 - ch, d.ntw - 1 - cw};
            const splitcnn_status_t r = launch_tc(1, Lo, Li, g, dy, wsp, g.L.cin, nullptr, dx, relu_src, 0, p0, p1, st,
                                                  nullptr, &ph);
            if (r != SPLITCNN_OK) return r;
            wsp += (((int64_t)g.L.cin * d.nth * d.ntw * Lo.Cpad * 2 + 1023) / 1024) * 1024;
        }
    return SPLITCNN_OK;
}

// ============================================================ weight gradient (tcgen05, MN-major)
// dW[co][r][c][ci] = sum over pixels of dY[pix][co] * X~[pix shifted by (r, c)][ci]
// GEMM with M = co (a block of 128 = two 64-channel dY boxes), K = pixels, and N = a set of B BLOCKS:
// each block is one TMA box of the input X at one tap's shift and one channel chunk of `cbox`
// channels, so one accumulator tile can cover several taps and the dY tile is loaded once for all
// of them.  Both operands are MN-major (pixels are rows): SW128 / SW64 / SW32 / no-swizzle for
// cbox = 64 / 32 / 16 / 8.  Split-K over pixel boxes of all patches; fp32 partial tiles go to the
// workspace and a fixed-order reduction sums them (deterministic).
constexpr int WG_ROWS = 64;    // pixels per K stage (4 MMAs of K = 16)
constexpr int WG_MAXBLK = 32;  // B blocks per tile

struct TcWgradParams {
    CUtensorMap mapDY[TC_MAXP];
    CUtensorMap mapX[TC_MAXP];
    int box_prefix[TC_MAXP + 1];
    int pt[TC_MAXP], pl[TC_MAXP];
    int nhb[TC_MAXP], nwb[TC_MAXP];
    int npatch;
    int BW, BH, BNn, rows_box;
    int kh, kw, s;
    int x3d;                        // X maps are 3-D (8-channel rows merged: coordinate 8*w)
    int cbox;                       // channels per B block
    int nchunk;                     // channel chunks per tap (Cpi / cbox)
    int bpt;                        // real blocks per tile
    int bpt_pad;                    // blocks per tile incl. zero blocks (N = bpt_pad * cbox, multiple of 16)
    int nblocks;                    // KT * nchunk
    int nco_blk, ntb, ntiles;       // tiles = nco_blk * ntb
    int boxes_per_split, nsplit;
    int Cout, Cpi;
    int stages;
    uint32_t tmem_cols;
    uint32_t b_layout, b_lbo, b_sbo, b_kstep, b_box_bytes;
    float *part;                    // [nsplit][Cout][kh][kw][Cpi]
};

__global__ void __launch_bounds__(192, 1) wgrad_tc_kernel(const __grid_constant__ TcWgradParams p) {
    extern __shared__ uint8_t smem_raw[];
    uint8_t *smem = (uint8_t *)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
    const int S = p.stages;
    const uint32_t a_stage = 2u * WG_ROWS * 128u;  // 128 co = two 64-channel blocks
    const uint32_t b_stage = (uint32_t)p.bpt_pad * p.b_box_bytes;
    const uint32_t b_stage_al = (b_stage + 1023u) & ~1023u;
    uint8_t *sA = smem;
    uint8_t *sB = smem + (size_t)S * a_stage;
    uint64_t *full = (uint64_t *)(sB + (size_t)S * b_stage_al);
    uint64_t *empty = full + S;
    uint64_t *tfull = empty + S;
    uint32_t *tmem_slot = (uint32_t *)(tfull + 1);
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;

    // rows >= rows_box and the zero blocks are never written by TMA: zero them once so they add 0
    {
        uint4 *z = (uint4 *)smem;
        const int n16 = (int)(((size_t)S * (a_stage + b_stage_al)) / 16);
        for (int i = threadIdx.x; i < n16; i += blockDim.x) z[i] = make_uint4(0, 0, 0, 0);
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    }
    if (warp == 0 && lane == 0) {
        for (int s = 0; s < S; ++s) {
            tc::mbar_init(&full[s], 1);
            tc::mbar_init(&empty[s], 1);
        }
        tc::mbar_init(&tfull[0], 1);
        tc::fence_barrier_init();
    }
    if (warp == 1) tc::tmem_alloc_dyn(tmem_slot, p.tmem_cols);
    tc::tc_fence_before();
    __syncthreads();
    tc::tc_fence_after();
    const uint32_t tmem_base = *tmem_slot;

    // work item: z-major so CTAs running together share the same pixels (L2 reuse)
    const int tile = blockIdx.x % p.ntiles, z = blockIdx.x / p.ntiles;
    const int tb = tile % p.ntb, co_blk = tile / p.ntb;
    const int blk0 = tb * p.bpt;
    const int nblk = min(p.bpt, p.nblocks - blk0);
    const int total_boxes = p.box_prefix[p.npatch];
    const int b0 = z * p.boxes_per_split, b1 = min(total_boxes, b0 + p.boxes_per_split);

    if (warp == 0) {
        if (lane == 0) {
            int stage = 0;
            uint32_t ph = 0;
            int ql = 0;
            // the upper 64-channel dY block is skipped when it is all out of bounds (Cout <= 64): its
            // shared memory stays zero from the clear above, so its accumulator rows add nothing
            const int nh = co_blk * 128 + 64 < p.Cout ? 2 : 1;
            const uint32_t tx = (uint32_t)nh * p.rows_box * 128u + (uint32_t)nblk * p.rows_box * p.cbox * 2u;
            for (int b = b0; b < b1; ++b) {
                while (b >= p.box_prefix[ql + 1]) ++ql;
                int idx = b - p.box_prefix[ql];
                const int wb = idx % p.nwb[ql];
                idx /= p.nwb[ql];
                const int hb = idx % p.nhb[ql], nb = idx / p.nhb[ql];
                const int ow0 = wb * p.BW, oh0 = hb * p.BH, n0 = nb * p.BNn;
                tc::mbar_wait(&empty[stage], ph ^ 1);
                tc::mbar_arrive_expect_tx(&full[stage], tx);
                uint8_t *a = sA + (size_t)stage * a_stage;
                uint8_t *bb = sB + (size_t)stage * b_stage_al;
                for (int h = 0; h < nh; ++h)
                    tc::tma_load_4d(a + h * WG_ROWS * 128, &p.mapDY[ql], &full[stage], co_blk * 128 + h * 64, ow0, oh0, n0);
                for (int k = 0; k < nblk; ++k) {
                    const int blk = blk0 + k;
                    const int tap = blk / p.nchunk, ch = blk - tap * p.nchunk;
                    const int r = tap / p.kw, c = tap - r * p.kw;
                    const int wx = ow0 * p.s - p.pl[ql] + c, hx = oh0 * p.s - p.pt[ql] + r;
                    if (p.x3d)
                        tc::tma_load_3d(bb + k * p.b_box_bytes, &p.mapX[ql], &full[stage], 8 * wx, hx, n0);
                    else
                        tc::tma_load_4d(bb + k * p.b_box_bytes, &p.mapX[ql], &full[stage], ch * p.cbox, wx, hx, n0);
                }
                if (++stage == S) { stage = 0; ph ^= 1; }
            }
        }
    } else if (warp == 1) {
        {   // converged warp; elect.sync issues
            const uint32_t idesc = tc::idesc_bf16(128, p.bpt_pad * p.cbox, 1, 1);
            int stage = 0;
            uint32_t ph = 0;
            for (int b = b0; b < b1; ++b) {
                tc::mbar_wait(&full[stage], ph);
                tc::tc_fence_after();
                const uint32_t a_base = tc::smem_u32(sA + (size_t)stage * a_stage);
                const uint32_t b_base = tc::smem_u32(sB + (size_t)stage * b_stage_al);
                const uint64_t a0 = tc::smem_desc(a_base, WG_ROWS * 128, 1024, 2);
                const uint64_t bd0 = tc::smem_desc(b_base, p.b_lbo, p.b_sbo, p.b_layout);
#pragma unroll
                for (int j = 0; j < WG_ROWS / 16; ++j)
                    tc::mma_bf16_ws(tmem_base, a0 + (uint64_t)(128 * j), bd0 + (uint64_t)((p.b_kstep >> 4) * j), idesc,
                                 (b != b0 || j) ? 1u : 0u);
                tc::mma_commit_ws(&empty[stage]);
                if (++stage == S) { stage = 0; ph ^= 1; }
            }
            tc::mma_commit_ws(&tfull[0]);
        }
    } else {
        const int quad = warp & 3;
        const int co = co_blk * 128 + quad * 32 + lane;
        const bool any = b1 > b0;
        if (any) {
            tc::mbar_wait(&tfull[0], 0);
            tc::tc_fence_after();
        }
        const uint32_t tacc = tmem_base + ((uint32_t)(quad * 32) << 16);
        const int KT = p.kh * p.kw;
        const int ncols = nblk * p.cbox;
        for (int cc = 0; cc < ncols; cc += 16) {
            float v[16];
            if (any) {
                tc::tmem_ld16(tacc + cc, v);
            } else {
#pragma unroll
                for (int e = 0; e < 16; ++e) v[e] = 0.f;
            }
            if (co >= p.Cout) continue;
#pragma unroll
            for (int g = 0; g < 2; ++g) {
                const int col = cc + 8 * g;
                if (col >= ncols) break;
                const int blk = blk0 + col / p.cbox;
                const int tap = blk / p.nchunk, ch = blk - tap * p.nchunk;
                float *dst = p.part + ((((int64_t)z * p.Cout + co) * KT + tap) * p.Cpi) + ch * p.cbox + (col % p.cbox);
                float4 *d4 = reinterpret_cast<float4 *>(dst);
                d4[0] = make_float4(v[8 * g], v[8 * g + 1], v[8 * g + 2], v[8 * g + 3]);
                d4[1] = make_float4(v[8 * g + 4], v[8 * g + 5], v[8 * g + 6], v[8 * g + 7]);
            }
        }
    }
    tc::tc_fence_before();
    __syncthreads();
    tc::tc_fence_after();
    if (warp == 1) tc::tmem_dealloc(tmem_base, p.tmem_cols);
}

// ------------------------------------------------------------ halo weight gradient (stride 1, 3 taps per row)
// Same GEMM as above, but the kw taps of one kernel row r share ONE input box: the X tile for output
// rows [h0, h0+BH) x 8 output columns is loaded with kw-1 halo columns (8+kw-1 pixels wide).  In the
// MN-major SW128 layout a pixel is a 128-byte smem row, so the operand of tap (r, c) is the same tile
// viewed c rows further on, and the kw taps are kw MN-blocks of ONE MMA with LBO = 128 B (N = kw*64).
// The output-row K groups of 8 pixels sit Wp = 8+kw-1 rows apart (SBO = Wp*128 B).  The SW128 swizzle
// is address-based, so any 128-byte row offset is a valid operand start (probed: scripts/umma_probe.cu).
// Per stage: 2 dY boxes + 1 X box for BH*8 pixels (3 TMA ops vs 2+kw).
struct TcWgHaloParams {
    CUtensorMap mapDY[TC_MAXP];
    CUtensorMap mapX[TC_MAXP];
    int box_prefix[TC_MAXP + 1];
    int pt[TC_MAXP], pl[TC_MAXP];
    int nhb[TC_MAXP], nwb[TC_MAXP];
    int npatch, BH, BNn, kh, kw;
    int nco_blk, nchunk, ntiles, boxes_per_split, nsplit;
    int Cout, Cpi, stages;
    int rpack;    // Cout <= 64: row-pair packing (below)
    uint32_t xrow;  // bytes per X pixel row in smem: 128 (64-channel chunks), 64 / 32 (32- / 16-channel levels:
                    // SW64 / SW32 MN-major, MN block = the level's channels), 64 in 2-CTA mode (channel halves)
    uint32_t tmem_cols;
    float *part;  // [nsplit][Cout][kh][kw][Cpi]
};
// Row-pair packing (Cout <= 64, where the upper 64 rows of the M = 128 MMA would be padding): the upper dY
// block is the SAME dY loaded one output row further down, so against the X box of kernel row r those rows
// accumulate sum_oh dY[oh + 1] X~[oh + r - pt] = the contribution of kernel row r - 1.  A tile then serves
// kernel rows (r, r - 1): ceil(kh / 2) tiles instead of kh.  The pixel boxes start one output row early
// (oh0 = hb * BH - 1), so the shifted block also sees output row 0; the extra row of the unshifted block is
// dY row -1, zero-filled by TMA.

// CTA2: a cluster of 2 runs one tile of 256 output channels (each CTA: its own 128-channel dY block
// as A) with cta_group::2 MMAs (M = 256); B is split by input channel -- each CTA loads 32 of the
// chunk's 64 channels (SW64 rows of 64 B), so D column n < kw*32 is (tap n/32, ci n%32) of the
// leader's half and n >= kw*32 the peer's.  Halves each CTA's smem operand traffic per MMA.
template <bool CTA2>
__global__ void __launch_bounds__(192, 1) wgrad_halo_kernel(const __grid_constant__ TcWgHaloParams p) {
    extern __shared__ uint8_t smem_raw[];
    uint8_t *smem = smem_raw + ((1024u - (tc::smem_u32(smem_raw) & 1023u)) & 1023u);
    const int S = p.stages;
    // pixels per stage: BNn images x BH output rows x 8 output columns; for a FIXED kernel row r the X
    // box has exactly BH rows per image, so the K groups (n, h) stay Wp rows apart across images too
    const int rows = p.BNn * p.BH * 8;
    const int Wp = 8 + p.kw - 1;
    const uint32_t a_blk = (uint32_t)rows * 128u;     // one 64-channel dY block
    // Cout <= 64 without row packing: the upper dY block is all out of bounds -- not loaded, and not even
    // given space (the MMA's rows 64..127 read the next stage's bytes; those accumulator rows are never stored)
    const uint32_t a_stage = (p.Cout <= 64 && !p.rpack ? 1u : 2u) * a_blk;
    const uint32_t xrow = p.xrow;                       // bytes per X pixel row (16, 32 or 64 channels)
    // row-packed: ONE X box of BH + kh - 1 rows (one image) serves every kernel row (views r * Wp rows on)
    const int xh = p.rpack ? p.BH + p.kh - 1 : p.BH;
    const uint32_t b_bytes = (uint32_t)Wp * xh * p.BNn * xrow;
    const uint32_t b_stage = (b_bytes + 1023u) & ~1023u;
    uint8_t *sA = smem;
    uint8_t *sB = smem + (size_t)S * a_stage;
    uint64_t *full = (uint64_t *)(sB + (size_t)S * b_stage);
    uint64_t *empty = full + S;
    uint64_t *tfull = empty + S;
    uint32_t *tmem_slot = (uint32_t *)(tfull + 1);
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const uint32_t rank = CTA2 ? tc::cluster_ctarank() : 0u;
    const bool leader = rank == 0;
    if (warp == 0 && lane == 0) {
        for (int s = 0; s < S; ++s) {
            tc::mbar_init(&full[s], 1);
            tc::mbar_init(&empty[s], 1);
        }
        tc::mbar_init(&tfull[0], 1);
        tc::fence_barrier_init();
    }
    if (warp == 1) {
        if (CTA2) tc::tmem_alloc2(tmem_slot, p.tmem_cols);
        else tc::tmem_alloc_dyn(tmem_slot, p.tmem_cols);
    }
    tc::tc_fence_before();
    if (CTA2) tc::cluster_sync_all();
    else __syncthreads();
    tc::tc_fence_after();
    const uint32_t tmem_base = *tmem_slot;

    // CTA2: work item = blockIdx.x / 2 over (co pair, kernel row, chunk) x split; ntiles counts pairs
    const int item = CTA2 ? (int)(blockIdx.x >> 1) : (int)blockIdx.x;
    const int tile = item % p.ntiles, z = item / p.ntiles;
    const int ch = tile % p.nchunk;
    const int nr = p.rpack ? 1 : p.kh;                              // kernel-row tiles (row-packed: all rows)
    const int nv = p.rpack ? (p.kh + 1) / 2 : 1;                    // accumulators (kernel-row pairs) per tile
    const int r = p.rpack ? 0 : (tile / p.nchunk) % p.kh;
    const int co_blk = CTA2 ? 2 * (tile / (p.nchunk * nr)) + (int)rank : tile / (p.nchunk * nr);
    const int total_boxes = p.box_prefix[p.npatch];
    const int b0 = z * p.boxes_per_split, b1 = min(total_boxes, b0 + p.boxes_per_split);
    const int cw = CTA2 ? 64 : (int)(xrow / 2);                     // channels per tap block of D (both CTAs)
    const int N = p.kw * cw;

    if (warp == 0) {
        if (lane == 0) {
            int stage = 0, ql = 0;
            uint32_t ph = 0;
            const bool hi = p.Cout > 64 || p.rpack;
            const uint32_t tx = (hi ? 2u : 1u) * a_blk + b_bytes;
            for (int b = b0; b < b1; ++b) {
                while (b >= p.box_prefix[ql + 1]) ++ql;
                int idx = b - p.box_prefix[ql];
                const int wb = idx % p.nwb[ql];
                idx /= p.nwb[ql];
                const int hb = idx % p.nhb[ql], n = (idx / p.nhb[ql]) * p.BNn;
                const int ow0 = wb * 8, oh0 = hb * p.BH - p.rpack;
                tc::mbar_wait_sleep(&empty[stage], ph ^ 1);
                uint8_t *a = sA + (size_t)stage * a_stage;
                if (CTA2) {   // own dY block + own channel half of X; bytes land on the leader's barrier
                    const uint32_t fb = tc::mapa_shared(&full[stage], 0);
                    if (leader) tc::mbar_arrive_expect_tx(&full[stage], 2 * tx);
                    tc::tma2_load_4d(a, &p.mapDY[ql], fb, co_blk * 128, ow0, oh0, n);
                    tc::tma2_load_4d(a + a_blk, &p.mapDY[ql], fb, co_blk * 128 + 64, ow0, oh0, n);
                    tc::tma2_load_4d(sB + (size_t)stage * b_stage, &p.mapX[ql], fb, ch * 64 + (int)rank * 32,
                                     ow0 - p.pl[ql], oh0 - p.pt[ql] + r, n);
                    if (++stage == S) { stage = 0; ph ^= 1; }
                    continue;
                }
                tc::mbar_arrive_expect_tx(&full[stage], tx);
                tc::tma_load_4d(a, &p.mapDY[ql], &full[stage], co_blk * 128, ow0, oh0, n);
                if (p.rpack) tc::tma_load_4d(a + a_blk, &p.mapDY[ql], &full[stage], 0, ow0, oh0 + 1, n);
                else if (hi) tc::tma_load_4d(a + a_blk, &p.mapDY[ql], &full[stage], co_blk * 128 + 64, ow0, oh0, n);
                tc::tma_load_4d(sB + (size_t)stage * b_stage, &p.mapX[ql], &full[stage], ch * 64, ow0 - p.pl[ql],
                                oh0 - p.pt[ql] + r, n);   // row-packed: r = 0, the box spans all kh rows
                if (++stage == S) { stage = 0; ph ^= 1; }
            }
        }
    } else if (warp == 1) {
        {   // converged warp; elect.sync issues
            const uint32_t idesc = tc::idesc_bf16(CTA2 ? 256 : 128, N, 1, 1);
            int stage = 0;
            uint32_t ph = 0;
            for (int b = b0; b < (leader ? b1 : b0); ++b) {
                tc::mbar_wait(&full[stage], ph);
                tc::tc_fence_after();
                const uint32_t a_base = tc::smem_u32(sA + (size_t)stage * a_stage);
                const uint32_t b_base = tc::smem_u32(sB + (size_t)stage * b_stage);
                // A: dY, MN-major: 8-pixel K groups at 1 KB, the second 64-co block at LBO = a_blk
                // B: X halo view, MN-major: tap c = MN block c at LBO = 128 B, K groups (output rows)
                //    at SBO = Wp rows; 16 pixels = 2 output rows.  Per-MMA descriptors = base + constant.
                const uint64_t a0 = tc::smem_desc(a_base, a_blk, 1024, 2);
                if (CTA2) {   // SW64 MN-major X: MN blocks of 32 channels, tap c = 1 row (64 B) further on
                    const uint64_t bd0 = tc::smem_desc(b_base, 64, (uint32_t)Wp * 64u, 4);
                    const uint64_t bstep = (uint64_t)(Wp * 8);   // 2 rows of Wp pixels x 64 B, >> 4
                    for (int j = 0; j < rows / 16; ++j)
                        tc::mma2_bf16_ws(tmem_base, a0 + (uint64_t)(128 * j), bd0 + bstep * j, idesc, (b != b0 || j) ? 1u : 0u);
                    tc::mma2_commit_mc_ws(&empty[stage]);
                } else {
                    // (16 / 32-channel levels: SW32 / SW64 MN-major, tap c = c pixel rows of xrow bytes on)
                    const uint32_t lay = xrow == 128u ? 2u : xrow == 64u ? 4u : 6u;
                    const uint64_t bd0 = tc::smem_desc(b_base, xrow, (uint32_t)Wp * xrow, lay);
                    const uint64_t bstep = (uint64_t)(2 * Wp * (xrow >> 4));   // 2 rows of Wp pixels, >> 4
                    // accumulator v (row-packed): X view of kernel row kh-1-2v (its rows 0..63) and kh-2-2v
                    // (rows 64..127, the shifted dY block) = the box viewed (kh-1-2v)*Wp pixel rows on
                    for (int v = 0; v < nv; ++v) {
                        const uint64_t bv = bd0 + (uint64_t)(p.rpack ? (p.kh - 1 - 2 * v) * Wp * (int)(xrow >> 4) : 0);
                        for (int j = 0; j < rows / 16; ++j)
                            tc::mma_bf16_ws(tmem_base + (uint32_t)(v * N), a0 + (uint64_t)(128 * j), bv + bstep * j, idesc,
                                            (b != b0 || j) ? 1u : 0u);
                    }
                    tc::mma_commit_ws(&empty[stage]);
                }
                if (++stage == S) { stage = 0; ph ^= 1; }
            }
            if (leader) {
                if (CTA2) tc::mma2_commit_mc_ws(&tfull[0]);
                else tc::mma_commit_ws(&tfull[0]);
            }
        }
    } else {
        const int quad = warp & 3;
        // row-packed: accumulator v, rows 0..63 = kernel row kh-1-2v, rows 64..127 = kh-2-2v (same channels)
        const int co = p.rpack ? (quad & 1) * 32 + lane : co_blk * 128 + quad * 32 + lane;
        const bool any = b1 > b0;
        if (any) {
            tc::mbar_wait(&tfull[0], 0);
            tc::tc_fence_after();
        }
        const uint32_t tacc = tmem_base + ((uint32_t)(quad * 32) << 16);
        const int KT = p.kh * p.kw;
        for (int vc = 0; vc < nv * N; vc += 16) {
            const int cc = vc % N;
            const int rr = p.rpack ? p.kh - 1 - 2 * (vc / N) - (quad >= 2 ? 1 : 0) : r;
            float v[16];
            if (any) {
                tc::tmem_ld16(tacc + vc, v);
            } else {
#pragma unroll
                for (int e = 0; e < 16; ++e) v[e] = 0.f;
            }
            if (co >= p.Cout || rr < 0) continue;
            // D column -> (tap, input channel); CTA2: the first kw*32 columns are the leader's channel half
            int c, ci;
            if (CTA2) {
                const int hb = cc >= p.kw * 32 ? 1 : 0, n = cc - hb * p.kw * 32;
                c = n >> 5;
                ci = ch * 64 + hb * 32 + (n & 31);
            } else {
                c = cc / cw;
                ci = ch * 64 + (cc % cw);
            }
            float4 *d4 = reinterpret_cast<float4 *>(p.part + (((int64_t)z * p.Cout + co) * KT + rr * p.kw + c) * p.Cpi + ci);
#pragma unroll
            for (int e = 0; e < 4; ++e) d4[e] = make_float4(v[4 * e], v[4 * e + 1], v[4 * e + 2], v[4 * e + 3]);
        }
    }
    tc::tc_fence_before();
    if (CTA2) tc::cluster_sync_all();
    else __syncthreads();
    tc::tc_fence_after();
    if (warp == 1) {
        if (CTA2) tc::tmem_dealloc2(tmem_base, p.tmem_cols);
        else tc::tmem_dealloc(tmem_base, p.tmem_cols);
    }
}

// ------------------------------------------------------------ narrow-input weight gradient (Cin_pad = 8)
// dW[co][tap][ci] for an 8-channel input (VGG conv1_1, C = 3 padded to 8): per stage one dY tile
// (BH output rows x 8 columns, MN-major SW128) and ONE X tile of (BH + kh - 1) rows x (8 + kw - 1)
// pixels x 8 channels loaded with 16-byte pixel rows merged into 3-D rows.  In the no-swizzle
// MN-major layout a core matrix is 8 pixels x 16 B, so the operand of tap t is the X tile viewed
// o_t = r*Wp + c pixels further on; two taps form the two 8-channel MN blocks of one N = 16 MMA
// (block stride SBO = (o_t1 - o_t0)*16 B, output-row K groups at LBO = Wp*16 B).
struct TcWgNarrowParams {
    CUtensorMap mapDY[TC_MAXP];
    CUtensorMap mapX[TC_MAXP];
    int box_prefix[TC_MAXP + 1];
    int pt[TC_MAXP], pl[TC_MAXP];
    int nhb[TC_MAXP], nwb[TC_MAXP];
    int npatch, BH, kh, kw;
    int nco_blk, boxes_per_split, nsplit;
    int Cout, stages;
    uint32_t tmem_cols;
    float *part;  // [nsplit][Cout][kh][kw][8]
};

__global__ void __launch_bounds__(192, 1) wgrad_narrow_kernel(const __grid_constant__ TcWgNarrowParams p) {
    extern __shared__ uint8_t smem_raw[];
    uint8_t *smem = (uint8_t *)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
    const int S = p.stages;
    const int rows = p.BH * 8;
    const int Wp = 8 + p.kw - 1, Hp = p.BH + p.kh - 1;
    const int KT = p.kh * p.kw, npairs = (KT + 1) / 2;
    const uint32_t a_blk = (uint32_t)rows * 128u;
    // Cout <= 64: one dY channel block per stage; the MMA's upper 64 rows then read the next stage's
    // bytes and produce accumulator rows for channels >= Cout, which are never stored
    const uint32_t a_stage = (p.Cout <= 64 ? 1u : 2u) * a_blk;
    const uint32_t b_bytes = (uint32_t)Wp * Hp * 16u;
    const uint32_t b_stage = (b_bytes + 1023u) & ~1023u;
    uint8_t *sA = smem;
    uint8_t *sB = smem + (size_t)S * a_stage;
    uint64_t *full = (uint64_t *)(sB + (size_t)S * b_stage);
    uint64_t *empty = full + S;
    uint64_t *tfull = empty + S;
    uint32_t *tmem_slot = (uint32_t *)(tfull + 1);
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    if (warp == 0 && lane == 0) {
        for (int s = 0; s < S; ++s) {
            tc::mbar_init(&full[s], 1);
            tc::mbar_init(&empty[s], 1);
        }
        tc::mbar_init(&tfull[0], 1);
        tc::fence_barrier_init();
    }
    if (warp == 1) tc::tmem_alloc_dyn(tmem_slot, p.tmem_cols);
    tc::tc_fence_before();
    __syncthreads();
    tc::tc_fence_after();
    const uint32_t tmem_base = *tmem_slot;
    const int co_blk = blockIdx.x % p.nco_blk, z = blockIdx.x / p.nco_blk;
    const int total_boxes = p.box_prefix[p.npatch];
    const int b0 = z * p.boxes_per_split, b1 = min(total_boxes, b0 + p.boxes_per_split);

    if (warp == 0) {
        if (lane == 0) {
            int stage = 0, ql = 0;
            uint32_t ph = 0;
            for (int b = b0; b < b1; ++b) {
                while (b >= p.box_prefix[ql + 1]) ++ql;
                int idx = b - p.box_prefix[ql];
                const int wb = idx % p.nwb[ql];
                idx /= p.nwb[ql];
                const int hb = idx % p.nhb[ql], n = idx / p.nhb[ql];
                const int ow0 = wb * 8, oh0 = hb * p.BH;
                tc::mbar_wait_sleep(&empty[stage], ph ^ 1);
                const bool hi = co_blk * 128 + 64 < p.Cout;     // upper 64-channel block has real channels
                tc::mbar_arrive_expect_tx(&full[stage], (hi ? 2u : 1u) * a_blk + b_bytes);
                uint8_t *a = sA + (size_t)stage * a_stage;
                tc::tma_load_4d(a, &p.mapDY[ql], &full[stage], co_blk * 128, ow0, oh0, n);
                if (hi) tc::tma_load_4d(a + a_blk, &p.mapDY[ql], &full[stage], co_blk * 128 + 64, ow0, oh0, n);
                tc::tma_load_3d(sB + (size_t)stage * b_stage, &p.mapX[ql], &full[stage], 8 * (ow0 - p.pl[ql]),
                                oh0 - p.pt[ql], n);
                if (++stage == S) { stage = 0; ph ^= 1; }
            }
        }
    } else if (warp == 1) {
        {   // converged warp; elect.sync issues
            // per kernel row r: the kw column taps are kw 8-channel MN blocks of ONE MMA (consecutive
            // pixels, SBO = 16 B); output-row K groups at LBO = Wp*16 B; N = kw*8 rounded up to 16
            const int NR = ((p.kw * 8 + 15) / 16) * 16;
            const uint32_t idesc = tc::idesc_bf16(128, NR, 1, 1);
            int stage = 0;
            uint32_t ph = 0;
            for (int b = b0; b < b1; ++b) {
                tc::mbar_wait(&full[stage], ph);
                tc::tc_fence_after();
                const uint32_t a_base = tc::smem_u32(sA + (size_t)stage * a_stage);
                const uint32_t b_base = tc::smem_u32(sB + (size_t)stage * b_stage);
                const uint64_t a0 = tc::smem_desc(a_base, a_blk, 1024, 2);
                const uint64_t bd0 = tc::smem_desc(b_base, (uint32_t)Wp * 16u, 16, 0);
                for (int j = 0; j < rows / 16; ++j)
                    for (int r = 0; r < p.kh; ++r)
                        tc::mma_bf16_ws(tmem_base + (uint32_t)(r * NR), a0 + (uint64_t)(128 * j),
                                        bd0 + (uint64_t)((2 * j + r) * Wp), idesc, (b != b0 || j) ? 1u : 0u);
                tc::mma_commit_ws(&empty[stage]);
                if (++stage == S) { stage = 0; ph ^= 1; }
            }
            tc::mma_commit_ws(&tfull[0]);
        }
    } else {
        const int quad = warp & 3;
        const int co = co_blk * 128 + quad * 32 + lane;
        const bool any = b1 > b0;
        if (any) {
            tc::mbar_wait(&tfull[0], 0);
            tc::tc_fence_after();
        }
        const uint32_t tacc = tmem_base + ((uint32_t)(quad * 32) << 16);
        const int NR = ((p.kw * 8 + 15) / 16) * 16;
        for (int r = 0; r < p.kh; ++r)
            for (int cc = 0; cc < NR; cc += 16) {
                float v[16];
                if (any) {
                    tc::tmem_ld16(tacc + (uint32_t)(r * NR + cc), v);
                } else {
#pragma unroll
                    for (int e = 0; e < 16; ++e) v[e] = 0.f;
                }
                if (co >= p.Cout) continue;
#pragma unroll
                for (int h = 0; h < 2; ++h) {
                    const int c = (cc >> 3) + h;          // column tap of this 8-channel block
                    if (c >= p.kw) break;
                    float4 *d4 = reinterpret_cast<float4 *>(p.part + (((int64_t)z * p.Cout + co) * KT + r * p.kw + c) * 8);
                    d4[0] = make_float4(v[8 * h], v[8 * h + 1], v[8 * h + 2], v[8 * h + 3]);
                    d4[1] = make_float4(v[8 * h + 4], v[8 * h + 5], v[8 * h + 6], v[8 * h + 7]);
                }
            }
    }
    tc::tc_fence_before();
    __syncthreads();
    tc::tc_fence_after();
    if (warp == 1) tc::tmem_dealloc(tmem_base, p.tmem_cols);
}

namespace {

struct WgradCfg {
    TileShape ts;
    int x3d, cbox, nchunk, nblocks, bpt, bpt_pad, ntb, nco_blk, ntiles, total_boxes, nsplit, boxes_per_split;
};

// Split-K count of a weight-gradient launch: enough splits to occupy the SMs, but not more than pays
// for the fp32 partials they write and the reduction reads back (2 * Z * |dW| * 4 bytes of HBM):
// minimise  waves * (boxes per split) * (MMA time per box)  +  partial traffic / HBM bandwidth.
static int choose_splits(long total_boxes, int ntiles, double box_flops, double dw_elems, int zcap) {
    const double sm_flops = 8192.0 * 1.8e9, hbm = 6.0e12;
    int bestZ = 1;
    double best = -1.0;
    for (int Z = 1; Z <= zcap; ++Z) {
        const long bps = (total_boxes + Z - 1) / Z;
        const long nsplit = (total_boxes + bps - 1) / bps;
        const long waves = ((long)ntiles * nsplit + num_sms() - 1) / num_sms();
        const double t = (double)waves * bps * box_flops / sm_flops + 2.0 * nsplit * dw_elems * 4.0 / hbm;
        if (best < 0 || t < best * 0.98) { best = t; bestZ = Z; }
    }
    return bestZ;
}

WgradCfg wgrad_cfg(const Level &Li, const Level &Lo, const LayerGeom &g, int p0, int p1) {
    WgradCfg c{};
    const int N = Lo.N, s = g.L.sh, KT = g.L.kh * g.L.kw;
    c.cbox = std::min(Li.Cpad, 64);
    c.x3d = (c.cbox == 8 && s == 1) ? 1 : 0;
    std::vector<std::pair<int, int>> ext;
    for (int q = p0; q < p1; ++q) ext.push_back({Lo.ph(q / Lo.nw()), Lo.pw(q % Lo.nw())});
    // pixel box of <= 64 rows (WG_ROWS) minimising the box count
    TileShape best{1, 1, 1};
    long best_n = -1;
    int maxh = 1, maxw = 1;
    for (auto &e : ext) { maxh = std::max(maxh, e.first); maxw = std::max(maxw, e.second); }
    const int wlim = std::min(std::min(maxw, WG_ROWS), c.x3d ? 32 : 256 / s);
    for (int bw = 1; bw <= wlim; ++bw)
        for (int bh = 1; bh <= std::min(maxh, 256 / s) && bw * bh <= WG_ROWS; ++bh) {
            const int bn = std::min(WG_ROWS / (bw * bh), N);
            long n = 0;
            for (auto &e : ext) n += (long)((N + bn - 1) / bn) * ((e.first + bh - 1) / bh) * ((e.second + bw - 1) / bw);
            if (best_n < 0 || n < best_n || (n == best_n && bw > best.BW)) { best_n = n; best = {bw, bh, bn}; }
        }
    c.ts = best;
    c.total_boxes = (int)best_n;
    c.nchunk = Li.Cpad / c.cbox;
    c.nblocks = KT * c.nchunk;
    const int maxb = std::min(WG_MAXBLK, 256 / c.cbox);
    c.ntb = (c.nblocks + maxb - 1) / maxb;
    c.bpt = (c.nblocks + c.ntb - 1) / c.ntb;
    c.bpt_pad = c.bpt;
    while ((c.bpt_pad * c.cbox) % 16) ++c.bpt_pad;  // MMA N multiple of 16
    c.nco_blk = (g.L.cout + 127) / 128;
    c.ntiles = c.nco_blk * c.ntb;
    int Z = std::max(1, (2 * num_sms() + c.ntiles - 1) / c.ntiles);
    Z = std::min(Z, std::max(1, c.total_boxes / 4));  // >= 4 boxes per split
    Z = std::min(Z, 296);   // (a single-tile layer takes one split per SM: a cap of 128 left 20 SMs idle)
    Z = choose_splits(c.total_boxes, c.ntiles, 2.0 * 128 * c.bpt_pad * c.cbox * c.ts.BW * c.ts.BH * c.ts.BNn,
                          (double)g.L.cout * KT * Li.Cpad, Z);
    c.boxes_per_split = (c.total_boxes + Z - 1) / Z;
    c.nsplit = (c.total_boxes + c.boxes_per_split - 1) / c.boxes_per_split;
    return c;
}

}  // namespace

namespace {

struct WgHaloCfg {
    int BH, BNn, nco_blk, nchunk, ntiles, total_boxes, nsplit, boxes_per_split, rpack;
};

int wgrad_rpack(const LayerGeom &g) { return (g.L.cout <= 64 && g.L.kh >= 2) ? 1 : 0; }

bool wgrad_halo_ok(const Level &Li, const Level &Lo, const LayerGeom &g) {
    // 16- / 32-channel inputs: one MN block of the level's channels per tap, N = kw * Cpad (a multiple of 16)
    const bool narrow = (Li.Cpad == 16 || Li.Cpad == 32) && (g.L.kw * Li.Cpad) % 16 == 0;
    return g.L.sh == 1 && g.L.sw == 1 && g.L.kw >= 2 && g.L.kw <= 4 && (Li.Cpad % 64 == 0 || narrow) && Lo.Cpad % 64 == 0;
}

WgHaloCfg wgrad_halo_cfg(const Level &Li, const Level &Lo, const LayerGeom &g, int p0, int p1) {
    WgHaloCfg c{};
    long best = -1;
    int maxh = 1;
    c.rpack = wgrad_rpack(g);   // row-pair packing (see TcWgHaloParams)
    for (int q = p0; q < p1; ++q) maxh = std::max(maxh, Lo.ph(q / Lo.nw()) + c.rpack);
    // BH x BNn x 8 pixels per stage (<= 128, a multiple of 16 for the K = 16 MMA steps); row-packed boxes
    // hold one image (its X box is BH + kh - 1 rows tall, so K groups of consecutive images are not Wp apart)
    for (int bh = 1; bh <= std::min(16, maxh); ++bh)
        for (int bn = 1; bn * bh * 8 <= 128 && bn <= (c.rpack ? 1 : Lo.N); ++bn) {
            if ((bh * bn) % 2) continue;
            long n = 0;
            for (int q = p0; q < p1; ++q)
                n += (long)((Lo.N + bn - 1) / bn) * ((Lo.ph(q / Lo.nw()) + c.rpack + bh - 1) / bh) *
                     ((Lo.pw(q % Lo.nw()) + 7) / 8);
            // cost ~ boxes x (fixed per-box cost + MMA rows): fewer, fuller boxes win
            const long cost = n * (bh * bn * 8 + 256);
            if (best < 0 || cost < best) { best = cost; c.BH = bh; c.BNn = bn; c.total_boxes = (int)n; }
        }
    c.nco_blk = (g.L.cout + 127) / 128;
    c.nchunk = std::max(1, Li.Cpad / 64);
    c.ntiles = c.nco_blk * (c.rpack ? 1 : g.L.kh) * c.nchunk;
    int Z = std::max(1, (2 * num_sms() + c.ntiles - 1) / c.ntiles);
    Z = std::min(Z, std::max(1, c.total_boxes / 4));
    Z = std::min(Z, 296);   // (the row-packed 64-channel layers are ONE tile: 148 splits, not 128 -- all SMs)
    Z = choose_splits(c.total_boxes, c.ntiles, 2.0 * 128 * g.L.kw * std::min(64, Li.Cpad) * c.BH * c.BNn * 8,
                          (double)g.L.cout * g.L.kh * g.L.kw * Li.Cpad, Z);
    c.boxes_per_split = (c.total_boxes + Z - 1) / Z;
    c.nsplit = (c.total_boxes + c.boxes_per_split - 1) / c.boxes_per_split;
    return c;
}

}  // namespace

namespace {

struct WgNarrowCfg {
    int BH, nco_blk, total_boxes, nsplit, boxes_per_split;
};

bool wgrad_narrow_ok(const Level &Li, const Level &Lo, const LayerGeom &g) {
    return Li.Cpad == 8 && g.L.sh == 1 && g.L.sw == 1 && g.L.kw <= 8 && g.L.kh * g.L.kw <= 16 && Lo.Cpad % 64 == 0;
}

WgNarrowCfg wgrad_narrow_cfg(const Level &Lo, const LayerGeom &g, int p0, int p1) {
    WgNarrowCfg c{};
    long best = -1;
    for (int bh = 2; bh <= 16; bh += 2) {
        long n = 0;
        for (int q = p0; q < p1; ++q)
            n += (long)Lo.N * ((Lo.ph(q / Lo.nw()) + bh - 1) / bh) * ((Lo.pw(q % Lo.nw()) + 7) / 8);
        const long cost = n * (bh * 8 + 256);
        if (best < 0 || cost < best) { best = cost; c.BH = bh; c.total_boxes = (int)n; }
    }
    c.nco_blk = (g.L.cout + 127) / 128;
    int Z = std::max(1, (2 * num_sms() + c.nco_blk - 1) / c.nco_blk);
    Z = std::min(Z, std::max(1, c.total_boxes / 4));
    Z = std::min(Z, 296);
    c.boxes_per_split = (c.total_boxes + Z - 1) / Z;
    c.nsplit = (c.total_boxes + c.boxes_per_split - 1) / c.boxes_per_split;
    return c;
}

}  // namespace

static bool wgrad_tc_ok(const Level &Li, const Level &Lo, const LayerGeom &g) {
    return a_channels_ok(Li.Cpad) && Lo.Cpad % 64 == 0 && g.L.sh == g.L.sw && g.L.sh <= 2;
}

// which weight-gradient kernel takes a layer: 2 narrow (8-channel input), 1 halo, 0 generic
static int wgrad_path(const Level &Li, const Level &Lo, const LayerGeom &g) {
    if (wgrad_narrow_ok(Li, Lo, g)) return 2;
    if (wgrad_halo_ok(Li, Lo, g)) return 1;
    return 0;
}

// upper bound of the split count of ONE launch (any group of <= TC_MAXP patches): see the *_cfg Z caps
static int wgrad_zbound(int path, const Level &Li, const LayerGeom &g) {
    const int nco = (g.L.cout + 127) / 128;
    int ntiles;
    if (path == 2) return std::max(1, std::min(296, (2 * num_sms() + nco - 1) / nco));
    if (path == 1) ntiles = nco * (wgrad_rpack(g) ? 1 : g.L.kh) * std::max(1, Li.Cpad / 64);
    else {
        const int cbox = std::min(Li.Cpad, 64), nblocks = g.L.kh * g.L.kw * (Li.Cpad / cbox);
        const int maxb = std::min(WG_MAXBLK, 256 / cbox);
        ntiles = nco * ((nblocks + maxb - 1) / maxb);
    }
    return std::max(1, std::min(296, (2 * num_sms() + ntiles - 1) / ntiles));
}

size_t wgrad_tc_ws_bytes(const Level &Li, const Level &Lo, const LayerGeom &g) {
    // every launch (group of <= TC_MAXP patches) of a call writes its split partials at its own z
    // offset and ONE fixed-order reduction sums them all: [Zmax][dW]; the db column sums reuse the space
    const int path = wgrad_path(Li, Lo, g);
    const int64_t ngroups = (Lo.npatch() + TC_MAXP - 1) / TC_MAXP;
    const int64_t zmax = ngroups * wgrad_zbound(path, Li, g);
    const int64_t nW = (int64_t)g.L.cout * g.L.kh * g.L.kw * Li.Cpad;
    // + a separate region for the db column-sum partials (computed concurrently, see launch_conv_wgrad_tc)
    const size_t dbp = (((size_t)9 * 4 * 148 * g.L.cout * sizeof(float)) + 255) & ~(size_t)255;   // colsum rows + folded rows
    return (((size_t)zmax * nW * sizeof(float) + 255) & ~(size_t)255) + dbp + 256;
}

// Library-owned side stream per device and host thread (fork/join through events, so the caller's stream
// semantics are kept, and CUDA-graph capture records the fork as a parallel branch; per thread, so two host
// threads never interleave records of the same fork / join event).
struct SideStream {
    cudaStream_t s = nullptr;
    cudaEvent_t fork = nullptr, join = nullptr;
};
static SideStream &side_stream() {
    static thread_local SideStream ss[16];
    int dev = 0;
    cudaGetDevice(&dev);
    SideStream &r = ss[dev & 15];
    if (!r.s) {
        cudaStreamCreateWithFlags(&r.s, cudaStreamNonBlocking);
        cudaEventCreateWithFlags(&r.fork, cudaEventDisableTiming);
        cudaEventCreateWithFlags(&r.join, cudaEventDisableTiming);
    }
    return r;
}

int launch_db_partials(splitcnn_dtype_t dt, const Level &Lo, const void *dy, float *part, int cout, int p0, int p1,
                       cudaStream_t st);
void launch_reduce(const float *part, int Z, int64_t n, float *out, float beta, cudaStream_t st);

splitcnn_status_t launch_conv_wgrad_tc(const Level &Li, const Level &Lo, const LayerGeom &g, const void *x, const void *dy,
                                       float *dw, float *db, float beta, void *ws, int p0, int p1, cudaStream_t st) {
    if (!get_encode()) return fail(SPLITCNN_ERR_CUDA, "cuTensorMapEncodeTiled unavailable");
    auto encode = encode_cached;
    const int KT = g.L.kh * g.L.kw, s = g.L.sh;
    const int64_t nW = (int64_t)g.L.cout * KT * Li.Cpad;
    float *part = (float *)ws;
    static bool attr_set = false;
    const int path = wgrad_path(Li, Lo, g);
    const int64_t zcap = (int64_t)((Lo.npatch() + TC_MAXP - 1) / TC_MAXP) * wgrad_zbound(path, Li, g);
    int zoff = 0;   // split partials written so far (all launches of this call)
    int gend = p1;  // end of the patch range left for the generic kernel
    // db = column sums of dY: HBM-bound, while the wgrad GEMM is not -- run it concurrently on a side
    // stream (forked after dY's producer, joined before this call returns), into its own partial region
    float *part_db = (float *)((char *)ws + ((((size_t)zcap * nW * sizeof(float)) + 255) & ~(size_t)255));
    SideStream *ss = nullptr;
    if (db) {
        ss = &side_stream();
        cudaEventRecord(ss->fork, st);
        cudaStreamWaitEvent(ss->s, ss->fork, 0);
    }
    // every exit joins the side stream back into the caller's (error returns included: an unjoined fork
    // would invalidate a graph capture and let the db partials race with the next call's workspace)
    struct Join {
        SideStream *ss;
        cudaStream_t st;
        ~Join() {
            if (!ss) return;
            cudaEventRecord(ss->join, ss->s);
            cudaStreamWaitEvent(st, ss->join, 0);
        }
    } join_guard{ss, st};
    bool db_launched = false;
    auto launch_db = [&]() {
        if (!db || db_launched) return;
        db_launched = true;
        const int Zd = launch_db_partials(SPLITCNN_BF16, Lo, dy, part_db, g.L.cout, p0, p1, ss->s);
        launch_reduce(part_db, Zd, g.L.cout, db, beta, ss->s);
    };
    if (path == 2) {
        static bool narrow_attr = false;
        for (int g0 = p0; g0 < p1; g0 += TC_MAXP) {
            const int g1 = std::min(p1, g0 + TC_MAXP);
            WgNarrowCfg c = wgrad_narrow_cfg(Lo, g, g0, g1);
            static thread_local TcWgNarrowParams P;
            std::memset(&P, 0, sizeof(P));
            P.npatch = g1 - g0;
            P.BH = c.BH; P.kh = g.L.kh; P.kw = g.L.kw;
            P.nco_blk = c.nco_blk; P.boxes_per_split = c.boxes_per_split; P.nsplit = c.nsplit;
            P.Cout = g.L.cout;
            const int Wp = 8 + g.L.kw - 1, Hp = c.BH + g.L.kh - 1;
            const uint32_t a_stage = (g.L.cout <= 64 ? 1u : 2u) * c.BH * 8u * 128u;
            const uint32_t b_stage = ((uint32_t)Wp * Hp * 16u + 1023u) & ~1023u;
            const uint32_t stage_bytes = a_stage + b_stage;
            // two co-resident CTAs per SM (grid = 2 x SMs) hide each other's TMA latency when the
            // stages fit in half the shared memory
            const uint32_t budget = (4u * stage_bytes <= 100u * 1024u) ? 100u * 1024u : 200u * 1024u;
            P.stages = std::min<int>(8, (int)(budget / stage_bytes));
            uint32_t cols = 32;
            while (cols < (uint32_t)(g.L.kh * (((g.L.kw * 8 + 15) / 16) * 16))) cols <<= 1;
            P.tmem_cols = cols;
            P.part = part + (int64_t)zoff * nW;
            int boxes = 0;
            for (int q = g0; q < g1; ++q) {
                const int ql = q - g0, i = q / Lo.nw(), j = q % Lo.nw();
                const int ho = Lo.ph(i), wo = Lo.pw(j), hp = Li.ph(i), wp = Li.pw(j);
                P.pt[ql] = g.pad_h[2 * i];
                P.pl[ql] = g.pad_w[2 * j];
                P.nhb[ql] = (ho + c.BH - 1) / c.BH;
                P.nwb[ql] = (wo + 7) / 8;
                P.box_prefix[ql] = boxes;
                boxes += Lo.N * P.nhb[ql] * P.nwb[ql];
                {
                    const int C = Lo.Cpad;
                    void *base = (char *)dy + Lo.offset(i, j) * 2;
                    cuuint64_t dims[4] = {(cuuint64_t)C, (cuuint64_t)wo, (cuuint64_t)ho, (cuuint64_t)Lo.N};
                    cuuint64_t strides[3] = {(cuuint64_t)C * 2, (cuuint64_t)wo * C * 2, (cuuint64_t)ho * wo * C * 2};
                    cuuint32_t box[4] = {64, 8, (cuuint32_t)c.BH, 1};
                    cuuint32_t es[4] = {1, 1, 1, 1};
                    if (encode(&P.mapDY[ql], CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 4, base, dims, strides, box, es,
                               CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                               CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS)
                        return fail(SPLITCNN_ERR_CUDA, "cuTensorMapEncodeTiled(dY narrow) failed");
                }
                {
                    void *base = (char *)x + Li.offset(i, j) * 2;
                    cuuint64_t d3[3] = {(cuuint64_t)wp * 8, (cuuint64_t)hp, (cuuint64_t)Li.N};
                    cuuint64_t s3[2] = {(cuuint64_t)wp * 16, (cuuint64_t)hp * wp * 16};
                    cuuint32_t b3[3] = {(cuuint32_t)(8 * Wp), (cuuint32_t)Hp, 1};
                    cuuint32_t e3[3] = {1, 1, 1};
                    if (encode(&P.mapX[ql], CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 3, base, d3, s3, b3, e3,
                               CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                               CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS)
                        return fail(SPLITCNN_ERR_CUDA, "cuTensorMapEncodeTiled(X narrow) failed");
                }
            }
            P.box_prefix[P.npatch] = boxes;
            const size_t smem = 1024 + (size_t)P.stages * stage_bytes + 256;
            if (!narrow_attr) {
                cudaFuncSetAttribute(wgrad_narrow_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024);
                narrow_attr = true;
            }
            wgrad_narrow_kernel<<<c.nco_blk * c.nsplit, 192, smem, st>>>(P);
            count_launch();
            launch_db();
            cudaError_t e = cudaGetLastError();
            if (e != cudaSuccess) return fail(SPLITCNN_ERR_CUDA, std::string("wgrad_narrow_kernel: ") + cudaGetErrorString(e));
            zoff += c.nsplit;
        }
        gend = p0;
    } else if (path == 1) {
        static bool halo_attr = false;
        for (int g0 = p0; g0 < p1; g0 += TC_MAXP) {
            const int g1 = std::min(p1, g0 + TC_MAXP);
            WgHaloCfg c = wgrad_halo_cfg(Li, Lo, g, g0, g1);
            static thread_local TcWgHaloParams P;
            std::memset(&P, 0, sizeof(P));
            P.npatch = g1 - g0;
            P.BH = c.BH; P.BNn = c.BNn; P.kh = g.L.kh; P.kw = g.L.kw;
            P.nco_blk = c.nco_blk; P.nchunk = c.nchunk; P.ntiles = c.ntiles;
            P.boxes_per_split = c.boxes_per_split; P.nsplit = c.nsplit;
            P.Cout = g.L.cout; P.Cpi = Li.Cpad;
            P.rpack = c.rpack;
            // 2-CTA pairs of 128-channel output blocks when the channels pair up
            const bool cta2 = g.L.cout % 256 == 0 && Li.Cpad % 64 == 0;
            if (cta2) P.ntiles = c.ntiles / 2;
            const int Wp = 8 + g.L.kw - 1;
            P.xrow = cta2 ? 64u : (uint32_t)std::min(Li.Cpad, 64) * 2u;
            const uint32_t a_stage = (g.L.cout <= 64 && !c.rpack ? 1u : 2u) * c.BH * c.BNn * 8u * 128u;
            const int xh = c.rpack ? c.BH + g.L.kh - 1 : c.BH;
            const uint32_t b_stage = ((uint32_t)Wp * xh * c.BNn * P.xrow + 1023u) & ~1023u;
            const uint32_t stage_bytes = a_stage + b_stage;
            P.stages = std::min<int>(8, (int)((200u * 1024u) / stage_bytes));
            P.tmem_cols = c.rpack ? 512 : 256;
            P.part = part + (int64_t)zoff * nW;
            int boxes = 0;
            for (int q = g0; q < g1; ++q) {
                const int ql = q - g0, i = q / Lo.nw(), j = q % Lo.nw();
                const int ho = Lo.ph(i), wo = Lo.pw(j), hp = Li.ph(i), wp = Li.pw(j);
                P.pt[ql] = g.pad_h[2 * i];
                P.pl[ql] = g.pad_w[2 * j];
                P.nhb[ql] = (ho + c.rpack + c.BH - 1) / c.BH;
                P.nwb[ql] = (wo + 7) / 8;
                P.box_prefix[ql] = boxes;
                boxes += ((Lo.N + c.BNn - 1) / c.BNn) * P.nhb[ql] * P.nwb[ql];
                {
                    const int C = Lo.Cpad;
                    void *base = (char *)dy + Lo.offset(i, j) * 2;
                    cuuint64_t dims[4] = {(cuuint64_t)C, (cuuint64_t)wo, (cuuint64_t)ho, (cuuint64_t)Lo.N};
                    cuuint64_t strides[3] = {(cuuint64_t)C * 2, (cuuint64_t)wo * C * 2, (cuuint64_t)ho * wo * C * 2};
                    cuuint32_t box[4] = {64, 8, (cuuint32_t)c.BH, (cuuint32_t)c.BNn};
                    cuuint32_t es[4] = {1, 1, 1, 1};
                    if (encode(&P.mapDY[ql], CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 4, base, dims, strides, box, es,
                               CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                               CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS)
                        return fail(SPLITCNN_ERR_CUDA, "cuTensorMapEncodeTiled(dY halo) failed");
                }
                {
                    const int C = Li.Cpad;
                    void *base = (char *)x + Li.offset(i, j) * 2;
                    cuuint64_t dims[4] = {(cuuint64_t)C, (cuuint64_t)wp, (cuuint64_t)hp, (cuuint64_t)Li.N};
                    cuuint64_t strides[3] = {(cuuint64_t)C * 2, (cuuint64_t)wp * C * 2, (cuuint64_t)hp * wp * C * 2};
                    cuuint32_t box[4] = {P.xrow / 2u, (cuuint32_t)Wp, (cuuint32_t)xh, (cuuint32_t)c.BNn};
                    cuuint32_t es[4] = {1, 1, 1, 1};
                    if (encode(&P.mapX[ql], CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 4, base, dims, strides, box, es,
                               CU_TENSOR_MAP_INTERLEAVE_NONE, swz_for((int)P.xrow),
                               CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS)
                        return fail(SPLITCNN_ERR_CUDA, "cuTensorMapEncodeTiled(X halo) failed");
                }
            }
            P.box_prefix[P.npatch] = boxes;
            const size_t smem = 1024 + (size_t)P.stages * stage_bytes + 256;
            if (!halo_attr) {
                cudaFuncSetAttribute(wgrad_halo_kernel<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024);
                cudaFuncSetAttribute(wgrad_halo_kernel<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024);
                halo_attr = true;
            }
            if (cta2) {
                cudaLaunchConfig_t cfg = {};
                cfg.gridDim = dim3((unsigned)(2 * P.ntiles * c.nsplit));
                cfg.blockDim = dim3(192);
                cfg.dynamicSmemBytes = smem;
                cfg.stream = st;
                cudaLaunchAttribute at[1];
                at[0].id = cudaLaunchAttributeClusterDimension;
                at[0].val.clusterDim.x = 2;
                at[0].val.clusterDim.y = 1;
                at[0].val.clusterDim.z = 1;
                cfg.attrs = at;
                cfg.numAttrs = 1;
                cudaLaunchKernelEx(&cfg, wgrad_halo_kernel<true>, P);
            } else {
                wgrad_halo_kernel<false><<<c.ntiles * c.nsplit, 192, smem, st>>>(P);
            }
            count_launch();
            launch_db();
            cudaError_t e = cudaGetLastError();
            if (e != cudaSuccess) return fail(SPLITCNN_ERR_CUDA, std::string("wgrad_halo_kernel: ") + cudaGetErrorString(e));
            zoff += c.nsplit;
        }
        gend = p0;  // done: skip the generic path below
    }
    for (int g0 = p0; g0 < gend; g0 += TC_MAXP) {
        const int g1 = std::min(gend, g0 + TC_MAXP);
        WgradCfg c = wgrad_cfg(Li, Lo, g, g0, g1);
        static thread_local TcWgradParams P;
        std::memset(&P, 0, sizeof(P));
        P.npatch = g1 - g0;
        P.BW = c.ts.BW; P.BH = c.ts.BH; P.BNn = c.ts.BNn; P.rows_box = c.ts.BW * c.ts.BH * c.ts.BNn;
        P.kh = g.L.kh; P.kw = g.L.kw; P.s = s;
        P.x3d = c.x3d; P.cbox = c.cbox; P.nchunk = c.nchunk; P.bpt = c.bpt; P.bpt_pad = c.bpt_pad;
        P.nblocks = c.nblocks; P.nco_blk = c.nco_blk; P.ntb = c.ntb; P.ntiles = c.ntiles;
        P.boxes_per_split = c.boxes_per_split; P.nsplit = c.nsplit;
        P.Cout = g.L.cout; P.Cpi = Li.Cpad;
        const uint32_t row_bytes = (uint32_t)c.cbox * 2u;
        P.b_box_bytes = WG_ROWS * row_bytes;
        P.b_layout = layout_for((int)row_bytes);
        if (row_bytes == 16) {        // no swizzle, MN-major: SBO = MN-block stride, LBO = 8-row K-group stride
            P.b_sbo = P.b_box_bytes;
            P.b_lbo = 128;
        } else {                      // swizzled MN-major: LBO = MN-block stride, SBO = 8-row K-group stride
            P.b_lbo = P.b_box_bytes;
            P.b_sbo = 8u * row_bytes;
        }
        P.b_kstep = 16u * row_bytes;
        const uint32_t b_stage_al = ((uint32_t)c.bpt_pad * P.b_box_bytes + 1023u) & ~1023u;
        const uint32_t stage_bytes = 2u * WG_ROWS * 128u + b_stage_al;
        P.stages = std::min<int>(8, (int)((200u * 1024u) / stage_bytes));
        uint32_t cols = 32;
        while (cols < (uint32_t)(c.bpt_pad * c.cbox)) cols <<= 1;
        P.tmem_cols = cols;
        P.part = part + (int64_t)zoff * nW;
        int boxes = 0;
        for (int q = g0; q < g1; ++q) {
            const int ql = q - g0, i = q / Lo.nw(), j = q % Lo.nw();
            const int ho = Lo.ph(i), wo = Lo.pw(j), hp = Li.ph(i), wp = Li.pw(j);
            P.pt[ql] = g.pad_h[2 * i];
            P.pl[ql] = g.pad_w[2 * j];
            P.nhb[ql] = (ho + c.ts.BH - 1) / c.ts.BH;
            P.nwb[ql] = (wo + c.ts.BW - 1) / c.ts.BW;
            P.box_prefix[ql] = boxes;
            boxes += ((Lo.N + c.ts.BNn - 1) / c.ts.BNn) * P.nhb[ql] * P.nwb[ql];
            {
                const int C = Lo.Cpad;
                void *base = (char *)dy + Lo.offset(i, j) * 2;
                cuuint64_t dims[4] = {(cuuint64_t)C, (cuuint64_t)wo, (cuuint64_t)ho, (cuuint64_t)Lo.N};
                cuuint64_t strides[3] = {(cuuint64_t)C * 2, (cuuint64_t)wo * C * 2, (cuuint64_t)ho * wo * C * 2};
                cuuint32_t box[4] = {64, (cuuint32_t)c.ts.BW, (cuuint32_t)c.ts.BH, (cuuint32_t)c.ts.BNn};
                cuuint32_t es[4] = {1, 1, 1, 1};
                if (encode(&P.mapDY[ql], CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 4, base, dims, strides, box, es,
                           CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                           CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS)
                    return fail(SPLITCNN_ERR_CUDA, "cuTensorMapEncodeTiled(dY) failed");
            }
            {
                const int C = Li.Cpad;
                void *base = (char *)x + Li.offset(i, j) * 2;
                CUresult r;
                if (c.x3d) {  // 8-channel pixels merged into rows: dims (8*wp, hp, N), box (8*BW, BH, BNn)
                    cuuint64_t dims[3] = {(cuuint64_t)wp * 8, (cuuint64_t)hp, (cuuint64_t)Li.N};
                    cuuint64_t strides[2] = {(cuuint64_t)wp * 16, (cuuint64_t)hp * wp * 16};
                    cuuint32_t box[3] = {(cuuint32_t)(c.ts.BW * 8), (cuuint32_t)c.ts.BH, (cuuint32_t)c.ts.BNn};
                    cuuint32_t es[3] = {1, 1, 1};
                    r = encode(&P.mapX[ql], CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 3, base, dims, strides, box, es,
                               CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                               CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
                } else {
                    cuuint64_t dims[4] = {(cuuint64_t)C, (cuuint64_t)wp, (cuuint64_t)hp, (cuuint64_t)Li.N};
                    cuuint64_t strides[3] = {(cuuint64_t)C * 2, (cuuint64_t)wp * C * 2, (cuuint64_t)hp * wp * C * 2};
                    cuuint32_t box[4] = {(cuuint32_t)c.cbox, (cuuint32_t)(c.ts.BW * s), (cuuint32_t)(c.ts.BH * s),
                                         (cuuint32_t)c.ts.BNn};
                    cuuint32_t es[4] = {1, (cuuint32_t)s, (cuuint32_t)s, 1};
                    r = encode(&P.mapX[ql], CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 4, base, dims, strides, box, es,
                               CU_TENSOR_MAP_INTERLEAVE_NONE, swz_for((int)row_bytes), CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                               CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
                }
                if (r != CUDA_SUCCESS) return fail(SPLITCNN_ERR_CUDA, "cuTensorMapEncodeTiled(X) failed");
            }
        }
        P.box_prefix[P.npatch] = boxes;
        const size_t smem = 1024 + (size_t)P.stages * stage_bytes + 256;
        if (!attr_set) {
            cudaFuncSetAttribute(wgrad_tc_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024);
            attr_set = true;
        }
        wgrad_tc_kernel<<<c.ntiles * c.nsplit, 192, smem, st>>>(P);
        count_launch();
        launch_db();
        cudaError_t e = cudaGetLastError();
        if (e != cudaSuccess) return fail(SPLITCNN_ERR_CUDA, std::string("wgrad_tc_kernel: ") + cudaGetErrorString(e));
        zoff += c.nsplit;
    }
    if (zoff > zcap) return fail(SPLITCNN_ERR_UNSUPPORTED, "wgrad split partials exceed the workspace bound");
    // ONE fixed-order sum of every launch's split partials (z ascending) into dW: bitwise
    // reproducible, and beta = 1 gives exactly 2x whatever the number of launches
    launch_reduce(part, zoff, nW, dw, beta, st);
    if (db) {
        launch_db();                              // (no GEMM launch when the range is empty; join: join_guard)
        cudaError_t e = cudaGetLastError();
        if (e != cudaSuccess) return fail(SPLITCNN_ERR_CUDA, std::string("db column sums: ") + cudaGetErrorString(e));
    }
    return SPLITCNN_OK;
}


// ============================================================ fp32 storage on the tensor cores
// SPLITCNN_TF32: one kind::tf32 pass (operands truncated to TF32 by the MMA, fp32 accumulate).
// SPLITCNN_FP32 (fp32-accurate): 3xTF32 -- each operand v = hi + lo with hi = v with the low 13 mantissa
// bits cleared (exactly a TF32 value) and lo = v - hi (exact in fp32); y = lo*W_hi + hi*W_lo + hi*W_hi
// as three kind::tf32 passes accumulated in fp32 by the direct epilogue (small terms first; bias, ReLU
// and the dgrad mask after the last pass).  The dropped lo*lo term and lo's own TF32 truncation are
// ~2^-22 of the product.
// Weight gradients: bf16 operand splitting on the bf16 wgrad kernels -- v = v1 + v2 (+ v3), v_k bf16
// (v1 = bf16(v), v2 = bf16(v - v1), v3 = bf16(v - v1 - v2)); every bf16 x bf16 product is exact in fp32,
// and the pair products summed are those of i + j <= 1 (TF32, 3 products, ~2^-16 of each product) or
// i + j <= 2 (FP32, 6 products, ~2^-24).  db = sum of dY in fp32.

__global__ void tf32_hilo_kernel(const float4 *__restrict__ x, float4 *__restrict__ hi, float4 *__restrict__ lo, int64_t n4) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n4; i += (int64_t)gridDim.x * blockDim.x) {
        const float4 v = x[i];
        float4 h;
        h.x = __uint_as_float(__float_as_uint(v.x) & 0xFFFFE000u);
        h.y = __uint_as_float(__float_as_uint(v.y) & 0xFFFFE000u);
        h.z = __uint_as_float(__float_as_uint(v.z) & 0xFFFFE000u);
        h.w = __uint_as_float(__float_as_uint(v.w) & 0xFFFFE000u);
        hi[i] = h;
        lo[i] = make_float4(v.x - h.x, v.y - h.y, v.z - h.z, v.w - h.w);
    }
}

__global__ void bf16_terms_kernel(const float4 *__restrict__ x, __nv_bfloat16 *__restrict__ t, int64_t n4, int64_t stride,
                                  int nterms) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n4; i += (int64_t)gridDim.x * blockDim.x) {
        float r[4];
        const float4 v = x[i];
        r[0] = v.x; r[1] = v.y; r[2] = v.z; r[3] = v.w;
        for (int k = 0; k < nterms; ++k) {
            __nv_bfloat16 b[4];
#pragma unroll
            for (int e = 0; e < 4; ++e) {
                b[e] = __float2bfloat16_rn(r[e]);
                r[e] -= __bfloat162float(b[e]);      // exact: the bf16 value is the leading part of r
            }
            *reinterpret_cast<uint2 *>(t + k * stride + 4 * i) = *reinterpret_cast<const uint2 *>(b);
        }
    }
}

static size_t al256(size_t b) { return (b + 255) & ~(size_t)255; }
#define F32TC_TRY(x)                              \
    do {                                          \
        const splitcnn_status_t r_ = (x);         \
        if (r_ != SPLITCNN_OK) return r_;         \
    } while (0)

static void hilo(const float *x, float *hi, float *lo, int64_t n, cudaStream_t st) {
    if (n <= 0) return;
    const int64_t n4 = n / 4;       // levels and weights hold multiples of 8 elements
    tf32_hilo_kernel<<<(unsigned)std::max<int64_t>(1, std::min<int64_t>((n4 + 255) / 256, 148 * 16)), 256, 0, st>>>(
        (const float4 *)x, (float4 *)hi, (float4 *)lo, n4);
    count_launch();
}

static void bf16_terms(const float *x, __nv_bfloat16 *t, int64_t n, int64_t stride, int nterms, cudaStream_t st) {
    if (n <= 0) return;
    const int64_t n4 = n / 4;
    bf16_terms_kernel<<<(unsigned)std::max<int64_t>(1, std::min<int64_t>((n4 + 255) / 256, 148 * 16)), 256, 0, st>>>(
        (const float4 *)x, t, n4, stride, nterms);
    count_launch();
}

static int64_t lvl_off(const Level &L, int q) { return q >= L.npatch() ? L.total() : L.offset(q / L.nw(), q % L.nw()); }

size_t f32tc_ws_bytes(int op, splitcnn_dtype_t dt, const Level &Li, const Level &Lo, const LayerGeom &g) {
    const size_t wf = (size_t)g.L.cout * g.L.kh * g.L.kw * Li.Cpad * 4;              // forward weights, fp32
    const size_t wb = (size_t)g.L.cin * g.L.kh * g.L.kw * Lo.Cpad * 4;               // flipped (dgrad) weights
    if (op == 0) return dt == SPLITCNN_FP32 ? 2 * al256((size_t)Li.total() * 4) + 2 * al256(wf) : 0;
    if (op == 1) {
        const size_t flip = al256(conv_tc_ws_bytes(1, Li, Lo, g, dt));
        return dt == SPLITCNN_FP32 ? flip + 2 * al256((size_t)Lo.total() * 4) + 2 * al256(wb) : flip;
    }
    const int nt = dt == SPLITCNN_TF32 ? 2 : 3;
    return nt * al256((size_t)Li.total() * 2) + nt * al256((size_t)Lo.total() * 2) + al256(wgrad_tc_ws_bytes(Li, Lo, g)) +
           al256((size_t)9 * 4 * 148 * g.L.cout * sizeof(float));
}

splitcnn_status_t launch_conv_fwd_f32tc(splitcnn_dtype_t dt, const Level &Li, const Level &Lo, const LayerGeom &g,
                                        const void *x, const void *w, const float *bias, void *y, int relu, int p0, int p1,
                                        void *ws, cudaStream_t st) {
    if (dt == SPLITCNN_TF32) return launch_conv_fwd_tc(Li, Lo, g, x, w, bias, y, relu, p0, p1, st, SPLITCNN_TF32, 0);
    const int64_t nw = (int64_t)g.L.cout * g.L.kh * g.L.kw * Li.Cpad;
    char *p = (char *)ws;
    float *xhi = (float *)p; p += al256((size_t)Li.total() * 4);
    float *xlo = (float *)p; p += al256((size_t)Li.total() * 4);
    float *whi = (float *)p; p += al256((size_t)nw * 4);
    float *wlo = (float *)p;
    const int64_t o0 = lvl_off(Li, p0), o1 = lvl_off(Li, p1);
    hilo((const float *)x + o0, xhi + o0, xlo + o0, o1 - o0, st);
    hilo((const float *)w, whi, wlo, nw, st);
    F32TC_TRY(launch_conv_fwd_tc(Li, Lo, g, xlo, whi, nullptr, y, 0, p0, p1, st, SPLITCNN_TF32, 0));
    F32TC_TRY(launch_conv_fwd_tc(Li, Lo, g, xhi, wlo, nullptr, y, 0, p0, p1, st, SPLITCNN_TF32, 1));
    return launch_conv_fwd_tc(Li, Lo, g, xhi, whi, bias, y, relu, p0, p1, st, SPLITCNN_TF32, 1);
}

splitcnn_status_t launch_conv_dgrad_f32tc(splitcnn_dtype_t dt, const Level &Li, const Level &Lo, const LayerGeom &g,
                                          const void *dy, const void *w, void *dx, const void *relu_src, int p0, int p1,
                                          void *ws, cudaStream_t st) {
    if (dt == SPLITCNN_TF32) return launch_conv_dgrad_tc(Li, Lo, g, dy, w, dx, relu_src, ws, p0, p1, st, SPLITCNN_TF32, 0);
    const int kh = g.L.kh, kw = g.L.kw;
    const int64_t nw = (int64_t)g.L.cin * kh * kw * Lo.Cpad;
    char *p = (char *)ws;
    float *wt = (float *)p; p += al256(conv_tc_ws_bytes(1, Li, Lo, g, dt));
    float *ghi = (float *)p; p += al256((size_t)Lo.total() * 4);
    float *glo = (float *)p; p += al256((size_t)Lo.total() * 4);
    float *whi = (float *)p; p += al256((size_t)nw * 4);
    float *wlo = (float *)p;
    flip_weights<float>(w, wt, g, Li.Cpad, Lo.Cpad, 0, 0, 1, kh, kw, st);
    const int64_t o0 = lvl_off(Lo, p0), o1 = lvl_off(Lo, p1);
    hilo((const float *)dy + o0, ghi + o0, glo + o0, o1 - o0, st);
    hilo(wt, whi, wlo, nw, st);
    F32TC_TRY(launch_tc(1, Lo, Li, g, glo, whi, g.L.cin, nullptr, dx, nullptr, 0, p0, p1, st, nullptr, nullptr, 1, 0));
    F32TC_TRY(launch_tc(1, Lo, Li, g, ghi, wlo, g.L.cin, nullptr, dx, nullptr, 0, p0, p1, st, nullptr, nullptr, 1, 1));
    return launch_tc(1, Lo, Li, g, ghi, whi, g.L.cin, nullptr, dx, relu_src, 0, p0, p1, st, nullptr, nullptr, 1, 1);
}

splitcnn_status_t launch_conv_wgrad_f32tc(splitcnn_dtype_t dt, const Level &Li, const Level &Lo, const LayerGeom &g,
                                          const void *x, const void *dy, float *dw, float *db, float beta, void *ws,
                                          int p0, int p1, cudaStream_t st) {
    const int nt = dt == SPLITCNN_TF32 ? 2 : 3;
    char *p = (char *)ws;
    const int64_t sx = (int64_t)(al256((size_t)Li.total() * 2) / 2), sg = (int64_t)(al256((size_t)Lo.total() * 2) / 2);
    __nv_bfloat16 *xt = (__nv_bfloat16 *)p; p += nt * sx * 2;
    __nv_bfloat16 *gt = (__nv_bfloat16 *)p; p += nt * sg * 2;
    void *wgws = p; p += al256(wgrad_tc_ws_bytes(Li, Lo, g));
    float *partdb = (float *)p;
    const int64_t xo0 = lvl_off(Li, p0), xo1 = lvl_off(Li, p1), go0 = lvl_off(Lo, p0), go1 = lvl_off(Lo, p1);
    bf16_terms((const float *)x + xo0, xt + xo0, xo1 - xo0, sx, nt, st);
    bf16_terms((const float *)dy + go0, gt + go0, go1 - go0, sg, nt, st);
    static const int prs[6][2] = {{0, 0}, {0, 1}, {1, 0}, {0, 2}, {1, 1}, {2, 0}};
    const int npr = nt == 2 ? 3 : 6;
    for (int k = 0; k < npr; ++k)
        F32TC_TRY(launch_conv_wgrad_tc(Li, Lo, g, xt + prs[k][0] * sx, gt + prs[k][1] * sg, dw, nullptr, k == 0 ? beta : 1.f,
                                 wgws, p0, p1, st));
    if (db) {
        const int Zd = launch_db_partials(SPLITCNN_FP32, Lo, dy, partdb, g.L.cout, p0, p1, st);
        launch_reduce(partdb, Zd, g.L.cout, db, beta, st);
    }
    return SPLITCNN_OK;
}

}  // namespace splitcnn
