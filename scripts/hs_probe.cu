// Per-tile handshake cost of the warp-specialised conv kernel's MMA <-> epilogue pipeline, isolated from
// loads and stores: one CTA per SM, warp 1 issues `kmma` groups of 4 tcgen05.mma 128x64x16 (operands
// resident, zero) per tile into one of 2*nacc TMEM accumulators and commits; two 4-warp epilogue groups
// take alternate tiles: wait, [tcgen05.ld 64 columns + st.shared 128 B per row], arrive.  flags: 1 named
// barriers per tile (as the staging epilogue), 2 TMEM -> smem copy, 4 fence.proxy.async per tile,
// 8 bulk store of the 16 KB staging tile to global memory (a 2 GB ring), 16 wait for the previous store's
// smem reads before refilling the staging tile (as the real epilogue), 32 a ring of 4 staging tiles per
// group (wait for the store 3 back instead of the last one).
// mflags (MMA side): 1 no accumulator-empty wait (epilogue off), 2 no tcgen05 fence after the wait,
// 4 accumulate flag always 1, 8 one accumulator for every tile, 16 no per-tile commit (one at the end),
// 32 two issuing warps (warps 1 and 0 take alternate tiles, each with its own accumulators and commits).
//   nvcc -gencode arch=compute_100a,code=sm_100a -I paper_conf_asplos_jinh19_b200/csrc -o /tmp/hs scripts/hs_probe.cu
#include <cstdio>
#include <cstdint>
#include <cstdlib>
#include "tc_ptx.cuh"

using namespace splitcnn;

__global__ void __launch_bounds__(320, 1) hs(int tiles, int kmma, int nacc, int flags, int mflags, unsigned long long *cyc, uint8_t *gout, long long gbytes) {
    extern __shared__ uint8_t smem_raw[];
    uint8_t *smem = smem_raw + ((1024u - (tc::smem_u32(smem_raw) & 1023u)) & 1023u);
    uint8_t *sA = smem;            // 128 x 128 B
    uint8_t *sB = smem + 16384;    // 64 x 128 B
    uint8_t *sY = smem + 32768;    // 8 staging tiles of 128 x 128 B
    __shared__ __align__(8) uint64_t tfull[8], tempty[8], done[2];
    __shared__ uint32_t slot;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    for (int i = threadIdx.x; i < 32768 / 16; i += blockDim.x) reinterpret_cast<uint4 *>(smem)[i] = make_uint4(0, 0, 0, 0);
    if (threadIdx.x == 0) {
        for (int a = 0; a < 8; ++a) { tc::mbar_init(&tfull[a], 1); tc::mbar_init(&tempty[a], 4); }
        tc::mbar_init(&done[0], 1);
        tc::mbar_init(&done[1], 1);
        tc::fence_barrier_init();
    }
    const uint32_t cols = 2u * nacc * 64u < 32u ? 32u : (2u * nacc * 64u);
    if (warp == 1) tc::tmem_alloc_dyn(&slot, cols);
    tc::fence_proxy_async_smem();
    tc::tc_fence_before();
    __syncthreads();
    tc::tc_fence_after();
    const uint32_t tb = slot;
    const unsigned long long t0 = clock64();
    if (warp == 1 || (warp == 0 && (mflags & 32))) {
        const int tstep = (mflags & 32) ? 2 : 1, tstart = (mflags & 32) ? (warp == 1 ? 0 : 1) : 0;
        const uint32_t idesc = tc::idesc_bf16(128, 64);
        const uint64_t a0 = tc::smem_desc(tc::smem_u32(sA), 16, 1024, 2);
        const uint64_t b0 = tc::smem_desc(tc::smem_u32(sB), 16, 1024, 2);
        for (int t = tstart; t < tiles; t += tstep) {
            const int g = t & 1, k = t >> 1, j = nacc == 1 ? 0 : k & 1, u = nacc == 1 ? k : k >> 1, s = g * nacc + j;
            if (!(mflags & 1)) tc::mbar_wait(&tempty[s], (u & 1) ^ 1);
            if (!(mflags & 2)) tc::tc_fence_after();
            const uint32_t d = tb + (mflags & 8 ? 0u : (uint32_t)s * 64u);
            for (int m = 0; m < kmma; ++m) tc::mma_bf16_x4_ws(d, a0, b0, idesc, (m != 0 || (mflags & 4)) ? 1u : 0u);
            if (!(mflags & 16)) tc::mma_commit_ws(&tfull[s]);
        }
        tc::mma_commit_ws(&done[warp]);
        tc::mbar_wait(&done[warp], 0);
    } else if (warp >= 2 && !(mflags & 1)) {
        const int g = (warp - 2) >> 2, quad = warp & 3, row = quad * 32 + lane;
        for (int t = g, k = 0; t < tiles; t += 2, ++k) {
            const int j = nacc == 1 ? 0 : k & 1, u = nacc == 1 ? k : k >> 1, s = g * nacc + j;
            uint8_t *stg = sY + (g * 4 + ((flags & 32) ? (k & 3) : 0)) * 16384;
            if ((flags & 16) && lane == 0 && warp == 2 + 4 * g) {
                if (flags & 32) tc::bulk_wait_read3();
                else tc::bulk_wait_read0();
            }
            if (flags & 1) tc::named_bar_sync(1 + g, 128);
            tc::mbar_wait(&tfull[s], u & 1);
            tc::tc_fence_after();
            if (flags & 2) {
                const uint32_t ta = tb + (uint32_t)s * 64u + ((uint32_t)(quad * 32) << 16);
                uint8_t *dst = stg + row * 128;
                for (int cc = 0; cc < 64; cc += 32) {
                    uint32_t r[2][16];
                    tc::tmem_ld16_nw(ta + cc, r[0]);
                    tc::tmem_ld16_nw(ta + cc + 16, r[1]);
                    tc::tmem_wait_ld();
#pragma unroll
                    for (int q = 0; q < 4; ++q) {
                        const uint32_t *v = r[q >> 1] + 8 * (q & 1);
                        uint4 o;
                        o.x = v[0] ^ v[1]; o.y = v[2] ^ v[3]; o.z = v[4] ^ v[5]; o.w = v[6] ^ v[7];
                        *reinterpret_cast<uint4 *>(dst + ((cc * 2 + 16 * q) ^ ((row & 7) << 4))) = o;
                    }
                }
            }
            tc::tc_fence_before();
            __syncwarp();
            if (lane == 0) tc::mbar_arrive(&tempty[s]);
            if (flags & 4) tc::fence_proxy_async_smem();
            if (flags & 1) tc::named_bar_sync(1 + g, 128);
            if ((flags & 8) && lane == 0 && warp == 2 + 4 * g) {
                const long long off = (((long long)blockIdx.x * tiles + t) * 16384) % gbytes;
                asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], 16384;" ::"l"(gout + off),
                             "r"(tc::smem_u32(stg)) : "memory");
                tc::bulk_commit();
            }
        }
        if ((flags & 8) && lane == 0 && warp == 2 + 4 * g) tc::bulk_wait0();
    }
    if (threadIdx.x == 32) {
        const unsigned long long t1 = clock64();
        cyc[blockIdx.x] = t1 - t0;
    }
    __syncthreads();
    tc::tc_fence_before();
    __syncthreads();
    tc::tc_fence_after();
    if (warp == 1) tc::tmem_dealloc(tb, cols);
}

int main(int argc, char **argv) {
    const int tiles = 4096;
    unsigned long long *cyc;
    cudaMalloc(&cyc, 148 * sizeof(unsigned long long));
    const size_t smem = 1024 + 32768 + 8 * 16384;
    const long long gbytes = 2048LL << 20;
    uint8_t *gout;
    cudaMalloc(&gout, gbytes);
    cudaFuncSetAttribute(hs, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    struct V { int km, na, fl, mf; };
    const V vs[] = {{9, 2, 31, 32}, {9, 2, 63, 32}, {1, 2, 31, 32}, {1, 2, 63, 32}, {0, 2, 27, 32}, {0, 2, 59, 32},
                    {0, 2, 8, 32}};
    for (const V &v : vs) {
            {
                const int km = v.km, na = v.na, fl = v.fl;
                hs<<<148, 320, smem>>>(tiles, km, na, fl, v.mf, cyc, gout, gbytes);
                cudaEvent_t e0, e1;
                cudaEventCreate(&e0);
                cudaEventCreate(&e1);
                cudaEventRecord(e0);
                hs<<<148, 320, smem>>>(tiles, km, na, fl, v.mf, cyc, gout, gbytes);
                cudaEventRecord(e1);
                cudaEventSynchronize(e1);
                float ms;
                cudaEventElapsedTime(&ms, e0, e1);
                unsigned long long h[148];
                cudaMemcpy(h, cyc, sizeof(h), cudaMemcpyDeviceToHost);
                printf("kmma %d (MMA floor %4d cyc) nacc %d flags %d mflags %2d: %.0f SM cycles per tile (MMA warp clock64), "
                       "%.0f at 1965 MHz from events (%.3f ms) %s\n", km, km * 4 * 48, na, fl, v.mf, (double)h[0] / tiles,
                       ms * 1e-3 * 1.965e9 / tiles, ms, cudaGetErrorString(cudaGetLastError()));
            }
    }
    return 0;
}
