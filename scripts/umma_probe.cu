// umma_probe.cu -- hardware probe: can a tcgen05 smem descriptor start at a ROW offset inside a
// 128B-swizzle atom (with or without the descriptor's base-offset field)?  Needed for halo reuse
// (one loaded input tile serving all taps of a 3x3 window through row-shifted operand views).
//
// Case K: A is K-major SW128 (rows = M, 128 B = 64 bf16 of K), shift in M by `off` rows.
// Case MN: A is MN-major SW128 (rows = K, 128 B = 64 bf16 of M), shift in K by `off` rows.
// B is K-major SW128 [N=64][K=64].  One 128 x 64 x 64 product per run, compared with a CPU GEMM.
//   nvcc -gencode arch=compute_100a,code=sm_100a -o /tmp/umma_probe scripts/umma_probe.cu && /tmp/umma_probe
#include <cuda_bf16.h>
#include <cstdio>
#include <cstdlib>
#include <cstdint>
#include <cmath>
#include <vector>

__device__ __forceinline__ uint32_t s32(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }

__device__ __forceinline__ uint64_t desc(uint32_t saddr, uint32_t lbo, uint32_t sbo, uint32_t layout, uint32_t base_off) {
    uint64_t d = 0;
    d |= (uint64_t)((saddr >> 4) & 0x3FFF);
    d |= (uint64_t)((lbo >> 4) & 0x3FFF) << 16;
    d |= (uint64_t)((sbo >> 4) & 0x3FFF) << 32;
    d |= (uint64_t)1 << 46;
    d |= (uint64_t)(base_off & 7) << 49;
    d |= (uint64_t)(layout & 7) << 61;
    return d;
}

// mode 0: A K-major (global A is [rowsA][64] with K contiguous); mode 1: A MN-major (global A is [rowsK][64 M... 128 M in 2 blocks])
__global__ void probe(const __nv_bfloat16 *A, const __nv_bfloat16 *B, float *D, int mode, int off, int base_off, int sbo_rows) {
    extern __shared__ __align__(1024) uint8_t smem[];
    uint8_t *sA = smem;                 // up to 2 x 32 KB
    uint8_t *sB = smem + 65536;         // 8 KB
    __shared__ uint64_t bar;
    __shared__ uint32_t tslot;
    const int tid = threadIdx.x;
    // fill smem with the TMA SW128 address-based swizzle: 16B unit u of row r at r*128 + ((u ^ (r&7))*16)
    if (mode == 0) {
        // A: 256 rows x 64 K
        for (int i = tid; i < 256 * 8; i += blockDim.x) {
            const int r = i / 8, u = i % 8;
            *(uint4 *)(sA + r * 128 + ((u ^ (r & 7)) * 16)) = *(const uint4 *)(A + r * 64 + u * 8);
        }
    } else {
        // A MN-major: two M-blocks of 64; each block: 256 K-rows x 64 M (128 B), blocks at 32 KB
        for (int i = tid; i < 2 * 256 * 8; i += blockDim.x) {
            const int blk = i / (256 * 8), rem = i % (256 * 8), r = rem / 8, u = rem % 8;
            *(uint4 *)(sA + blk * 32768 + r * 128 + ((u ^ (r & 7)) * 16)) = *(const uint4 *)(A + (blk * 256 + r) * 64 + u * 8);
        }
    }
    for (int i = tid; i < 64 * 8; i += blockDim.x) {
        const int r = i / 8, u = i % 8;
        *(uint4 *)(sB + r * 128 + ((u ^ (r & 7)) * 16)) = *(const uint4 *)(B + r * 64 + u * 8);
    }
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    if (tid == 0) {
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(s32(&bar)));
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    if (tid < 32) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 64;" ::"r"(s32(&tslot)));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    asm volatile("tcgen05.fence::before_thread_sync;");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;");
    const uint32_t tmem = tslot;
    if (tid == 0) {
        // idesc: f32 D, bf16 A/B, A major = mode, B K-major, N=64, M=128
        const uint32_t idesc = (1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)mode << 15) | ((64u >> 3) << 17) | ((128u >> 4) << 24);
        for (int j = 0; j < 4; ++j) {
            uint64_t ad, bd;
            if (mode == 0) ad = desc(s32(sA) + off * 128 + 32 * j, 16, sbo_rows * 128, 2, base_off);
            else ad = desc(s32(sA) + off * 128 + 2048 * j, 32768, 1024, 2, base_off);
            bd = desc(s32(sB) + 32 * j, 16, 1024, 2, 0);
            asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
                         "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(tmem),
                         "l"(ad), "l"(bd), "r"(idesc), "r"(j));
        }
        asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(s32(&bar)));
    }
    asm volatile("{\n\t.reg .pred P1;\nW:\n\tmbarrier.try_wait.parity.shared::cta.b64 P1, [%0], 0;\n\t@!P1 bra W;\n\t}" ::"r"(s32(&bar)));
    asm volatile("tcgen05.fence::after_thread_sync;");
    const int warp = tid / 32, lane = tid % 32;
    for (int c = 0; c < 64; c += 16) {
        uint32_t r[16];
        asm volatile("tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
                     : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
                       "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15])
                     : "r"(tmem + ((uint32_t)(warp * 32) << 16) + c));
        asm volatile("tcgen05.wait::ld.sync.aligned;");
        for (int e = 0; e < 16; ++e) D[(warp * 32 + lane) * 64 + c + e] = __uint_as_float(r[e]);
    }
    asm volatile("tcgen05.fence::before_thread_sync;");
    __syncthreads();
    if (tid < 32) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 64;" ::"r"(tmem));
}

int main() {
    const int nA = 2 * 256 * 64;
    std::vector<__nv_bfloat16> hA(nA), hB(64 * 64);
    std::vector<float> fA(nA), fB(64 * 64);
    srand(1);
    for (int i = 0; i < nA; ++i) { fA[i] = (float)(rand() % 17 - 8) / 8.f; hA[i] = __float2bfloat16(fA[i]); }
    for (int i = 0; i < 64 * 64; ++i) { fB[i] = (float)(rand() % 17 - 8) / 8.f; hB[i] = __float2bfloat16(fB[i]); }
    __nv_bfloat16 *dA, *dB;
    float *dD;
    cudaMalloc(&dA, nA * 2); cudaMalloc(&dB, 64 * 64 * 2); cudaMalloc(&dD, 128 * 64 * 4);
    cudaMemcpy(dA, hA.data(), nA * 2, cudaMemcpyHostToDevice);
    cudaMemcpy(dB, hB.data(), 64 * 64 * 2, cudaMemcpyHostToDevice);
    cudaFuncSetAttribute(probe, cudaFuncAttributeMaxDynamicSharedMemorySize, 80 * 1024);
    std::vector<float> hD(128 * 64);
    for (int mode = 0; mode < 2; ++mode)
        for (int off : {0, 1, 2, 3, 7, 8, 10, 16, 17})
            for (int bo : {0, 1, 2, 3, 7}) {
                if (bo && off == 0) continue;
                cudaMemset(dD, 0, 128 * 64 * 4);
                probe<<<1, 128, 80 * 1024>>>(dA, dB, dD, mode, off, bo, 8);
                cudaError_t e = cudaDeviceSynchronize();
                if (e != cudaSuccess) { printf("mode %d off %d bo %d: CUDA error %s\n", mode, off, bo, cudaGetErrorString(e)); return 1; }
                cudaMemcpy(hD.data(), dD, 128 * 64 * 4, cudaMemcpyDeviceToHost);
                double maxerr = 0;
                for (int m = 0; m < 128; ++m)
                    for (int n = 0; n < 64; ++n) {
                        double ref = 0;
                        for (int k = 0; k < 64; ++k) {
                            double a = mode == 0 ? fA[(m + off) * 64 + k]                       // row m+off, K k
                                                 : fA[((m / 64) * 256 + k + off) * 64 + (m % 64)];  // K row k+off, M m
                            ref += a * fB[n * 64 + k];
                        }
                        maxerr = fmax(maxerr, fabs(ref - hD[m * 64 + n]));
                    }
                printf("mode %s off %2d base_off %d : max|err| = %g %s\n", mode == 0 ? "K-major " : "MN-major", off, bo, maxerr,
                       maxerr < 1e-3 ? "MATCH" : "");
            }
    // K-major A with 8-row M groups SBO = sbo rows apart (halo views): M row m -> A row (m/8)*sbo + m%8 + off
    for (int sbo : {8, 9, 10, 12, 16})
        for (int off : {0, 1, 2, 3}) {
            cudaMemset(dD, 0, 128 * 64 * 4);
            probe<<<1, 128, 80 * 1024>>>(dA, dB, dD, 0, off, 0, sbo);
            cudaDeviceSynchronize();
            cudaMemcpy(hD.data(), dD, 128 * 64 * 4, cudaMemcpyDeviceToHost);
            double maxerr = 0;
            for (int m = 0; m < 128; ++m)
                for (int n = 0; n < 64; ++n) {
                    const int row = (m / 8) * sbo + m % 8 + off;
                    if (row >= 256) continue;
                    double ref = 0;
                    for (int k = 0; k < 64; ++k) ref += fA[row * 64 + k] * fB[n * 64 + k];
                    maxerr = fmax(maxerr, fabs(ref - hD[m * 64 + n]));
                }
            printf("K-major SBO %2d rows off %d : max|err| = %g %s\n", sbo, off, maxerr, maxerr < 1e-3 ? "MATCH" : "");
        }
    return 0;
}
