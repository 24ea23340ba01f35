// Raw tcgen05.mma throughput with operands resident in shared memory (no TMA, no epilogue): how fast can the
// tensor core consume SS-mode bf16 MMAs of M = 128 and N = 64 / 128 / 256 (1-CTA), i.e. is the N = 64 conv
// (conv1_2) bound by the MMA's shared-memory operand reads?  One CTA per SM, ITERS x 4 MMAs (K = 64 per
// group of 4) into one TMEM accumulator, one commit.  nvcc -gencode arch=compute_100a,code=sm_100a -I
// paper_conf_asplos_jinh19_b200/csrc -o /tmp/mma_probe scripts/mma_probe.cu && /tmp/mma_probe
#include <cstdio>
#include <cstdint>
#include "tc_ptx.cuh"

using namespace splitcnn;

template <int N>
__global__ void __launch_bounds__(128, 1) probe(int iters, unsigned long long *cyc) {
    extern __shared__ uint8_t smem_raw[];
    uint8_t *smem = smem_raw + ((1024u - (tc::smem_u32(smem_raw) & 1023u)) & 1023u);
    uint8_t *sA = smem;                 // 128 rows x 128 B (64 bf16), SW128 K-major
    uint8_t *sB = smem + 16384;         // N rows x 128 B
    __shared__ __align__(8) uint64_t bar;
    __shared__ uint32_t slot;
    for (int i = threadIdx.x; i < (16384 + N * 128) / 16; i += blockDim.x)
        reinterpret_cast<uint4 *>(smem)[i] = make_uint4(0, 0, 0, 0);
    if (threadIdx.x == 0) { tc::mbar_init(&bar, 1); tc::fence_barrier_init(); }
    if (threadIdx.x < 32) tc::tmem_alloc_dyn(&slot, 512);
    tc::tc_fence_before();
    __syncthreads();
    tc::tc_fence_after();
    const uint32_t d = slot;
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    __syncthreads();
    unsigned long long t0 = clock64();
    if (threadIdx.x < 32) {
        const uint32_t idesc = tc::idesc_bf16(128, N);
        const uint64_t a0 = tc::smem_desc(tc::smem_u32(sA), 16, 1024, 2);
        const uint64_t b0 = tc::smem_desc(tc::smem_u32(sB), 16, 1024, 2);
        for (int i = 0; i < iters; ++i) tc::mma_bf16_x4_ws(d, a0, b0, idesc, i != 0);
        tc::mma_commit_ws(&bar);
        tc::mbar_wait(&bar, 0);
    }
    __syncthreads();
    unsigned long long t1 = clock64();
    if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
    tc::tc_fence_before();
    __syncthreads();
    tc::tc_fence_after();
    if (threadIdx.x < 32) tc::tmem_dealloc(d, 512);
}

template <int N>
void run(int iters) {
    unsigned long long *cyc;
    cudaMalloc(&cyc, 148 * sizeof(unsigned long long));
    const size_t smem = 1024 + 16384 + N * 128;
    cudaFuncSetAttribute(probe<N>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    probe<N><<<148, 128, smem>>>(iters, cyc);
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    cudaEventRecord(e0);
    probe<N><<<148, 128, smem>>>(iters, cyc);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms;
    cudaEventElapsedTime(&ms, e0, e1);
    unsigned long long h[148];
    cudaMemcpy(h, cyc, sizeof(h), cudaMemcpyDeviceToHost);
    const double flop = 2.0 * 128 * N * 64 * (double)iters * 148;
    printf("M=128 N=%3d: %.3f ms, %.1f TFLOP/s, %.0f cycles/SM for %d x 4 MMAs -> %.1f cycles per 128x%dx16 MMA "
           "(floor 128*N/256 = %d), %s\n", N, ms, flop / ms / 1e9, (double)h[0], iters, (double)h[0] / (4.0 * iters), N,
           128 * N / 256, cudaGetErrorString(cudaGetLastError()));
    cudaFree(cyc);
}

int main() {
    run<64>(20000);
    run<128>(10000);
    run<256>(5000);
    return 0;
}
