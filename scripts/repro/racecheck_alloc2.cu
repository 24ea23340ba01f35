// Minimal repro for the compute-sanitizer racecheck reports on the library's 2-CTA kernels: a cluster of two
// CTAs that ONLY allocates tensor memory with tcgen05.alloc.cta_group::2 (address written to shared memory by
// the instruction), fences, cluster-barriers, reads the address, and frees it -- no TMA, no MMA, no other
// shared-memory traffic.  Variant 1 does the same with cta_group::1 and a CTA barrier.
//   nvcc -gencode arch=compute_100a,code=sm_100a -o /tmp/race scripts/repro/racecheck_alloc2.cu
//   compute-sanitizer --tool racecheck /tmp/race N   (N = 1, 2, 3, 4)
#include <cstdio>
#include <cstdint>
#include <cstdlib>

__device__ __forceinline__ uint32_t smem_u32(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }

__global__ void __cluster_dims__(2, 1, 1) alloc2_kernel(uint32_t *out) {
    __shared__ uint32_t slot;
    if (threadIdx.x < 32) {
        asm volatile("tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(&slot)), "r"(64)
                     : "memory");
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::2.sync.aligned;" ::: "memory");
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    asm volatile("barrier.cluster.arrive.aligned; barrier.cluster.wait.aligned;" ::: "memory");
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    const uint32_t taddr = slot;
    if (threadIdx.x == 0) out[blockIdx.x] = taddr;
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    asm volatile("barrier.cluster.arrive.aligned; barrier.cluster.wait.aligned;" ::: "memory");
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    if (threadIdx.x < 32)
        asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, %1;" ::"r"(taddr), "r"(64) : "memory");
}

__global__ void alloc1_kernel(uint32_t *out) {
    __shared__ uint32_t slot;
    if (threadIdx.x < 32) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(&slot)), "r"(64)
                     : "memory");
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    const uint32_t taddr = slot;
    if (threadIdx.x == 0) out[blockIdx.x] = taddr;
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    if (threadIdx.x < 32) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(taddr), "r"(64) : "memory");
}

// variant 3: the cross-CTA mbarrier handshake of the 2-CTA kernels (epilogue -> leader's accumulator-empty
// barrier): CTA 1's thread arrives remotely on CTA 0's mbarrier (mapa + mbarrier.arrive.shared::cluster),
// CTA 0 waits on it with try_wait.parity.  No other shared-memory traffic.
__global__ void __cluster_dims__(2, 1, 1) remote_arrive_kernel(uint32_t *out) {
    __shared__ __align__(8) uint64_t bar;
    uint32_t rank;
    asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(rank));
    if (threadIdx.x == 0) {
        asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(&bar)), "r"(1) : "memory");
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    asm volatile("barrier.cluster.arrive.aligned; barrier.cluster.wait.aligned;" ::: "memory");
    if (rank == 1 && threadIdx.x == 0) {
        uint32_t remote;
        asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(remote) : "r"(smem_u32(&bar)), "r"(0));
        asm volatile("mbarrier.arrive.release.cluster.shared::cluster.b64 _, [%0];" ::"r"(remote) : "memory");
    }
    if (rank == 0 && threadIdx.x == 0) {
        asm volatile("{\n\t.reg .pred P1;\nW:\n\tmbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n\t@!P1 bra W;\n\t}"
                     ::"r"(smem_u32(&bar)), "r"(0) : "memory");
        out[blockIdx.x] = 1;
    }
    asm volatile("barrier.cluster.arrive.aligned; barrier.cluster.wait.aligned;" ::: "memory");
}

// variant 4: the library kernels' exact prologue -- 320 threads, 1024-aligned dynamic shared memory of ~215 KB,
// thread 0 initialising mbarriers next to the TMEM-address slot while warp 1 runs the cta_group::2 alloc, all
// threads staging a bias vector, then the fences + cluster barrier, the read of the slot, and the teardown.
__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(320, 1) prologue_kernel(uint32_t *out, uint32_t bar_off) {
    extern __shared__ uint8_t smem_raw[];
    uint8_t *smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
    uint64_t *bars = (uint64_t *)(smem + bar_off);
    uint32_t *slot = (uint32_t *)(bars + 24);
    float *sbias = (float *)(smem + bar_off + 512);
    const int warp = threadIdx.x >> 5;
    if (threadIdx.x == 0) {
        for (int i = 0; i < 24; ++i)
            asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(&bars[i])), "r"(1) : "memory");
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    for (int i = threadIdx.x; i < 256; i += blockDim.x) sbias[i] = 0.5f * i;
    if (warp == 1) {
        asm volatile("tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(slot)), "r"(512)
                     : "memory");
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::2.sync.aligned;" ::: "memory");
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    asm volatile("barrier.cluster.arrive.aligned; barrier.cluster.wait.aligned;" ::: "memory");
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    const uint32_t taddr = *slot;
    if (threadIdx.x == 0) out[blockIdx.x] = taddr + (uint32_t)sbias[3];
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    asm volatile("barrier.cluster.arrive.aligned; barrier.cluster.wait.aligned;" ::: "memory");
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    if (warp == 1)
        asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, %1;" ::"r"(taddr), "r"(512) : "memory");
}

int main(int argc, char **argv) {
    const int variant = argc > 1 ? atoi(argv[1]) : 2;
    uint32_t *d;
    cudaMalloc(&d, 64 * sizeof(uint32_t));
    if (variant == 4) {
        const size_t smem = 215 * 1024;
        cudaFuncSetAttribute(prologue_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        prologue_kernel<<<16, 320, smem>>>(d, 200 * 1024);
    } else if (variant == 3) remote_arrive_kernel<<<16, 128>>>(d);
    else if (variant == 2) alloc2_kernel<<<16, 128>>>(d);
    else alloc1_kernel<<<16, 128>>>(d);
    cudaError_t e = cudaDeviceSynchronize();
    uint32_t h[16];
    cudaMemcpy(h, d, sizeof(h), cudaMemcpyDeviceToHost);
    printf("variant %d: %s, taddr[0..3] = %u %u %u %u\n", variant, cudaGetErrorString(e), h[0], h[1], h[2], h[3]);
    return e != cudaSuccess;
}
