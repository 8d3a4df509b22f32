// Microbenchmark: HBM read throughput of TMA bulk copies of runs of L bytes
// gathered like k_probe gathers a co-partition: each item is NRUN runs, run k
// taken from chunk region k (stride REGION bytes) at a per-item offset, copied
// into one of three shared-memory stages (one mbarrier per stage).  Items are
// spread over the grid like the probe's (item i -> CTA i % grid).  Prints GB/s
// per run length.  Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tma_runs tools/tma_runs.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t smem_u32(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }

__global__ void __launch_bounds__(256) k_gather(const char *src, size_t bytes_total, int L, int nrun, size_t region,
                                              int items, unsigned long long *sink, int nw) {
    extern __shared__ __align__(128) char sm[];
    __shared__ __align__(8) uint64_t bar[3];
    const int lane = threadIdx.x & 31;
    if (threadIdx.x == 0) {
        for (int s = 0; s < 3; ++s) asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&bar[s])));
        asm volatile("fence.mbarrier_init.release.cluster;");
    }
    __syncthreads();
    const int stage_bytes = L * nrun;
    const size_t nregions = bytes_total / region;
    unsigned long long acc = 0;
    int j = 0;
    for (int it = blockIdx.x; it < items; it += gridDim.x, ++j) {
        const int s = j % 3;
        if (j >= 3) {  // wait for the stage's previous load, consume a word
            asm volatile("{\n\t.reg .pred p;\n\tW%=:\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t@!p bra W%=;\n\t}" ::"r"(
                             smem_u32(&bar[s])),
                         "r"((uint32_t)(((j / 3) - 1) & 1)));
            acc += sm[s * stage_bytes + lane];
            __syncwarp();
        }
        if (threadIdx.x == 0)
            asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(&bar[s])),
                         "r"((uint32_t)stage_bytes));
        __syncthreads();  // the stage is free for every issuing warp, its byte count armed
        const int w = threadIdx.x >> 5;
        if (w < nw) {
            // item it: chunk regions base..base+nrun-1, run offset within the region by item
            const size_t base = ((size_t)it * 7919 % (nregions - nrun));
            const size_t off = ((size_t)it * 2654435761u) % (region - L) & ~(size_t)15;
            for (int k = w * 32 + lane; k < nrun; k += 32 * nw) {
                const char *g = src + (base + k) * region + off;
                asm volatile(
                    "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                        smem_u32(sm + s * stage_bytes + k * L)),
                    "l"(g), "r"(L), "r"(smem_u32(&bar[s]))
                    : "memory");
            }
        }
    }
    for (int q = 0; q < 3 && q < j; ++q) {  // drain
        const int jj = j - 1 - q, s = jj % 3;
        asm volatile("{\n\t.reg .pred p;\n\tW%=:\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t@!p bra W%=;\n\t}" ::"r"(
                         smem_u32(&bar[s])),
                     "r"((uint32_t)((jj / 3) & 1)));
    }
    if (acc == 12345) *sink = acc;
}

int main() {
    const size_t total = 8ull << 30, region = 98304 + 4096;
    char *src;
    unsigned long long *sink;
    cudaMalloc(&src, total);
    cudaMalloc(&sink, 8);
    cudaMemset(src, 1, total);
    int nsm;
    cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0);
    const int runs[] = {256, 512, 768, 1024, 1536, 2048, 3072, 6144};
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    printf("warps run_bytes runs_per_item item_KB GB/s\n");
    for (int nw : {1, 2, 4, 8})
    for (int L : runs) {
        const int stage = 65536;          // bytes per item (one probe side pair ~ 64 KB)
        const int nrun = stage / L;
        const int items = (int)(4ull * 1024 * 1024 * 1024 / stage);  // 4 GB moved
        cudaFuncSetAttribute(k_gather, cudaFuncAttributeMaxDynamicSharedMemorySize, 3 * stage);
        for (int rep = 0; rep < 2; ++rep) {
            cudaEventRecord(a);
            k_gather<<<nsm, 256, 3 * stage>>>(src, total, L, nrun, region, items, sink, nw);
            cudaEventRecord(b);
            cudaEventSynchronize(b);
            float ms;
            cudaEventElapsedTime(&ms, a, b);
            if (rep) printf("%d %d %d %d %.1f\n", nw, L, nrun, stage / 1024, (double)items * stage / (ms * 1e6));
        }
    }
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) printf("error %s\n", cudaGetErrorString(e));
    return 0;
}
