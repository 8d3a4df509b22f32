// Microbenchmark: throughput of many small shared -> global bulk copies
// (cp.async.bulk.global.shared::cta) issued the way a per-partition write-out
// would issue them: each CTA (one per SM, 1024 threads) owns P = 1024
// "partitions"; per round every partition stores B bytes at its own cursor
// (partition regions spread over a large buffer), the copies issued by NW
// warps (each lane issues its partitions' copies).  Compared against the same
// pattern written with 32-byte st.global.v8 stores by all 32 warps.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o build/tma_store_bench tools/tma_store_bench.cu
#include <cstdint>
#include <cstdio>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t smem_u32(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }

__global__ void __launch_bounds__(1024, 1) k_bulk(char *dst, size_t region, int B, int rounds, int nw) {
    extern __shared__ __align__(128) char sm[];
    const int P = 1024;
    for (int i = threadIdx.x; i < 64 * 1024 / 4; i += blockDim.x) reinterpret_cast<uint32_t *>(sm)[i] = i;
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    __syncthreads();
    const int w = threadIdx.x >> 5, lane = threadIdx.x & 31;
    if (w < nw) {
        for (int r = 0; r < rounds; ++r) {
            for (int p = w * 32 + lane; p < P; p += 32 * nw) {
                char *g = dst + ((size_t)blockIdx.x * P + p) * region + (size_t)r * B;
                const char *s = sm + ((p * 64) & (32 * 1024 - 1));
                asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(g), "r"(smem_u32(s)),
                             "r"(B)
                             : "memory");
            }
            asm volatile("cp.async.bulk.commit_group;" ::: "memory");
            // keep at most a few groups in flight per thread (the shared source is reused)
            asm volatile("cp.async.bulk.wait_group.read 4;" ::: "memory");
        }
        asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
    }
}

// one lane per issuing warp issues copies back to back (operands of one thread:
// no per-lane serialisation loop), unrolled by 4
__global__ void __launch_bounds__(1024, 1) k_bulk1(char *dst, size_t region, int B, int rounds, int nw) {
    extern __shared__ __align__(128) char sm[];
    const int P = 1024;
    for (int i = threadIdx.x; i < 64 * 1024 / 4; i += blockDim.x) reinterpret_cast<uint32_t *>(sm)[i] = i;
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    __syncthreads();
    const int w = threadIdx.x >> 5, lane = threadIdx.x & 31;
    if (w < nw && lane == 0) {
        for (int r = 0; r < rounds; ++r) {
#pragma unroll 4
            for (int p = w; p < P; p += nw) {
                char *g = dst + ((size_t)blockIdx.x * P + p) * region + (size_t)r * B;
                const char *s = sm + ((p * 64) & (32 * 1024 - 1));
                asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(g), "r"(smem_u32(s)),
                             "r"(B)
                             : "memory");
            }
            asm volatile("cp.async.bulk.commit_group;" ::: "memory");
            asm volatile("cp.async.bulk.wait_group.read 4;" ::: "memory");
        }
        asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
    }
}

__global__ void __launch_bounds__(1024, 1) k_stg(char *dst, size_t region, int B, int rounds) {
    extern __shared__ __align__(128) char sm[];
    const int P = 1024;
    for (int i = threadIdx.x; i < 64 * 1024 / 4; i += blockDim.x) reinterpret_cast<uint32_t *>(sm)[i] = i;
    __syncthreads();
    const int G = B / 32;  // 32-byte groups per partition per round
    for (int r = 0; r < rounds; ++r) {
        for (int u = threadIdx.x; u < P * G; u += blockDim.x) {
            const int p = u / G, j = u % G;
            char *g = dst + ((size_t)blockIdx.x * P + p) * region + (size_t)r * B + j * 32;
            const uint4 a = *reinterpret_cast<const uint4 *>(sm + ((u * 32) & (64 * 1024 - 1)));
            const uint4 b = *reinterpret_cast<const uint4 *>(sm + ((u * 32 + 16) & (64 * 1024 - 1)));
            asm volatile("st.global.v8.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8};" ::"l"(g), "r"(a.x), "r"(a.y), "r"(a.z),
                         "r"(a.w), "r"(b.x), "r"(b.y), "r"(b.z), "r"(b.w)
                         : "memory");
        }
        __syncthreads();
    }
}

int main() {
    int nsm = 0;
    cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0);
    const size_t total = 16ull << 30;
    char *dst;
    if (cudaMalloc(&dst, total) != cudaSuccess) return 1;
    const size_t region = total / ((size_t)nsm * 1024) / 256 * 256;  // ~110 KB per partition
    cudaFuncSetAttribute(k_bulk, cudaFuncAttributeMaxDynamicSharedMemorySize, 64 * 1024);
    cudaFuncSetAttribute(k_stg, cudaFuncAttributeMaxDynamicSharedMemorySize, 64 * 1024);
    cudaFuncSetAttribute(k_bulk1, cudaFuncAttributeMaxDynamicSharedMemorySize, 64 * 1024);
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    for (int B : {48, 64, 96, 128}) {
        const int rounds = (int)(region / B) < 512 ? (int)(region / B) : 512;
        const double bytes = (double)nsm * 1024 * B * rounds;
        for (int nw : {1, 2, 4, 8, 32}) {
            k_bulk<<<nsm, 1024, 64 * 1024>>>(dst, region, B, rounds, nw);
            cudaEventRecord(a);
            k_bulk<<<nsm, 1024, 64 * 1024>>>(dst, region, B, rounds, nw);
            cudaEventRecord(b);
            cudaEventSynchronize(b);
            float ms;
            cudaEventElapsedTime(&ms, a, b);
            printf("bulk  B=%4d nw=%2d: %8.1f GB/s  %6.2f cyc/copy/SM (at 1.965 GHz)  %s\n", B, nw, bytes / ms / 1e6,
                   ms * 1e-3 * 1.965e9 / (1024.0 * rounds), cudaGetErrorString(cudaGetLastError()));
        }
        for (int nw : {1, 2, 4, 8, 16}) {
            k_bulk1<<<nsm, 1024, 64 * 1024>>>(dst, region, B, rounds, nw);
            cudaEventRecord(a);
            k_bulk1<<<nsm, 1024, 64 * 1024>>>(dst, region, B, rounds, nw);
            cudaEventRecord(b);
            cudaEventSynchronize(b);
            float ms;
            cudaEventElapsedTime(&ms, a, b);
            printf("bulk1 B=%4d nw=%2d: %8.1f GB/s  %6.2f cyc/copy/SM (one lane per warp)  %s\n", B, nw, bytes / ms / 1e6,
                   ms * 1e-3 * 1.965e9 / (1024.0 * rounds), cudaGetErrorString(cudaGetLastError()));
        }
        if (B % 32) continue;
        k_stg<<<nsm, 1024, 64 * 1024>>>(dst, region, B, rounds);
        cudaEventRecord(a);
        k_stg<<<nsm, 1024, 64 * 1024>>>(dst, region, B, rounds);
        cudaEventRecord(b);
        cudaEventSynchronize(b);
        float ms;
        cudaEventElapsedTime(&ms, a, b);
        printf("stg   B=%4d      : %8.1f GB/s  %6.2f cyc/partition-run/SM\n", B, bytes / ms / 1e6,
               ms * 1e-3 * 1.965e9 / (1024.0 * rounds));
    }
    return 0;
}
