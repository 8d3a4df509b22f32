// Transfer-size sweep (the B200 analogue of PAPER.md Fig. 4, §4.1 P:549-559:
// bandwidth of a link against the packet size, 2 KB .. 16 MB there).
// Three ways of moving `size`-byte packets from a source buffer to a
// destination buffer, scattered over 1 GiB (packet k at a pseudo-random
// packet slot, as the shuffle's per-partition runs are):
//   ce   : one cudaMemcpyAsync (copy engine) per packet, back to back;
//   sm   : the in-kernel path the shuffle uses — warps copy packets with
//          16-byte loads and stores (148 x 4 CTAs of 256 threads);
//   bulk : a TMA bulk copy global -> shared -> global per packet (one warp
//          lane per packet).
// The destination is GPU 1's memory (peer access, NVLink/NVSwitch) when a
// second GPU is visible, else GPU 0's own memory (then every byte is read
// and written in the same HBM: the sizes where throughput saturates are the
// point, not the absolute numbers).
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o build/transfer_sweep tools/transfer_sweep.cu
#include <cstdint>
#include <cstdio>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t smem_u32(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }
__host__ __device__ inline uint64_t slot_of(uint64_t k, uint64_t nslots) { return (k * 0x9E3779B97F4A7C15ull >> 20) % nslots; }

__global__ void k_sm(const char *src, char *dst, uint64_t size, uint64_t npk, uint64_t nslots) {
    // 16-byte pieces in order: consecutive lanes take consecutive pieces of a
    // packet (several packets per warp when packets are small)
    const uint64_t per = size / 16, n = npk * per;
    for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += gridDim.x * (uint64_t)blockDim.x) {
        const uint64_t k = i / per, j = i - k * per;
        const uint64_t o = slot_of(k, nslots) * per + j;
        reinterpret_cast<uint4 *>(dst)[o] = __ldcs(reinterpret_cast<const uint4 *>(src) + o);
    }
}

__global__ void __launch_bounds__(256) k_bulk(const char *src, char *dst, uint32_t size, uint64_t npk, uint64_t nslots) {
    extern __shared__ __align__(128) char sm[];
    __shared__ __align__(8) uint64_t bar[8];
    const int w = threadIdx.x >> 5, lane = threadIdx.x & 31;
    if (lane == 0) asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&bar[w])));
    asm volatile("fence.mbarrier_init.release.cluster;");
    __syncthreads();
    char *buf = sm + (size_t)w * size;  // one packet buffer per warp (lane 0 moves it)
    uint32_t ph = 0;
    const uint64_t warp = blockIdx.x * 8ull + w, nw = gridDim.x * 8ull;
    if (lane) return;
    for (uint64_t k = warp; k < npk; k += nw, ph ^= 1) {
        const uint64_t o = slot_of(k, nslots) * size;
        asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");  // buffer free
        asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(&bar[w])), "r"(size));
        asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                         smem_u32(buf)), "l"(src + o), "r"(size), "r"(smem_u32(&bar[w])) : "memory");
        asm volatile("{\n\t.reg .pred p;\n\tW%=:\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t@!p bra W%=;\n\t}" ::"r"(
                         smem_u32(&bar[w])), "r"(ph) : "memory");
        asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(dst + o), "r"(smem_u32(buf)), "r"(size)
                     : "memory");
        asm volatile("cp.async.bulk.commit_group;" ::: "memory");
    }
    asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
}

int main() {
    int ndev = 0, nsm = 0;
    cudaGetDeviceCount(&ndev);
    cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0);
    const uint64_t total = 1ull << 30;
    char *src, *dst;
    cudaSetDevice(0);
    cudaMalloc(&src, total);
    cudaMemset(src, 1, total);
    int peer = 0;
    if (ndev > 1) {
        cudaDeviceCanAccessPeer(&peer, 0, 1);
        if (peer) {
            cudaDeviceEnablePeerAccess(1, 0);
            cudaSetDevice(1);
            cudaMalloc(&dst, total);
            cudaDeviceEnablePeerAccess(0, 0);
            cudaSetDevice(0);
        }
    }
    if (!peer) cudaMalloc(&dst, total);
    printf("# destination: %s\n", peer ? "GPU 1 (peer)" : "GPU 0 (same HBM: read + write)");
    printf("%10s %12s %12s %12s\n", "size", "ce_GB/s", "sm_GB/s", "bulk_GB/s");
    cudaStream_t s;
    cudaStreamCreate(&s);
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    cudaFuncSetAttribute(k_bulk, cudaFuncAttributeMaxDynamicSharedMemorySize, 8 * 16384);
    for (uint64_t size = 32; size <= (16ull << 20); size *= 2) {  // (packets of 16 MB: 64 per GiB)
        const uint64_t nslots = total / size;
        const uint64_t npk_ce = nslots < 8192 ? nslots : 8192;  // copy-engine calls per measurement
        const uint64_t npk = nslots;                            // kernels move the whole GiB
        float ms_ce = 0, ms_sm = 0, ms_bulk = -1;
        for (int rep = 0; rep < 2; ++rep) {
            cudaEventRecord(a, s);
            for (uint64_t k = 0; k < npk_ce; ++k) {
                const uint64_t o = slot_of(k, nslots) * size;
                cudaMemcpyAsync(dst + o, src + o, size, peer ? cudaMemcpyDefault : cudaMemcpyDeviceToDevice, s);
            }
            cudaEventRecord(b, s);
            cudaEventSynchronize(b);
            cudaEventElapsedTime(&ms_ce, a, b);
            if (size >= 16) {
                cudaEventRecord(a, s);
                k_sm<<<nsm * 4, 256, 0, s>>>(src, dst, size, npk, nslots);
                cudaEventRecord(b, s);
                cudaEventSynchronize(b);
                cudaEventElapsedTime(&ms_sm, a, b);
            }
            if (size <= 16384) {
                cudaEventRecord(a, s);
                k_bulk<<<nsm, 256, 8 * size, s>>>(src, dst, (uint32_t)size, npk, nslots);
                cudaEventRecord(b, s);
                cudaEventSynchronize(b);
                cudaEventElapsedTime(&ms_bulk, a, b);
            }
        }
        const double gb_ce = npk_ce * size / (ms_ce * 1e6), gb_sm = npk * size / (ms_sm * 1e6);
        const double gb_bulk = ms_bulk > 0 ? npk * size / (ms_bulk * 1e6) : 0.0;
        printf("%10llu %12.1f %12.1f %12.1f %s\n", (unsigned long long)size, gb_ce, gb_sm, gb_bulk,
               cudaGetErrorString(cudaGetLastError()));
    }
    return 0;
}
