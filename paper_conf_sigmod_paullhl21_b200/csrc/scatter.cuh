// scatter.cuh — phase a3: global partitioning step 1 + data distribution,
// fused: every tuple is written straight into its owner's receive buffer.
#pragma once

#include "common.cuh"
#include "tma.cuh"

namespace mgj {

template <typename K> struct ScatCfg {
    using Tup = typename TupT<K>::T;
    static constexpr int TMAX = SCAT_T8 * 4 / (int)sizeof(K);     // 8192 (4-byte) / 4096 (8-byte) tuples
    static constexpr int VMAX = TMAX / SCATTER_THREADS;           // tuples per thread per sub-tile
};

// Sub-tile size for P partitions: keeps stages + sorted buffer + per-partition
// arrays inside 227 KB of shared memory.
__host__ __device__ inline int scat_subtile(int P, int key_bytes) {
    const int tmax = SCAT_T8 * 4 / key_bytes;
    return P <= 1024 ? tmax : tmax / 2;
}

__host__ __device__ inline size_t scat_smem_bytes(int P, int key_bytes) {
    const size_t T = (size_t)scat_subtile(P, key_bytes);
    return 2 * 2 * T * key_bytes     // two input stages, keys + payloads
           + T * 2 * key_bytes       // partition-sorted sub-tile
           + (size_t)P * 4           // bins
           + (size_t)P * 8 * 2;      // wbase, base
}

// ---------------------------------------------------------------------------
// a3 (§3.2 "Global partitioning phase" step 1, P:408-416 — "each
// thread ... reads a unique input tuple, determines the index for the tuple
// after partitioning based on the histogram and then writes the tuple" —
// after Rui et al. [38]; step 3 data distribution, P:405-407 and §4).
//
// B200 form: one persistent CTA per SM processes tile c = blockIdx.x of R and
// then of S, in sub-tiles of T tuples brought into shared memory by TMA bulk
// copies (double-buffered, two sub-tiles ahead).  Each sub-tile is counting-
// sorted by digit1 in shared memory (one SMEM atomic per tuple gives the rank
// in its bin), then written out in sorted order so that each warp store
// covers a few contiguous runs.  The destination of every tuple is exact:
// owner(p)'s receive buffer at send_off[p] (a2) + tile_base[c][p] (a1 tile
// prefix) + the running count of p in this tile, so no global atomics and no
// buffer flushes are needed.  On NVSwitch the owner may be another GPU: the
// same store goes over NVLink (a peer-mapped address); the paper's packets,
// routing buffers and multi-hop routing (§4) have no role on a one-hop
// fabric.  The last CTA raises SIG_DATA at every peer after a system fence.
// ---------------------------------------------------------------------------
template <typename K>
__global__ void __launch_bounds__(SCATTER_THREADS, 1) k_scatter(Ctx c) {
    using Tup = typename TupT<K>::T;
    constexpr int VMAX = ScatCfg<K>::VMAX;
    constexpr int TB = (int)sizeof(Tup);
    extern __shared__ __align__(128) unsigned char smem[];
    const int P = c.P;
    const int T = scat_subtile(P, (int)sizeof(K));
    const int V = T / SCATTER_THREADS;
    K *const stage0 = reinterpret_cast<K *>(smem);  // [2][keys T | payloads T]
    auto skey = [&](int s) { return stage0 + (size_t)s * 2 * T; };
    auto spay = [&](int s) { return stage0 + (size_t)s * 2 * T + T; };
    Tup *sorted = reinterpret_cast<Tup *>(stage0 + (size_t)4 * T);
    uint32_t *bins = reinterpret_cast<uint32_t *>(sorted + T);
    unsigned long long *wbase = reinterpret_cast<unsigned long long *>(bins + P);
    unsigned long long *base = wbase + P;
    __shared__ __align__(8) uint64_t bar[2];
    __shared__ uint32_t tmp[33];
    const int tid = threadIdx.x;
    const int tile = blockIdx.x;
    const int ok = *(volatile int32_t *)&c.meta[MT_OK];

    uint64_t lo[2], hi[2];
    uint32_t nsub[2];
    for (int r = 0; r < 2; ++r) {
        tile_range(c.n_in[r], c.G, tile, lo[r], hi[r]);
        nsub[r] = ok ? (uint32_t)((hi[r] - lo[r] + T - 1) / T) : 0;
    }
    const uint32_t ntot = nsub[0] + nsub[1];
    if (tid == 0) {
        mbar_init(&bar[0], 1);
        mbar_init(&bar[1], 1);
        fence_mbar_init();
    }
    __syncthreads();
    const uint64_t pol = policy_evict_first();

    // sub-tile g of the R-then-S sequence -> (rel, first tuple, length)
    auto subtile = [&](uint32_t g, int &rel, uint64_t &first, uint32_t &len) {
        rel = g < nsub[0] ? 0 : 1;
        const uint32_t j = rel ? g - nsub[0] : g;
        first = lo[rel] + (uint64_t)j * T;
        len = (uint32_t)min((uint64_t)T, hi[rel] - first);
    };
    auto issue = [&](uint32_t g) {  // thread 0: TMA the 16-byte-aligned body of sub-tile g
        int rel;
        uint64_t first;
        uint32_t len;
        subtile(g, rel, first, len);
        const uint32_t body = len & ~(uint32_t)(16 / sizeof(K) - 1);
        const uint32_t bytes = body * (uint32_t)sizeof(K);
        uint64_t *b = &bar[g & 1];
        mbar_arrive_expect_tx(b, 2 * bytes);
        if (bytes) {
            tma_load_1d(skey(g & 1), static_cast<const K *>(c.in_key[rel]) + first, bytes, b, pol);
            tma_load_1d(spay(g & 1), static_cast<const K *>(c.in_pay[rel]) + first, bytes, b, pol);
        }
    };
    auto set_base = [&](int rel) {  // destination of this tile's first tuple of each partition
        const uint32_t *tb = c.tile_base + ((size_t)rel * c.G + tile) * P;
        const uint64_t *so = c.send_off + (size_t)rel * P;
        for (int p = tid; p < P; p += SCATTER_THREADS) {
            const int own = c.owner[p];
            base[p] = (unsigned long long)(c.arena[own] + c.lay.recv[rel]) + (so[p] + tb[p]) * (uint64_t)TB;
        }
    };

    if (tid == 0) {
        if (ntot > 0) issue(0);
        if (ntot > 1) issue(1);
    }
    int cur_rel = -1;
    for (uint32_t g = 0; g < ntot; ++g) {
        int rel;
        uint64_t first;
        uint32_t len;
        subtile(g, rel, first, len);
        if (rel != cur_rel) {  // (previous sub-tile's write-out is ordered by the barriers below)
            __syncthreads();
            set_base(rel);
            cur_rel = rel;
        }
        const int s = g & 1;
        mbar_wait(&bar[s], (g >> 1) & 1);
        const uint32_t body = len & ~(uint32_t)(16 / sizeof(K) - 1);
        const K *gk = static_cast<const K *>(c.in_key[rel]) + first;
        const K *gp = static_cast<const K *>(c.in_pay[rel]) + first;
        K kk[VMAX], pp[VMAX];
#pragma unroll
        for (int v = 0; v < VMAX; ++v) {
            const uint32_t i = tid + v * SCATTER_THREADS;
            if (v < V && i < body) {
                kk[v] = skey(s)[i];
                pp[v] = spay(s)[i];
            } else if (v < V && i < len) {  // < 4 trailing tuples of the relation
                kk[v] = gk[i];
                pp[v] = gp[i];
            }
        }
        for (int p = tid; p < P; p += SCATTER_THREADS) bins[p] = 0;
        __syncthreads();  // stage s consumed, bins cleared
        if (tid == 0 && g + 2 < ntot) issue(g + 2);
        uint32_t rp[VMAX];  // rank in bin << 16 | partition
#pragma unroll
        for (int v = 0; v < VMAX; ++v) {
            const uint32_t i = tid + v * SCATTER_THREADS;
            if (v < V && i < len) {
                const uint32_t p = digit1(kk[v], P);
                rp[v] = (atomicAdd(&bins[p], 1u) << 16) | p;
            }
        }
        __syncthreads();
        block_excl_scan_u32(bins, P, tmp);
        for (int p = tid; p < P; p += SCATTER_THREADS) {
            const uint32_t o = bins[p], e = (p + 1 < P) ? bins[p + 1] : len;
            const unsigned long long b = base[p];
            wbase[p] = b - (unsigned long long)o * TB;
            base[p] = b + (unsigned long long)(e - o) * TB;
        }
#pragma unroll
        for (int v = 0; v < VMAX; ++v) {
            const uint32_t i = tid + v * SCATTER_THREADS;
            if (v < V && i < len) {
                Tup t;
                t.x = kk[v];
                t.y = pp[v];
                sorted[bins[rp[v] & 0xffffu] + (rp[v] >> 16)] = t;
            }
        }
        __syncthreads();
        for (uint32_t i = tid; i < len; i += SCATTER_THREADS) {
            const Tup t = sorted[i];
            Tup *dst = reinterpret_cast<Tup *>(wbase[digit1(t.x, P)] + (unsigned long long)i * TB);
            *dst = t;
        }
    }

    // ---- every CTA: make its (peer) stores visible, the last one signals ----
    __threadfence_system();
    __syncthreads();
    if (tid == 0) {
        const uint32_t t = atomicAdd(&c.ticket[TK_SCAT_DONE], 1u);
        if (t == gridDim.x - 1) {
            __threadfence_system();
            signal_all(c, SIG_DATA);
        }
    }
}

}  // namespace mgj
