// scatter.cuh — phase a3: global partitioning step 1 + data distribution,
// fused: every tuple is written straight into its owner's receive buffer.
#pragma once

#include "common.cuh"
#include "tma.cuh"

namespace mgj {

template <typename K> struct ScatCfg {
    using Tup = typename TupT<K>::T;
    static constexpr int TMAX = SCAT_T8 * 4 / (int)sizeof(K);  // 8192 (4-byte) / 4096 (8-byte) tuples
    static constexpr int VMAX = TMAX / SCATTER_THREADS;        // tuples per thread per sub-tile
};

// Sub-tile size and per-partition carry capacity for P partitions (shared
// memory stays within 227 KB).  The carry holds the < 32-byte tail of each
// partition's output so that global stores cover whole 32-byte sectors.
__host__ __device__ inline int scat_subtile(int P, int key_bytes) {
    const int tmax = SCAT_T8 * 4 / key_bytes;
    return P <= 1024 ? tmax : tmax / 2;
}
__host__ __device__ inline int scat_carry(int P, int tuple_bytes) { return P <= 2048 ? 32 / tuple_bytes - 1 : 0; }

__host__ __device__ inline size_t scat_smem_bytes(int P, int key_bytes) {
    const size_t T = (size_t)scat_subtile(P, key_bytes);
    const size_t TB = 2 * (size_t)key_bytes;
    const size_t CC = (size_t)scat_carry(P, (int)TB);
    return 2 * T * key_bytes      // input stage: keys + payloads
           + (T + CC * P) * TB    // partition-sorted sub-tile (+ carried tails)
           + (size_t)P * 4 * 4    // bins, pos, lim, ccount
           + (size_t)P * 8 * 2    // wb, base
           + (size_t)P * CC * TB; // carry
}

// ---------------------------------------------------------------------------
// a3 (§3.2 "Global partitioning phase" step 1, P:408-416 — "each
// thread ... reads a unique input tuple, determines the index for the tuple
// after partitioning based on the histogram and then writes the tuple" —
// after Rui et al. [38]; step 3 data distribution, P:405-407 and §4).
//
// B200 form: one persistent CTA per SM processes tile c = blockIdx.x of R and
// then of S, in sub-tiles of T tuples brought into shared memory by a TMA
// bulk copy issued one sub-tile ahead.  Each sub-tile is counting-sorted by
// digit1 in shared memory (one SMEM atomic per tuple gives the rank in its
// bin) and written out in sorted order, so each warp store covers a few
// contiguous runs.  Destinations are exact: owner(p)'s receive buffer at
// send_off[p] (a2) + tile_base[c][p] (a1 tile prefix) + the running count of
// p in this tile — no global atomics.  Every partition keeps its < 32-byte
// tail in shared memory until the next sub-tile completes the sector, so
// (except at tile boundaries) every store covers whole 32-byte sectors and
// DRAM never sees a partial-sector read-modify-write.  On NVSwitch the owner
// may be another GPU: the same store goes over NVLink to a peer-mapped
// address; the paper's packets, routing buffers and multi-hop routing (§4)
// have no role on a one-hop fabric.  The last CTA raises SIG_DATA at every
// peer after a system fence.
// ---------------------------------------------------------------------------
template <typename K>
__global__ void __launch_bounds__(SCATTER_THREADS, 1) k_scatter(Ctx c) {
    using Tup = typename TupT<K>::T;
    constexpr int VMAX = ScatCfg<K>::VMAX;
    constexpr int TB = (int)sizeof(Tup);
    typedef unsigned long long ull;
    extern __shared__ __align__(128) unsigned char smem[];
    const int P = c.P;
    const int T = scat_subtile(P, (int)sizeof(K));
    const int V = T / SCATTER_THREADS;
    const int CC = scat_carry(P, TB);
    K *const skey = reinterpret_cast<K *>(smem);
    K *const spay = skey + T;
    Tup *const sorted = reinterpret_cast<Tup *>(spay + T);
    uint32_t *const bins = reinterpret_cast<uint32_t *>(sorted + T + (size_t)CC * P);
    uint32_t *const pos = bins + P;
    uint32_t *const lim = pos + P;
    uint32_t *const ccount = lim + P;
    ull *const wb = reinterpret_cast<ull *>(ccount + P);
    ull *const base = wb + P;
    Tup *const carry = reinterpret_cast<Tup *>(base + P);
    __shared__ __align__(8) uint64_t bar;
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
        mbar_init(&bar, 1);
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
        mbar_arrive_expect_tx(&bar, 2 * bytes);
        if (bytes) {
            tma_load_1d(skey, static_cast<const K *>(c.in_key[rel]) + first, bytes, &bar, pol);
            tma_load_1d(spay, static_cast<const K *>(c.in_pay[rel]) + first, bytes, &bar, pol);
        }
    };
    auto set_base = [&](int rel) {  // destination of this tile's first tuple of each partition
        const uint32_t *tb = c.tile_base + ((size_t)rel * c.G + tile) * P;
        const uint64_t *so = c.send_off + (size_t)rel * P;
        for (int p = tid; p < P; p += SCATTER_THREADS) {
            const int own = c.owner[p];
            base[p] = (ull)(c.arena[own] + c.lay.recv[rel]) + (so[p] + tb[p]) * (uint64_t)TB;
            ccount[p] = 0;
        }
    };
    auto flush_carry = [&]() {  // end of a relation: write the remaining tails
        for (int p = tid; p < P; p += SCATTER_THREADS)
            for (uint32_t k = 0; k < ccount[p]; ++k)
                reinterpret_cast<Tup *>(base[p])[k] = carry[(size_t)p * CC + k];
    };

    if (tid == 0 && ntot > 0) issue(0);
    int cur_rel = -1;
    for (uint32_t g = 0; g < ntot; ++g) {
        int rel;
        uint64_t first;
        uint32_t len;
        subtile(g, rel, first, len);
        if (rel != cur_rel) {
            __syncthreads();
            if (cur_rel >= 0) flush_carry();
            __syncthreads();
            set_base(rel);
            cur_rel = rel;
        }
        mbar_wait(&bar, g & 1);
        const uint32_t body = len & ~(uint32_t)(16 / sizeof(K) - 1);
        const K *gk = static_cast<const K *>(c.in_key[rel]) + first;
        const K *gp = static_cast<const K *>(c.in_pay[rel]) + first;
        K kk[VMAX], pp[VMAX];
#pragma unroll
        for (int v = 0; v < VMAX; ++v) {
            const uint32_t i = tid + v * SCATTER_THREADS;
            if (v < V && i < body) {
                kk[v] = skey[i];
                pp[v] = spay[i];
            } else if (v < V && i < len) {  // < 4 trailing tuples of the relation
                kk[v] = gk[i];
                pp[v] = gp[i];
            }
        }
        for (int p = tid; p < P; p += SCATTER_THREADS) bins[p] = 0;
        __syncthreads();  // S1: stage consumed, bins cleared
        if (tid == 0 && g + 1 < ntot) issue(g + 1);
        uint32_t rp[VMAX];  // rank in bin << 16 | partition
#pragma unroll
        for (int v = 0; v < VMAX; ++v) {
            const uint32_t i = tid + v * SCATTER_THREADS;
            if (v < V && i < len) {
                const uint32_t p = digit1(kk[v], P);
                rp[v] = (atomicAdd(&bins[p], 1u) << 16) | p;
            }
        }
        __syncthreads();  // S2
        for (int p = tid; p < P; p += SCATTER_THREADS) bins[p] += ccount[p];
        __syncthreads();
        const uint32_t ttot = block_excl_scan_u32(bins, P, tmp);
        for (int p = tid; p < P; p += SCATTER_THREADS) {
            const uint32_t o = bins[p];
            const uint32_t tp = ((p + 1 < P) ? bins[p + 1] : ttot) - o;
            const uint32_t cc = ccount[p];
            const ull G = base[p];
            const ull end = G + (ull)tp * TB;
            const ull aend = CC ? (end & ~31ull) : end;
            const uint32_t L = aend > G ? (uint32_t)((aend - G) / TB) : 0;
            lim[p] = o + L;
            wb[p] = G - (ull)o * TB;
            base[p] = G + (ull)L * TB;
            for (uint32_t k = 0; k < cc; ++k) sorted[o + k] = carry[(size_t)p * CC + k];
            pos[p] = o + cc;
            ccount[p] = tp - L;
        }
        __syncthreads();  // S3
#pragma unroll
        for (int v = 0; v < VMAX; ++v) {
            const uint32_t i = tid + v * SCATTER_THREADS;
            if (v < V && i < len) {
                Tup t;
                t.x = kk[v];
                t.y = pp[v];
                sorted[pos[rp[v] & 0xffffu] + (rp[v] >> 16)] = t;
            }
        }
        __syncthreads();  // S4
        for (uint32_t i = tid; i < ttot; i += SCATTER_THREADS) {
            const Tup t = sorted[i];
            const uint32_t p = digit1(t.x, P);
            const uint32_t l = lim[p];
            if (i < l) reinterpret_cast<Tup *>(wb[p] + (ull)i * TB)[0] = t;
            else carry[(size_t)p * CC + (i - l)] = t;
        }
    }
    __syncthreads();
    if (cur_rel >= 0) flush_carry();

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
