// scatter.cuh — phase a3: global partitioning step 1 + data distribution,
// fused: every tuple is written straight into its owner's receive buffer.
#pragma once

#include "common.cuh"

namespace mgj {

// ---------------------------------------------------------------------------
// a3 (§3.2 "Global partitioning phase" step 1, after Rui
// et al. [38]; step 3 data distribution, P:405-407 and §4).  On NVSwitch every
// pair of GPUs is one hop, so the paper's packets, routing buffers and
// adaptive multi-hop routing (§4) reduce to this: each CTA stages tuples in
// a shared-memory write-combining line per global partition and, when a line
// is full, reserves L slots in the owner's receive range with one atomic and
// writes the line there (a peer store over NVLink when the owner is another
// GPU).  The receive layout per relation is: owned p ascending, then source
// rank ascending, exactly tiled by the plan's offsets.  Order inside a
// (source rank, p) range is unspecified (reading C17).
//
// Persistent grid (1 CTA/SM, 1024 threads); input batches are claimed
// dynamically; each thread holds SCATTER_V tuples loaded with 16-byte
// streaming loads, prefetching the next batch while the current one is
// placed.  The last CTA raises SIG_DATA at every peer after a system fence.
// ---------------------------------------------------------------------------
template <typename K>
__global__ void __launch_bounds__(SCATTER_THREADS, 1) k_scatter(Ctx c) {
    using Tup = typename TupT<K>::T;
    constexpr int V = SCATTER_V;
    constexpr int NW = SCATTER_THREADS / 32;
    extern __shared__ __align__(16) unsigned char smem[];
    const int P = c.P, L = c.line_tuples;
    Tup *buf = reinterpret_cast<Tup *>(smem);
    uint32_t *cnt = reinterpret_cast<uint32_t *>(buf + (size_t)P * L);
    uint16_t *flist = reinterpret_cast<uint16_t *>(cnt + P);
    __shared__ uint32_t s_nf[2], s_batch[2];
    __shared__ int s_ok;
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    if (tid == 0) {
        s_ok = *(volatile int32_t *)&c.meta[MT_OK];
        s_nf[0] = s_nf[1] = 0;
    }
    __syncthreads();
    uint32_t gr = 0;  // global round counter (parity of the flush-list counter)

    for (int rel = 0; rel < 2 && s_ok; ++rel) {
        const uint64_t n = c.n_in[rel];
        const K *keys = static_cast<const K *>(c.in_key[rel]);
        const K *pays = static_cast<const K *>(c.in_pay[rel]);
        const uint32_t nb = (uint32_t)((n + SCATTER_BATCH - 1) / SCATTER_BATCH);
        const uint64_t *soff = c.send_off + (size_t)rel * P;
        uint32_t *gcur = c.gcur + (size_t)rel * P;
        const uint64_t recv_off = c.lay.recv[rel];
        for (int i = tid; i < P; i += SCATTER_THREADS) cnt[i] = 0;

        auto load = [&](uint32_t b, K (&kk)[V], K (&pp)[V]) {
            const uint64_t base = (uint64_t)b * SCATTER_BATCH + (uint64_t)tid * V;
            if (b < nb && base + V <= n) {
                if (sizeof(K) == 4) {
                    uint4 a = __ldcs(reinterpret_cast<const uint4 *>(keys + base));
                    uint4 d = __ldcs(reinterpret_cast<const uint4 *>(pays + base));
                    kk[0] = (K)a.x; kk[1] = (K)a.y; kk[2] = (K)a.z; kk[3] = (K)a.w;
                    pp[0] = (K)d.x; pp[1] = (K)d.y; pp[2] = (K)d.z; pp[3] = (K)d.w;
                } else {
#pragma unroll
                    for (int h = 0; h < V / 2; ++h) {
                        ulonglong2 a = __ldcs(reinterpret_cast<const ulonglong2 *>(keys + base) + h);
                        ulonglong2 d = __ldcs(reinterpret_cast<const ulonglong2 *>(pays + base) + h);
                        kk[2 * h] = (K)a.x; kk[2 * h + 1] = (K)a.y;
                        pp[2 * h] = (K)d.x; pp[2 * h + 1] = (K)d.y;
                    }
                }
            } else {
#pragma unroll
                for (int v = 0; v < V; ++v) {
                    const bool ok = b < nb && base + v < n;
                    kk[v] = ok ? keys[base + v] : (K)0;
                    pp[v] = ok ? pays[base + v] : (K)0;
                }
            }
        };

        // Write the nf full lines listed in flist: one reservation atomic per line.
        auto flush_lines = [&](uint32_t nf, uint32_t round) {
            const int epw = 32 / L, sub = lane / L, li = lane % L;
            for (uint32_t e0 = (uint32_t)warp * 32; e0 < nf; e0 += NW * 32) {
                const uint32_t e = e0 + lane;
                uint32_t p = 0, own = 0;
                uint64_t off = 0;
                if (e < nf) {
                    p = flist[e];
                    off = soff[p] + atomicAdd(&gcur[p], (uint32_t)L);
                    own = (uint32_t)c.owner[p];
                }
                const uint32_t ne = min(32u, nf - e0);
                for (uint32_t j = 0; j < ne; j += epw) {
                    const uint32_t sl = j + sub;
                    const uint32_t pj = __shfl_sync(0xffffffffu, p, sl & 31);
                    const uint64_t oj = __shfl_sync(0xffffffffu, off, sl & 31);
                    const uint32_t ow = __shfl_sync(0xffffffffu, own, sl & 31);
                    if (sl < ne) {
                        Tup *dst = reinterpret_cast<Tup *>(c.arena[ow] + recv_off) + oj + li;
                        *dst = buf[(size_t)pj * L + li];
                    }
                }
            }
        };

        uint32_t it = 0;
        if (tid == 0) s_batch[0] = atomicAdd(&c.ticket[TK_SCAT_R + rel], 1u);
        __syncthreads();
        uint32_t b = s_batch[0];
        K kk[V], pp[V];
        load(b, kk, pp);
        while (b < nb) {
            ++it;
            if (tid == 0) s_batch[it & 1] = atomicAdd(&c.ticket[TK_SCAT_R + rel], 1u);
            __syncthreads();
            const uint32_t bn = s_batch[it & 1];
            K kn[V], pn[V];
            load(bn, kn, pn);  // prefetch the next batch while this one is placed

            const uint64_t base = (uint64_t)b * SCATTER_BATCH + (uint64_t)tid * V;
            uint32_t pd[V], pos[V];
#pragma unroll
            for (int v = 0; v < V; ++v) {
                if (base + v < n) {
                    pd[v] = digit1(kk[v], P);
                    pos[v] = atomicAdd(&cnt[pd[v]], 1u);
                } else {
                    pd[v] = 0;
                    pos[v] = 0xffffffffu;
                }
            }
            for (uint32_t r = 0;; ++r, ++gr) {
                const uint32_t lo = r * (uint32_t)L, hi = lo + (uint32_t)L;
                int more = 0;
#pragma unroll
                for (int v = 0; v < V; ++v) {
                    if (pos[v] >= lo && pos[v] < hi) {
                        Tup t;
                        t.x = kk[v];
                        t.y = pp[v];
                        buf[(size_t)pd[v] * L + (pos[v] - lo)] = t;
                        if (pos[v] == hi - 1) flist[atomicAdd(&s_nf[gr & 1], 1u)] = (uint16_t)pd[v];
                    } else if (pos[v] != 0xffffffffu && pos[v] >= hi) {
                        more = 1;
                    }
                }
                __syncthreads();
                const uint32_t nf = s_nf[gr & 1];
                if (tid == 0) s_nf[(gr + 1) & 1] = 0;
                flush_lines(nf, r);
                more = __syncthreads_or(more);
                if (!more) break;
            }
            ++gr;
            for (int i = tid; i < P; i += SCATTER_THREADS) cnt[i] &= (uint32_t)(L - 1);
#pragma unroll
            for (int v = 0; v < V; ++v) {
                kk[v] = kn[v];
                pp[v] = pn[v];
            }
            b = bn;
        }
        __syncthreads();
        // drain partially filled lines
        for (int p0 = warp * 32; p0 < P; p0 += NW * 32) {
            const int p = p0 + lane;
            const uint32_t m = p < P ? cnt[p] : 0;
            uint64_t off = 0;
            uint32_t own = 0;
            if (m) {
                off = soff[p] + atomicAdd(&gcur[p], m);
                own = (uint32_t)c.owner[p];
            }
            uint32_t msk = __ballot_sync(0xffffffffu, m > 0);
            while (msk) {
                const int src = __ffs(msk) - 1;
                msk &= msk - 1;
                const uint32_t mm = __shfl_sync(0xffffffffu, m, src);
                const uint64_t oo = __shfl_sync(0xffffffffu, off, src);
                const uint32_t ow = __shfl_sync(0xffffffffu, own, src);
                if ((uint32_t)lane < mm) {
                    Tup *dst = reinterpret_cast<Tup *>(c.arena[ow] + recv_off) + oo + lane;
                    *dst = buf[(size_t)(p0 + src) * L + lane];
                }
            }
        }
        __syncthreads();
        if (tid == 0) s_nf[gr & 1] = 0;
        __syncthreads();
    }

    // ---- every CTA: make its peer stores visible, the last one signals ----
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
