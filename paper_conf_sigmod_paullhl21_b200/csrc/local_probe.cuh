// local_probe.cuh — phase a4 (local radix partitioning of the received
// segments), phase a5 (shared-memory build/probe) and a6 (cross-rank sum).
#pragma once

#include "common.cuh"

namespace mgj {

template <typename K> struct LocalCfg {
    using Tup = typename TupT<K>::T;
    static constexpr int V = LOCAL_V * 8 / (int)sizeof(Tup);  // 16 (8-byte) / 8 (16-byte) tuples per thread
    static constexpr int C = V * LOCAL_THREADS;                // chunk size: 8192 / 4096 tuples
};

// ---------------------------------------------------------------------------
// a4 (§3.2 "Local partitioning"): the received data of
// each owned global partition p is partitioned again by the next B2 key bits
// so that every R co-partition fits the shared-memory hash table of a5.
// B200 form: each CTA takes one chunk of C consecutive received tuples of a
// segment, counting-sorts it by digit2 in shared memory (one SMEM atomic per
// tuple gives both the bin count and the tuple's rank in its bin) and writes
// the chunk back contiguously, plus its 2^B2+1 sub-partition offsets.  The
// pass needs no global histogram and a chunk can be processed as soon as it
// has arrived (the property P:455-468 asks of [44]); co-partition q of p is
// the concatenation of the q-runs of p's chunks.  One pass suffices for every
// configured size; R runs larger than the table are handled
// by chunked builds in a5 (the skew case of P:450-452).
// Grid: persistent over all chunks of both relations.
// ---------------------------------------------------------------------------
template <typename K>
__global__ void __launch_bounds__(LOCAL_THREADS, 2) k_local(Ctx c) {
    using Tup = typename TupT<K>::T;
    constexpr int V = LocalCfg<K>::V;
    constexpr int C = LocalCfg<K>::C;
    extern __shared__ __align__(16) unsigned char smem[];
    Tup *sbuf = reinterpret_cast<Tup *>(smem);
    uint32_t *bins = reinterpret_cast<uint32_t *>(sbuf + C);  // [Q]
    __shared__ uint32_t tmp[33];
    __shared__ int s_pi;
    const int tid = threadIdx.x;
    if (!c.meta[MT_OK]) return;
    const int P = c.P, plo = c.meta[MT_PLO], phi = c.meta[MT_PHI], B2 = c.meta[MT_B2];
    const int Q = 1 << B2, np = phi - plo;
    const uint32_t nch_r = (uint32_t)c.meta[MT_NCH_R], nch_s = (uint32_t)c.meta[MT_NCH_S];
    const uint32_t total = nch_r + nch_s;
    for (uint32_t ci = blockIdx.x; ci < total; ci += gridDim.x) {
        const int rel = ci < nch_r ? 0 : 1;
        const uint32_t li = rel ? ci - nch_r : ci;
        const uint32_t *cb = c.chunk_base + rel * (P + 1);
        if (tid == 0) {  // owned partition of this chunk: last pi with cb[pi] <= li
            int lo = 0, hi = np - 1;
            while (lo < hi) {
                const int mid = (lo + hi + 1) >> 1;
                if (cb[mid] <= li) lo = mid; else hi = mid - 1;
            }
            s_pi = lo;
        }
        for (int i = tid; i < Q; i += LOCAL_THREADS) bins[i] = 0;
        __syncthreads();
        const int pi = s_pi, p = plo + pi;
        const uint64_t k = li - cb[pi];
        const uint64_t start = c.seg_start[rel * P + p] + k * C;
        const uint32_t len = (uint32_t)min((uint64_t)C, c.seg_len[rel * P + p] - k * C);
        const Tup *src = reinterpret_cast<const Tup *>(c.arena[c.rank] + c.lay.recv[rel]) + start;
        Tup *dst = static_cast<Tup *>(c.local[rel]) + start;
        Tup t[V];
        uint32_t qr[V];  // (rank in bin) << 16 | digit2
#pragma unroll
        for (int j = 0; j < V; ++j) {
            const uint32_t i = tid + j * LOCAL_THREADS;
            if (i < len) t[j] = __ldcs(src + i);
        }
#pragma unroll
        for (int j = 0; j < V; ++j) {
            const uint32_t i = tid + j * LOCAL_THREADS;
            if (i < len) {
                const uint32_t q = digit2(t[j].x, c.B1, Q);
                qr[j] = (atomicAdd(&bins[q], 1u) << 16) | q;
            }
        }
        __syncthreads();
        block_excl_scan_u32(bins, Q, tmp);
        uint16_t *coff = c.chunk_off[rel] + (size_t)li * (Q + 1);
        uint32_t *cop = c.cop_count + ((size_t)rel * P + pi) * Q;
        for (int i = tid; i <= Q; i += LOCAL_THREADS) {
            const uint32_t b = i < Q ? bins[i] : len;
            coff[i] = (uint16_t)b;
            if (i < Q) {
                const uint32_t e = (i + 1 < Q) ? bins[i + 1] : len;
                if (e > b) atomicAdd(&cop[i], e - b);
            }
        }
#pragma unroll
        for (int j = 0; j < V; ++j) {
            const uint32_t i = tid + j * LOCAL_THREADS;
            if (i < len) sbuf[bins[qr[j] & 0xffffu] + (qr[j] >> 16)] = t[j];
        }
        __syncthreads();
        for (uint32_t i = tid; i < len; i += LOCAL_THREADS) __stcs(dst + i, sbuf[i]);
        __syncthreads();
    }
}

// ---------------------------------------------------------------------------
// Probe work items: co-partition (p, q) becomes ceil(|R_pq|/PROBE_CAP) x
// ceil(|S_pq|/PROBE_S_TARGET) items, so an oversized R co-partition is built
// in table-sized chunks (block nested loop over R chunks, the "both
// relations heavily skewed" case of P:450-452) and a heavy S co-partition is
// probed by many CTAs.
// ---------------------------------------------------------------------------
__global__ void k_itemize(Ctx c) {
    if (!c.meta[MT_OK]) return;
    const int P = c.P, plo = c.meta[MT_PLO], phi = c.meta[MT_PHI];
    const int Q = 1 << c.meta[MT_B2];
    const uint64_t total = (uint64_t)(phi - plo) * Q;
    for (uint64_t idx = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; idx < total;
         idx += (uint64_t)gridDim.x * blockDim.x) {
        const uint32_t pi = (uint32_t)(idx / Q), q = (uint32_t)(idx % Q);
        const uint32_t r = c.cop_count[(size_t)pi * Q + q];
        const uint32_t s = c.cop_count[((size_t)P + pi) * Q + q];
        if (r == 0 || s == 0) continue;
        const uint32_t nr = (r + PROBE_CAP - 1) / PROBE_CAP;
        const uint32_t ns = (s + PROBE_S_TARGET - 1) / PROBE_S_TARGET;
        const uint64_t n = (uint64_t)nr * ns;
        const uint32_t base = atomicAdd(&c.ticket[TK_ITEMS], (uint32_t)n);
        if ((uint64_t)base + n > c.max_items) {
            set_err(c, MGJ_ECAPACITY);
            continue;
        }
        for (uint32_t a = 0; a < nr; ++a)
            for (uint32_t b = 0; b < ns; ++b) {
                Item it;
                it.pi = pi;
                it.q = q;
                it.r_lo = (uint32_t)((uint64_t)r * a / nr);
                it.r_hi = (uint32_t)((uint64_t)r * (a + 1) / nr);
                it.s_lo = (uint32_t)((uint64_t)s * b / ns);
                it.s_hi = (uint32_t)((uint64_t)s * (b + 1) / ns);
                c.items[base + a * ns + b] = it;
            }
    }
}

// Walk the q-runs of owned partition pi (= p - p_lo) of relation rel in
// logical order (chunk order) and hand every part of a run that falls in the
// logical range [lo, hi) to a warp: f(src, n, first) is called by all 32
// lanes of one warp for n consecutive tuples at src whose first tuple has
// logical index lo + first.  Chunk runs are staged PROBE_WIN at a time.
template <typename Tup, typename F>
__device__ inline void for_runs(const Ctx &c, int rel, int pi, int p, uint32_t q, int Q, uint32_t lo, uint32_t hi,
                                int C, uint32_t *rlen, uint32_t *rpos, uint32_t *tmp, F &&f) {
    const int tid = threadIdx.x, warp = tid >> 5, nw = blockDim.x >> 5;
    const uint32_t *cbp = c.chunk_base + rel * (c.P + 1);
    const uint32_t cb = cbp[pi], nch = cbp[pi + 1] - cb;
    const uint16_t *coff = c.chunk_off[rel] + (size_t)cb * (Q + 1);
    const Tup *base = static_cast<const Tup *>(c.local[rel]) + c.seg_start[rel * c.P + p];
    uint32_t logical = 0;
    for (uint32_t w0 = 0; w0 < nch && logical < hi; w0 += PROBE_WIN) {
        const uint32_t wn = min((uint32_t)PROBE_WIN, nch - w0);
        for (uint32_t k = tid; k < wn; k += blockDim.x) {
            const uint16_t *row = coff + (size_t)(w0 + k) * (Q + 1);
            const uint32_t s = row[q], e = row[q + 1];
            rlen[k] = e - s;
            rpos[k] = (w0 + k) * (uint32_t)C + s;
        }
        __syncthreads();
        const uint32_t tot = block_excl_scan_u32(rlen, (int)wn, tmp);
        for (uint32_t k = warp; k < wn; k += nw) {
            const uint32_t a = logical + rlen[k];
            const uint32_t b = logical + (k + 1 < wn ? rlen[k + 1] : tot);
            const uint32_t x0 = max(a, lo), x1 = min(b, hi);
            if (x0 < x1) f(base + rpos[k] + (x0 - a), x1 - x0, x0 - lo);
        }
        logical += tot;
        __syncthreads();
    }
}

// ---------------------------------------------------------------------------
// a5 (§3.2 "Probe"): per work item, the R slice of
// co-partition (p, q) is gathered into shared memory and a chained hash
// table is built over it (the SMEM hash-table variant of P:471-472, which the
// north star asks for; the paper's nested loop is its degenerate form), then
// the S slice streams through: one warp per run, lanes walk chains and
// compare full keys.  count += 1 and checksum += a*C + b (mod 2^64) for every
// equal-key pair; with MAT the item's matches are first counted, one
// reservation is taken in the output, and a second pass over the (L2-
// resident) S slice writes the (key, payR, payS) triples at exact positions.
// ---------------------------------------------------------------------------
template <typename K, bool MAT>
__global__ void __launch_bounds__(PROBE_THREADS) k_probe(Ctx c) {
    using Tup = typename TupT<K>::T;
    constexpr int C = LocalCfg<K>::C;
    constexpr int T = PROBE_CAP;
    constexpr int LOGT = 12;
    constexpr uint32_t EMPTY = 0xffffffffu;
    static_assert((1 << LOGT) == T, "table size");
    extern __shared__ __align__(16) unsigned char smem[];
    Tup *rt = reinterpret_cast<Tup *>(smem);
    uint32_t *head = reinterpret_cast<uint32_t *>(rt + PROBE_CAP);
    uint32_t *nxt = head + T;
    uint32_t *rlen = nxt + PROBE_CAP;
    uint32_t *rpos = rlen + PROBE_WIN;
    __shared__ uint32_t tmp[33];
    __shared__ unsigned long long s_base;
    __shared__ uint32_t s_cur, s_m;
    __shared__ int s_write;
    if (!c.meta[MT_OK]) return;
    const int tid = threadIdx.x, lane = tid & 31;
    const int plo = c.meta[MT_PLO], B2 = c.meta[MT_B2];
    const int Q = 1 << B2, shift = c.B1 + B2;
    const uint32_t nitems = min(__ldcg(&c.ticket[TK_ITEMS]), c.max_items);
    unsigned long long my_cnt = 0, my_chk = 0;

    for (uint32_t it = blockIdx.x; it < nitems; it += gridDim.x) {
        const Item I = c.items[it];
        const int pi = (int)I.pi, p = plo + pi;
        const uint32_t nr = I.r_hi - I.r_lo;
        for (int i = tid; i < T; i += PROBE_THREADS) head[i] = EMPTY;
        for_runs<Tup>(c, 0, pi, p, I.q, Q, I.r_lo, I.r_hi, C, rlen, rpos, tmp,
                      [&](const Tup *src, uint32_t n, uint32_t first) {
                          for (uint32_t x = lane; x < n; x += 32) rt[first + x] = src[x];
                      });
        for (uint32_t i = tid; i < nr; i += PROBE_THREADS) nxt[i] = atomicExch(&head[tab_hash(rt[i].x, shift, LOGT)], i);
        __syncthreads();

        if (!MAT) {
            for_runs<Tup>(c, 1, pi, p, I.q, Q, I.s_lo, I.s_hi, C, rlen, rpos, tmp,
                          [&](const Tup *src, uint32_t n, uint32_t) {
                              for (uint32_t x = lane; x < n; x += 32) {
                                  const Tup s = src[x];
                                  for (uint32_t i = head[tab_hash(s.x, shift, LOGT)]; i != EMPTY; i = nxt[i]) {
                                      const Tup r = rt[i];
                                      if (r.x == s.x) {
                                          ++my_cnt;
                                          my_chk += chk_term(r.y, s.y);
                                      }
                                  }
                              }
                          });
        } else {
            uint32_t m = 0;
            for_runs<Tup>(c, 1, pi, p, I.q, Q, I.s_lo, I.s_hi, C, rlen, rpos, tmp,
                          [&](const Tup *src, uint32_t n, uint32_t) {
                              for (uint32_t x = lane; x < n; x += 32) {
                                  const Tup s = src[x];
                                  for (uint32_t i = head[tab_hash(s.x, shift, LOGT)]; i != EMPTY; i = nxt[i]) {
                                      const Tup r = rt[i];
                                      if (r.x == s.x) {
                                          ++m;
                                          my_chk += chk_term(r.y, s.y);
                                      }
                                  }
                              }
                          });
            my_cnt += m;
            if (tid == 0) s_m = 0;
            __syncthreads();
            const uint32_t wm = (uint32_t)warp_sum(m);
            if (lane == 0 && wm) atomicAdd(&s_m, wm);
            __syncthreads();
            if (tid == 0) {
                const uint32_t M = s_m;
                s_cur = 0;
                s_base = M ? atomicAdd(&c.acc[2], (unsigned long long)M) : 0;
                s_write = M && (s_base + M <= c.out_cap);
                if (M && !s_write) set_err(c, MGJ_ECAPACITY);
            }
            __syncthreads();
            if (s_write) {
                K *ok = static_cast<K *>(c.out_key);
                K *oa = static_cast<K *>(c.out_a);
                K *ob = static_cast<K *>(c.out_b);
                const unsigned long long base = s_base;
                for_runs<Tup>(c, 1, pi, p, I.q, Q, I.s_lo, I.s_hi, C, rlen, rpos, tmp,
                              [&](const Tup *src, uint32_t n, uint32_t) {
                                  for (uint32_t x0 = 0; x0 < n; x0 += 32) {
                                      const uint32_t x = x0 + lane;
                                      Tup s;
                                      uint32_t i = EMPTY;
                                      if (x < n) {
                                          s = src[x];
                                          i = head[tab_hash(s.x, shift, LOGT)];
                                      }
                                      while (__any_sync(0xffffffffu, i != EMPTY)) {
                                          bool hit = false;
                                          Tup r;
                                          if (i != EMPTY) {
                                              r = rt[i];
                                              hit = r.x == s.x;
                                              i = nxt[i];
                                          }
                                          const uint32_t bal = __ballot_sync(0xffffffffu, hit);
                                          if (bal) {
                                              uint32_t wb = 0;
                                              if (lane == 0) wb = atomicAdd(&s_cur, (uint32_t)__popc(bal));
                                              wb = __shfl_sync(0xffffffffu, wb, 0);
                                              if (hit) {
                                                  const unsigned long long pos =
                                                      base + wb + __popc(bal & ((1u << lane) - 1u));
                                                  ok[pos] = (K)s.x;
                                                  oa[pos] = (K)r.y;
                                                  ob[pos] = (K)s.y;
                                              }
                                          }
                                      }
                                  }
                              });
            }
        }
        __syncthreads();
    }
    my_cnt = warp_sum(my_cnt);
    my_chk = warp_sum(my_chk);
    if (lane == 0 && (my_cnt || my_chk)) {
        atomicAdd(&c.acc[0], my_cnt);
        atomicAdd(&c.acc[1], my_chk);
    }
}

// ---------------------------------------------------------------------------
// a6: count = sum_g count_g, checksum = sum_g checksum_g (mod 2^64), split in
// two so that several ranks can share one stream (virtual ranks):
//  k_publish (end of mgj_join): store this rank's (count, checksum, n_out,
//    status) in every peer's arena and raise SIG_RES there;
//  k_gather (mgj_result): wait for every rank's SIG_RES and sum the N entries
//    (order-free, bit-exact).
// ---------------------------------------------------------------------------
__global__ void k_publish(Ctx c) {
    if (threadIdx.x != 0 || blockIdx.x != 0) return;
    const int32_t st = *(volatile int32_t *)c.err;
    const unsigned long long v[4] = {__ldcg(&c.acc[0]), __ldcg(&c.acc[1]), __ldcg(&c.acc[2]),
                                     (unsigned long long)(uint32_t)st};
    for (int d = 0; d < c.world; ++d) {
        volatile unsigned long long *rm =
            reinterpret_cast<unsigned long long *>(c.arena[d] + c.lay.resmail) + c.rank * 4;
        rm[0] = v[0];
        rm[1] = v[1];
        rm[2] = v[2];
        rm[3] = v[3];
    }
    __threadfence_system();
    signal_all(c, SIG_RES);
}

__global__ void k_gather(Ctx c) {
    if (threadIdx.x != 0 || blockIdx.x != 0) return;
    unsigned long long cnt = 0, chk = 0;
    int32_t gst = 0;
    if (!wait_all_flags(c, SIG_RES)) {
        gst = MGJ_EPEER;
    } else {
        const volatile unsigned long long *rm =
            reinterpret_cast<const unsigned long long *>(c.arena[c.rank] + c.lay.resmail);
        for (int g = 0; g < c.world; ++g) {
            cnt += rm[g * 4 + 0];
            chk += rm[g * 4 + 1];
            const int32_t s = (int32_t)(uint32_t)rm[g * 4 + 3];
            if (gst == 0 && s != 0) gst = s;
        }
    }
    c.result[0] = cnt;
    c.result[1] = chk;
    c.result[2] = __ldcg(&c.acc[2]);
    c.result[3] = (unsigned long long)(uint32_t)gst;
}

}  // namespace mgj
