// local_probe.cuh — phase a4 (local radix partitioning of the received
// segments), phase a5 (shared-memory build/probe) and a6 (cross-rank sum).
#pragma once

#include "common.cuh"
#include "tma.cuh"

namespace mgj {

// (Probe variants measured in round 1 and not kept, against 1.96 ms at M2:
// L2 bulk prefetch of later items' runs 2.40-2.53 ms, cp.async instead of
// bulk copies 4.64, lane copies of short runs (Zipf z = 1: 3.13-3.55 vs
// 2.80), an even R + S split between the producers 2.35, a software-
// pipelined packed probe 2.02, two S slots per step 2.00, the packed table
// for 8-byte keys 3.04 vs 2.82 at M5.  Round 2, against 1.885 ms: fewer
// instructions per match 1.902, S slots in batches of 2 / 4 per thread
// 2.015 / 2.116, head exchanges 2 / 4 at a time 1.899 / 1.889, the build of
// item j+1 beside the probe of item j in a second table 2.86 — the consumers
// are busy 94% of the time and the copies keep up.)

template <typename K> struct Layout {
    using Tup = typename TupT<K>::T;
    static constexpr int TB = (int)sizeof(Tup);
    static constexpr int ALIGN = 16 / TB;  // tuples per 16 bytes: runs are padded to this (2 / 1)
};

// Run q of a chunk, decoded from the chunk's offset row E (reading of the
// padded layout written by k_local): first slot, slots (padded length) and
// valid tuples.  For 8-byte tuples E[q] = start | (count odd), E[Q] = end.
template <int ALIGN>
__device__ __forceinline__ void decode_run(uint32_t e0, uint32_t e1, uint32_t &start, uint32_t &slots,
                                           uint32_t &valid) {
    if (ALIGN == 2) {
        start = e0 & ~1u;
        slots = (e1 & ~1u) - start;
        valid = slots - (e0 & 1u);
    } else {
        start = e0;
        slots = e1 - e0;
        valid = slots;
    }
}

// Two chunk buffers that alternate roles (TMA load target of chunk j+1 /
// sorted output of chunk j), plus two alternating bin-counter arrays and the
// run starts.
__host__ __device__ inline size_t local_smem_bytes(int C, int Qmax, int TB) {
    return 2 * (size_t)(C + Qmax + 2) * TB + 3 * (size_t)Qmax * 4;
}

// Chunk descriptors for the local pass: chunk ci of owned partition pi covers
// received tuples [start, start + len).
struct ChunkDesc {
    uint64_t start;
    uint32_t len;
    uint32_t pi;
};

__global__ void k_chunkmap(Ctx c, ChunkDesc *desc) {
    if (!c.meta[MT_OK]) return;
    const int P = c.P, np = c.meta[MT_NP];
    const uint32_t nch_r = (uint32_t)c.meta[MT_NCH_R], total = nch_r + (uint32_t)c.meta[MT_NCH_S];
    // the table k_plan built: chunks of C tuples, or of C 32-byte units with the compressed shuffle
    const uint64_t C = (uint64_t)(c.comp ? c.chunk_units : (c.meta[MT_BA] ? c.chunk_tuples1s : c.chunk_tuples));
    for (uint32_t ci = blockIdx.x * blockDim.x + threadIdx.x; ci < total; ci += gridDim.x * blockDim.x) {
        const int rel = ci < nch_r ? 0 : 1;
        const uint32_t li = rel ? ci - nch_r : ci;
        const uint32_t *cb = c.chunk_base + (size_t)rel * c.cb_stride;
        int lo = 0, hi = np - 1;
        while (lo < hi) {
            const int mid = (lo + hi + 1) >> 1;
            if (__ldg(cb + mid) <= li) lo = mid; else hi = mid - 1;
        }
        const uint32_t j = li - cb[lo];
        const uint32_t *pc = c.piece_chunk + ((size_t)rel * P + lo) * (MAX_RANKS + 1);
        int g = 0;
        while (c.ext && g + 1 < MAX_RANKS && pc[g + 1] <= j) ++g;  // piece holding chunk j of partition lo (P2P: one)
        const uint64_t k = j - pc[g];
        const size_t pidx = ((size_t)rel * P + lo) * MAX_RANKS + g;
        ChunkDesc d;
        d.start = c.piece_start[pidx] + k * C;
        d.len = (uint32_t)min(C, (uint64_t)c.piece_len[pidx] - k * C);
        d.pi = (uint32_t)lo;
        desc[ci] = d;
        if (c.stream && rel == 1) {
            // NEXT-3: the S rounds this chunk needs.  A P2P segment holds the
            // sources' pieces back to back (sources ascending; a broadcast
            // partition's S only this rank's own): sources g_lo..g_hi overlap
            // the chunk; those before g_hi end inside it (all their rounds),
            // g_hi needs the rounds whose first offset lies below the chunk's end
            const int pg = c.plist[lo];
            const uint64_t o0 = k * C, o1 = o0 + d.len;
            int glo = c.rank, ghi = c.rank;
            uint64_t base_hi = 0;
            if (!c.bcast[pg]) {
                const uint32_t *cnt = reinterpret_cast<const uint32_t *>(c.arena[c.rank] + (c.comp ? c.lay.umail : c.lay.mail));
                uint64_t b = 0;
                glo = -1;
                for (int s = 0; s < c.world; ++s) {
                    const uint64_t e = b + __ldcg(cnt + (size_t)(s * 2 + 1) * P + pg);
                    if (e > o0 && b < o1) {
                        if (glo < 0) glo = s;
                        ghi = s;
                        base_hi = b;
                    }
                    b = e;
                }
                if (glo < 0) glo = ghi = c.rank;  // (an empty chunk: none)
            }
            int rh = 0;
            while (rh + 1 < c.nrounds && base_hi + __ldcg(rb_first(c.arena[ghi], c.lay, P, rh + 1, pg)) < o1) ++rh;
            c.cwait[li] = (uint32_t)(glo << 8 | ghi << 4 | rh);
            atomicAdd(&c.rcount[glo < ghi ? c.nrounds - 1 : rh], 1u);
        }    }
}

// NEXT-3: the S chunks in round order (a counting sort by the last round each
// needs; the order inside a round is free: outputs are placed by chunk index).
__global__ void k_chunkorder(Ctx c) {
    if (!c.meta[MT_OK] || !c.stream) return;
    __shared__ uint32_t base[STREAM_RMAX];
    if (threadIdx.x == 0) {
        uint32_t a = 0;
        for (int r = 0; r < STREAM_RMAX; ++r) base[r] = a, a += __ldcg(&c.rcount[r]);
    }
    __syncthreads();
    const uint32_t nch_s = (uint32_t)c.meta[MT_NCH_S];
    for (uint32_t li = blockIdx.x * blockDim.x + threadIdx.x; li < nch_s; li += gridDim.x * blockDim.x) {
        const uint32_t w = c.cwait[li];
        const int r = ((w >> 8) & 15u) < ((w >> 4) & 15u) ? c.nrounds - 1 : (int)(w & 15u);
        c.corder[base[r] + atomicAdd(&c.rcount[STREAM_RMAX + r], 1u)] = li;
    }
}

// NEXT-3: thread-level wait until every source rank g_lo..g_hi of a chunk
// has stored every non-empty S tile of the rounds the chunk needs for this
// run (w = g_lo << 8 | g_hi << 4 | rh: all rounds of g < g_hi, rounds 0..rh
// of g_hi; the sources' counters, polled over NVLink), then order the async
// proxy's (TMA) reads of the received tuples after it.
__device__ inline void stream_wait(const Ctx &c, uint32_t w) {
    const int glo = (int)((w >> 8) & 15u), ghi = (int)((w >> 4) & 15u), rh = (int)(w & 15u);
    const uint64_t t0 = globaltimer();
    for (int g = glo; g <= ghi; ++g) {
        for (int r = 0; r <= (g < ghi ? c.nrounds - 1 : rh); ++r) {
            const uint64_t want = c.epoch << 32 | __ldcg(rb_ntile(c.arena[g], c.lay) + r);
            const uint64_t *f = reinterpret_cast<const uint64_t *>(rdone_ptr(c.arena[g], c.lay, r));
            while (ld_acquire_sys(f) < want) {
                if (globaltimer() - t0 > c.timeout_ns) {
                    set_err(c, MGJ_EPEER);
                    return;
                }
                __nanosleep(64);
            }
        }
    }
    fence_proxy_async_global();
}

// ---------------------------------------------------------------------------
// Two-level local partitioning (multi-pass a4).
// One chunked pass writes one run per (chunk, sub-partition), so an owned
// partition of nch chunks leaves each co-partition in nch runs of ~C/Q
// tuples.  At N = 8 (M2) an owner's partitions are 8x larger than at N = 1
// and the runs shrink to a dozen tuples, which the probe cannot fetch
// efficiently.  Then (k_plan sets BA > 0) a first pass (k_local_split, the
// chunked sort by the BA key bits above B1, each chunk stored in place with
// its run offsets, like the paper's histogram-free local pass) leaves every
// (owned partition, BA-bit digit) sub-partition v as one run per chunk of
// ~C/2^BA tuples; k_planA numbers the chunks of the second pass (ceil of each
// sub-partition's padded size, counted by the first pass, over C2), k_emit2
// cuts each sub-partition's runs into those chunks, and the chunked pass
// (k_local_second) gathers a chunk's runs by bulk copies and partitions it by
// the remaining B2 - BA bits.  No pass only counts.
// ---------------------------------------------------------------------------
__device__ __forceinline__ uint32_t nch_local(const Ctx &c, int rel) {
    return (uint32_t)c.meta[c.meta[MT_BA] ? MT_NCHB_R + rel : MT_NCH_R + rel];
}

// A chunk of the second pass: the slots [(k0, a0), (k1, a1)) of sub-partition
// v's runs, run k being sub-partition v's run in first-pass chunk k (chunk
// indices of the relation, ascending), a a slot offset inside it.
struct ChunkDescB {
    uint32_t v, k0, a0, k1, a1, len;
};

// Chunk table of the second pass: first chunk of every sub-partition v (the
// exclusive scan of ceil(padded size / C2)); the first pass's table of the
// owned partitions is kept in chunk_base1 for k_emit2.  One CTA.
__global__ void __launch_bounds__(1024) k_planA(Ctx c) {
    extern __shared__ uint64_t sv[];  // [L+1] then u32 [L+1]
    __shared__ uint32_t tmp32[33];
    if (!c.meta[MT_OK] || !c.meta[MT_BA]) return;
    const int BA = c.meta[MT_BA];
    const int np = c.meta[MT_NP], L = np << BA;
    const int tid = threadIdx.x;
    uint32_t *nch = reinterpret_cast<uint32_t *>(sv + L + 1);
    const uint64_t C = (uint64_t)c.chunk_tuples2;  // the chunked pass after the first pass
    uint32_t tot_ch[2];
    bool bad = false;
    for (int rel = 0; rel < 2; ++rel) {
        const uint32_t *h = c.hA + (size_t)rel * c.vcap;
        uint32_t *cb = c.chunk_base + (size_t)rel * c.cb_stride;
        for (int i = tid; i <= np; i += blockDim.x) c.chunk_base1[(size_t)rel * c.cb_stride + i] = cb[i];
        for (int v = tid; v <= L; v += blockDim.x) {
            const uint32_t n = v < L ? __ldcg(h + v) : 0;
            nch[v] = (uint32_t)((n + C - 1) / C);
        }
        __syncthreads();  // (the first pass's table is copied before it is overwritten)
        tot_ch[rel] = block_excl_scan_u32(nch, L + 1, tmp32);
        bad |= tot_ch[rel] > c.max_chunks;
        for (int v = tid; v <= L; v += blockDim.x) cb[v] = nch[v];
        __syncthreads();
    }
    if (tid == 0) {
        c.meta[MT_NCHB_R] = (int)tot_ch[0];
        c.meta[MT_NCHB_S] = (int)tot_ch[1];
        c.meta[MT_NLP] = L;
        if (bad) {
            set_err(c, MGJ_ECAPACITY);
            c.meta[MT_OK] = 0;
        }
    }
}

// The second pass's chunk descriptors: one warp per (relation, sub-partition
// v) walks v's runs in first-pass chunk order (32 at a time, a warp scan of
// their padded sizes) and cuts them at every multiple of C2: chunk s of v is
// the slots [s * C2, min((s + 1) * C2, total)) of the concatenated runs.
template <typename K>
__global__ void k_emit2(Ctx c, ChunkDescB *descB) {
    constexpr int ALIGN = Layout<K>::ALIGN;
    if (!c.meta[MT_OK] || !c.meta[MT_BA]) return;
    const int BA = c.meta[MT_BA], QA = 1 << BA;
    const int L = c.meta[MT_NLP];
    const uint32_t C2 = (uint32_t)c.chunk_tuples2;
    const uint32_t nchb_r = (uint32_t)c.meta[MT_NCHB_R];
    const int lane = threadIdx.x & 31;
    const uint32_t warps = (gridDim.x * blockDim.x) >> 5;
    for (uint32_t w = (blockIdx.x * blockDim.x + threadIdx.x) >> 5; w < 2u * (uint32_t)L; w += warps) {
        const int rel = w >= (uint32_t)L, v = (int)(w - (rel ? L : 0));
        const int pi = v >> BA, a = v & (QA - 1);
        const uint32_t *cb1 = c.chunk_base1 + (size_t)rel * c.cb_stride;
        const uint32_t kb = __ldcg(cb1 + pi), ke = __ldcg(cb1 + pi + 1);
        const uint32_t out0 = (rel ? nchb_r : 0u) + __ldcg(c.chunk_base + (size_t)rel * c.cb_stride + v);
        const uint16_t *E = c.eoffA[rel];
        uint32_t pre = 0;  // slots of v's runs before this batch
        for (uint32_t k0 = kb; k0 < ke; k0 += 32) {
            const uint32_t k = k0 + lane;
            uint32_t slots = 0, st = 0, valid = 0;
            if (k < ke) decode_run<ALIGN>(E[(size_t)k * EA_STRIDE + a], E[(size_t)k * EA_STRIDE + a + 1], st, slots, valid);
            uint32_t incl = slots;
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                const uint32_t y = __shfl_up_sync(0xffffffffu, incl, o);
                if (lane >= o) incl += y;
            }
            const uint32_t lo = pre + incl - slots, hi = pre + incl;  // this run: [lo, hi) of v's slots
            // every chunk boundary s * C2 inside [lo, hi): chunk s starts here, chunk s - 1 ends here
            for (uint32_t s = (lo + C2 - 1) / C2; s * C2 < hi; ++s) {
                ChunkDescB *d = descB + out0 + s;
                d->v = (uint32_t)v;
                d->k0 = k;
                d->a0 = s * C2 - lo;
                if (s > 0) {
                    ChunkDescB *e = d - 1;
                    e->k1 = k;
                    e->a1 = s * C2 - lo;
                    e->len = C2;
                }
            }
            pre += __shfl_sync(0xffffffffu, incl, 31);
            (void)valid;
        }
        if (lane == 0 && pre > 0) {  // the last chunk ends after v's last run
            const uint32_t s = (pre - 1) / C2;
            ChunkDescB *d = descB + out0 + s;
            d->k1 = ke;
            d->a1 = 0;
            d->len = pre - s * C2;
        }
    }
}

// ---------------------------------------------------------------------------
// a4 (§3.2 "Local partitioning"): the received data of
// each owned global partition p is partitioned again by the next B2 key bits
// so that every R co-partition fits a shared-memory hash table.
// B200 form: a persistent CTA per SM streams chunks of C received tuples in
// by TMA (double-buffered, two chunks ahead), counting-sorts each chunk by
// its digit in shared memory (one SMEM atomic per tuple gives bin count and
// rank), and streams the sorted chunk out by TMA bulk store.  Runs are
// padded to 16 bytes so the probe can fetch them with bulk copies.  No global
// histogram is needed and a chunk can be processed as soon as it has arrived
// — the property the paper takes [44] for.
//  MODE = LM_SINGLE (the only pass, BA = 0) / LM_SECOND (after a first
//    pass): the chunked pass.  digit = the B2 - BA key bits above B1 + BA,
//    one bulk store per chunk, run offsets to E[(Q+1)*chunk_base[v] +
//    q*nch_v + k] (contiguous per (v, q)).  LM_SECOND gathers its chunk from
//    the first pass's runs of sub-partition v (k_emit2's descriptors, one
//    bulk copy per run piece) and drops the first pass's padding tuples
//    (digit1 != p).
//  MODE = LM_SPLIT (first pass of two-level partitioning): digit = the BA
//    bits above B1; the sorted chunk is stored in place (chunk li at
//    mid + li * chunk_region1) with its run offsets in eoffA, and each run's
//    padded size is added to its sub-partition's total (hA).
// Each instance returns at once when the run's BA does not select it.
// R co-partitions larger than the table are built in pieces by a5
// (P:450-452's skew case).
// ---------------------------------------------------------------------------
enum LocalMode { LM_SINGLE = 0, LM_SPLIT = 1, LM_SECOND = 2 };

template <int MODE> struct LocalDesc { using T = ChunkDesc; };
template <> struct LocalDesc<2> { using T = ChunkDescB; };

template <typename K, int MODE, int RSEL = 2, bool COMP = false, bool STRM = false>
__device__ __forceinline__ void local_body(const Ctx &c, const typename LocalDesc<MODE>::T *cdesc) {
    static_assert(!COMP || (MODE == LM_SINGLE && sizeof(K) == 4), "compressed input: single pass, 4-byte keys");
    using Desc = typename LocalDesc<MODE>::T;
    constexpr bool SPLIT = MODE == LM_SPLIT;
    using Tup = typename Layout<K>::Tup;
    constexpr int TB = Layout<K>::TB, ALIGN = Layout<K>::ALIGN;
    constexpr int VMAX = local_vmax(TB);
    extern __shared__ __align__(128) unsigned char smem[];
    __shared__ __align__(8) uint64_t bar[2];
    __shared__ Desc sdesc[2];
    __shared__ uint32_t tmp[33];
    const int BA = MODE == LM_SINGLE ? 0 : c.meta[MT_BA];
    const int tid = threadIdx.x;
    // LM_SECOND has its own chunk geometry (fan-out <= 2^(b2_max - 1): larger chunks fit)
    const int C = MODE == LM_SECOND ? c.chunk_tuples2 : (SPLIT ? c.chunk_tuples1s : c.chunk_tuples);
    const int CR = MODE == LM_SECOND ? c.chunk_region2 : c.chunk_region, V = C / LOCAL_THREADS;
    const int P = c.P, Q = 1 << (SPLIT ? BA : c.meta[MT_QB]);
    const int shift = SPLIT ? c.B1 : c.B1 + BA;  // digit = (key >> shift) & (Q - 1)
    const int Qmax = 1 << c.b2_max;  // stride of the co-partition size table
    const int QL = MODE == LM_SECOND ? 1 << c.qm2_bits : (SPLIT ? 1 << MAX_BA : Qmax);  // bins / padding in shared memory
    const int BUF = C + QL + 2;  // slots per buffer
    Tup *const buf0 = reinterpret_cast<Tup *>(smem);
    auto buf = [&](int x) { return buf0 + (size_t)x * BUF; };
    uint32_t *const bins2 = reinterpret_cast<uint32_t *>(buf0 + (size_t)2 * BUF);  // [2][QL], chunk j uses j & 1
    uint32_t *const abin = bins2 + 2 * QL;
    const uint32_t nch_r = SPLIT ? (uint32_t)c.meta[MT_NCH_R] : nch_local(c, 0);
    const uint32_t total = nch_r + (SPLIT ? (uint32_t)c.meta[MT_NCH_S] : nch_local(c, 1));
    // chunks of R [0, nch_r), of S [nch_r, total); RSEL picks R (0), S (1) or both (2)
    const uint32_t c0 = RSEL == 1 ? nch_r : 0u, c1 = RSEL == 0 ? nch_r : total;
    const uint32_t span = c1 - c0;
    const uint32_t mine = span > blockIdx.x ? (span - blockIdx.x + gridDim.x - 1) / gridDim.x : 0;
    // NEXT-3 streaming (S pass beside S's scatter): the chunks in round order,
    // each loaded once the scatter rounds it needs are complete
    static_assert(!STRM || (RSEL == 1 && MODE == LM_SINGLE), "streaming: S's single pass");
    constexpr bool strm = STRM;
    auto cidx = [&](uint32_t j) -> uint32_t {
        const uint32_t k = blockIdx.x + j * gridDim.x;
        return c0 + (strm ? __ldcg(c.corder + k) : k);
    };
    constexpr bool from_mid = MODE == LM_SECOND;
    // source of a chunk: a receive buffer (this rank's, or a broadcast
    // partition root's for its R side: piece_src)
    auto chunk_src = [&](int rel, uint64_t start) -> const Tup * {
        return reinterpret_cast<const Tup *>(c.arena[piece_src(start)] + c.lay.recv[rel]) + piece_off(start);
    };
    if (tid == 0) {
        mbar_init(&bar[0], 1);
        mbar_init(&bar[1], 1);
        fence_mbar_init();
    }
    for (int q = tid; q < 2 * QL; q += LOCAL_THREADS) bins2[q] = 0;
    __syncthreads();
    const uint64_t pol = policy_evict_first();
    constexpr int LI = 32;  // the thread that issues the chunk loads (and the chunked pass's stores)
    // LM_SECOND: warps issuing a chunk's run copies (measured at B1 = 7 / 8-byte keys at
    // B1 = 6, local pass: 1 warp 6.28 / 6.79 ms, 2 6.20 / 6.32, 4 6.25 / 6.11, 8 6.27 / 6.15)
    constexpr int GW = 4;
    // thread LI: TMA chunk j (16-byte-aligned superset) into buffer j & 1
    auto issue = [&](uint32_t j, const Desc &d) {
        const uint32_t ci = cidx(j);
        const int rel = ci < nch_r ? 0 : 1;
        if (strm) stream_wait(c, __ldcg(c.cwait + (ci - c0)));
        sdesc[j & 1] = d;
        uint64_t *b = &bar[j & 1];
        if constexpr (from_mid) {
            // the pieces of sub-partition d.v's runs, back to back: the issuing
            // warps' lanes take 32 runs at a time (their offsets loaded in
            // parallel, destinations by a warp scan); piece i is copied by lane i
            // of issuing warp i mod GW, so the copies issue from GW warps at once
            const int lane = tid & 31, gw = (tid >> 5) - (LI >> 5);
            if (tid == LI) mbar_arrive_expect_tx(b, d.len * TB);
            named_bar_sync(2, 32 * GW);  // the expected bytes are set before any copy lands
            const int a = (int)(d.v & ((1u << BA) - 1));
            const uint16_t *E = c.eoffA[rel];
            const Tup *mid = static_cast<const Tup *>(c.mid[rel]);
            uint32_t at = 0;
            for (uint32_t kb = d.k0; kb <= d.k1; kb += 32) {
                const uint32_t k = kb + lane;
                uint32_t pc = 0;
                size_t src = 0;
                if (k <= d.k1 && !(k == d.k1 && d.a1 == 0)) {
                    uint32_t st, slots, valid;
                    decode_run<ALIGN>(__ldcg(E + (size_t)k * EA_STRIDE + a), __ldcg(E + (size_t)k * EA_STRIDE + a + 1), st,
                                      slots, valid);
                    const uint32_t alo = k == d.k0 ? d.a0 : 0u, ahi = k == d.k1 ? d.a1 : slots;
                    if (ahi > alo) {
                        pc = ahi - alo;
                        src = (size_t)k * c.chunk_region1 + st + alo;
                    }
                }
                uint32_t incl = pc;
#pragma unroll
                for (int o = 1; o < 32; o <<= 1) {
                    const uint32_t y = __shfl_up_sync(0xffffffffu, incl, o);
                    if (lane >= o) incl += y;
                }
                if (pc && (lane % GW) == gw) tma_load_1d(buf(j & 1) + at + incl - pc, mid + src, pc * TB, b, pol);
                at += __shfl_sync(0xffffffffu, incl, 31);
            }
            return;
        } else if constexpr (COMP) {  // whole 32-byte units
            const uint32_t bytes = d.len * 32u;
            mbar_arrive_expect_tx(b, bytes);
            if (bytes)
                tma_load_1d(buf(j & 1), c.arena[piece_src(d.start)] + c.lay.recv[rel] + piece_off(d.start) * 32, bytes, b,
                            pol);
            return;
        }
        else {
            const uint64_t st = piece_off(d.start);
            const uint64_t g0 = st & ~(uint64_t)(ALIGN - 1);
            const uint64_t g1 = (st + d.len + ALIGN - 1) & ~(uint64_t)(ALIGN - 1);
            const uint32_t bytes = (uint32_t)((g1 - g0) * TB);
            mbar_arrive_expect_tx(b, bytes);
            if (bytes) tma_load_1d(buf(j & 1), chunk_src(rel, d.start) - (st - g0), bytes, b, pol);
        }
    };
    Desc nxt{};
    // (the second pass issues its run pieces with GW whole warps from LI's on)
    auto issuer = [&]() { return from_mid ? (unsigned)((tid >> 5) - (LI >> 5)) < (unsigned)GW : tid == LI; };
    if (issuer()) {
        if (mine > 0) issue(0, cdesc[cidx(0)]);
        if (mine > 1) nxt = cdesc[cidx(1)];
    }
    for (uint32_t j = 0; j < mine; ++j) {
        const uint32_t ci = cidx(j);
        const int rel = ci < nch_r ? 0 : 1;
        const uint32_t li = rel ? ci - nch_r : ci;
        const int X = j & 1;
        uint32_t *const bins = bins2 + X * QL;  // zero (cleared during chunk j - 1)
        mbar_wait(&bar[X], (j >> 1) & 1);
        const Desc d = sdesc[X];
        uint32_t skip = 0, dpi = 0;  // slots before the chunk's first tuple; its (sub-)partition
        if constexpr (from_mid) {
            dpi = d.v;
        } else {
            skip = (uint32_t)(d.start & (ALIGN - 1));
            dpi = d.pi;
        }
        const uint32_t len = d.len;
        // partition of this chunk's tuples (a first pass's padding tuples lie in another one)
        const uint32_t p = (uint32_t)c.plist[from_mid ? dpi >> BA : dpi];
        Tup t[VMAX];
        uint32_t cvalid = 0;  // COMP: bit v set if t[v] holds a decoded tuple
        if constexpr (COMP) {
            // NEXT-1 decode: this thread's units tid, tid + 1024 of the chunk, CU_N
            // entries each: key = (entry's low 32 - B1 bits) << B1 | p, payload =
            // the unit's (rank, tile) first row id + the entry's row offset
            const int kb = 32 - c.B1;
#pragma unroll
            for (int k = 0; k < VMAX / CU_N; ++k) {
                const uint32_t un = tid + k * LOCAL_THREADS;
                if (un < len) {
                    const uint4 lo4 = *reinterpret_cast<const uint4 *>(reinterpret_cast<const char *>(buf(X)) + un * 32u);
                    const uint4 hi4 = *reinterpret_cast<const uint4 *>(reinterpret_cast<const char *>(buf(X)) + un * 32u + 16);
                    const unsigned long long a[4] = {(unsigned long long)lo4.x | (unsigned long long)lo4.y << 32,
                                                     (unsigned long long)lo4.z | (unsigned long long)lo4.w << 32,
                                                     (unsigned long long)hi4.x | (unsigned long long)hi4.y << 32,
                                                     (unsigned long long)hi4.z | (unsigned long long)hi4.w << 32};
                    const uint32_t meta = hi4.w, nv = meta & 7u;
                    const uint32_t tb = __ldg(c.rowbase + ((size_t)rel * MAX_RANKS + ((meta >> 3) & 7u)) * c.G + (meta >> 6));
#pragma unroll
                    for (int e = 0; e < CU_N; ++e) {
                        const unsigned long long en = unit_entry(a, e);
                        t[k * CU_N + e].x = (K)((((uint32_t)en & ((1u << kb) - 1u)) << c.B1) | p);
                        t[k * CU_N + e].y = (K)(tb + (uint32_t)(en >> kb));
                        if ((uint32_t)e < nv) cvalid |= 1u << (k * CU_N + e);
                    }
                }
            }
        } else {
#pragma unroll
            for (int v = 0; v < VMAX; ++v) {
                const uint32_t i = tid + v * LOCAL_THREADS;
                if (v < V && i < len) t[v] = buf(X)[skip + i];
            }
        }
        uint32_t rq[VMAX];  // rank << 16 | digit (0xffffffff: dropped)
#pragma unroll
        for (int v = 0; v < VMAX; ++v) {
            const uint32_t i = tid + v * LOCAL_THREADS;
            rq[v] = 0xffffffffu;
            const bool have = COMP ? ((cvalid >> v) & 1u) != 0 : (v < V && i < len);
            if (have && (!from_mid || digit1(t[v].x, P) == p)) {
                const uint32_t q = digit2(t[v].x, shift, Q);
                rq[v] = (atomicAdd(&bins[q], 1u) << 16) | q;
            }
        }
        __syncthreads();  // S1: buffer X consumed (it becomes this chunk's sorted output), bins final
        // chunk j+1 -> buffer X^1 once chunk j-1's stores have read it; the issuing
        // thread (warp 1, LI) also issues the chunk's bulk store, warp 0 scans meanwhile
        if (issuer() && j + 1 < mine) {
            if (tid == LI) bulk_wait_read0();  // (issue's barrier orders the other issuers after it)
            issue(j + 1, nxt);
            if (j + 2 < mine) nxt = cdesc[cidx(j + 2)];
        }
        if (tid >= 32) {  // the other bin array (last read by chunk j-1 before its S3) for chunk j+1
            uint32_t *const bn = bins2 + (X ^ 1) * QL;
            for (int q = tid - 32; q < Q; q += LOCAL_THREADS - 32) bn[q] = 0;
        }
        if (tid < 32) {  // one warp: padded run starts (exclusive scan over the Q bins)
            const int per = (Q + 31) / 32, q0 = tid * per;
            uint32_t sum = 0;
            for (int q = q0; q < min(Q, q0 + per); ++q) sum += (bins[q] + ALIGN - 1) & ~(uint32_t)(ALIGN - 1);
            uint32_t incl = sum;
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                const uint32_t y = __shfl_up_sync(0xffffffffu, incl, o);
                if (tid >= o) incl += y;
            }
            uint32_t run = incl - sum;
            for (int q = q0; q < min(Q, q0 + per); ++q) {
                abin[q] = run;
                run += (bins[q] + ALIGN - 1) & ~(uint32_t)(ALIGN - 1);
            }
            if (tid == 31) tmp[0] = incl;
        }
        __syncthreads();  // S2b
        const uint32_t tot = tmp[0];
        if (SPLIT) {  // run offsets of the chunk stored in place; padded run sizes per sub-partition
            uint16_t *E = c.eoffA[rel] + (size_t)li * EA_STRIDE;
            for (int q = tid; q <= Q; q += LOCAL_THREADS) {
                if (q < Q) {
                    const uint32_t n = bins[q];
                    E[q] = (uint16_t)(abin[q] | (ALIGN == 2 ? (n & 1u) : 0u));
                    if (n)
                        atomicAdd(&c.hA[(size_t)rel * c.vcap + ((size_t)dpi << BA) + q],
                                  (n + ALIGN - 1) & ~(uint32_t)(ALIGN - 1));
                } else {
                    E[q] = (uint16_t)tot;
                }
            }
        } else {
            const uint32_t *cb = c.chunk_base + (size_t)rel * c.cb_stride;
            const uint32_t cbp = cb[dpi], nchp = cb[dpi + 1] - cbp;
            uint16_t *E = c.eoff[rel] + (size_t)(Q + 1) * cbp + (li - cbp);
            uint32_t *cop = c.cop_slots + (size_t)rel * P * Qmax + (size_t)dpi * Q;
            for (int q = tid; q <= Q; q += LOCAL_THREADS) {
                if (q < Q) {
                    const uint32_t n = bins[q];
                    E[(size_t)q * nchp] = (uint16_t)(abin[q] | (ALIGN == 2 ? (n & 1u) : 0u));
                    if (n) atomicAdd(&cop[q], (n + ALIGN - 1) & ~(uint32_t)(ALIGN - 1));
                } else {
                    E[(size_t)q * nchp] = (uint16_t)tot;
                }
            }
        }
        Tup *const sorted = buf(X);
#pragma unroll
        for (int v = 0; v < VMAX; ++v) {
            if (rq[v] != 0xffffffffu) {
                const uint32_t q = rq[v] & 0xffffu, r = rq[v] >> 16;
                sorted[abin[q] + r] = t[v];
                // 16-byte padding slot of an odd run: a tuple whose key has its
                // lowest bit flipped, i.e. lies in another global partition, so
                // it never equals a real key of this co-partition; the probe
                // skips S padding slots (bitmap), R padding is inert, and the
                // chunked pass drops a first pass's padding (DESIGN.md §2 R2)
                if (ALIGN == 2 && r == 0 && (bins[q] & 1u)) {
                    Tup pad = t[v];
                    pad.x ^= (rel == 1 && P >= 4) ? 2 : 1;
                    sorted[abin[q] + bins[q]] = pad;
                }
            }
        }
        fence_proxy_async_smem();
        __syncthreads();  // S3
        if (tid == LI && tot) {  // the sorted chunk in place: first pass -> mid, else -> local
            Tup *dst = SPLIT ? static_cast<Tup *>(c.mid[rel]) + (size_t)li * c.chunk_region1
                             : static_cast<Tup *>(c.local[rel]) + (size_t)li * CR;
            tma_store_1d(dst, sorted, tot * TB);
            bulk_commit();
        }
    }
    bulk_wait0();
}

// The first pass of two-level local partitioning (a no-op unless k_plan chose
// BA > 0).
template <typename K>
__global__ void __launch_bounds__(LOCAL_THREADS, 1) k_local_split(Ctx c, const ChunkDesc *cdesc) {
    if (!c.meta[MT_OK] || !c.meta[MT_BA]) return;
    trace_begin(c, MGJ_TR_LOCAL_SPLIT);
    local_body<K, LM_SPLIT>(c, cdesc);
    trace_end(c, MGJ_TR_LOCAL_SPLIT);
}

// The chunked pass over the first pass's sub-partitions (a no-op when BA = 0).
template <typename K>
__global__ void __launch_bounds__(LOCAL_THREADS, 1) k_local_second(Ctx c, const ChunkDescB *descB) {
    if (!c.meta[MT_OK] || !c.meta[MT_BA]) return;
    trace_begin(c, MGJ_TR_LOCAL_SECOND);
    local_body<K, LM_SECOND>(c, descB);
    trace_end(c, MGJ_TR_LOCAL_SECOND);
}

// The single chunked pass over the owned partitions (a no-op when BA > 0):
// the chunks of R (rsel 0), of S (1) or of both (2).  With the shuffle
// overlapped (§8(e)), R's launch first waits for every rank's R tuples
// (SIG_DATA_R) and runs beside the scatter of S on the SMs it leaves free.
template <typename K, int RSEL, bool COMP = false, bool STRM = false>
__global__ void __launch_bounds__(LOCAL_THREADS, 1) k_local(Ctx c, const ChunkDesc *cdesc) {
    if (!c.meta[MT_OK] || c.meta[MT_BA]) return;
    // timeline stamps for the overlapped launches only: in the single launch
    // over both relations (the one-GPU path) they cost a 4-byte spill
    constexpr int id = RSEL == 0 ? MGJ_TR_LOCAL_R : MGJ_TR_LOCAL_S;
    if constexpr (RSEL != 2) trace_begin(c, id);
    local_body<K, LM_SINGLE, RSEL, COMP, STRM>(c, cdesc);
    if constexpr (RSEL != 2) trace_end(c, id);
}

// ---------------------------------------------------------------------------
// Probe work items.  A pipeline stage holds 2 * cap slots shared by the two
// sides: R from slot 0 (at most cap slots: one shared-memory table), S from
// slot soff.  Co-partition (p, q) is one item when R <= cap and R + S fit the
// stage (the common case, whatever the |R|:|S| ratio); otherwise R is cut
// into slices of cap slots and S into slices of the rest of the stage (at
// even slot offsets), and every R slice is paired with every S slice: an
// oversized R co-partition is built in table-sized pieces (block nested loop
// over R slices — the "both relations heavily skewed" case of P:450-452) and
// a heavy S co-partition is spread over many CTAs.
// ---------------------------------------------------------------------------
struct ItemX {
    Item it;
    uint32_t cb[2], nch[2];  // first chunk / chunk count of p per relation
    uint32_t soff;           // stage slot where the S side starts (>= the R side's slots)
};

// Walk the q-runs of one side in chunk order and cut it into slices of at
// most `cap` slots and `maxp` chunk pieces; call emit(slice) for each.
template <int ALIGN, typename F>
__device__ inline void walk_side(const uint16_t *E0, const uint16_t *E1, uint32_t nch, uint32_t cap,
                                 uint32_t maxp, F &&emit) {
    uint32_t acc = 0, npc = 0;
    Side cur{0, 0, 0, 0};
    for (uint32_t k = 0; k < nch; ++k) {
        uint32_t st, slots, valid;
        decode_run<ALIGN>(E0[k], E1[k], st, slots, valid);
        uint32_t a = 0;
        do {
            if (npc == maxp || (acc == cap && a < slots)) {
                cur.k1 = k;
                cur.a1 = a;
                emit(cur);
                cur = Side{k, a, 0, 0};
                acc = 0;
                npc = 0;
            }
            const uint32_t take = min(slots - a, cap - acc);
            acc += take;
            a += take;
            ++npc;
        } while (a < slots);
    }
    if (acc > 0) {
        cur.k1 = nch;
        cur.a1 = 0;
        emit(cur);
    }
}

template <typename K>
__global__ void k_itemize(Ctx c) {
    constexpr int ALIGN = Layout<K>::ALIGN;
    if (!c.meta[MT_OK]) return;
    trace_begin(c, MGJ_TR_ITEMIZE);
    const int P = c.P, Qmax = 1 << c.b2_max;
    const int Q = 1 << c.meta[MT_QB];  // sub-partitions of the chunked pass
    const uint32_t cap = (uint32_t)c.probe_slots;
    ItemX *items = reinterpret_cast<ItemX *>(c.items);
    const uint64_t total = (uint64_t)c.meta[MT_NLP] * Q;
    for (uint64_t idx = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; idx < total;
         idx += (uint64_t)gridDim.x * blockDim.x) {
        const uint32_t pi = (uint32_t)(idx / Q), q = (uint32_t)(idx % Q);
        const uint32_t r = c.cop_slots[(size_t)pi * Q + q];
        const uint32_t s = c.cop_slots[(size_t)P * Qmax + (size_t)pi * Q + q];
        if (r == 0 || s == 0) continue;
        ItemX x;
        x.it.pi = pi;
        x.it.q = q;
        for (int rel = 0; rel < 2; ++rel) {
            const uint32_t *cb = c.chunk_base + (size_t)rel * c.cb_stride;
            x.cb[rel] = cb[pi];
            x.nch[rel] = cb[pi + 1] - cb[pi];
        }
        if (r <= cap && r + s <= 2 * cap && x.nch[0] <= PROBE_MAXP && x.nch[1] <= PROBE_MAXP) {
            x.it.r = Side{0, 0, x.nch[0], 0};
            x.it.s = Side{0, 0, x.nch[1], 0};
            x.soff = r;
            const uint32_t b = atomicAdd(&c.ticket[TK_ITEMS], 1u);
            if (b < c.max_items) {
                items[b] = x;
            } else {  // the probe must not read reserved-but-unwritten items: it is skipped
                set_err(c, MGJ_ECAPACITY);
                c.meta[MT_OK] = 0;
            }
            continue;
        }
        // slow path: slice both sides, pair every R slice with every S slice
        const uint16_t *E[2][2];
        for (int rel = 0; rel < 2; ++rel) {
            E[rel][0] = c.eoff[rel] + (size_t)(Q + 1) * x.cb[rel] + (size_t)q * x.nch[rel];
            E[rel][1] = E[rel][0] + x.nch[rel];
        }
        const uint32_t rcap = r < cap ? r : cap, scap = 2 * cap - rcap;  // both even
        x.soff = rcap;
        uint32_t nr = 0, ns = 0;
        walk_side<ALIGN>(E[0][0], E[0][1], x.nch[0], rcap, PROBE_MAXP, [&](const Side &) { ++nr; });
        walk_side<ALIGN>(E[1][0], E[1][1], x.nch[1], scap, PROBE_MAXP, [&](const Side &) { ++ns; });
        const uint64_t n = (uint64_t)nr * ns;
        const uint32_t b = atomicAdd(&c.ticket[TK_ITEMS], (uint32_t)min(n, (uint64_t)0x7fffffffu));
        if ((uint64_t)b + n > c.max_items) {
            set_err(c, MGJ_ECAPACITY);
            c.meta[MT_OK] = 0;
            continue;
        }
        uint32_t ir = 0;
        walk_side<ALIGN>(E[0][0], E[0][1], x.nch[0], rcap, PROBE_MAXP, [&](const Side &rs) {
            uint32_t is = 0;
            walk_side<ALIGN>(E[1][0], E[1][1], x.nch[1], scap, PROBE_MAXP, [&](const Side &ss) {
                ItemX y = x;
                y.it.r = rs;
                y.it.s = ss;
                items[b + (uint64_t)ir * ns + is] = y;
                ++is;
            });
            ++ir;
        });
    }
    trace_end(c, MGJ_TR_ITEMIZE);
}

__host__ __device__ inline size_t probe_smem_bytes(int slots, int TB) {
    return (size_t)PROBE_NST * 2 * slots * TB  // stages (R then S, 2 * slots each)
           + (size_t)PROBE_NST * (2 * slots / 32 + 1) * 4  // S padding-slot bitmaps
           + 4096 * 4                          // head
           + (size_t)slots * 2;                // next
}

// ---------------------------------------------------------------------------
// a5 (§3.2 "Probe"): the co-partitions of R and S with
// the same partition id are joined; the paper notes the nested-loop and the
// shared-memory hash-table variants perform alike and the north
// star asks for the hash table.  Warp-specialised, PROBE_NST-stage pipeline:
//  - warps 0..PROBE_NP-1 (producers, items round-robin) read the run offsets
//    of their next item and issue one TMA bulk copy per (chunk, relation)
//    run into a free stage, packing the runs back to back;
//  - the other warps (consumers) build a chained hash table over the stage's
//    R slots (head entries tagged with the item, so the table is never
//    cleared), then stream the S slots through it: count += 1 and
//    checksum += a*C + b (mod 2^64) for every equal-key pair.  Padding slots
//    hold keys of another partition and never match.  With MAT the item's
//    matches are counted, one output reservation is taken, and a second pass
//    over the S slots in shared memory writes (key, payR, payS).
// ---------------------------------------------------------------------------
template <typename K, bool MAT>
__global__ void __launch_bounds__(PROBE_THREADS, 1) k_probe(Ctx c) {
    using Tup = typename Layout<K>::Tup;
    constexpr int TB = Layout<K>::TB;
    constexpr int LOGT = 12, T = 1 << LOGT;
    constexpr uint16_t END = 0xffff;
    constexpr int NCONS = PROBE_THREADS - 32 * PROBE_NP;
    extern __shared__ __align__(128) unsigned char smem[];
    __shared__ __align__(8) uint64_t full[PROBE_NST], empty[PROBE_NST];
    __shared__ uint32_t totals[PROBE_NST][2];
    __shared__ uint32_t stage_p[PROBE_NST];  // global partition (digit1) of the stage's item
    __shared__ uint32_t stage_soff[PROBE_NST];  // slot where the stage's S side starts
    __shared__ uint32_t s_wtot[32];
    __shared__ unsigned long long s_base;
    __shared__ int s_write;
    if (!c.meta[MT_OK]) return;
    const int SL = c.probe_slots;
    Tup *stages = reinterpret_cast<Tup *>(smem);  // [NST][2 * SL]: R from 0, S from the item's soff
    const int PW = 2 * SL / 32 + 1;  // words per S padding bitmap
    uint32_t *padbits = reinterpret_cast<uint32_t *>(stages + (size_t)PROBE_NST * 2 * SL);  // [NST][PW]
    uint32_t *head = padbits + PROBE_NST * PW;
    uint16_t *nxt = reinterpret_cast<uint16_t *>(head + T);
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const int B2 = c.meta[MT_B2];
    // S padding slots (8-byte tuples): with P >= 4 their key has bit 1 flipped
    // and R's bit 0 (k_local), so neither can equal any key of the other side
    // and S padding is probed harmlessly; only P < 4 needs the skip bitmap
    const bool SBITS = Layout<K>::ALIGN == 2 && c.P < 4;
    const int BAp = c.meta[MT_BA];
    // packed table (B1 + B2 >= 16, so khi = key >> (B1 + B2) fits the key's
    // width minus 16 bits): the build overwrites each R slot's key with
    // (khi << 16 | next), so a chain step is one shared load of the slot
    // that yields khi, the next link and the payload.  All
    // real keys of a co-partition share their low B1 + B2 bits, so equal khi
    // means equal keys; padding slots (digit1 != p) are left out on both sides.
    // (8-byte keys: measured slower packed, 3.04 vs 2.82 ms at M5 size: the
    // 64-bit shifts and compares cost more issue slots than the link load saves)
    const bool packed = sizeof(K) == 4 && c.B1 + B2 >= 16;
    const int P = c.P;
    const int Q = 1 << c.meta[MT_QB], shift = c.B1 + B2;  // Q: runs per chunk of the chunked pass
    const uint32_t nitems = min(__ldcg(&c.ticket[TK_ITEMS]), c.max_items);
    const uint32_t mine = nitems > blockIdx.x ? (nitems - blockIdx.x + gridDim.x - 1) / gridDim.x : 0;
    const ItemX *items = reinterpret_cast<const ItemX *>(c.items);
    if (tid == 0) {
        for (int s = 0; s < PROBE_NST; ++s) {
            mbar_init(&full[s], PROBE_PPI);
            mbar_init(&empty[s], 1);
        }
        fence_mbar_init();
    }
    for (int i = tid; i < T; i += PROBE_THREADS) head[i] = 0;
    __syncthreads();

    if (warp < PROBE_NP) {
        // ------------------------------------------------------- producers
        // two warps per item stream: warp & 1 issues the item's R runs, the
        // other its S runs (one warp's bulk copies issue one after another;
        // tools/tma_runs.cu)
        constexpr int ALIGN = Layout<K>::ALIGN;
        const uint64_t pol = policy_evict_first();
        constexpr int NPI = PROBE_NP / PROBE_PPI;  // item streams (<= PROBE_NST)
        const int pw = warp / PROBE_PPI;
        const int rel = warp & 1;
        ItemX x;
        if (pw < (int)mine) x = items[blockIdx.x + pw * gridDim.x];
        for (uint32_t j = pw; j < mine; j += NPI) {
            ItemX xn;
            if (j + NPI < mine) xn = items[blockIdx.x + (j + NPI) * gridDim.x];  // prefetch
            const int s = j % PROBE_NST;
            if (j >= PROBE_NST) mbar_wait(&empty[s], ((j / PROBE_NST) - 1) & 1);
            uint32_t *pb = padbits + s * PW;
            if (SBITS && rel == 1) {
                for (int w = lane; w < PW; w += 32) pb[w] = 0;
                __syncwarp();
            }
            const Side sd = rel ? x.it.s : x.it.r;
            const uint32_t xcb = rel ? x.cb[1] : x.cb[0], xnch = rel ? x.nch[1] : x.nch[0];  // no local memory
            const uint16_t *E0 = (rel ? c.eoff[1] : c.eoff[0]) + (size_t)(Q + 1) * xcb + (size_t)x.it.q * xnch;
            const uint16_t *E1 = E0 + xnch;
            const uint32_t kend = min(sd.k1, xnch - 1);
            const uint32_t np = sd.k0 <= kend ? kend - sd.k0 + 1 : 0;
            Tup *dstbase = stages + (size_t)s * 2 * SL + (rel ? x.soff : 0);
            const Tup *lbase = static_cast<const Tup *>(rel ? c.local[1] : c.local[0]);
            uint32_t run = 0;
            // run offsets of the next batch of 32 runs are loaded while this
            // batch is scanned and issued (items of heavy partitions have
            // hundreds of runs: one load latency per batch otherwise)
            uint32_t en0 = 0, en1 = 0;
            if (lane < np) en0 = E0[sd.k0 + lane], en1 = E1[sd.k0 + lane];
            for (uint32_t m0 = 0; m0 < np; m0 += 32) {
                const uint32_t m = m0 + lane;
                uint32_t sz = 0, pad = 0xffffffffu;
                uint64_t src = 0;
                const uint32_t ec0 = en0, ec1 = en1;
                if (m + 32 < np) en0 = E0[sd.k0 + m + 32], en1 = E1[sd.k0 + m + 32];
                if (m < np) {
                    const uint32_t k = sd.k0 + m;
                    uint32_t st, slots, v;
                    decode_run<ALIGN>(ec0, ec1, st, slots, v);
                    const uint32_t alo = (k == sd.k0) ? sd.a0 : 0;
                    const uint32_t ahi = (k == sd.k1) ? sd.a1 : slots;
                    if (ahi > alo) {
                        sz = ahi - alo;
                        src = (uint64_t)(xcb + k) * (BAp ? c.chunk_region2 : c.chunk_region) + st + alo;
                    }
                    pad = (SBITS && rel == 1 && v < slots && v >= alo && v < ahi) ? v - alo : 0xffffffffu;
                }
                uint32_t incl = sz;
#pragma unroll
                for (int o = 1; o < 32; o <<= 1) {
                    const uint32_t y = __shfl_up_sync(0xffffffffu, incl, o);
                    if (lane >= o) incl += y;
                }
                const uint32_t dst = run + incl - sz;
                const uint32_t gsum = __shfl_sync(0xffffffffu, incl, 31);
                if (lane == 0 && gsum)
                    asm volatile("mbarrier.expect_tx.relaxed.cta.shared::cta.b64 [%0], %1;" ::"r"(
                                     smem_u32(&full[s])),
                                 "r"(gsum * TB)
                                 : "memory");
                __syncwarp();
                if (sz) tma_load_1d(dstbase + dst, lbase + src, sz * TB, &full[s], pol);
                if (pad != 0xffffffffu) atomicOr(&pb[(dst + pad) >> 5], 1u << ((dst + pad) & 31));
                run += gsum;
            }
            if (lane == 0) totals[s][rel] = run;
            if (lane == 0 && rel == 0) {
                stage_p[s] = (uint32_t)c.plist[BAp ? x.it.pi >> BAp : x.it.pi];
                stage_soff[s] = x.soff;
            }
            __syncwarp();
            if (lane == 0) mbar_arrive(&full[s]);
            x = xn;
        }
        return;
    }

    // ------------------------------------------------------------ consumers
    const int ct = tid - 32 * PROBE_NP;
    unsigned long long my_cnt = 0, my_chk = 0, my_dig = 0;  // count, checksum, pair digest
    uint32_t tag = 0;
    // stage and parity advance incrementally; barrier addresses computed once
    // 4-byte keys: the per-item shared addresses pinned in registers, not re-derived
    // from the shared window (S2R SR_CgaCtaId) for every item (measured at M2: probe
    // 1.887 -> 1.849 ms; the 8-byte instances would spill)
    constexpr bool pin = sizeof(K) == 4;
    const uint32_t full_at = pin ? smem_pin(&full[0]) : smem_u32(&full[0]);
    const uint32_t empty_at = pin ? smem_pin(&empty[0]) : smem_u32(&empty[0]);
    const uint32_t tot_at = pin ? smem_pin(&totals[0][0]) : 0u;  // per-stage item fields
    const uint32_t sp_at = pin ? smem_pin(&stage_p[0]) : 0u;
    const uint32_t so_at = pin ? smem_pin(&stage_soff[0]) : 0u;
    int s = 0;
    uint32_t ph = 0;
    for (uint32_t j = 0; j < mine; ++j) {
        if (++tag == 0x10000u) {  // tag wrap: clear the table once every 65535 items
            for (int i = ct; i < T; i += NCONS) head[i] = 0;
            named_bar_sync(1, NCONS);
            tag = 1;
        }
        mbar_wait_at(full_at + 8u * s, ph);
        const Tup *rt = stages + (size_t)s * 2 * SL;
        const Tup *st = rt + (pin ? lds_u32_at(so_at + 4u * s) : stage_soff[s]);
        const uint32_t rtot = pin ? lds_u32_at(tot_at + 8u * s) : totals[s][0];
        const uint32_t stot = pin ? lds_u32_at(tot_at + 8u * s + 4u) : totals[s][1];
        const uint32_t pitem = pin ? lds_u32_at(sp_at + 4u * s) : stage_p[s];
        auto fold = [](K khi) {  // table index from khi (identity for dense keys below 2^12)
            if constexpr (sizeof(K) == 4) {
                return ((uint32_t)khi ^ ((uint32_t)khi >> LOGT)) & (uint32_t)(T - 1);
            } else {
                const uint32_t f = (uint32_t)khi ^ (uint32_t)((unsigned long long)khi >> 32);
                return (f ^ (f >> LOGT) ^ (f >> (2 * LOGT))) & (uint32_t)(T - 1);
            }
        };
        // head entry of khi: the same index as fold(), computed as a byte offset
        // in three instructions (shift, shift, xor-and) for 4-byte keys
        auto hp = [&](K khi) -> uint32_t * {
            if constexpr (sizeof(K) == 4) {
                const uint32_t off = (((uint32_t)khi << 2) ^ ((uint32_t)khi >> (LOGT - 2))) & (uint32_t)((T - 1) << 2);
                return reinterpret_cast<uint32_t *>(reinterpret_cast<char *>(head) + off);
            } else {
                return head + fold(khi);
            }
        };
        // build
        if (packed) {
            K *rw = reinterpret_cast<K *>(stages + (size_t)s * 2 * SL);
            for (uint32_t slot = ct; slot < rtot; slot += NCONS) {
                const K k = rt[slot].x;
                if (((uint32_t)k & (uint32_t)(P - 1)) != pitem) continue;  // R padding slot
                const K khi = k >> shift;
                const uint32_t old = atomicExch(hp(khi), (tag << 16) | slot);
                const uint32_t ox = old ^ (tag << 16);  // < 2^16: a slot of this item
                rw[2 * slot] = (K)min(ox, (uint32_t)END) |  // a stale head (>= 2^16) ends the chain
                               (khi << 16);
            }
        } else {
            for (uint32_t slot = ct; slot < rtot; slot += NCONS) {
                const uint32_t h = tab_hash(rt[slot].x, shift, LOGT);
                const uint32_t old = atomicExch(&head[h], (tag << 16) | slot);
                nxt[slot] = (old >> 16) == tag ? (uint16_t)(old & 0xffffu) : END;
            }
        }
        named_bar_sync(1, NCONS);
        const uint32_t *pb = padbits + s * PW;
        // every R payload matching S slot x: f(payR)
        auto walk = [&](uint32_t x, const Tup &sv, auto &&f) {
            if (packed) {
                const K k = sv.x;
                if (((uint32_t)k & (uint32_t)(P - 1)) != pitem) return;  // S padding slot
                const K khi = k >> shift;
                const uint32_t hv = *hp(khi);
                // a head of this item has tag << 16 | slot: xor leaves the slot; a stale
                // head (another tag) leaves a value >= 2^16, which ends the walk like END
                for (uint32_t i = hv ^ (tag << 16); i < END;) {
                    const Tup rv = rt[i];
                    const K l = rv.x;
                    if ((l >> 16) == khi) f((K)rv.y, i);
                    i = (uint32_t)l & 0xffffu;
                }
            } else {
                if (SBITS && ((pb[x >> 5] >> (x & 31)) & 1u)) return;  // padding slot (P < 4 only)
                const uint32_t hv = head[tab_hash(sv.x, shift, LOGT)];
                for (uint32_t i = (hv >> 16) == tag ? (hv & 0xffffu) : END; i != END; i = nxt[i]) {
                    const Tup rv = rt[i];
                    if (rv.x == sv.x) f((K)rv.y, i);
                }
            }
        };
        // probe
        uint32_t m_item = 0;
        uint32_t x0 = ct;
        // MAT: the first match of each of this thread's S slots is kept (R slot
        // index) so the write pass needs no second walk unless a slot matched
        // more than once (duplicate R keys: the warp re-walks instead)
        constexpr int KMAX = (PROBE_SLOTS8 + NCONS - 1) / NCONS;  // S slots per consumer thread
        uint16_t mi[MAT ? KMAX : 1];
        bool ovf = false;
        if (MAT) {
#pragma unroll
            for (int k = 0; k < KMAX; ++k) {
                const uint32_t x = ct + k * NCONS;
                mi[k] = END;
                if (x < stot) {
                    const Tup sv = st[x];
                    walk(x, sv, [&](K a, uint32_t i) {
                        ++m_item;
                        my_chk += chk_term(a, (K)sv.y);
                        my_dig += dig_term(a, (K)sv.y);
                        if (mi[k] == END) mi[k] = (uint16_t)i;
                        else ovf = true;
                    });
                }
            }
            for (uint32_t x = ct + KMAX * NCONS; x < stot; x += NCONS) {  // beyond the record: re-walk
                const Tup sv = st[x];
                walk(x, sv, [&](K a, uint32_t) {
                    ++m_item;
                    my_chk += chk_term(a, (K)sv.y);
                    my_dig += dig_term(a, (K)sv.y);
                    ovf = true;
                });
            }
        } else if (packed && sizeof(K) == 4) {
            // 4-byte keys, packed table, count + checksum only: shared addresses
            // kept as 32-bit byte offsets (one LEA per access) and the S slots
            // walked by pointer increment
            const uint32_t rt_s = smem_u32(rt), tagsh = tag << 16;
            const uint32_t mP = (uint32_t)(P - 1);
            uint32_t sa = smem_u32(st + x0);
            const uint32_t se = smem_u32(st + stot);
            for (; sa < se; sa += NCONS * (uint32_t)sizeof(Tup)) {
                uint32_t k, b;
                asm("ld.shared.v2.u32 {%0,%1}, [%2];" : "=r"(k), "=r"(b) : "r"(sa));
                if ((k & mP) != pitem) continue;  // S padding slot
                const uint32_t khi = k >> shift;
                for (uint32_t i = *hp((K)khi) ^ tagsh; i < END;) {
                    uint32_t l, a;
                    asm("ld.shared.v2.u32 {%0,%1}, [%2];" : "=r"(l), "=r"(a) : "r"(rt_s + i * 8u));
                    if ((l >> 16) == khi) {
                        ++m_item;
                        my_chk += chk_term((K)a, (K)b);
                        my_dig += dig_term((K)a, (K)b);
                    }
                    i = l & 0xffffu;
                }
            }
        } else {
            for (uint32_t x = x0; x < stot; x += NCONS) {
                const Tup sv = st[x];
                walk(x, sv, [&](K a, uint32_t) {
                    ++m_item;
                    my_chk += chk_term(a, (K)sv.y);
                    my_dig += dig_term(a, (K)sv.y);
                });
            }
        }
        my_cnt += m_item;
        if (MAT) {
            // exact output positions: exclusive scan of the per-thread match
            // counts of the pass above, one reservation per item, then each
            // thread re-walks the same S slots and writes its matches in order
            const int cwi = ct >> 5;
            uint32_t incl = m_item;
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                const uint32_t y = __shfl_up_sync(0xffffffffu, incl, o);
                if (lane >= o) incl += y;
            }
            if (lane == 31) s_wtot[cwi] = incl;
            named_bar_sync(1, NCONS);
            if (ct < 32) {
                uint32_t v = ct < NCONS / 32 ? s_wtot[ct] : 0;
#pragma unroll
                for (int o = 1; o < 32; o <<= 1) {
                    const uint32_t y = __shfl_up_sync(0xffffffffu, v, o);
                    if (ct >= o) v += y;
                }
                if (ct < NCONS / 32) s_wtot[ct] = v;
                if (ct == 31) {
                    s_base = v ? atomicAdd(&c.acc[2], (unsigned long long)v) : 0;
                    s_write = v && (s_base + v <= c.out_cap);
                    if (v && !s_write) set_err(c, MGJ_ECAPACITY);
                }
            }
            named_bar_sync(1, NCONS);
            // write pass, warp-synchronous: every chain step of the warp's 32 S
            // slots emits its matches at consecutive positions of the warp's
            // reservation (ballot + popc), so each store instruction covers
            // consecutive output elements
            const unsigned long long wlo = cwi ? s_wtot[cwi - 1] : 0;
            K *ok = static_cast<K *>(c.out_key);
            K *oa = static_cast<K *>(c.out_a);
            K *ob = static_cast<K *>(c.out_b);
            const uint32_t lt = (1u << lane) - 1u;
            const bool wovf = __any_sync(0xffffffffu, ovf);
            if (s_write && s_wtot[cwi] > wlo && !wovf) {  // from the recorded matches
                unsigned long long wpos = s_base + wlo;
#pragma unroll
                for (int k = 0; k < KMAX; ++k) {
                    const bool has = mi[k] != END;
                    const uint32_t mask = __ballot_sync(0xffffffffu, has);
                    if (has) {
                        const unsigned long long q = wpos + __popc(mask & lt);
                        const Tup sv = st[ct + k * NCONS];
                        ok[q] = (K)sv.x;
                        oa[q] = (K)rt[mi[k]].y;
                        ob[q] = (K)sv.y;
                    }
                    wpos += __popc(mask);
                }
            } else if (s_write && s_wtot[cwi] > wlo) {
                unsigned long long wpos = s_base + wlo;
                for (uint32_t xb = (uint32_t)(ct & ~31); xb < stot; xb += NCONS) {
                    const uint32_t x = xb + lane;
                    Tup sv{};
                    uint32_t i = END;
                    K khi = 0;
                    if (x < stot) {
                        sv = st[x];
                        if (packed) {
                            const K k = sv.x;
                            if (((uint32_t)k & (uint32_t)(P - 1)) == pitem) {
                                khi = k >> shift;
                                const uint32_t hv = *hp(khi);
                                i = (hv >> 16) == tag ? (hv & 0xffffu) : END;
                            }
                        } else if (!(SBITS && ((pb[x >> 5] >> (x & 31)) & 1u))) {
                            const uint32_t hv = head[tab_hash(sv.x, shift, LOGT)];
                            i = (hv >> 16) == tag ? (hv & 0xffffu) : END;
                        }
                    }
                    while (__any_sync(0xffffffffu, i != END)) {
                        bool match = false;
                        K a = 0;
                        if (i != END) {
                            const Tup rv = rt[i];
                            if (packed) {
                                const K l = rv.x;
                                match = (l >> 16) == khi;
                                i = (uint32_t)l & 0xffffu;
                            } else {
                                match = rv.x == sv.x;
                                i = nxt[i];
                            }
                            a = (K)rv.y;
                        }
                        const uint32_t mask = __ballot_sync(0xffffffffu, match);
                        if (match) {
                            const unsigned long long q = wpos + __popc(mask & lt);
                            ok[q] = (K)sv.x;
                            oa[q] = a;
                            ob[q] = (K)sv.y;
                        }
                        wpos += __popc(mask);
                    }
                }
            }
        }
        named_bar_sync(1, NCONS);  // stage s and the table are free
        if (ct == 0) mbar_arrive_at(empty_at + 8u * s);
        if (++s == PROBE_NST) s = 0, ph ^= 1u;
    }
    my_cnt = warp_sum(my_cnt);
    my_chk = warp_sum(my_chk);
    my_dig = warp_sum(my_dig);
    if (lane == 0 && (my_cnt || my_chk || my_dig)) {
        atomicAdd(&c.acc[0], my_cnt);
        atomicAdd(&c.acc[1], my_chk);
        atomicAdd(&c.acc[3], my_dig);
    }
}

// ---------------------------------------------------------------------------
// a6: count = sum_g count_g, checksum = sum_g checksum_g, digest = sum_g
// digest_g (mod 2^64), the last step of mgj_join.  Thread 0 stores this
// rank's (count, checksum, n_out, status, digest) into every peer's result
// mailbox, raises SIG_RES there, waits for every rank's SIG_RES and sums the
// N entries (order-free, bit-exact).  Mailbox reuse across runs is safe: a
// rank publishes run e+1 only after k_plan(e+1) saw every rank's SIG_HIST of
// e+1, which each rank raises after its own k_reduce(e) (stream order).
// ---------------------------------------------------------------------------
__global__ void k_reduce(Ctx c) {
    if (threadIdx.x != 0 || blockIdx.x != 0) return;
    trace_begin(c, MGJ_TR_REDUCE);
    const int32_t st = *(volatile int32_t *)c.err;
    const unsigned long long v[5] = {__ldcg(&c.acc[0]), __ldcg(&c.acc[1]), __ldcg(&c.acc[2]),
                                     (unsigned long long)(uint32_t)st, __ldcg(&c.acc[3])};
    if (c.world == 1) {  // one rank: the local sums are the global ones (no mailbox round trip)
        c.result[0] = v[0];
        c.result[1] = v[1];
        c.result[2] = v[2];
        c.result[3] = v[3];
        c.result[4] = v[4];
        trace_end(c, MGJ_TR_REDUCE);
        return;
    }
    for (int d = 0; d < c.world; ++d) {
        volatile unsigned long long *rm =
            reinterpret_cast<unsigned long long *>(c.arena[d] + c.lay.resmail) + c.rank * RES_W;
        for (int i = 0; i < 5; ++i) rm[i] = v[i];
    }
    __threadfence_system();
    signal_all(c, SIG_RES);
    unsigned long long cnt = 0, chk = 0, dig = 0;
    int32_t gst = 0;
    if (!wait_all_flags(c, SIG_RES)) {
        gst = MGJ_EPEER;
    } else {
        const volatile unsigned long long *rm =
            reinterpret_cast<const unsigned long long *>(c.arena[c.rank] + c.lay.resmail);
        for (int g = 0; g < c.world; ++g) {
            cnt += rm[g * RES_W + 0];
            chk += rm[g * RES_W + 1];
            dig += rm[g * RES_W + 4];
            const int32_t s = (int32_t)(uint32_t)rm[g * RES_W + 3];
            if (gst == 0 && s != 0) gst = s;
        }
    }
    c.result[0] = cnt;
    c.result[1] = chk;
    c.result[2] = v[2];
    c.result[3] = (unsigned long long)(uint32_t)gst;
    c.result[4] = dig;
    trace_end(c, MGJ_TR_REDUCE);
}

}  // namespace mgj
