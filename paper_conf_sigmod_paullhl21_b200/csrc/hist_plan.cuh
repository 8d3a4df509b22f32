// hist_plan.cuh — phase a1 (radix histogram fused with its all-gather) and
// phase a2 (partition -> GPU assignment and exact receive offsets).
#pragma once

#include "common.cuh"
#include "scatter.cuh"  // scat_geom: the sub-tiles a1 counts
#include "tma.cuh"

namespace mgj {

constexpr int HIST_NB = 3;  // k_hist: TMA ring depth at most (sub-tiles in flight per CTA; 2 CTAs per SM)
// ring depth for sub-tiles of T keys: about 96 KB in flight per CTA, 2..HIST_NB deep
// k_hist reads a scatter sub-tile of T keys in HN blocks of T / HN keys (two for
// 16384 4-byte keys: a 64 KB ring entry would leave room for one CTA per SM)
__host__ __device__ inline int hist_halves(int T, int key_bytes) { return T * key_bytes > 49152 ? 2 : 1; }
__host__ __device__ inline int hist_nb(int T, int key_bytes) {
    const int nb = 98304 / (T * key_bytes);
    return nb < 2 ? 2 : (nb > HIST_NB ? HIST_NB : nb);
}

// ---------------------------------------------------------------------------
// a1: per-GPU radix histogram (§3.2 "Histogram generation",
// P:356-370, built in shared memory after Rui et al. [38]; bin count from the
// Eq. 1 analogue).  H[rel][p] = #{t in rel_g : digit1(t.key) = p}.
// hist_split CTAs share tile c of R and of S (two k_hist CTAs per SM)
// (the tiles the scatter kernel processes); each counts a contiguous run of
// the scatter's sub-tiles, whose key columns a TMA ring brings into shared
// memory HIST_NB sub-tiles ahead.  Per sub-tile it stores the u16 counts (the
// scatter lays each sub-tile out from them before reading it) and folds
// them into the tile histogram (exact scatter offsets) and the rank
// histogram.  The last CTA
// stores the rank histogram into every peer's arena mailbox and raises
// SIG_HIST there (histogram exchange X4 fused).
// ---------------------------------------------------------------------------
// The fused exchange of a1 (one CTA): the rank histogram (and, compressed,
// the unit counts) and the job-wide configuration words into every peer's
// mailbox, then SIG_HIST everywhere.
// Job-wide configuration word checked equal on every rank by k_plan: B1, the
// compressed shuffle and, with chunk streaming, the tile geometry the round
// counts assume (tiles per relation, S scatter CTAs).
__device__ __forceinline__ uint64_t cfg_word(const Ctx &c) {
    return (uint64_t)(c.B1 | c.comp << 8 | c.stream << 9) |
           (c.stream ? ((uint64_t)c.G << 16 | (uint64_t)c.sgrid << 40) : 0ull);
}

__device__ inline void publish_hist(const Ctx &c) {
    const int P = c.P;
    for (int d = 0; d < c.world; ++d) {
        uint32_t *mb = reinterpret_cast<uint32_t *>(c.arena[d] + c.lay.mail) + (size_t)c.rank * 2 * P;
        for (int j = threadIdx.x; j < 2 * P; j += blockDim.x) mb[j] = __ldcg(&c.rank_hist[j]);
        if (c.comp) {
            uint32_t *ub = reinterpret_cast<uint32_t *>(c.arena[d] + c.lay.umail) + (size_t)c.rank * 2 * P;
            for (int j = threadIdx.x; j < 2 * P; j += blockDim.x) ub[j] = __ldcg(&c.rank_units[j]);
        }
        // this rank's job-wide configuration words, checked equal on every rank by k_plan
        if (threadIdx.x < 4) {
            const uint64_t w[4] = {c.recv_cap[0], c.recv_cap[1], c.lay.total, cfg_word(c)};
            reinterpret_cast<uint64_t *>(c.arena[d] + c.lay.cfgmail)[c.rank * 4 + threadIdx.x] = w[threadIdx.x];
        }
    }
    __threadfence_system();
    __syncthreads();
    if (threadIdx.x == 0) signal_all(c, SIG_HIST);
}

template <typename K>
__global__ void __launch_bounds__(HIST_THREADS, 2) k_hist(Ctx c) {
    extern __shared__ __align__(128) unsigned char hsm[];  // ring[NB][TB] keys | sub[P] | acc[P]
    __shared__ __align__(8) uint64_t bar[HIST_NB];
    const int P = c.P, T = c.scat_T, HN = hist_halves(T, sizeof(K)), TB = T / HN, NB = hist_nb(TB, sizeof(K));
    // blocks per sub-tile = 1 << hs; ring slot and parity advance by counters: runtime
    // divisions per block (b / HN, b % NB) cost 14% more instructions (measured at M2
    // with 16384-key sub-tiles: 775 -> 739 us; 12288-key sub-tiles in one block: 731 us)
    const int hs = HN == 2 ? 1 : 0;
    K *const ring = reinterpret_cast<K *>(hsm);  // NB entries of TB keys (block b: half b % HN of sub-tile b / HN)
    uint32_t *const sub = reinterpret_cast<uint32_t *>(ring + (size_t)NB * TB);
    uint32_t *const acc = sub + P;
    const int tid = threadIdx.x, HS = c.hist_split, tile = blockIdx.x / HS, part = blockIdx.x % HS;
    constexpr int LU = 16 / (int)sizeof(K);
    uint64_t lo0, hi0, lo1, hi1;
    tile_range(c.n_in[0], c.G, tile, lo0, hi0);
    tile_range(c.n_in[1], c.G, tile, lo1, hi1);
    // hist_split CTAs share a tile: contiguous runs of its sub-tiles
    const uint32_t ns0 = (uint32_t)((hi0 - lo0 + T - 1) / T), ns1 = (uint32_t)((hi1 - lo1 + T - 1) / T);
    const uint32_t ja0 = ns0 * part / HS, jb0 = ns0 * (part + 1) / HS;
    const uint32_t ja1 = ns1 * part / HS, jb1 = ns1 * (part + 1) / HS;
    const uint32_t nsub0 = jb0 - ja0;
    const uint32_t ntot = nsub0 + (jb1 - ja1);
    auto subtile = [&](uint32_t g, int &rel, uint32_t &j, uint64_t &first, uint32_t &len) {
        rel = g < nsub0 ? 0 : 1;
        j = rel ? g - nsub0 + ja1 : g + ja0;
        first = (rel ? lo1 : lo0) + (uint64_t)j * T;
        len = (uint32_t)min((uint64_t)T, (rel ? hi1 : hi0) - first);
    };
    const uint64_t pol = policy_evict_first();
    auto block = [&](uint32_t b, int &rel, uint32_t &j, uint64_t &first, uint32_t &len) {  // keys of block b
        uint32_t slen;
        subtile(b >> hs, rel, j, first, slen);
        const uint32_t o = (b & (uint32_t)(HN - 1)) * (uint32_t)TB;
        first += o;
        len = slen > o ? min(slen - o, (uint32_t)TB) : 0u;
    };
    auto issue = [&](uint32_t b, int slot) {  // thread 0: TMA the 16-byte-aligned body of block b's keys
        int rel;
        uint32_t j, len;
        uint64_t first;
        block(b, rel, j, first, len);
        uint64_t *br = &bar[slot];
        const uint32_t bytes = (len & ~(uint32_t)(LU - 1)) * (uint32_t)sizeof(K);
        mbar_arrive_expect_tx(br, bytes);
        if (bytes)
            tma_load_1d(ring + (size_t)slot * TB, static_cast<const K *>(c.in_key[rel]) + first, bytes, br, pol);
    };
    const uint32_t nblk = ntot * (uint32_t)HN;
    trace_begin(c, MGJ_TR_HIST);
    for (int i = tid; i < 2 * P; i += blockDim.x) sub[i] = 0;
    if (tid == 0) {
        for (int i = 0; i < NB; ++i) mbar_init(&bar[i], 1);
        fence_mbar_init();
        for (uint32_t b = 0; b < nblk && b < (uint32_t)NB; ++b) issue(b, (int)b);
    }
    __syncthreads();
    const uint32_t m = (uint32_t)(P - 1);
    auto flush_acc = [&](int rel) {  // tile histogram (this CTA owns the tile) and rank histogram
        uint32_t *th = c.tile_hist + ((size_t)rel * c.G + tile) * P;
        for (int p = tid; p < P; p += blockDim.x) {
            const uint32_t x = acc[p];
            if (x) {
                atomicAdd(&th[p], x);
                atomicAdd(&c.rank_hist[rel * P + p], x);
            }
            acc[p] = 0;
        }
    };
    int slot = 0;
    uint32_t phase = 0;  // ring slot of block b (b mod NB) and its barrier's parity (b / NB odd)
    for (uint32_t b = 0; b < nblk; ++b) {
        int rel;
        uint32_t j, len;
        uint64_t first;
        block(b, rel, j, first, len);
        const uint32_t g = b >> hs;  // the sub-tile
        const K *buf = ring + (size_t)slot * TB;
        mbar_wait(&bar[slot], phase);
        const uint32_t body = len & ~(uint32_t)(LU - 1);
        for (uint32_t i0 = (uint32_t)tid * LU; i0 < body; i0 += (uint32_t)blockDim.x * LU) {
            const uint4 v = *reinterpret_cast<const uint4 *>(buf + i0);
            if (sizeof(K) == 4) {
                atomicAdd(&sub[v.x & m], 1u);
                atomicAdd(&sub[v.y & m], 1u);
                atomicAdd(&sub[v.z & m], 1u);
                atomicAdd(&sub[v.w & m], 1u);
            } else {  // two 8-byte keys: low words are .x and .z
                atomicAdd(&sub[v.x & m], 1u);
                atomicAdd(&sub[v.z & m], 1u);
            }
        }
        if (tid < (int)(len - body))  // < LU trailing tuples of the relation: from global
            atomicAdd(&sub[digit1(static_cast<const K *>(c.in_key[rel])[first + body + tid], P)], 1u);
        // (measured, not kept: the last warp done reading a slot refilling it instead of
        // this barrier, M2 727 -> 755 us with 12288-key sub-tiles)
        __syncthreads();  // counts final; ring slot b % NB free
        if (tid == 0 && b + NB < nblk) issue(b + NB, slot);
        if (++slot == NB) slot = 0, phase ^= 1u;
        if ((b & (uint32_t)(HN - 1)) != (uint32_t)(HN - 1)) continue;  // the sub-tile's other block comes next
        // sub-tile histogram (u16 pairs) for the scatter's layout, then fold into acc
        uint32_t *o32 = reinterpret_cast<uint32_t *>(c.sub_hist + (((size_t)rel * c.G + tile) * c.sub_ns + j) * P);
        if constexpr (sizeof(K) == 4) {  // wide shared accesses, four bins per thread (measured at M2: pairs of
                                         // bins 0.83 -> 0.78 ms, then four bins; slower for 8-byte keys,
                                         // 0.71 -> 0.75, which keep the scalar fold)
            for (int q = tid; q < P / 4; q += blockDim.x) {  // 16-byte accesses, four bins (P >= 4 below)
                const uint4 x = reinterpret_cast<const uint4 *>(sub)[q];
                reinterpret_cast<uint2 *>(o32)[q] = make_uint2(x.x | x.y << 16, x.z | x.w << 16);
                uint4 a = reinterpret_cast<const uint4 *>(acc)[q];
                a.x += x.x;
                a.y += x.y;
                a.z += x.z;
                a.w += x.w;
                reinterpret_cast<uint4 *>(acc)[q] = a;
                reinterpret_cast<uint4 *>(sub)[q] = make_uint4(0u, 0u, 0u, 0u);
            }
            if (P < 4 && tid < P / 2) {  // P = 2
                const uint32_t x0 = sub[0], x1 = sub[1];
                o32[0] = x0 | x1 << 16;
                acc[0] += x0;
                acc[1] += x1;
                sub[0] = sub[1] = 0;
            }
        } else {
            for (int q = tid; q < P / 2; q += blockDim.x) {
                const uint32_t x0 = sub[2 * q], x1 = sub[2 * q + 1];
                o32[q] = x0 | x1 << 16;
                acc[2 * q] += x0;
                acc[2 * q + 1] += x1;
                sub[2 * q] = 0;
                sub[2 * q + 1] = 0;
            }
        }
        if (g + 1 == nsub0 || g + 1 == ntot) {  // end of a relation's tile
            __syncthreads();
            flush_acc(rel);
        }
        __syncthreads();
    }

    // ---- fused exchange: the last CTA publishes the rank histogram ----
    trace_end(c, MGJ_TR_HIST);
    __threadfence();
    __syncthreads();
    __shared__ int last;
    if (threadIdx.x == 0) last = (atomicAdd(&c.ticket[TK_HIST], 1u) == gridDim.x * gridDim.y - 1);
    __syncthreads();
    // compressed shuffle / chunk streaming: k_tilescan publishes (unit counts, round boundaries)
    if (!last || c.comp || c.stream) return;
    __threadfence();
    publish_hist(c);
}

// Exclusive prefix of the per-tile histograms over tiles: tile c's tuples of
// partition p start at send_off[p] + tile_base[rel][c][p] in the owner's
// receive range (deterministic placement; one thread per (rel, p)).
// With the compressed shuffle (NEXT-1) a tile's run of partition p is
// ceil(count / CU_N) 32-byte units, and tile_base counts units; the last block
// then publishes the histograms with the rank's unit totals (publish_hist).
__global__ void k_tilescan(Ctx c) {
    const int idx = blockIdx.x * blockDim.x + threadIdx.x;
    auto val = [&](uint32_t v) { return c.comp ? (v + CU_N - 1) / CU_N : v; };
    if (!c.stream) {
        // one warp per (rel, p): the tiles' counts loaded 32 at a time and
        // scanned across the lanes (measured at M2: 27 us with a thread per
        // (rel, p) walking the tiles one after another, 8 us like this)
        const int w = idx >> 5, lane = threadIdx.x & 31;
        if (w < 2 * c.P) {
            const int rel = w / c.P, p = w % c.P;
            const uint32_t *src = c.tile_hist + (size_t)rel * c.G * c.P + p;
            uint32_t *dst = c.tile_base + (size_t)rel * c.G * c.P + p;
            uint32_t run = 0;
            for (int t0 = 0; t0 < c.G; t0 += 32) {
                const int t = t0 + lane;
                const uint32_t v = t < c.G ? val(__ldcg(src + (size_t)t * c.P)) : 0u;
                uint32_t incl = v;
#pragma unroll
                for (int o = 1; o < 32; o <<= 1) {
                    const uint32_t y = __shfl_up_sync(0xffffffffu, incl, o);
                    if (lane >= o) incl += y;
                }
                if (t < c.G) dst[(size_t)t * c.P] = run + incl - v;
                run += __shfl_sync(0xffffffffu, incl, 31);
            }
            if (c.comp && lane == 0) c.rank_units[w] = run;
        }
    } else if (idx < 2 * c.P) {
        const int rel = idx / c.P, p = idx % c.P;
        const size_t stride = c.P;
        const uint32_t *src = c.tile_hist + (size_t)rel * c.G * c.P + p;
        uint32_t *dst = c.tile_base + (size_t)rel * c.G * c.P + p;
        uint32_t run = 0;
        int t = 0;
        if (c.stream && rel == 1) {
            // NEXT-3: S round boundaries — offset of round r's first tile in this
            // rank's piece of p (round r = tiles [r * sgrid, (r + 1) * sgrid)),
            // read by p's owner to tell which rounds a received chunk needs
            for (int r = 0; r < c.nrounds; ++r) {
                *rb_first(c.arena[c.rank], c.lay, c.P, r, p) = run;
                const int t1 = min(c.G, (r + 1) * c.sgrid);
                for (; t + 4 <= t1; t += 4) {
                    const uint32_t v0 = src[(t + 0) * stride], v1 = src[(t + 1) * stride];
                    const uint32_t v2 = src[(t + 2) * stride], v3 = src[(t + 3) * stride];
                    dst[(t + 0) * stride] = run;
                    run += val(v0);
                    dst[(t + 1) * stride] = run;
                    run += val(v1);
                    dst[(t + 2) * stride] = run;
                    run += val(v2);
                    dst[(t + 3) * stride] = run;
                    run += val(v3);
                }
                for (; t < t1; ++t) {
                    dst[t * stride] = run;
                    run += val(src[t * stride]);
                }
            }
            for (int r = p; r < c.nrounds; r += c.P) {  // round r's non-empty tiles, its counter opened
                const int u0 = r * c.sgrid, u1 = min(c.G, (r + 1) * c.sgrid);
                uint32_t nt = (uint32_t)(u1 - u0);
                if (c.n_in[1] < 8ull * (uint64_t)c.G) {  // small input: some tiles are empty
                    nt = 0;
                    for (int u = u0; u < u1; ++u) {
                        uint64_t lo, hi;
                        tile_range(c.n_in[1], c.G, u, lo, hi);
                        nt += hi > lo;
                    }
                }
                rb_ntile(c.arena[c.rank], c.lay)[r] = nt;
                *rdone_ptr(c.arena[c.rank], c.lay, r) = c.epoch << 32;
            }
        }
        for (; t + 4 <= c.G; t += 4) {
            const uint32_t v0 = src[(t + 0) * stride], v1 = src[(t + 1) * stride];
            const uint32_t v2 = src[(t + 2) * stride], v3 = src[(t + 3) * stride];
            dst[(t + 0) * stride] = run;
            run += val(v0);
            dst[(t + 1) * stride] = run;
            run += val(v1);
            dst[(t + 2) * stride] = run;
            run += val(v2);
            dst[(t + 3) * stride] = run;
            run += val(v3);
        }
        for (; t < c.G; ++t) {
            const uint32_t v = src[t * stride];
            dst[t * stride] = run;
            run += val(v);
        }
        if (c.comp) c.rank_units[idx] = run;
    }
    if (!c.comp && !c.stream) return;
    __shared__ int last;
    __threadfence();
    __syncthreads();
    if (threadIdx.x == 0) last = atomicAdd(&c.ticket[TK_TSCAN], 1u) == gridDim.x - 1;
    __syncthreads();
    if (!last) return;
    __threadfence();
    publish_hist(c);
}

// ---------------------------------------------------------------------------
// a2 formulas, shared by the device plan kernel and mgj_plan_host.
// Owner of global partition p (reduced form, DESIGN.md
// §4): contiguous ranges of p cut where the cumulative tuple count (both
// relations, all ranks) crosses multiples of total/N, using the partition's
// midpoint; identity ranges p*N/P for uniform data.
// ---------------------------------------------------------------------------
__host__ __device__ inline int owner_of(uint64_t cum_before, uint64_t T, uint64_t total, int N, int p, int P) {
    if (total == 0) return (int)(((uint64_t)p * (uint64_t)N) / (uint64_t)P);
    const uint64_t o = ((2 * cum_before + T) * (uint64_t)N) / (2 * total);
    return o >= (uint64_t)N ? N - 1 : (int)o;
}

// Selective broadcast of partition p (the paper's
// assignment step P:418-444 after Track-Join: a partition is migrated or
// selectively broadcast, whichever moves fewer tuples; heavy hitters
// P:386-395).  Broadcasting R_p to every rank and keeping S_p where it is
// moves (N-1)|R_p| tuples; single-owner hash partitioning moves about
// (N-1)/N (|R_p| + |S_p|).  Broadcast wins when (N-1)|R_p| < |S_p| (both
// sides times N, the R_p terms collected).  cfg: < 0 never; 0 (auto) only
// heavy partitions, |S_p| >= 2 |S| / P, so uniform data never broadcasts;
// > 0 every partition that passes the traffic test.  Never with one rank.
__host__ __device__ inline bool bcast_of(uint64_t r, uint64_t s, uint64_t s_total, int N, int P, int cfg) {
    if (N < 2 || cfg < 0 || s == 0) return false;
    if ((uint64_t)(N - 1) * r >= s) return false;
    return cfg > 0 || s * (uint64_t)P >= 2 * s_total;
}

// The histogram as a simplified Bloom filter: a partition with no
// R or no S tuple anywhere cannot produce a match, so none of its tuples is
// shuffled, partitioned or probed.  P2P shuffle only.
__host__ __device__ inline bool skip_of(uint64_t r, uint64_t s) { return (r == 0) != (s == 0); }

// Placement-aware assignment (NEXT-2, Track-Join migration): partitions in
// order go to their preferred rank (the one holding most of their tuples)
// unless its assigned weight would pass cap = 9/8 of the mean, then to the
// least-loaded rank.  Shared by k_plan (thread 0) and mgj_plan_host.
#pragma nv_exec_check_disable  // host lambdas from mgj_plan_host, device lambdas from k_plan
template <typename WF, typename BF>
__host__ __device__ inline void assign_greedy(int N, int P, WF weight, BF pref, int32_t *owner) {
    uint64_t load[MAX_RANKS] = {}, total = 0;
    for (int p = 0; p < P; ++p) total += weight(p);
    const uint64_t cap = total / (uint64_t)N + total / (8ull * (uint64_t)N) + 1;
    for (int p = 0; p < P; ++p) {
        const uint64_t w = weight(p);
        int d = pref(p);
        if (w && load[d] + w > cap) {
            d = 0;
            for (int g = 1; g < N; ++g)
                if (load[g] < load[d]) d = g;
        }
        owner[p] = d;
        load[d] += w;
    }
}

// Weight of p in the owner ranges: a broadcast partition's S stays spread
// over the ranks, its owner (the root, which receives R_p) gets R_p + S_p/N.
__host__ __device__ inline uint64_t owner_weight(uint64_t r, uint64_t s, bool bc, int N) {
    return bc ? r + (s + (uint64_t)N - 1) / (uint64_t)N : r + s;
}

__host__ __device__ inline int ceil_log2_u64(uint64_t x) {
    int l = 0;
    while (l < 63 && (1ull << l) < x) ++l;
    return l;
}

// B2: R co-partitions that fit one shared-memory table (cap slots: the
// largest owned R partition sets this bound, against the full capacity — a
// co-partition a little above it is sliced, rarely), and, on average, R + S
// co-partitions of at most 2 * target tuples (one probe stage shared by the
// two sides, target = cap minus headroom for run padding and spread; the mean
// R + S of the owned partitions sets this bound: a heavy-hitter partition
// cannot be split by radix bits, its S side is sliced over several items).
// (Against the target, the max bound doubled the fan-out of random 8-byte keys
// whose largest partition exceeds the mean by a few sigma: M5 probe 2.8 ms.)
__host__ __device__ inline int choose_b2(uint64_t max_r, uint64_t mean_rs, int b2_cfg, int b2_max, uint64_t target,
                                         uint64_t cap) {
    if (b2_cfg > 0) return b2_cfg < b2_max ? b2_cfg : b2_max;
    int b = ceil_log2_u64((max_r + cap - 1) / cap);
    const int bs = ceil_log2_u64((mean_rs + 2 * target - 1) / (2 * target));
    if (bs > b) b = bs;
    if (b > b2_max) b = b2_max;
    return b;
}

// ---------------------------------------------------------------------------
// a2 device plan: one CTA of 1024 threads.  Every rank computes the same
// broadcast flags, owner[] and receive sizes from the same all-gathered
// histograms, plus its own send offsets (u64 tuples into the destination's
// receive buffer), its owned partitions, the local radix bits B2 and the
// chunk table of the local pass.
// Receive layout of rank d.  R: the partitions of d's range ascending, each
// [source rank ascending] (a broadcast partition's R lands at its root, the
// range owner, like any other).  S: the non-broadcast partitions of d's range
// ascending, each [source ascending], then every broadcast partition
// ascending with d's own S tuples only.  Owned list of d (plist): its range,
// then the broadcast partitions outside it; the R side of those is read from
// the root's receive buffer by the local pass (a pull broadcast).
// ---------------------------------------------------------------------------
__global__ void __launch_bounds__(1024) k_plan(Ctx c) {
    extern __shared__ uint64_t sp[];
    const int P = c.P, N = c.world, tid = threadIdx.x;
    uint64_t *tot0 = sp, *tot1 = sp + P, *pre0 = sp + 2 * P, *pre1 = sp + 3 * P, *cum = sp + 4 * P;
    int32_t *own = reinterpret_cast<int32_t *>(sp + 5 * P);
    uint32_t *chn = reinterpret_cast<uint32_t *>(own + P);  // [P+1] scratch scans (u32)
    uint8_t *bcf = reinterpret_cast<uint8_t *>(chn + P + 1);  // [P] broadcast flags
    // compressed shuffle: the receive layout counts 32-byte units, ownership still tuples
    // (present only with compression, P <= 1024: P = 4096 would not fit shared memory otherwise)
    const int PU = c.comp ? P : 0;
    uint64_t *ut0 = reinterpret_cast<uint64_t *>((reinterpret_cast<uintptr_t>(bcf + P) + 7) & ~(uintptr_t)7), *ut1 = ut0 + PU;
    __shared__ uint64_t tmp[33];
    __shared__ uint32_t tmp32[33];
    __shared__ int first[MAX_RANKS], endp[MAX_RANKS];
    __shared__ int ok, cap_bad, nbc;
    __shared__ unsigned long long maxr, sumrs, stot, bcs[MAX_RANKS];
    trace_begin(c, MGJ_TR_PLAN);
    if (tid == 0) {
        ok = wait_all_flags(c, SIG_HIST);
        cap_bad = 0;
        maxr = 0;
        sumrs = 0;
        stot = 0;
        nbc = 0;
    }
    if (tid < MAX_RANKS) first[tid] = endp[tid] = P, bcs[tid] = 0;
    __syncthreads();
    if (tid == 0 && ok) {
        // the capacities and the arena layout are job-wide (mgj.h): every rank
        // must have planned with the same ones, else peers store at offsets
        // that differ from the receiver's layout
        const uint64_t *cf = reinterpret_cast<const uint64_t *>(c.arena[c.rank] + c.lay.cfgmail);
        const uint64_t w[4] = {c.recv_cap[0], c.recv_cap[1], c.lay.total, cfg_word(c)};
        for (int g = 0; g < N && ok; ++g)
            for (int i = 0; i < 4; ++i)
                if (__ldcg(cf + g * 4 + i) != w[i]) {
                    set_err(c, MGJ_EINVAL);
                    ok = 0;
                    break;
                }
    }
    __syncthreads();
    if (!ok) {
        if (tid == 0) c.meta[MT_OK] = 0;
        return;
    }
    const uint32_t *mail = reinterpret_cast<const uint32_t *>(c.arena[c.rank] + c.lay.mail);
    auto H = [&](int g, int rel, int p) -> uint32_t { return __ldcg(mail + (size_t)(g * 2 + rel) * P + p); };
    const uint32_t *umail = reinterpret_cast<const uint32_t *>(c.arena[c.rank] + c.lay.umail);
    // layout counts: tuples, or 32-byte units with the compressed shuffle
    auto HL = [&](int g, int rel, int p) -> uint32_t {
        return c.comp ? __ldcg(umail + (size_t)(g * 2 + rel) * P + p) : H(g, rel, p);
    };
    auto LT = [&](int rel, int p) -> uint64_t { return c.comp ? (rel ? ut1[p] : ut0[p]) : (rel ? tot1[p] : tot0[p]); };
    {
        unsigned long long st = 0;
        for (int p = tid; p < P; p += blockDim.x) {
            uint64_t t0 = 0, t1 = 0, u0 = 0, u1 = 0;
            for (int g = 0; g < N; ++g) t0 += H(g, 0, p), t1 += H(g, 1, p);
            if (c.comp)
                for (int g = 0; g < N; ++g) u0 += HL(g, 0, p), u1 += HL(g, 1, p);
            const bool sk = !c.ext && skip_of(t0, t1);
            c.pskip[p] = sk;
            if (sk) t0 = t1 = u0 = u1 = 0;  // a skipped partition is absent from every layout
            tot0[p] = t0;
            pre0[p] = c.comp ? u0 : t0;
            tot1[p] = t1;
            if (c.comp) ut0[p] = u0, ut1[p] = u1;
            st += t1;
        }
        st = warp_sum(st);
        if ((tid & 31) == 0 && st) atomicAdd(&stot, st);
    }
    __syncthreads();
    const int bcfg = c.ext ? -1 : c.bcast_cfg;
    for (int p = tid; p < P; p += blockDim.x) {
        const bool bc = bcast_of(tot0[p], tot1[p], stot, N, P, bcfg);
        bcf[p] = bc;
        c.bcast[p] = bc;
        pre1[p] = bc ? 0 : LT(1, p);  // S layout: broadcast partitions are not in the owner's range part
        cum[p] = owner_weight(tot0[p], tot1[p], bc, N);
        chn[p] = bc ? HL(c.rank, 1, p) : 0u;  // this rank's own S of broadcast partitions (never skipped)
        if (bc) {
            atomicAdd(&nbc, 1);
            for (int d = 0; d < N; ++d) atomicAdd(&bcs[d], (unsigned long long)HL(d, 1, p));
        }
    }
    __syncthreads();
    block_excl_scan_u64(pre0, P, tmp);
    block_excl_scan_u64(pre1, P, tmp);
    block_excl_scan_u32(chn, P, tmp32);  // chn[p] = own S of broadcast partitions before p
    const uint64_t total = block_excl_scan_u64(cum, P, tmp);
    for (int p = tid; p < P; p += blockDim.x) {
        const int o = owner_of(cum[p], owner_weight(tot0[p], tot1[p], bcf[p], N), total, N, p, P);
        own[p] = o;
        c.owner[p] = o;
    }
    __syncthreads();
    for (int p = tid; p < P; p += blockDim.x) {
        if (p == 0 || own[p - 1] != own[p]) first[own[p]] = p;
        if (p == P - 1 || own[p + 1] != own[p]) endp[own[p]] = p + 1;
    }
    __syncthreads();
    // S tuples of this rank's own range part (non-broadcast), where its broadcast part starts
    const uint64_t s_range_me = first[c.rank] < P ? pre1[endp[c.rank] - 1] + (bcf[endp[c.rank] - 1] ? 0 : LT(1, endp[c.rank] - 1)) - pre1[first[c.rank]] : 0;
    for (int p = tid; p < P; p += blockDim.x) {
        const int f = first[own[p]];
        uint64_t m0 = 0, m1 = 0;
        for (int g = 0; g < c.rank; ++g) m0 += HL(g, 0, p), m1 += HL(g, 1, p);
        const uint64_t b0 = pre0[p] - pre0[f];
        const uint64_t b1 = bcf[p] ? s_range_me + chn[p] : pre1[p] - pre1[f];
        if (!c.ext) {
            c.send_off[p] = b0 + m0;
            c.send_off[P + p] = bcf[p] ? b1 : b1 + m1;  // broadcast partition: S goes to this rank itself
        }
        c.seg_start[p] = b0;
        c.seg_start[P + p] = b1;
        c.seg_len[p] = LT(0, p);
        c.seg_len[P + p] = bcf[p] ? HL(c.rank, 1, p) : LT(1, p);
    }
    if (tid < 2 * MAX_RANKS) {
        const int d = tid >> 1, rel = tid & 1;
        uint64_t size = 0;
        if (d < N && first[d] < P) {
            const uint64_t *pre = rel ? pre1 : pre0;
            const int l = endp[d] - 1;
            const uint64_t last = rel ? (bcf[l] ? 0 : LT(1, l)) : LT(0, l);
            size = pre[l] + last - pre[first[d]];
        }
        if (d < N && rel) size += bcs[d];
        c.recv_size[rel * MAX_RANKS + d] = size;
        if (size > (c.comp ? c.recv_cap_u[rel] : c.recv_cap[rel])) atomicOr(&cap_bad, 1);
        // EXTERNAL: the send arena holds this rank's whole input per relation
        // in a region of recv_cap tuples
        if (c.ext && d == 0 && c.n_in[rel] > c.recv_cap[rel]) atomicOr(&cap_bad, 1);
    }
    int plo = first[c.rank] < P ? first[c.rank] : 0;
    int phi = first[c.rank] < P ? endp[c.rank] : 0;
    __syncthreads();
    // owned list: the range, then the broadcast partitions outside it (ascending)
    for (int p = tid; p < P; p += blockDim.x) chn[p] = (bcf[p] && (p < plo || p >= phi)) ? 1u : 0u;
    __syncthreads();
    const int nout = (int)block_excl_scan_u32(chn, P, tmp32);
    int nr = phi - plo, np = nr + nout;
    for (int p = tid; p < P; p += blockDim.x) {
        if (p >= plo && p < phi) c.plist[p - plo] = p;
        else if (bcf[p]) c.plist[nr + chn[p]] = p;
    }
    __syncthreads();
    if (c.assign) {
        // Placement-aware assignment (NEXT-2; the paper's migration step after
        // Track-Join [34]): with uniform one-hop costs a partition's
        // cheapest single destination is the rank that already holds most of
        // its tuples (of R for a broadcast partition, whose S stays spread), so
        // it moves there unless that rank's assigned weight would pass 9/8 of
        // the mean, then to the least-loaded rank (thread 0, partitions in
        // order: deterministic, the same on every rank; host mirror
        // mgj_plan_host).  Owners are no longer contiguous ranges: the layout
        // of rank d is its partitions ascending (one block scan per rank and
        // relation), then, for S, its own tuples of broadcast partitions.
        uint8_t *best = reinterpret_cast<uint8_t *>(ut1 + PU);  // [P] (after the unit totals, if any)
        for (int p = tid; p < P; p += blockDim.x) {
            int b = 0;
            uint64_t hb = 0;
            for (int g = 0; g < N; ++g) {
                const uint64_t h = (uint64_t)H(g, 0, p) + (bcf[p] ? 0u : H(g, 1, p));
                if (h > hb) hb = h, b = g;
            }
            best[p] = (uint8_t)b;
        }
        __syncthreads();
        if (tid == 0) assign_greedy(N, P, [&](int p) { return owner_weight(tot0[p], tot1[p], bcf[p], N); },
                                    [&](int p) { return (int)best[p]; }, own);
        __syncthreads();
        for (int p = tid; p < P; p += blockDim.x) c.owner[p] = own[p];
        __shared__ unsigned long long rsum[2][MAX_RANKS];
        for (int rel = 0; rel < 2; ++rel)
            for (int d = 0; d < N; ++d) {
                for (int p = tid; p < P; p += blockDim.x)
                    cum[p] = (own[p] == d && !(rel && bcf[p])) ? LT(rel, p) : 0;
                __syncthreads();
                const uint64_t tot_d = block_excl_scan_u64(cum, P, tmp);
                for (int p = tid; p < P; p += blockDim.x) {
                    if (own[p] != d || (rel && bcf[p])) continue;
                    uint64_t m = 0;  // this rank's tuples of p go after those of lower ranks
                    for (int g = 0; g < c.rank; ++g) m += HL(g, rel, p);
                    c.send_off[rel * P + p] = cum[p] + m;
                    if (rel == 0 || d == c.rank) c.seg_start[rel * P + p] = cum[p];
                }
                if (tid == 0) rsum[rel][d] = tot_d;
                __syncthreads();
            }
        // S of broadcast partitions: this rank's own tuples, after its assigned part
        for (int p = tid; p < P; p += blockDim.x) cum[p] = bcf[p] ? HL(c.rank, 1, p) : 0u;
        __syncthreads();
        block_excl_scan_u64(cum, P, tmp);
        for (int p = tid; p < P; p += blockDim.x)
            if (bcf[p]) c.send_off[P + p] = c.seg_start[P + p] = rsum[1][c.rank] + cum[p];
        __syncthreads();
        if (tid == 0) {
            cap_bad &= ~1;
            for (int d = 0; d < N; ++d)
                for (int rel = 0; rel < 2; ++rel) {
                    const uint64_t size = rsum[rel][d] + (rel ? bcs[d] : 0);
                    c.recv_size[rel * MAX_RANKS + d] = size;
                    if (size > (c.comp ? c.recv_cap_u[rel] : c.recv_cap[rel])) cap_bad |= 1;
                }
        }
        // owned list: the partitions assigned here, then the broadcast ones rooted elsewhere
        __syncthreads();
        for (int p = tid; p < P; p += blockDim.x) chn[p] = own[p] == c.rank ? 1u : 0u;
        __syncthreads();
        const int nmine = (int)block_excl_scan_u32(chn, P, tmp32);
        for (int p = tid; p < P; p += blockDim.x)
            if (own[p] == c.rank) c.plist[chn[p]] = p;
        __syncthreads();
        for (int p = tid; p < P; p += blockDim.x) chn[p] = (bcf[p] && own[p] != c.rank) ? 1u : 0u;
        __syncthreads();
        const int nb = (int)block_excl_scan_u32(chn, P, tmp32);
        for (int p = tid; p < P; p += blockDim.x)
            if (bcf[p] && own[p] != c.rank) c.plist[nmine + chn[p]] = p;
        plo = phi = nr = 0;
        np = nmine + nb;
        __syncthreads();
    }
    // per owned partition: R and S sizes of its received pieces
    auto own_p = [&](int i) -> int { return i < nr ? plo + i : c.plist[i]; };
    auto own_len = [&](int rel, int p) -> uint64_t { return rel ? (bcf[p] ? (uint64_t)H(c.rank, 1, p) : tot1[p]) : tot0[p]; };  // 0 if skipped
    {  // largest owned R partition and total owned R + S: warp reductions, one shared atomic per warp
        unsigned long long mr = 0, sr = 0;
        for (int i = tid; i < np; i += blockDim.x) {
            const int p = own_p(i);
            mr = max(mr, (unsigned long long)tot0[p]);
            sr += tot0[p] + own_len(1, p);
        }
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) {
            mr = max(mr, __shfl_xor_sync(0xffffffffu, mr, o));
            sr += __shfl_xor_sync(0xffffffffu, sr, o);
        }
        if ((tid & 31) == 0) {
            atomicMax(&maxr, mr);
            atomicAdd(&sumrs, sr);
        }
    }
    __syncthreads();
    const int B2 = choose_b2(maxr, np > 0 ? sumrs / (uint64_t)np : 0, c.b2_cfg, c.b2_max,
                             (uint64_t)c.probe_target, (uint64_t)c.probe_slots);
    // received pieces of every owned partition i: P2P — one piece per relation
    // (the whole segment, sources ascending inside it; a broadcast partition's
    // R piece in its root's buffer); EXTERNAL — one piece per source rank g,
    // the receive area being [g0 | g1 | ...], each [owned p ascending]
    const uint32_t *mine = mail + (size_t)c.rank * 2 * P;
    for (int rel = 0; rel < 2; ++rel) {
        uint64_t *ps = c.piece_start + (size_t)rel * P * MAX_RANKS;
        uint32_t *pl = c.piece_len + (size_t)rel * P * MAX_RANKS;
        if (!c.ext) {
            for (int i = tid; i < np; i += blockDim.x) {
                const int p = own_p(i);
                const uint64_t src = rel ? (uint64_t)c.rank : (uint64_t)own[p];
                // piece 0 only: with the P2P shuffle nothing reads pieces 1.. (chunk_table,
                // k_chunkmap); storing them was most of this kernel's time (LSU-bound)
                ps[(size_t)i * MAX_RANKS] = c.seg_start[rel * P + p] | src << PIECE_SRC_SHIFT;
                pl[(size_t)i * MAX_RANKS] = (uint32_t)(rel ? (bcf[p] ? (uint64_t)HL(c.rank, 1, p) : LT(1, p)) : LT(0, p));
            }
            continue;
        }
        uint64_t displ = 0;  // start of source g's block in this rank's receive area
        for (int g = 0; g < N; ++g) {
            for (int i = tid; i <= np; i += blockDim.x)
                chn[i] = i < np ? __ldcg(mail + (size_t)(g * 2 + rel) * P + plo + i) : 0;
            __syncthreads();
            const uint32_t from_g = block_excl_scan_u32(chn, np + 1, tmp32);
            for (int i = tid; i < np; i += blockDim.x) {
                ps[(size_t)i * MAX_RANKS + g] = (displ + chn[i]) | (uint64_t)c.rank << PIECE_SRC_SHIFT;
                pl[(size_t)i * MAX_RANKS + g] = __ldcg(mail + (size_t)(g * 2 + rel) * P + plo + i);
            }
            if (tid == 0) c.ext_counts[(1 * 2 + rel) * MAX_RANKS + g] = from_g;
            displ += from_g;
            __syncthreads();
        }
        // send side: owners are contiguous ascending ranges, so the send buffer
        // ordered by destination is ordered by partition: offsets = prefix of H_me
        for (int p = tid; p <= P; p += blockDim.x) {
            if (p < P) cum[p] = __ldcg(mine + rel * P + p);
        }
        __syncthreads();
        block_excl_scan_u64(cum, P, tmp);
        for (int p = tid; p < P; p += blockDim.x) c.send_off[rel * P + p] = cum[p];
        if (tid < N) {
            uint64_t cnt = 0;
            for (int p = first[tid]; p < endp[tid] && first[tid] < P; ++p) cnt += __ldcg(mine + rel * P + p);
            c.ext_counts[(0 * 2 + rel) * MAX_RANKS + tid] = cnt;
        }
        __syncthreads();
    }
    __syncthreads();
    // chunk table of the local pass: chunk_base[rel][i] = first chunk of owned partition i,
    // piece_chunk[rel][i][g] = first chunk of piece g inside i (chunks of C tuples)
    __shared__ int s_ba;
    uint32_t nch[2];
    auto chunk_table = [&](uint64_t C) {
        for (int rel = 0; rel < 2; ++rel) {
            const uint32_t *pl = c.piece_len + (size_t)rel * P * MAX_RANKS;
            uint32_t *pc = c.piece_chunk + (size_t)rel * P * (MAX_RANKS + 1);
            for (int i = tid; i <= np; i += blockDim.x) {
                uint32_t t = 0;
                if (i < np && !c.ext) {  // one piece (P2P)
                    pc[(size_t)i * (MAX_RANKS + 1)] = 0;
                    t = (uint32_t)((pl[(size_t)i * MAX_RANKS] + C - 1) / C);
                } else if (i < np) {
                    for (int g = 0; g < MAX_RANKS; ++g) {
                        pc[(size_t)i * (MAX_RANKS + 1) + g] = t;
                        t += (uint32_t)((pl[(size_t)i * MAX_RANKS + g] + C - 1) / C);
                    }
                    pc[(size_t)i * (MAX_RANKS + 1) + MAX_RANKS] = t;
                }
                chn[i] = t;
            }
            __syncthreads();
            nch[rel] = block_excl_scan_u32(chn, np + 1, tmp32);
            for (int i = tid; i <= np; i += blockDim.x) c.chunk_base[(size_t)rel * c.cb_stride + i] = chn[i];
            __syncthreads();
        }
    };
    chunk_table((uint64_t)(c.comp ? c.chunk_units : c.chunk_tuples));  // compressed: chunks of units
    if (c.comp) {
        // global row id of the first row of every (relation, rank, tile): rank
        // g holds rows [sum_{g' < g} n_g', + n_g) (reading C12), tile c its
        // local rows tile_range(n_g, G, c); the local pass adds a unit entry's
        // offset to rebuild the id payload
        __shared__ unsigned long long nrank[2][MAX_RANKS];
        if (tid < 2 * MAX_RANKS) nrank[tid / MAX_RANKS][tid % MAX_RANKS] = 0;
        __syncthreads();
        for (int x = tid; x < 2 * N * P; x += blockDim.x) {
            const int rel = x / (N * P), g = (x / P) % N, p = x % P;
            const uint32_t h = H(g, rel, p);
            if (h) atomicAdd(&nrank[rel][g], (unsigned long long)h);
        }
        __syncthreads();
        for (int x = tid; x < 2 * N * c.G; x += blockDim.x) {
            const int rel = x / (N * c.G), g = (x / c.G) % N, t = x % c.G;
            uint64_t row0 = 0, lo, hi;
            for (int h = 0; h < g; ++h) row0 += nrank[rel][h];
            tile_range(nrank[rel][g], c.G, t, lo, hi);
            c.rowbase[((size_t)rel * MAX_RANKS + g) * c.G + t] = (uint32_t)(row0 + lo);
            // an entry holds the row's offset in its tile in 12 + B1 bits
            if (hi - lo > (1ull << (12 + c.B1))) atomicOr(&cap_bad, 2);
        }
        __syncthreads();
    }
    if (tid == 0) {
        // two-level local partitioning: when the owned
        // partitions span more than LOCAL2_NCH chunks on average, a first
        // pass splits every owned partition into 2^BA sub-partitions (runs
        // stored in place per chunk), and the chunked pass then gathers each
        // sub-partition's runs and uses the remaining B2 - BA bits.  The mean, not the maximum: a few
        // heavy-hitter partitions (Zipf) are not helped by splitting the rest
        const uint32_t meannch = np ? (max(nch[0], nch[1]) + np - 1) / np : 0;
        int BA = 0;
        if (c.split_cfg > 0) {
            BA = c.split_cfg;
        } else if (c.split_cfg == 0 && meannch > (uint32_t)LOCAL2_NCH) {
            // sub-partitions of ~32 chunks; measured at N=8-sized partitions (B1 = 7, mean
            // 341 chunks): BA 4 12.13 ms > 3 12.30 > 5 12.42 > 2 13.34 (round 1, with a
            // counting pass and contiguous sub-partitions: 3 > 4 > 2)
            BA = ceil_log2_u64((meannch + 31) / 32);
            while (BA > 0 && (np << BA) > c.vcap) --BA;
        }
        if (BA > B2) BA = B2;
        if (BA > MAX_BA) BA = MAX_BA;
        if (!c.mid[0] || (np << BA) > c.vcap || c.comp) BA = 0;  // compressed: one local pass (it decodes)
        s_ba = BA;
    }
    __syncthreads();
    const int BA = s_ba;
    // the first pass (fan-out <= 2^MAX_BA) reads chunks of its own, larger size
    if (BA > 0 && c.chunk_tuples1s != c.chunk_tuples) chunk_table((uint64_t)c.chunk_tuples1s);
    if (tid == 0) {
        const bool fits = nch[0] <= c.max_chunks && nch[1] <= c.max_chunks;
        if (cap_bad & 2) set_err(c, MGJ_EINVAL);  // tiles too long for the compressed entry
        if (cap_bad || !fits) set_err(c, MGJ_ECAPACITY);
        c.meta[MT_PLO] = plo;
        c.meta[MT_PHI] = phi;
        c.meta[MT_NP] = np;
        c.meta[MT_NBC] = nbc;
        c.meta[MT_B2] = B2;
        c.meta[MT_NCH_R] = (int)nch[0];
        c.meta[MT_NCH_S] = (int)nch[1];
        c.meta[MT_CHUNK] = c.comp ? c.chunk_units : (BA ? c.chunk_tuples1s : c.chunk_tuples);
        c.meta[MT_BA] = BA;
        c.meta[MT_QB] = B2 - BA;
        c.meta[MT_NLP] = np;
        c.meta[MT_OK] = (cap_bad || !fits) ? 0 : 1;
    }
    trace_end(c, MGJ_TR_PLAN);
}

// Wait for every rank's flag `kind` (and `kind2` unless < 0).
__global__ void k_wait(Ctx c, int kind, int kind2) {
    if (threadIdx.x == 0 && blockIdx.x == 0 && wait_all_flags(c, kind) && kind2 >= 0) wait_all_flags(c, kind2);
}

}  // namespace mgj
