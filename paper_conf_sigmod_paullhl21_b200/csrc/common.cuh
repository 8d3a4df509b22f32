// common.cuh — shared device helpers, the per-run kernel context and the
// symmetric-arena layout of libmgj (B200 / sm_100a).
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>

#include "mgj.h"
#include "mgj_aux.h"

namespace mgj {

constexpr int MAX_RANKS = MGJ_MAX_RANKS;
constexpr int MAX_B1 = 12;              // 2^12 global partitions at most
constexpr int MAX_B2 = 11;              // local fan-out per pass
constexpr int HIST_THREADS = 512;
constexpr int SCATTER_THREADS = 1024;
constexpr int LOCAL_THREADS = 1024;
// local-pass tuples per thread (chunk C <= 12 * LOCAL_THREADS), 8-byte tuples
// (13 measured: local 3.24 vs 2.87 ms from spills)
constexpr int LOCAL_VMAX = 12;
__host__ __device__ constexpr int local_vmax(int tuple_bytes) { return LOCAL_VMAX * 8 / tuple_bytes; }
constexpr int PROBE_THREADS = 1024;     // warps 0..PROBE_NP-1 = TMA producers, the rest build/probe
constexpr int PROBE_NST = 3;            // pipeline stages (items in flight per CTA)
// producer warps per item: one per relation (four, two per relation, measured:
// Zipf z = 1 probe 2.71 -> 2.54 ms but M2 1.95 -> 2.24 ms, so two stay)
constexpr int PROBE_PPI = 2;
constexpr int PROBE_NP = PROBE_NST * PROBE_PPI;  // producer warps (item streams <= PROBE_NST: parity waits one phase ahead)
constexpr int PROBE_SLOTS8 = 4224;      // stage capacity per relation (slots) for 8-byte tuples; half for 16-byte
constexpr int PROBE_HEAD8 = 128;        // headroom: co-partition target = capacity - headroom (padding, spread)
constexpr int PROBE_MAXP = 1024;        // chunk pieces per relation per item
constexpr int MAX_BA = 6;               // two-level local partitioning: at most 2^6 sub-partitions per pass A
constexpr int LOCAL2_NCH = 256;         // a partition of more chunks than this gets the first local pass
constexpr int EA_STRIDE = (1 << MAX_BA) + 1;  // first-pass run offsets per chunk (2^BA runs + the end)
// sub-partitions of a first local pass: at most local2_vcap(P) in total
__host__ __device__ constexpr int local2_vcap(int P) { return 4 * P > 4096 ? 4 * P : 4096; }
constexpr uint64_t WAIT_TIMEOUT_NS = 20ull * 1000 * 1000 * 1000;  // default peer-signal wait bound

constexpr int RES_W = 8;  // u64 words per rank in the result mailbox (a6)
// NEXT-1 compressed shuffle: a 32-byte unit carries CU_N tuples as 44-bit
// entries (key >> B1 in the low 32 - B1 bits, the row's offset in its source
// tile above), plus (count, source rank, tile) in its top word
constexpr int CU_N = 5;
constexpr int CU_ENTRY_BITS = 44;
constexpr int CHUNK_UNITS = 2048;  // local-pass chunk with the compressed shuffle: 2 units per thread
// NEXT-3 chunk streaming: the S scatter's tiles complete in rounds (round r =
// the r-th tile of every scatter CTA); at most STREAM_RMAX rounds, tiles per
// scatter CTA STREAM_TPC (fewer if the rounds would exceed STREAM_RMAX)
constexpr int STREAM_RMAX = 16;
constexpr int STREAM_TPC = 4;
// peer flags: histograms published (a1), R / S tuples all stored (a3), partial sums published (a6)
enum Sig { SIG_HIST = 0, SIG_DATA_R = 1, SIG_RES = 2, SIG_DATA_S = 3, SIG_COUNT = 4 };
enum Ticket { TK_HIST = 0, TK_SCAT_R = 1, TK_SCAT_S = 2, TK_SCAT_DONE = 3, TK_ITEMS = 4,
              TK_PROBE = 5, TK_LOCAL = 6, TK_TSCAN = 7, TK_COUNT = 8 };
enum Meta { MT_PLO = 0, MT_PHI = 1, MT_B2 = 2, MT_OK = 3, MT_NCH_R = 4, MT_NCH_S = 5,
            MT_NITEMS = 6, MT_CHUNK = 7,
            MT_BA = 8,       // bits of the first local pass (0: single local pass)
            MT_QB = 9,       // bits of the (last) chunked local pass: B2 - BA
            MT_NLP = 10,     // partitions of the chunked local pass: owned partitions, or sub-partitions
            MT_NCHB_R = 11,  // chunks of the chunked pass after a first pass (R, S)
            MT_NCHB_S = 12,
            MT_NP = 13,      // owned partitions (the range + broadcast partitions outside it)
            MT_NBC = 14,     // broadcast partitions (selective broadcast, NEXT-2)
            MT_COUNT = 16 };

// Source rank of a received piece travels in the top byte of its start
// (starts are < 2^56 tuples): a broadcast partition's R piece lives in its
// root's receive buffer and is read from there by the local pass.
constexpr int PIECE_SRC_SHIFT = 56;
__host__ __device__ __forceinline__ uint64_t piece_off(uint64_t v) { return v & ((1ull << PIECE_SRC_SHIFT) - 1); }
__host__ __device__ __forceinline__ int piece_src(uint64_t v) { return (int)(v >> PIECE_SRC_SHIFT); }

// Arena layout (bytes from each rank's arena base; identical on all ranks).
struct Arena {
    uint64_t sig;      // u64 flags[SIG_COUNT][MAX_RANKS], written by peers
    uint64_t mail;     // u32 hist[MAX_RANKS][2][P]
    uint64_t resmail;  // u64 res[MAX_RANKS][RES_W] (count, checksum, n_out, status, pair digest)
    uint64_t cfgmail;  // u64 cfg[MAX_RANKS][4] (recv_cap R, recv_cap S, arena bytes, B1) published with a1
    uint64_t umail;    // u32 units[MAX_RANKS][2][P] (compress: 32-byte units per partition) published with a1
    uint64_t rbmail;   // u32 ntile[STREAM_RMAX], then rb[STREAM_RMAX][P]: this rank's S rounds (streaming)
    uint64_t rdone;    // u64 done[STREAM_RMAX]: epoch << 32 | this rank's S tiles of round r stored (streaming)
    uint64_t recv[2];  // received tuples of R, S
    uint64_t total;
};

// One probe work item: a slice of co-partition (p, q).  Each side is the
// half-open range of (chunk k, slot offset a) positions [(k0, a0), (k1, a1))
// over the q-runs of p's chunks (a counts padded 8/16-byte slots, even).
struct Side {
    uint32_t k0, a0, k1, a1;
};
struct Item {
    uint32_t pi;  // owned partition index (p - p_lo)
    uint32_t q;   // local sub-partition
    Side r, s;
};

// Everything a kernel needs, passed by value (param space).
struct Ctx {
    int32_t rank, world, B1, P, b2_cfg, b2_max;
    int32_t G;                    // tiles per relation (= scatter CTAs)
    int32_t hist_split;           // k_hist CTAs per tile
    int32_t chunk_tuples;         // local-pass chunk C (tuples)
    int32_t chunk_region;         // slots per chunk in the local buffer (C + 2^b2_max, even)
    int32_t chunk_tuples2;        // chunk of the chunked pass after a first pass (its fan-out is at
    int32_t chunk_region2;        //   most 2^(b2_max - 1), so its buffers leave room for larger chunks)
    int32_t qm2_bits;             // log2 of that fan-out bound
    int32_t chunk_tuples1s;       // chunk of the first (split) pass: fan-out <= 2^MAX_BA
    int32_t probe_slots;          // probe stage capacity per relation (slots)
    int32_t probe_target;         // co-partition size B2 aims at (tuples)
    int32_t materialize;
    int32_t ext;                  // shuffle mode EXTERNAL: scatter into send_buf, caller exchanges
    int32_t comp;                 // NEXT-1 compressed shuffle (units of CU_N entries, see scatter.cuh)
    int32_t assign;               // NEXT-2 placement-aware partition assignment (k_plan)
    int32_t chunk_units;          // compress: local-pass chunk in units
    int32_t stream;               // NEXT-3: S's local pass streams chunks as their scatter rounds complete
    int32_t sgrid;                //   S scatter CTAs (tiles per round)
    int32_t nrounds;              //   rounds of the S scatter: ceil(G / sgrid) <= STREAM_RMAX
    uint32_t *cwait;              //   [max_chunks] S chunk li: first source << 8 | last source << 4 | its last round
    uint32_t *corder;             //   [max_chunks] S chunks in round order
    uint32_t *rcount;             //   [2][STREAM_RMAX] S chunks per round, placement cursors (zeroed per run)
    uint32_t *rowbase;            // compress: [2][MAX_RANKS][G] global row id of each (rank, tile)'s first row
    uint32_t *rank_units;         // compress: [2][P] this rank's 32-byte units per partition
    uint32_t max_items;
    uint64_t epoch;
    uint64_t timeout_ns;          // bound on a wait for peer signals (mgj_config.peer_timeout_ms)
    uint64_t recv_cap[2];
    uint64_t recv_cap_u[2];       // compressed shuffle: receive capacity in 32-byte units
    uint64_t max_chunks;
    uint64_t out_cap;
    uint64_t mid_cap;             // slots of each first-pass output buffer (max_chunks * chunk_region1)
    int32_t vcap;                 // local2_vcap(P)
    int32_t cb_stride;            // entries per relation of chunk_base, chunk_base1 (vcap + 1)
    int32_t split_cfg;            // mgj_config.local_split_bits
    Arena lay;
    char *arena[MAX_RANKS];       // arena bases as mapped in this process
    const void *in_key[2];
    const void *in_pay[2];
    uint64_t n_in[2];
    // workspace (this rank's device memory)
    uint32_t *rank_hist;          // [2][P]
    uint32_t *tile_hist;          // [2][G][P] per-tile histograms (a1)
    uint32_t *tile_base;          // [2][G][P] exclusive prefix over tiles
    uint16_t *sub_hist;           // [2][G][sub_ns][P] per scatter sub-tile histograms (a1)
    int32_t scat_T;               // scatter sub-tile (tuples)
    int32_t sub_ns;               // sub-tiles per tile (capacity)
    uint32_t *ticket;             // [TK_COUNT]
    int32_t *meta;                // [MT_COUNT]
    int32_t *owner;               // [P] range owner (a broadcast partition's root)
    uint8_t *bcast;               // [P] selective broadcast flags (a2)
    uint8_t *pskip;               // [P] partitions with an empty side: never shuffled (histogram as a Bloom filter)
    int32_t *plist;               // [P] owned partitions: the range, then broadcast partitions outside it
    int32_t bcast_cfg;            // mgj_config.skew_bcast
    uint64_t *send_off;           // [2][P]
    uint64_t *seg_start;          // [2][P]
    uint64_t *seg_len;            // [2][P]
    uint64_t *recv_size;          // [2][MAX_RANKS]
    uint64_t *piece_start;        // [2][P][MAX_RANKS] received piece of owned partition pi from source g
    uint32_t *piece_len;          // [2][P][MAX_RANKS]
    uint32_t *piece_chunk;        // [2][P][MAX_RANKS+1] chunk prefix over the pieces of pi
    uint64_t *ext_counts;         // [2 (send, recv)][2 rel][MAX_RANKS] (EXTERNAL shuffle)
    uint32_t *chunk_base;         // [2][cb_stride] first chunk of each (sub-)partition of the chunked pass
    uint32_t *hA;                 // [2][vcap] first local pass: padded slots per sub-partition
    uint32_t *chunk_base1;        // [2][cb_stride] first chunk of each owned partition in the first pass
    uint16_t *eoffA[2];           // [chunks][EA_STRIDE] first pass: run offsets in each chunk's output
    void *mid[2];                 // first local pass output: chunk li at slot li * chunk_region1
    int32_t chunk_region1;        // slots per first-pass chunk region (chunk_tuples1s + 2^MAX_BA, even)
    uint16_t *eoff[2];            // run offsets, [(Q+1)*chunk_base[p] + q*nch_p + k]
    uint32_t *cop_slots;          // [2][P][2^b2_max] padded slots per co-partition
    Item *items;                  // [max_items]
    void *local[2];               // locally partitioned tuples (a4 output), chunk regions
    unsigned long long *acc;      // [4] local count, checksum, n_out, pair digest
    int32_t *err;                 // sticky device status
    unsigned long long *result;   // [8] global count, checksum; local n_out; status; global pair digest
    unsigned long long *trace;    // [MGJ_TRACE_COUNT][2] (UINT64_MAX - first start, last end) or null
    void *out_key, *out_a, *out_b;
};

// Tile c of G over n tuples: boundaries are multiples of 4 tuples (16-byte
// aligned for the TMA loads); the last tile ends at n.
__host__ __device__ __forceinline__ void tile_range(uint64_t n, int G, int c, uint64_t &lo, uint64_t &hi) {
    lo = (n * (uint64_t)c / (uint64_t)G) & ~3ull;
    hi = (c == G - 1) ? n : ((n * (uint64_t)(c + 1) / (uint64_t)G) & ~3ull);
}

template <typename K> struct TupT;
template <> struct TupT<uint32_t> { using T = uint2; };       // {key, payload}
template <> struct TupT<uint64_t> { using T = ulonglong2; };  // {key, payload}

__device__ __forceinline__ uint64_t *sig_ptr(char *arena, const Arena &lay, int kind, int g) {
    return reinterpret_cast<uint64_t *>(arena + lay.sig) + kind * MAX_RANKS + g;
}

__device__ __forceinline__ void st_release_sys(uint64_t *p, uint64_t v) {
    asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

__device__ __forceinline__ uint64_t ld_acquire_sys(const uint64_t *p) {
    uint64_t v;
    asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}


__device__ __forceinline__ uint64_t globaltimer() {
    uint64_t t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}

__device__ __forceinline__ void set_err(const Ctx &c, int code) { atomicCAS(c.err, 0, code); }

// Kernel timeline (mgj_config.trace): every CTA's thread 0 stamps its start
// and end; slot id keeps the earliest start (stored as UINT64_MAX - t so that
// a zeroed buffer is "empty" for max) and the latest end.
__device__ __forceinline__ void trace_begin(const Ctx &c, int id, bool who = threadIdx.x == 0) {
    if (c.trace && who) atomicMax(&c.trace[2 * id], ~(unsigned long long)globaltimer());
}
__device__ __forceinline__ void trace_end(const Ctx &c, int id, bool who = threadIdx.x == 0) {
    if (c.trace && who) atomicMax(&c.trace[2 * id + 1], (unsigned long long)globaltimer());
}

// Thread-0 helper: wait until every rank g raised flag `kind` for this epoch.
__device__ inline bool wait_all_flags(const Ctx &c, int kind) {
    const uint64_t t0 = globaltimer();
    for (int g = 0; g < c.world; ++g) {
        const uint64_t *f = sig_ptr(c.arena[c.rank], c.lay, kind, g);
        while (ld_acquire_sys(f) < c.epoch) {
            if (globaltimer() - t0 > c.timeout_ns) {
                set_err(c, MGJ_EPEER);
                return false;
            }
            __nanosleep(100);
        }
    }
    return true;
}

// NEXT-3 streaming, in the arena of source rank g: the completed S tiles of
// its round r (epoch << 32 | count: k_tilescan sets the epoch, each tile adds
// one; a later run's value compares above any earlier one), and the rounds'
// non-empty tiles and per-partition first offsets.
__device__ __forceinline__ unsigned long long *rdone_ptr(char *arena, const Arena &lay, int r) {
    return reinterpret_cast<unsigned long long *>(arena + lay.rdone) + r;
}
__device__ __forceinline__ uint32_t *rb_ntile(char *arena, const Arena &lay) {
    return reinterpret_cast<uint32_t *>(arena + lay.rbmail);
}
__device__ __forceinline__ uint32_t *rb_first(char *arena, const Arena &lay, int P, int r, int p) {
    return reinterpret_cast<uint32_t *>(arena + lay.rbmail) + STREAM_RMAX + (size_t)r * P + p;
}

// Raise flag `kind` of this rank at every peer (call after a system fence).
__device__ inline void signal_all(const Ctx &c, int kind) {
    for (int d = 0; d < c.world; ++d) st_release_sys(sig_ptr(c.arena[d], c.lay, kind, c.rank), c.epoch);
}

// Radix digits: digit1 = low B1 key bits (global partition), digit2 = the
// next B2 bits (local sub-partition); SURVEY.md §8 notation, reading C5.
template <typename T>
__device__ __forceinline__ uint32_t digit1(T k, int P) {
    return (uint32_t)k & (uint32_t)(P - 1);
}
template <typename T>
__device__ __forceinline__ uint32_t digit2(T k, int B1, int Q) {
    return (uint32_t)((unsigned long long)k >> B1) & (uint32_t)(Q - 1);
}

// Shared-memory hash of the key bits above the radix digits (a5).  A
// multiplicative (Weyl) hash; deliberately unrelated to the oracle's.
template <typename T>
__device__ __forceinline__ uint32_t tab_hash(T k, int shift, int logT) {
    if constexpr (sizeof(T) == 4) {
        return (((uint32_t)k >> shift) * 0x2545F491u) >> (32 - logT);
    } else {
        const unsigned long long v = (unsigned long long)k;
        const uint32_t x = (uint32_t)(v >> shift) ^ (uint32_t)(v >> 32) * 0x9E3779B1u;
        return (x * 0x2545F491u) >> (32 - logT);
    }
}

// Checksum term a*C + b (reading C3): C = 2^32 for 4-byte
// payloads, 0x9E3779B97F4A7C15 for 8-byte payloads.
template <typename T>
__device__ __forceinline__ unsigned long long chk_term(T a, T b) {
    if constexpr (sizeof(T) == 4) {
        return ((unsigned long long)(uint32_t)a << 32) + (uint32_t)b;
    } else {
        return (unsigned long long)a * 0x9E3779B97F4A7C15ull + (unsigned long long)b;
    }
}

// Pair-digest term a*b mod 2^64 (reading C3b): bilinear in the
// matched (R, S) pair, so a wrong pairing changes the digest even where the
// linear checksum cannot.
template <typename T>
__device__ __forceinline__ unsigned long long dig_term(T a, T b) {
    if constexpr (sizeof(T) == 4) {
        return (unsigned long long)(uint32_t)a * (uint32_t)b;
    } else {
        return (unsigned long long)a * (unsigned long long)b;
    }
}

// NEXT-1 unit (256 bits as four u64 words): entries e0..e4 of 44 bits at bit
// 44*i, then the unit's meta word (valid count | source rank << 3 | tile << 6)
// in bits 224..255.
__device__ __forceinline__ void unit_pack(const unsigned long long (&e)[CU_N], uint32_t meta,
                                          unsigned long long (&a)[4]) {
    a[0] = e[0] | (e[1] << 44);
    a[1] = (e[1] >> 20) | (e[2] << 24);
    a[2] = (e[2] >> 40) | (e[3] << 4) | (e[4] << 48);
    a[3] = (e[4] >> 16) | ((unsigned long long)meta << 32);
}
__device__ __forceinline__ unsigned long long unit_entry(const unsigned long long (&a)[4], int i) {
    constexpr unsigned long long M44 = (1ull << CU_ENTRY_BITS) - 1;
    switch (i) {
        case 0: return a[0] & M44;
        case 1: return (a[0] >> 44) | ((a[1] & ((1ull << 24) - 1)) << 20);
        case 2: return (a[1] >> 24) | ((a[2] & 0xFull) << 40);
        case 3: return (a[2] >> 4) & M44;
        default: return (a[2] >> 48) | ((a[3] & ((1ull << 28) - 1)) << 16);
    }
}

__device__ __forceinline__ unsigned long long warp_sum(unsigned long long v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    return v;
}

// Block-wide exclusive scan of u32 values in shared memory `a[0..n)`, n <= 32*blockDim.
// Uses `tmp` (>= 33 u32).  Returns the total.  All threads must call.
__device__ inline uint32_t block_excl_scan_u32(uint32_t *a, int n, uint32_t *tmp) {
    const int tid = threadIdx.x, nt = blockDim.x;
    const int per = (n + nt - 1) / nt;
    const int lo = min(n, tid * per), hi = min(n, lo + per);
    uint32_t s = 0;
    for (int i = lo; i < hi; ++i) s += a[i];
    // warp inclusive scan of s
    const int lane = tid & 31, w = tid >> 5;
    uint32_t x = s;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        uint32_t y = __shfl_up_sync(0xffffffffu, x, o);
        if (lane >= o) x += y;
    }
    if (lane == 31) tmp[w] = x;
    __syncthreads();
    if (w == 0) {
        const int nw = (nt + 31) >> 5;
        uint32_t v = lane < nw ? tmp[lane] : 0;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            uint32_t y = __shfl_up_sync(0xffffffffu, v, o);
            if (lane >= o) v += y;
        }
        if (lane < nw) tmp[lane] = v;  // inclusive per-warp totals
        if (lane == 31) tmp[32] = v;
    }
    __syncthreads();
    uint32_t run = x - s + (w > 0 ? tmp[w - 1] : 0);
    for (int i = lo; i < hi; ++i) {
        uint32_t v = a[i];
        a[i] = run;
        run += v;
    }
    uint32_t total = tmp[32];
    __syncthreads();
    return total;
}

// Same for u64 (plan kernel).
__device__ inline uint64_t block_excl_scan_u64(uint64_t *a, int n, uint64_t *tmp) {
    const int tid = threadIdx.x, nt = blockDim.x;
    const int per = (n + nt - 1) / nt;
    const int lo = min(n, tid * per), hi = min(n, lo + per);
    uint64_t s = 0;
    for (int i = lo; i < hi; ++i) s += a[i];
    const int lane = tid & 31, w = tid >> 5;
    uint64_t x = s;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        uint64_t y = __shfl_up_sync(0xffffffffu, x, o);
        if (lane >= o) x += y;
    }
    if (lane == 31) tmp[w] = x;
    __syncthreads();
    if (w == 0) {
        const int nw = (nt + 31) >> 5;
        uint64_t v = lane < nw ? tmp[lane] : 0;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            uint64_t y = __shfl_up_sync(0xffffffffu, v, o);
            if (lane >= o) v += y;
        }
        if (lane < nw) tmp[lane] = v;
        if (lane == 31) tmp[32] = v;
    }
    __syncthreads();
    uint64_t run = x - s + (w > 0 ? tmp[w - 1] : 0);
    for (int i = lo; i < hi; ++i) {
        uint64_t v = a[i];
        a[i] = run;
        run += v;
    }
    uint64_t total = tmp[32];
    __syncthreads();
    return total;
}

}  // namespace mgj
