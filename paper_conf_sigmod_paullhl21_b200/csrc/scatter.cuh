// scatter.cuh — phase a3: global partitioning step 1 + data distribution,
// fused: every tuple is written straight into its owner's receive buffer.
#pragma once

#include "common.cuh"
#include "tma.cuh"

namespace mgj {

// Scatter geometry for P partitions and a key width (kernel template
// arguments; the host picks the instance with scatter_kernel<K>(P)):
//   T   = sub-tile (tuples) staged in shared memory per step,
//   SG  = tuples per 32-byte sector group (the unit of a global store),
//   PPT = partitions owned by each of the 1024 threads (registers).
// With SG > 1 every partition's output leaves in whole 32-byte sectors: the
// < 32-byte tail of a partition waits (in registers of its owning thread)
// for the next sub-tile.  For P = 4096 the alignment padding would not fit
// shared memory, so SG = 1 (one tuple per store).
// (Measured alternatives, round 1, not kept: 4096-tuple sub-tiles in two
// 512-thread CTAs per SM with 16- or 32-byte groups, 9.2 / 6.2 ms; SoA
// staging with 4-byte random stores, 4.42 ms; register-staged sub-tiles
// without TMA, 4.73 ms; a per-group destination table, 4.36 ms; against
// 4.16 ms for this design at M2.)
struct ScatGeom {
    int T, SG, PPT, NT;
    int NH;  // key-stage pieces: the sub-tile's keys arrive in NH pieces through one stage of T / NH keys
             // (P <= 1024, 4-byte keys: 16384-tuple sub-tiles whose keys come in two halves; measured at
             // M2 against 12288 tuples with one key stage: scatter 3.79 -> 3.73 ms, k_hist, which counts
             // them in two 8192-key blocks, 0.73 -> 0.74 ms, step 9.34 -> 9.29 ms)
};
__host__ __device__ constexpr ScatGeom scat_geom(int P, int key_bytes) {
    return key_bytes == 4
               ? (P <= 1024 ? ScatGeom{16384, 4, 1, 1024, 2}
                  : P == 2048 ? ScatGeom{4096, 4, 2, 1024, 1} : ScatGeom{8192, 1, 4, 1024, 1})
               : (P <= 1024 ? ScatGeom{6144, 2, 1, 1024, 1} : P == 2048 ? ScatGeom{2048, 2, 2, 1024, 1}
                                                                         : ScatGeom{4096, 1, 4, 1024, 1});
}

// Per-partition write-out descriptor of the current sub-tile (8 bytes, one
// shared load per sector group): the destination tuple index of sorted slot
// 0 in the owner's receive buffer (modulo 2^32: slot s goes to didx + s), the
// end of the partition's valid slots, and the head group, if any, whose first
// h slots are not the partition's ((slot / SG) << 2 | h; 0xffff: none).  The
// owner's receive buffer comes from two small per-kernel tables (destination
// rank of each partition, base of each rank's receive buffer).
struct __align__(8) PInfo {
    uint32_t didx;
    uint16_t lim;
    uint16_t head;
};
constexpr uint16_t PI_NONE = 0xffff;

__host__ __device__ inline size_t scat_smem_bytes(int P, int key_bytes) {
    const ScatGeom g = scat_geom(P, key_bytes);
    const size_t TB = 2 * (size_t)key_bytes;
    return (size_t)g.T / g.NH * key_bytes                      // input stage: keys (payloads: L2 prefetch + loads)
           + ((size_t)g.T + 2 * (size_t)(g.SG - 1) * P) * TB  // partition-sorted sub-tile (+ carries, group padding)
           + (size_t)P * sizeof(PInfo)                         // write-out descriptors
           + (size_t)P * 4                                     // next free slot per partition
           + 2 * (size_t)MAX_RANKS * 8                         // receive-buffer base per (relation, rank)
           + 2 * (size_t)P;                                    // destination rank per (relation, partition)
}

// Block-wide exclusive scan of one register value per thread (<= 1024 threads).
__device__ __forceinline__ uint32_t block_scan_reg(uint32_t v, uint32_t *tmp, uint32_t &total) {
    const int tid = threadIdx.x, lane = tid & 31, w = tid >> 5;
    uint32_t x = v;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const uint32_t y = __shfl_up_sync(0xffffffffu, x, o);
        if (lane >= o) x += y;
    }
    if (lane == 31) tmp[w] = x;
    __syncthreads();
    if (w == 0) {
        uint32_t s = lane < (int)(blockDim.x >> 5) ? tmp[lane] : 0u;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const uint32_t y = __shfl_up_sync(0xffffffffu, s, o);
            if (lane >= o) s += y;
        }
        tmp[lane] = s;  // inclusive warp totals
    }
    __syncthreads();
    total = tmp[31];
    return x - v + (w ? tmp[w - 1] : 0);
}

// 16-byte shared load that the compiler keeps where it is written (not sunk
// into the branch that consumes it): the write-out issues its group and
// descriptor loads back to back.
__device__ __forceinline__ uint4 lds128(const void *p) {
    uint4 v;
    asm volatile("ld.volatile.shared.v4.u32 {%0,%1,%2,%3}, [%4];"
                 : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w)
                 : "r"(smem_u32(p)));
    return v;
}

// Shared-memory accesses on precomputed 32-bit shared addresses: with plain
// pointers the compiler re-derived the shared window base (S2R SR_CgaCtaId)
// inside the write-out loop, 6% of the kernel's stall samples (ncu, round 2).
__device__ __forceinline__ uint4 lds128_at(uint32_t a) {
    uint4 v;
    asm volatile("ld.shared.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "r"(a));
    return v;
}
__device__ __forceinline__ uint2 lds64_at(uint32_t a) {
    uint2 v;
    asm volatile("ld.shared.v2.u32 {%0,%1}, [%2];" : "=r"(v.x), "=r"(v.y) : "r"(a));
    return v;
}
__device__ __forceinline__ void sts_at(uint32_t a, const uint2 &v) {
    asm volatile("st.shared.v2.u32 [%0], {%1,%2};" ::"r"(a), "r"(v.x), "r"(v.y) : "memory");
}
__device__ __forceinline__ void sts_at(uint32_t a, const ulonglong2 &v) {
    asm volatile("st.shared.v2.u64 [%0], {%1,%2};" ::"r"(a), "l"(v.x), "l"(v.y) : "memory");
}
template <typename Tup> __device__ __forceinline__ Tup lds_tup(uint32_t a);
template <> __device__ __forceinline__ uint2 lds_tup<uint2>(uint32_t a) { return lds64_at(a); }
template <> __device__ __forceinline__ ulonglong2 lds_tup<ulonglong2>(uint32_t a) {
    ulonglong2 v;
    asm volatile("ld.shared.v2.u64 {%0,%1}, [%2];" : "=l"(v.x), "=l"(v.y) : "r"(a));
    return v;
}

template <int BYTES> struct Vec;
template <> struct Vec<8> { using T = uint2; };
template <> struct Vec<16> { using T = uint4; };
template <> struct Vec<32> { struct __align__(32) T { uint4 a, b; }; };

// One global store of a 8/16/32-byte group (32 bytes: a single 256-bit store).
template <int BYTES>
__device__ __forceinline__ void st_group(void *dst, const typename Vec<BYTES>::T &v) {
    if constexpr (BYTES == 32) {
        // L1::no_allocate: the scattered sectors are never read back here
        // (measured at M2: scatter 3.85 -> 3.80 ms; .cs streaming stores: no change)
        asm volatile("st.global.L1::no_allocate.v8.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8};" ::"l"(dst), "r"(v.a.x),
                     "r"(v.a.y), "r"(v.a.z), "r"(v.a.w), "r"(v.b.x), "r"(v.b.y), "r"(v.b.z), "r"(v.b.w)
                     : "memory");
    } else {
        *static_cast<typename Vec<BYTES>::T *>(dst) = v;
    }
}

// ---------------------------------------------------------------------------
// a3 (§3.2 "Global partitioning phase" step 1, P:408-416 — "each
// thread ... reads a unique input tuple, determines the index for the tuple
// after partitioning based on the histogram and then writes the tuple" —
// after Rui et al. [38]; step 3 data distribution, P:405-407 and §4).
//
// B200 form: one launch per relation (rel); persistent CTAs (1024 threads,
// one per SM) take tiles c = blockIdx.x, + gridDim.x, ... of that relation
// (one tile per CTA at full grid; fewer CTAs when the launch shares the GPU
// with the local pass of the other relation, §8(e) overlap) and stream each
// tile in sub-tiles of T tuples whose keys a TMA bulk copy brings into shared
// memory ahead of their use (NH = 2: in two halves through one stage, half 1
// arriving while half 0 is ranked; payloads: L2 prefetch, then registers).
// Per sub-tile:
//  1. thread t owns partitions t*PPT.. (PPT per thread) and keeps, in
//     registers, each one's destination cursor and its < 32-byte tail
//     (carry) from the previous sub-tile; a block scan of the per-partition
//     sizes (carry + new, rounded up to a 32-byte group; a1 counted them)
//     lays the partitions out group-aligned in `sorted`, the carry first;
//  2. each thread ranks its tuples in their digit1 bins (one shared atomic
//     each) and scatters them into `sorted`;
//  3. the sorted sub-tile is written out one 32-byte group per thread and
//     store (st.global.v8.b32): every complete group is a whole DRAM sector
//     at its final address — owner(p)'s receive buffer at send_off[p] (a2) +
//     tile_base[c][p] (a1 tile prefix) + the running count of p in this tile;
//     no global atomics.  An incomplete last group stays in `sorted` and its
//     owning thread reloads it as the next carry.
// A tile's first destination of a partition need not be group-aligned: the
// carry then starts with h placeholder slots (key = p) that are never stored
// (the head group is written tuple by tuple from slot h).  A tile's remaining
// tails are written tuple by tuple at its end.  On NVSwitch the owner may be
// another GPU: the same stores go over NVLink to a peer-mapped address; the
// paper's packets, routing buffers and multi-hop routing (§4) have no role on
// a one-hop fabric.  With N > 1 each CTA starts its write-out sweep at a
// different destination rank (rotated group order), so that the CTAs' stores
// spread over all peers' links instead of visiting the ranks in step.  The
// last CTA raises SIG_DATA_R / SIG_DATA_S at every peer after a system fence.
// ---------------------------------------------------------------------------
template <typename K, int T, int SG, int PPT, int NT, bool COMP = false, int NH = 1>
__global__ void __launch_bounds__(NT, 1) k_scatter(Ctx c, int rel0, int rel1) {
    using Tup = typename TupT<K>::T;
    constexpr int TB = (int)sizeof(Tup);
    constexpr int V = T / NT;                  // tuples per thread per sub-tile
    constexpr int LU = 16 / (int)sizeof(K);    // tuples per 16-byte stage vector
    constexpr int NU = V / LU;                 // vectors per thread
    static_assert(NU * LU == V && NU >= 1, "sub-tile");
    // NH = 2: the keys arrive in two halves of TH through a stage of TH keys (the
    // shared memory of a full key stage goes to the larger sorted sub-tile);
    // half h of the sub-tile is ranked while half h + 1 is loaded
    constexpr int TH = T / NH, VH = V / NH, NUH = NU / NH;
    static_assert(NH == 1 || (NH == 2 && !COMP && NUH * NH == NU && NUH >= 1), "key-stage halves");
    // COMP (NEXT-1): a group is one 32-byte unit of SG = CU_N encoded tuples
    static_assert(!COMP || (SG == CU_N && sizeof(K) == 4 && PPT == 1), "compressed scatter");
    constexpr int GB = COMP ? 32 : SG * TB;    // group bytes at the destination
    constexpr int CW = SG > 1 ? SG - 1 : 1;    // carry capacity (tuples)
    using GV = typename Vec<COMP ? 32 : SG * TB>::T;
    typedef unsigned long long ull;
    // `sorted` swizzle: the two 16-byte halves of every 32-byte group whose
    // index has bit 2 set are swapped, so that the write-out's 16-byte loads
    // (8 consecutive groups per quarter warp) hit distinct banks
    auto swz = [](uint32_t s) -> uint32_t {
        if constexpr (!COMP && SG > 1 && SG * sizeof(Tup) == 32) return s ^ (((s >> (SG == 4 ? 4 : 3)) & 1u) * (SG / 2));
        else return s;
    };
    extern __shared__ __align__(128) unsigned char smem[];
    const int P = c.P;
    K *const skey = reinterpret_cast<K *>(smem);  // stage: the sub-tile's keys
    Tup *const sorted = reinterpret_cast<Tup *>(smem + TH * sizeof(K));
    PInfo *const pinfo = reinterpret_cast<PInfo *>(sorted + T + 2 * (SG - 1) * P);  // 8-byte aligned
    uint32_t *const off = reinterpret_cast<uint32_t *>(pinfo + P);  // next free slot per partition
    unsigned long long *const obase = reinterpret_cast<unsigned long long *>(off + P);  // [2][MAX_RANKS]
    uint8_t *const own8 = reinterpret_cast<uint8_t *>(obase + 2 * MAX_RANKS);            // [2][P]
    // shared addresses pinned in registers for 4-byte keys (smem_pin; measured at M2:
    // scatter 3.795 -> 3.780 ms; the 8-byte-key instance would spill)
    auto pin = [](const void *p) -> uint32_t {
        if constexpr (sizeof(K) == 4) return smem_pin(p);
        else return smem_u32(p);
    };
    const uint32_t sorted_s = pin(sorted), pinfo_s = pin(pinfo);
    const uint32_t obase_s = pin(obase), own8_s = pin(own8);
    // receive-buffer base of partition pidx's owner (N > 1), from the two tables
    auto owner_base = [&](int rel, uint32_t pidx) -> unsigned long long {
        if constexpr (sizeof(K) != 4) return obase[rel * MAX_RANKS + own8[rel * P + pidx]];
        uint32_t o8, lo, hi;
        asm volatile("ld.shared.u8 %0, [%1];" : "=r"(o8) : "r"(own8_s + (uint32_t)rel * (uint32_t)P + pidx));
        asm volatile("ld.shared.v2.u32 {%0,%1}, [%2];" : "=r"(lo), "=r"(hi) : "r"(obase_s + ((uint32_t)rel * MAX_RANKS + o8) * 8u));
        return (unsigned long long)hi << 32 | lo;
    };
    auto saddr = [&](uint32_t x) -> uint32_t { return sorted_s + swz(x) * (uint32_t)TB; };
    auto sput = [&](uint32_t x, const Tup &t) { sts_at(saddr(x), t); };
    auto sget = [&](uint32_t x) -> Tup { return lds_tup<Tup>(saddr(x)); };
    __shared__ __align__(8) uint64_t bar;
    __shared__ uint32_t tmp[32];
    const int tid = threadIdx.x;
    const int ok = *(volatile int32_t *)&c.meta[MT_OK];

    for (int rel = rel0; rel <= rel1; ++rel) trace_begin(c, rel ? MGJ_TR_SCATTER_S : MGJ_TR_SCATTER_R);
    if (tid == 0) {
        mbar_init(&bar, 1);
        fence_mbar_init();
    }
    __syncthreads();
    const uint64_t pol = policy_evict_first();

    // This CTA's sub-tiles: tiles blockIdx.x + k * gridDim.x, each cut into
    // sub-tiles of T tuples.  A cursor (k, j) walks them in order.
    // This CTA's sub-tiles: for rel = rel0..rel1, tiles blockIdx.x + k *
    // gridDim.x of the relation, each cut into sub-tiles of T tuples.  A
    // cursor walks them in order (across the relation boundary, so the next
    // sub-tile is always prefetched).
    struct Cur {
        int rel, tile;
        uint32_t j, nsub;
        uint64_t lo, hi;  // the tile's tuple range (computed once per tile: 64-bit divisions)
    };
    auto at_tile = [&](int rel, int tile) -> Cur {  // first non-empty tile from (rel, tile) on
        Cur u{rel, tile, 0, 0, 0, 0};
        for (; u.rel <= rel1; ++u.rel, u.tile = (int)blockIdx.x) {
            const uint64_t n = ok ? c.n_in[u.rel] : 0;
            for (; u.tile < c.G; u.tile += gridDim.x) {
                tile_range(n, c.G, u.tile, u.lo, u.hi);
                u.nsub = (uint32_t)((u.hi - u.lo + T - 1) / T);
                if (u.nsub) return u;
            }
        }
        return u;  // u.rel > rel1: done
    };
    auto next_cur = [&](Cur u) -> Cur {
        if (u.j + 1 < u.nsub) {
            ++u.j;
            return u;
        }
        return at_tile(u.rel, u.tile + gridDim.x);
    };
    auto span = [&](const Cur &u, uint64_t &first, uint32_t &len) {
        first = u.lo + (uint64_t)u.j * T;
        len = (uint32_t)min((uint64_t)T, u.hi - first);
    };

    // per owned partition (registers): destination of the next group, carry
    uint32_t bidx[PPT];  // destination tuple index of the next group (owner's receive buffer, mod 2^32)
    uint8_t dstr[PPT];   // destination rank
    uint32_t cc[PPT], hd[PPT], lim[PPT];
    bool skp[PPT];  // partition skipped by the plan (an empty side): nothing is stored
    Tup carry[PPT][CW];
    bool pending = false;  // carries of the last sub-tile still sit in `sorted`
#pragma unroll
    for (int k = 0; k < PPT; ++k) bidx[k] = 0, dstr[k] = 0, cc[k] = 0, hd[k] = 0, lim[k] = 0, skp[k] = false;
    // per-kernel tables for the write-out: receive-buffer base of every (relation, rank) and the
    // destination rank of every (relation, partition) (read after the first layout barrier)
    if (tid < 2 * MAX_RANKS)
        obase[tid] = (tid % MAX_RANKS) < c.world ? (ull)(c.arena[tid % MAX_RANKS] + c.lay.recv[tid / MAX_RANKS]) : 0ull;
    for (int p = tid; p < P; p += NT) {
        own8[p] = (uint8_t)c.owner[p];
        own8[P + p] = (uint8_t)(c.bcast[p] ? c.rank : c.owner[p]);  // S of a broadcast partition stays here
    }

    // keys of half h of sub-tile u: [h * TH, h * TH + hlen)
    auto half_len = [&](uint32_t len, int h) -> uint32_t {
        return len > (uint32_t)(h * TH) ? min(len - (uint32_t)(h * TH), (uint32_t)TH) : 0u;
    };
    auto issue = [&](const Cur &u, int h) {  // thread 0: TMA the 16-byte-aligned body of half h of sub-tile u's keys
        uint64_t first;
        uint32_t len;
        span(u, first, len);
        const K *in_key = static_cast<const K *>(c.in_key[u.rel]);
        const K *in_pay = static_cast<const K *>(c.in_pay[u.rel]);
        const uint32_t kbytes = (half_len(len, h) & ~(uint32_t)(LU - 1)) * (uint32_t)sizeof(K);
        const uint32_t bytes = (len & ~(uint32_t)(LU - 1)) * (uint32_t)sizeof(K);
        mbar_arrive_expect_tx(&bar, kbytes);
        if (kbytes) tma_load_1d(skey, in_key + first + h * TH, kbytes, &bar, pol);
        if (h == 0 && bytes) {
            // payloads: brought into L2 now and loaded into registers while the
            // previous sub-tile is written out (the shared memory of a payload
            // stage goes to a 1.5x larger sub-tile instead; measured at M2:
            // scatter 4.12 -> 3.89 ms; without the L2 prefetch 4.65 ms)
            prefetch_l2(in_pay + first, bytes);
        }
    };
    // COMP: global row id of the rank's first row, a tile's first local row, and one entry
    auto cbase_rel = [&](int rel) -> uint32_t { return COMP ? __ldg(c.rowbase + ((size_t)rel * MAX_RANKS + c.rank) * c.G) : 0u; };
    auto tile_lo_of = [&](int rel, int tile) -> uint64_t {
        uint64_t lo, hi;
        tile_range(c.n_in[rel], c.G, tile, lo, hi);
        return lo;
    };
    const int kb = 32 - c.B1;  // key bits above the partition digit
    auto unit_enc = [&](uint32_t key, uint32_t pay, uint32_t tilebase) -> unsigned long long {
        return (unsigned long long)(key >> c.B1) | ((unsigned long long)(pay - tilebase) << kb);
    };
    bool bad_pay = false;  // COMP: a payload that is not its global row id
    auto fetch_carry = [&]() {  // the incomplete last groups of the previous sub-tile -> registers
        if (pending) {
#pragma unroll
            for (int k = 0; k < PPT; ++k)
#pragma unroll
                for (int i = 0; i < CW; ++i)
                    if (i < (int)cc[k]) carry[k][i] = sget(lim[k] - cc[k] + i);
            pending = false;
        }
    };
    auto flush = [&](int rel, int tile) {  // end of a tile: store the remaining tails
        fetch_carry();
        if constexpr (COMP) {  // one partial unit of cc entries
            if (!skp[0] && cc[0]) {
                unsigned long long e[CU_N], a[4];
                const uint32_t tb0 = cbase_rel(rel) + (uint32_t)tile_lo_of(rel, tile);
#pragma unroll
                for (int i = 0; i < CU_N; ++i)
                    e[i] = i < (int)cc[0] ? unit_enc((uint32_t)carry[0][i < CW ? i : 0].x, (uint32_t)carry[0][i < CW ? i : 0].y, tb0) : 0ull;
                unit_pack(e, cc[0] | (uint32_t)c.rank << 3 | (uint32_t)tile << 6, a);
                char *d = c.arena[dstr[0]] + c.lay.recv[rel] + (size_t)bidx[0] * 32;
                asm volatile("st.global.L1::no_allocate.v4.u64 [%0], {%1,%2,%3,%4};" ::"l"(d), "l"(a[0]), "l"(a[1]), "l"(a[2]), "l"(a[3]) : "memory");
            }
        } else {
#pragma unroll
            for (int k = 0; k < PPT; ++k)
#pragma unroll
                for (int i = 0; i < CW; ++i)
                    if (!skp[k] && i >= (int)hd[k] && i < (int)cc[k]) {
                        Tup *d = reinterpret_cast<Tup *>(c.arena[dstr[k]] + c.lay.recv[rel]);
                        d[(uint32_t)(bidx[k] + i)] = carry[k][i];
                    }
        }
    };
    auto set_base = [&](int rel, int tile) {  // destination of this tile's first tuple of each owned partition
        const uint32_t *tb = c.tile_base + ((size_t)rel * c.G + tile) * P;
        const uint64_t *so = c.send_off + (size_t)rel * P;
#pragma unroll
        for (int k = 0; k < PPT; ++k) {
            const int p = tid * PPT + k;
            cc[k] = hd[k] = 0;
            if (p < P) {
                // destination: the owner, or this rank itself for the S side of a
                // selectively broadcast partition (a2, NEXT-2)
                const int dst = (rel && c.bcast[p]) ? c.rank : c.owner[p];
                skp[k] = c.pskip[p] != 0;
                const uint64_t idx = so[p] + tb[p];  // COMP: in 32-byte units (runs start unit-aligned)
                const ull a = (ull)(c.arena[dst] + c.lay.recv[rel]) + idx * (uint64_t)TB;
                const uint32_t h = (SG > 1 && !COMP) ? (uint32_t)((a & (GB - 1)) / TB) : 0u;
                bidx[k] = (uint32_t)idx - h;  // may wrap below 0: placeholders are never stored
                dstr[k] = (uint8_t)dst;
                cc[k] = hd[k] = h;
#pragma unroll
                for (int i = 0; i < CW; ++i) {  // placeholders: digit1 = p, never stored
                    carry[k][i].x = (K)p;
                    carry[k][i].y = 0;
                }
            }
        }
    };

    // counts of sub-tile u for this thread's partitions (a1 wrote them, u16 per partition)
    auto load_counts = [&](const Cur &u, uint32_t (&out)[PPT]) {
#pragma unroll
        for (int k = 0; k < PPT; ++k) out[k] = 0;
        if (u.rel > rel1 || tid * PPT >= P) return;
        const uint16_t *src = c.sub_hist + (((size_t)u.rel * c.G + u.tile) * c.sub_ns + u.j) * P + tid * PPT;
        if constexpr (PPT == 1) {
            out[0] = __ldg(src);
        } else if constexpr (PPT == 2) {
            const uint32_t v = __ldg(reinterpret_cast<const uint32_t *>(src));
            out[0] = v & 0xffffu, out[1] = v >> 16;
        } else {
            const uint2 v = __ldg(reinterpret_cast<const uint2 *>(src));
            out[0] = v.x & 0xffffu, out[1] = v.x >> 16, out[2] = v.y & 0xffffu, out[3] = v.y >> 16;
        }
    };
    // payloads of sub-tile u (L2-resident since issue(u)), loaded into
    // registers while the previous sub-tile is written out
    // (half h = the vectors [h * NUH, (h + 1) * NUH) of every thread)
    K pp[V];
    auto load_pay = [&](const Cur &u, int h) {
        uint64_t first;
        uint32_t len;
        span(u, first, len);
        const K *gp = static_cast<const K *>(c.in_pay[u.rel]) + first;
        if (len == T) {
#pragma unroll
            for (int x = 0; x < NU; ++x) {
                if (x / NUH != h) continue;
                const uint4 b = __ldcs(reinterpret_cast<const uint4 *>(gp + (uint32_t)(x * NT + tid) * LU));
                memcpy(&pp[x * LU], &b, 16);
            }
        } else {
#pragma unroll
            for (int x = 0; x < NU; ++x) {
                if (x / NUH != h) continue;
#pragma unroll
                for (int e = 0; e < LU; ++e) {
                    const uint32_t i = (uint32_t)(x * NT + tid) * LU + e;
                    pp[x * LU + e] = i < len ? __ldcs(gp + i) : (K)0;
                }
            }
        }
    };
    // write-out rotation (N > 1): CTA b starts its sweep of the groups at rank
    // b mod N's share of them (owner ranges are contiguous in p, so in group order)
    const uint32_t rot_num = c.world > 1 ? (uint32_t)(blockIdx.x % c.world) : 0u;

    // NEXT-3 chunk streaming (S launch): every completed S tile counts once in
    // its round's counter in this rank's arena (after a system fence by every
    // thread that stored its tuples; one atomic by thread 0), which owners
    // poll before they start the local pass of a chunk the round fills.
    // (The condition is re-read from the parameters and the tile to count
    // kept in shared memory: more registers in the sub-tile loop spill.)
#define MGJ_SCAT_STRM (c.stream && rel0 == 1)
    auto sig_round = [&](int tile) {  // thread 0, after a system fence
        atomicAdd_system(rdone_ptr(c.arena[c.rank], c.lay, tile / c.sgrid), 1ull);
    };
    __shared__ int done_tile;  // an S tile whose stores are fenced, counted after the next barrier
    if (tid == 0) done_tile = -1;

    Cur u = at_tile(rel0, (int)blockIdx.x);
    uint32_t ncnt[PPT];
    load_counts(u, ncnt);
    if (u.rel <= rel1) {
        if (tid == 0) issue(u, 0);
        load_pay(u, 0);
    }
    int cur_tile = -1;       // (relation, tile) the partition state belongs to: rel * G + tile
    uint32_t nsub_done = 0;  // sub-tiles processed (the stage barrier's phase parity)
    for (; u.rel <= rel1; u = next_cur(u), ++nsub_done) {
        uint64_t first;
        uint32_t len;
        span(u, first, len);
        const Cur nx = next_cur(u);
        const uint32_t row0 = cbase_rel(u.rel);  // COMP: global row id of this rank's first row
        if (u.rel * c.G + u.tile != cur_tile) {  // thread-private partition state: no barrier needed
            if (cur_tile >= 0) {
                flush(cur_tile / c.G, cur_tile % c.G);
                if (MGJ_SCAT_STRM && cur_tile >= c.G) {
                    __threadfence_system();
                    if (tid == 0) done_tile = cur_tile - c.G;
                }
            }
            set_base(u.rel, u.tile);
            cur_tile = u.rel * c.G + u.tile;
        }
        fetch_carry();
        // lay out this sub-tile's partitions (known from a1): carry + new tuples, group-rounded
        uint32_t cnt[PPT], seg[PPT], tsum = 0;
#pragma unroll
        for (int k = 0; k < PPT; ++k) {
            cnt[k] = cc[k] + ncnt[k];
            seg[k] = COMP ? (cnt[k] + SG - 1) / SG * SG : (cnt[k] + SG - 1) & ~(uint32_t)(SG - 1);
            tsum += seg[k];
        }
        load_counts(nx, ncnt);  // prefetch (consumed next iteration)
        uint32_t total;
        uint32_t o = block_scan_reg(tsum, tmp, total);  // its barriers: the last write-out is done
        if (MGJ_SCAT_STRM && tid == 0 && done_tile >= 0) {  // every thread has fenced the tile's stores
            __threadfence_system();
            sig_round(done_tile);
            done_tile = -1;
        }
#pragma unroll
        for (int k = 0; k < PPT; ++k) {
            const int p = tid * PPT + k;
            if (p < P) {
#pragma unroll
                for (int i = 0; i < CW; ++i)
                    if (i < (int)cc[k]) sput(o + i, carry[k][i]);
                off[p] = o + cc[k];
                const uint32_t full = COMP ? cnt[k] / SG * SG : cnt[k] & ~(uint32_t)(SG - 1);
                PInfo in;
                in.didx = COMP ? bidx[k] - o / SG : bidx[k] - o;  // COMP: units
                in.lim = (uint16_t)(skp[k] ? o : o + cnt[k]);  // a skipped partition's groups are never stored
                in.head = (hd[k] && full) ? (uint16_t)((o / SG) << 2 | hd[k]) : PI_NONE;
                pinfo[p] = in;
                bidx[k] += COMP ? full / SG : full;
                if (full) hd[k] = 0;
                cc[k] = cnt[k] - full;
                lim[k] = o + cnt[k];
            }
            o += seg[k];
        }
        pending = SG > 1;
        K kk[V];
        const K *gk = static_cast<const K *>(c.in_key[u.rel]) + first;
#pragma unroll
        for (int h = 0; h < NH; ++h) {  // (NH = 2: half 0 ranked while half 1 arrives)
            mbar_wait(&bar, NH == 1 ? (nsub_done & 1) : (uint32_t)h);
            const uint32_t hl = half_len(len, h), body = hl & ~(uint32_t)(LU - 1);
            if (hl == (uint32_t)TH) {  // full half: branch-free vector loads
#pragma unroll
                for (int x = 0; x < NU; ++x) {
                    if (x / NUH != h) continue;
                    const uint4 a = *reinterpret_cast<const uint4 *>(skey + (uint32_t)((x - h * NUH) * NT + tid) * LU);
                    memcpy(&kk[x * LU], &a, 16);
                }
            } else {
#pragma unroll
                for (int x = 0; x < NU; ++x) {
                    if (x / NUH != h) continue;
#pragma unroll
                    for (int e = 0; e < LU; ++e) {  // < LU trailing tuples of the relation come from global
                        const uint32_t i = (uint32_t)((x - h * NUH) * NT + tid) * LU + e;  // index in the half
                        kk[x * LU + e] = i < body ? skey[i] : (i < hl ? gk[h * TH + i] : (K)0);
                    }
                }
            }
            __syncthreads();  // S1 (half 0: offsets and carries in place too): stage consumed
            if (tid == 0) {
                if (h + 1 < NH) issue(u, h + 1);
                else if (nx.rel <= rel1) issue(nx, 0);
            }
            if (h + 1 < NH) load_pay(u, h + 1);  // (in L2 since the sub-tile's first issue)
#pragma unroll
            for (int v = 0; v < V; ++v) {
                if (v / VH != h) continue;
                const uint32_t i = (uint32_t)((v / LU) * NT + tid) * LU + (v % LU);
                if (i < len) {
                    Tup t;
                    t.x = kk[v];
                    t.y = pp[v];
                    if constexpr (COMP) bad_pay |= (uint32_t)pp[v] != row0 + (uint32_t)(first + i);
                    sput(atomicAdd(&off[digit1(kk[v], P)], 1u), t);
                }
            }
        }
        __syncthreads();  // S2
        if (nx.rel <= rel1) load_pay(nx, 0);  // the ranking of this sub-tile has consumed pp
        // write-out: one group per thread per step, rotated by rank share for N > 1
        const uint32_t ngroups = total / SG;
        const ull ob_rel = (ull)(c.arena[0] + c.lay.recv[u.rel]);  // N = 1: the one receive buffer
        const uint32_t tbase = row0 + (uint32_t)u.lo;  // COMP: global row id of this tile's first row
        const uint32_t rot = c.world > 1 ? (uint32_t)(((uint64_t)ngroups * rot_num) / (uint32_t)c.world) : 0u;
        for (uint32_t w = tid; w < ngroups; w += NT) {
            const uint32_t gi = w + rot < ngroups ? w + rot : w + rot - ngroups;
            const uint32_t slot = gi * SG;
            if constexpr (COMP) {
                Tup tt[CU_N];
#pragma unroll
                for (int e = 0; e < CU_N; ++e) tt[e] = sget(slot + e);
                const uint32_t pidx = (uint32_t)tt[0].x & (uint32_t)(P - 1);
                const uint2 pv = lds64_at(pinfo_s + pidx * 8u);
                if (slot + SG <= (pv.y & 0xffffu)) {
                    const ull ob = c.world == 1 ? ob_rel : owner_base(u.rel, pidx);
                    unsigned long long e[CU_N], a[4];
#pragma unroll
                    for (int x = 0; x < CU_N; ++x) e[x] = unit_enc((uint32_t)tt[x].x, (uint32_t)tt[x].y, tbase);
                    unit_pack(e, (uint32_t)CU_N | (uint32_t)c.rank << 3 | (uint32_t)u.tile << 6, a);
                    char *dst = reinterpret_cast<char *>(ob + (ull)(uint32_t)(pv.x + slot / SG) * 32);
                    asm volatile("st.global.L1::no_allocate.v4.u64 [%0], {%1,%2,%3,%4};" ::"l"(dst), "l"(a[0]), "l"(a[1]), "l"(a[2]),
                                 "l"(a[3])
                                 : "memory");
                }
                continue;
            }
            GV gv;
            if constexpr (GB == 32) {  // two conflict-free 16-byte halves (swizzled)
                gv.a = lds128_at(saddr(slot));
                gv.b = lds128_at(saddr(slot + SG / 2));
            } else if constexpr (GB == 16) {
                gv = lds128_at(saddr(slot));
            } else {
                gv = lds64_at(saddr(slot));
            }
            const uint32_t pidx = reinterpret_cast<const uint32_t *>(&gv)[0] & (uint32_t)(P - 1);
            const uint2 pv = lds64_at(pinfo_s + pidx * 8u);
            const uint32_t plim = pv.y & 0xffffu, phead = pv.y >> 16;
            if (slot + SG <= plim) {
                const ull ob = c.world == 1 ? ob_rel : owner_base(u.rel, pidx);
                char *dst = reinterpret_cast<char *>(ob + (ull)(uint32_t)(pv.x + slot) * TB);
                if (phead == PI_NONE || (phead >> 2) * SG != slot) {
                    st_group<GB>(dst, gv);
                } else {
                    for (uint32_t i = phead & 3u; i < SG; ++i) reinterpret_cast<Tup *>(dst)[i] = sget(slot + i);
                }
            }
        }
    }
    if (cur_tile >= 0) flush(cur_tile / c.G, cur_tile % c.G);
    if (COMP && bad_pay) set_err(c, MGJ_EINVAL);

    // ---- every CTA: make its (peer) stores visible, the last one signals ----
    __threadfence_system();
    __syncthreads();
    for (int rel = rel0; rel <= rel1; ++rel) trace_end(c, rel ? MGJ_TR_SCATTER_S : MGJ_TR_SCATTER_R);
    if (tid == 0) {
        if (MGJ_SCAT_STRM && cur_tile >= c.G) sig_round(cur_tile - c.G);  // the last S tile (fenced above)
        const uint32_t t = atomicAdd(&c.ticket[rel0 ? TK_SCAT_S : TK_SCAT_R], 1u);
        if (t == gridDim.x - 1) {
            __threadfence_system();
            for (int rel = rel0; rel <= rel1; ++rel) signal_all(c, rel ? SIG_DATA_S : SIG_DATA_R);
        }
    }
}

#undef MGJ_SCAT_STRM

// The compressed-shuffle instance (NEXT-1): 4-byte keys, P <= 1024.
// (12288-tuple sub-tiles like the uncompressed instance, measured at M2:
// scatter 4.94 vs 5.36 ms with 8192, in spite of a 92-byte spill)
constexpr ScatGeom scat_geom_comp() { return ScatGeom{12288, CU_N, 1, 1024, 1}; }
inline size_t scat_smem_bytes_comp(int P) {
    const ScatGeom g = scat_geom_comp();
    return (size_t)g.T * 4 + ((size_t)g.T + 2 * (size_t)(g.SG - 1) * P) * 8 + (size_t)P * sizeof(PInfo) +
           (size_t)P * 4 + 2 * (size_t)MAX_RANKS * 8 + 2 * (size_t)P;
}
inline void (*scatter_kernel_comp())(Ctx, int, int) {
    constexpr ScatGeom g = scat_geom_comp();
    return k_scatter<uint32_t, g.T, g.SG, g.PPT, g.NT, true>;
}

template <typename K>
inline void (*scatter_kernel(int P))(Ctx, int, int) {
    constexpr ScatGeom g1 = scat_geom(1024, sizeof(K)), g2 = scat_geom(2048, sizeof(K)), g4 = scat_geom(4096, sizeof(K));
    if (P <= 1024) return k_scatter<K, g1.T, g1.SG, g1.PPT, g1.NT, false, g1.NH>;
    if (P == 2048) return k_scatter<K, g2.T, g2.SG, g2.PPT, g2.NT>;
    return k_scatter<K, g4.T, g4.SG, g4.PPT, g4.NT>;
}
inline int scatter_threads(int P, int key_bytes) { return scat_geom(P, key_bytes).NT; }
inline size_t scatter_smem_bytes(int P, int key_bytes) { return scat_smem_bytes(P, key_bytes); }

}  // namespace mgj
