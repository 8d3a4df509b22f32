// scatter.cuh — phase a3: global partitioning step 1 + data distribution,
// fused: every tuple is written straight into its owner's receive buffer.
#pragma once

#include "common.cuh"
#include "tma.cuh"

namespace mgj {

#ifndef SCAT_WO_UNROLL
#define SCAT_WO_UNROLL 1  // write-out groups per thread per step
#endif
#ifndef SCAT_ATOM_FIRST
#define SCAT_ATOM_FIRST 0  // rank all tuples of a thread before storing them
#endif

// Scatter geometry for P partitions and a key width (kernel template
// arguments; the host picks the instance with scatter_kernel<K>(P)):
//   T   = sub-tile (tuples) staged in shared memory per step,
//   SG  = tuples per 32-byte sector group (the unit of a global store),
//   PPT = partitions owned by each of the 1024 threads (registers).
// With SG > 1 every partition's output leaves in whole 32-byte sectors: the
// < 32-byte tail of a partition waits (in registers of its owning thread)
// for the next sub-tile.  For P = 4096 the alignment padding would not fit
// shared memory, so SG = 1 (one tuple per store).
#ifndef SCAT_GDST
#define SCAT_GDST 0  // per-group destination table written at layout time, no partition lookup in the write-out (measured slower: 4.36 vs 4.16 ms)
#endif

#ifndef SCAT_SOA
#define SCAT_SOA 0  // 4-byte keys: `sorted` held as key and payload arrays (4-byte random stores; measured slower: 4.42 vs 4.14 ms)
#endif
#ifndef SCAT_LDG
#define SCAT_LDG 0  // sub-tiles loaded straight into registers one sub-tile ahead, no shared-memory stage (measured slower: 4.73 vs 4.13 ms)
#endif
#ifndef SCAT_T4
#define SCAT_T4 8192  // sub-tile of the 4-byte-key, P <= 1024 instance
#endif
#ifndef SCAT_2CTA
#define SCAT_2CTA 0  // 4-byte keys, P <= 1024: two 512-thread CTAs per SM, 4096-tuple sub-tiles, 16-byte groups (measured slower: 9.2 vs 4.1 ms)
#endif
#ifndef SCAT_ALIAS
#define SCAT_ALIAS 0  // 4-byte keys, P <= 1024: two 512-thread CTAs per SM, stage aliased into the sorted buffer (measured: 6.2 vs 4.1 ms)
#endif
#ifndef SCAT_PROF
#define SCAT_PROF 0  // DIAGNOSTIC: thread 0 and 512 of CTA 0 print clock64 time per phase
#endif
#ifndef SCAT_RING
#define SCAT_RING 0  // EXPERIMENT ONLY (wrong results): full-group stores land modulo SCAT_RING bytes of the arena (L2-resident)
#endif
struct ScatGeom {
    int T, SG, PPT, NT;
    bool alias;  // stage inside the sorted buffer (two CTAs per SM)
};
__host__ __device__ constexpr ScatGeom scat_geom(int P, int key_bytes) {
    return key_bytes == 4
               ? (P <= 1024 ? (SCAT_ALIAS  ? ScatGeom{4096, 4, P <= 512 ? 1 : 2, 512, true}
                               : SCAT_2CTA ? ScatGeom{4096, 2, P <= 512 ? 1 : 2, 512, false}
                                           : ScatGeom{SCAT_T4, 4, 1, 1024, false})
                  : P == 2048 ? ScatGeom{4096, 4, 2, 1024, false} : ScatGeom{8192, 1, 4, 1024, false})
               : (P <= 1024 ? ScatGeom{4096, 2, 1, 1024, false} : P == 2048 ? ScatGeom{2048, 2, 2, 1024, false}
                                                                      : ScatGeom{4096, 1, 4, 1024, false});
}

// Per-partition write-out descriptor of the current sub-tile (16 bytes, one
// shared load per sector group).
struct __align__(16) PInfo {
    unsigned long long wb;  // destination address of sorted slot 0 (wb + slot * TB)
    uint32_t lim;           // end of the partition's valid slots in `sorted`
    uint32_t head;          // (slot << 2 | h) of a head group whose first h slots are not ours, else ~0
};

__host__ __device__ inline size_t scat_smem_bytes(int P, int key_bytes) {
    const ScatGeom g = scat_geom(P, key_bytes);
    const size_t TB = 2 * (size_t)key_bytes;
    return ((g.alias || SCAT_LDG) ? 0 : 2 * (size_t)g.T * key_bytes)  // input stage: keys + payloads (SoA)
           + ((size_t)g.T + 2 * (size_t)(g.SG - 1) * P) * TB  // partition-sorted sub-tile (+ carries, group padding)
           + ((SCAT_GDST && g.SG > 1) ? ((size_t)g.T + 2 * (size_t)(g.SG - 1) * P) / g.SG * 8  // group destinations
                                      : (size_t)P * sizeof(PInfo))
           + (size_t)P * 4;                                  // next free slot per partition
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

// Same with one barrier: every warp reduces the per-warp totals itself (its
// prefix and the block total) instead of one warp scanning them behind a
// second barrier.  `tmp` may be rewritten only after a later barrier.
__device__ __forceinline__ uint32_t block_scan_reg1(uint32_t v, uint32_t *tmp, uint32_t &total) {
    const int tid = threadIdx.x, lane = tid & 31, w = tid >> 5;
    uint32_t x = v;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const uint32_t y = __shfl_up_sync(0xffffffffu, x, o);
        if (lane >= o) x += y;
    }
    if (lane == 31) tmp[w] = x;
    __syncthreads();
    const uint32_t t = lane < (int)(blockDim.x >> 5) ? tmp[lane] : 0u;
    uint32_t pre = lane < w ? t : 0u, tot = t;
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        pre += __shfl_xor_sync(0xffffffffu, pre, o);
        tot += __shfl_xor_sync(0xffffffffu, tot, o);
    }
    total = tot;
    return x - v + pre;
}

#ifndef SCAT_SCAN1
#define SCAT_SCAN1 0  // one-barrier layout scan (measured neutral: 4.16 vs 4.16 ms)
#endif

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

#ifndef SCAT_EAGER
#define SCAT_EAGER 1  // write-out: both group halves and the whole descriptor loaded up front, 8-byte keys
                      // (measured: M5 scatter 3.725 -> 3.693 ms; 4-byte keys 4.155 -> 4.19, so not used there)
#endif

template <int BYTES> struct Vec;
template <> struct Vec<8> { using T = uint2; };
template <> struct Vec<16> { using T = uint4; };
template <> struct Vec<32> { struct __align__(32) T { uint4 a, b; }; };

// One global store of a 8/16/32-byte group (32 bytes: a single 256-bit store).
template <int BYTES>
__device__ __forceinline__ void st_group(void *dst, const typename Vec<BYTES>::T &v) {
    if constexpr (BYTES == 32) {
        asm volatile("st.global.v8.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8};" ::"l"(dst), "r"(v.a.x), "r"(v.a.y),
                     "r"(v.a.z), "r"(v.a.w), "r"(v.b.x), "r"(v.b.y), "r"(v.b.z), "r"(v.b.w)
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
// B200 form: one persistent CTA (1024 threads) per SM processes tile
// c = blockIdx.x of R and then of S, in sub-tiles of T tuples that a TMA
// bulk copy brings into shared memory one sub-tile ahead.  Per sub-tile:
//  1. each thread takes LU-tuple vectors of keys and payloads from the stage
//     and ranks every tuple in its digit1 bin (one shared atomic);
//  2. thread t owns partitions t*PPT.. (PPT per thread) and keeps, in
//     registers, each one's destination cursor and its < 32-byte tail
//     (carry) from the previous sub-tile; a block scan of the per-partition
//     sizes (carry + new, rounded up to a 32-byte group) lays the partitions
//     out group-aligned in `sorted`, the carry first;
//  3. tuples are scattered into `sorted`, then written out one 32-byte group
//     per thread and store (st.global.v8.b32): every complete group is a
//     whole DRAM sector at its final address — owner(p)'s receive buffer at
//     send_off[p] (a2) + tile_base[c][p] (a1 tile prefix) + the running
//     count of p in this tile; no global atomics.  An incomplete last group
//     stays in `sorted` and its owning thread reloads it as the next carry.
// A tile's first destination of a partition need not be group-aligned: the
// carry then starts with h placeholder slots (key = p) that are never stored
// (the head group is written tuple by tuple from slot h).  The relation's
// remaining tails are written tuple by tuple at its end.  On NVSwitch the
// owner may be another GPU: the same stores go over NVLink to a peer-mapped
// address; the paper's packets, routing buffers and multi-hop routing (§4)
// have no role on a one-hop fabric.  The last CTA raises SIG_DATA at every
// peer after a system fence.
// ---------------------------------------------------------------------------
template <typename K, int T, int SG, int PPT, int NT, bool ALIAS>
__global__ void __launch_bounds__(NT, NT <= 512 ? 2 : 1) k_scatter(Ctx c) {
    using Tup = typename TupT<K>::T;
    constexpr int TB = (int)sizeof(Tup);
    constexpr int V = T / NT;                  // tuples per thread per sub-tile
    constexpr int LU = 16 / (int)sizeof(K);    // tuples per 16-byte stage vector
    constexpr int NU = V / LU;                 // vectors per thread
    static_assert(NU * LU == V && NU >= 1, "sub-tile");
    constexpr int GB = SG * TB;                // group bytes
    constexpr int CW = SG > 1 ? SG - 1 : 1;    // carry capacity (tuples)
    constexpr uint32_t NONE = 0xffffffffu;
    using GV = typename Vec<GB>::T;
    typedef unsigned long long ull;
    // `sorted` swizzle: the two 16-byte halves of every 32-byte group whose
    // index has bit 2 set are swapped, so that the write-out's 16-byte loads
    // (8 consecutive groups per quarter warp) hit distinct banks
    // SOA (4-byte keys, 32-byte groups): `sorted` is a key array and a payload
    // array; the scatter's random stores are 4 bytes wide (fewer bank conflicts
    // than 8-byte ones) and the write-out interleaves 16 bytes of keys with 16
    // bytes of payloads into the group's 32-byte store (conflict-free, no swizzle)
    constexpr bool SOA = SCAT_SOA && sizeof(K) == 4 && SG == 4 && !ALIAS;
    auto swz = [](uint32_t s) -> uint32_t {
        if constexpr (SG > 1 && !SOA && SG * sizeof(Tup) == 32) return s ^ (((s >> (SG == 4 ? 4 : 3)) & 1u) * (SG / 2));
        else return s;
    };
    extern __shared__ __align__(128) unsigned char smem[];
    const int P = c.P;
    // ALIAS: the stage is the head of the sorted buffer (loaded after the write-out)
    // LDG: sub-tile g+1 is loaded into registers (16-byte streaming loads) while
    // g is laid out, ranked and written out; no stage, no TMA, no mbarrier
    constexpr bool LDG = SCAT_LDG && !ALIAS;
    Tup *const sorted = reinterpret_cast<Tup *>(smem + ((ALIAS || LDG) ? 0 : 2 * T * sizeof(K)));
    K *const skey = reinterpret_cast<K *>(ALIAS ? static_cast<void *>(sorted) : static_cast<void *>(smem));
    K *const spay = skey + T;
    // GD: the layout writes every group's destination (0: not stored; low bits:
    // h placeholder slots of a head group) so the write-out needs no lookup of
    // the group's partition; otherwise a per-partition descriptor (PInfo)
    constexpr bool GD = SCAT_GDST && SG > 1;
    constexpr bool EAGER = SCAT_EAGER && sizeof(K) == 8;
    PInfo *const pinfo = reinterpret_cast<PInfo *>(sorted + T + 2 * (SG - 1) * P);  // 16-byte aligned
    unsigned long long *const gdst = reinterpret_cast<unsigned long long *>(pinfo);
    uint32_t *const off = GD ? reinterpret_cast<uint32_t *>(gdst + (T + 2 * (SG - 1) * P) / SG)
                             : reinterpret_cast<uint32_t *>(pinfo + P);  // next free slot per partition
    K *const ks = reinterpret_cast<K *>(sorted);  // SOA: keys, then payloads
    K *const ps = ks + (T + 2 * (SG - 1) * P);
    auto sput = [&](uint32_t x, const Tup &t) {
        if constexpr (SOA) {
            ks[x] = t.x;
            ps[x] = t.y;
        } else {
            sorted[swz(x)] = t;
        }
    };
    auto sget = [&](uint32_t x) -> Tup {
        if constexpr (SOA) {
            Tup t;
            t.x = ks[x];
            t.y = ps[x];
            return t;
        } else {
            return sorted[swz(x)];
        }
    };
    __shared__ __align__(8) uint64_t bar;
    __shared__ uint32_t tmp[32];
    const int tid = threadIdx.x;
    const int tile = blockIdx.x;
    const int ok = *(volatile int32_t *)&c.meta[MT_OK];

    uint64_t lo0, hi0, lo1, hi1;  // scalars (no local-memory arrays)
    tile_range(c.n_in[0], c.G, tile, lo0, hi0);
    tile_range(c.n_in[1], c.G, tile, lo1, hi1);
    const uint32_t nsub0 = ok ? (uint32_t)((hi0 - lo0 + T - 1) / T) : 0;
    const uint32_t ntot = nsub0 + (ok ? (uint32_t)((hi1 - lo1 + T - 1) / T) : 0);
    if (tid == 0) {
        mbar_init(&bar, 1);
        fence_mbar_init();
    }
    __syncthreads();
    const uint64_t pol = policy_evict_first();

    // per owned partition (registers): destination of the next group, carry
    ull base[PPT];
    uint32_t cc[PPT], hd[PPT], lim[PPT];
    bool skp[PPT];  // partition skipped by the plan (an empty side): nothing is stored
    Tup carry[PPT][CW];
    bool pending = false;  // carries of the last sub-tile still sit in `sorted`
#pragma unroll
    for (int k = 0; k < PPT; ++k) base[k] = 0, cc[k] = 0, hd[k] = 0, lim[k] = 0, skp[k] = false;

    auto subtile = [&](uint32_t g, int &rel, uint64_t &first, uint32_t &len) {
        rel = g < nsub0 ? 0 : 1;
        const uint32_t j = rel ? g - nsub0 : g;
        first = (rel ? lo1 : lo0) + (uint64_t)j * T;
        len = (uint32_t)min((uint64_t)T, (rel ? hi1 : hi0) - first);
    };
    auto issue = [&](uint32_t g) {  // thread 0: TMA the 16-byte-aligned body of sub-tile g
        int rel;
        uint64_t first;
        uint32_t len;
        subtile(g, rel, first, len);
        const uint32_t bytes = (len & ~(uint32_t)(LU - 1)) * (uint32_t)sizeof(K);
        mbar_arrive_expect_tx(&bar, 2 * bytes);
        if (bytes) {
            tma_load_1d(skey, static_cast<const K *>(c.in_key[rel]) + first, bytes, &bar, pol);
            tma_load_1d(spay, static_cast<const K *>(c.in_pay[rel]) + first, bytes, &bar, pol);
        }
    };
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
    auto flush = [&]() {  // end of a relation: store the remaining tails tuple by tuple
        fetch_carry();
#pragma unroll
        for (int k = 0; k < PPT; ++k)
#pragma unroll
            for (int i = 0; i < CW; ++i)
                if (!skp[k] && i >= (int)hd[k] && i < (int)cc[k]) reinterpret_cast<Tup *>(base[k])[i] = carry[k][i];
    };
    auto set_base = [&](int rel) {  // destination of this tile's first tuple of each owned partition
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
                const ull a = (ull)(c.arena[dst] + c.lay.recv[rel]) + (so[p] + tb[p]) * (uint64_t)TB;
                const uint32_t h = SG > 1 ? (uint32_t)((a & (GB - 1)) / TB) : 0u;
                base[k] = a - (ull)h * TB;
                cc[k] = hd[k] = h;
#pragma unroll
                for (int i = 0; i < CW; ++i) {  // placeholders: digit1 = p, never stored
                    carry[k][i].x = (K)p;
                    carry[k][i].y = 0;
                }
            }
        }
    };

    // counts of sub-tile g for this thread's partitions (a1 wrote them, u16 per partition)
    auto load_counts = [&](uint32_t g, uint32_t (&out)[PPT]) {
#pragma unroll
        for (int k = 0; k < PPT; ++k) out[k] = 0;
        if (g >= ntot || tid * PPT >= P) return;
        const int rel = g < nsub0 ? 0 : 1;
        const uint32_t j = rel ? g - nsub0 : g;
        const uint16_t *src = c.sub_hist + (((size_t)rel * c.G + tile) * c.sub_ns + j) * P + tid * PPT;
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
    K kn[V], pn[V];  // LDG: the next sub-tile
    auto fetch = [&](uint32_t g) {
        int rel;
        uint64_t first;
        uint32_t len;
        subtile(g, rel, first, len);
        const K *gk = static_cast<const K *>(c.in_key[rel]) + first;
        const K *gp = static_cast<const K *>(c.in_pay[rel]) + first;
        if (len == T) {
#pragma unroll
            for (int u = 0; u < NU; ++u) {
                const uint32_t i0 = (uint32_t)(u * NT + tid) * LU;
                const uint4 a = __ldcs(reinterpret_cast<const uint4 *>(gk + i0));
                const uint4 b = __ldcs(reinterpret_cast<const uint4 *>(gp + i0));
                memcpy(&kn[u * LU], &a, 16);
                memcpy(&pn[u * LU], &b, 16);
            }
        } else {
#pragma unroll
            for (int u = 0; u < NU; ++u) {
#pragma unroll
                for (int e = 0; e < LU; ++e) {
                    const uint32_t i = (uint32_t)(u * NT + tid) * LU + e;
                    kn[u * LU + e] = i < len ? __ldcs(gk + i) : (K)0;
                    pn[u * LU + e] = i < len ? __ldcs(gp + i) : (K)0;
                }
            }
        }
    };
    uint32_t ncnt[PPT];
    load_counts(0, ncnt);
    if (LDG) {
        if (ntot > 0) fetch(0);
    } else if (tid == 0 && ntot > 0) {
        issue(0);
    }
    int cur_rel = -1;
    unsigned long long pt[7] = {0, 0, 0, 0, 0, 0, 0};
    long long pc = clock64();
    auto PT = [&](int i) {
        if (SCAT_PROF) {
            const long long n = clock64();
            pt[i] += (unsigned long long)(n - pc);
            pc = n;
        }
    };
    for (uint32_t g = 0; g < ntot; ++g) {
        int rel;
        uint64_t first;
        uint32_t len;
        subtile(g, rel, first, len);
        if (rel != cur_rel) {  // thread-private partition state: no barrier needed
            if (SCAT_PROF && blockIdx.x == 0 && (tid == 0 || tid == 512))
        printf("SCATPROF tid %d subtiles %u: top %llu scan %llu layout %llu tmawait %llu read+S1 %llu rank+S2 %llu writeout %llu\n",
               tid, ntot, pt[0], pt[1], pt[2], pt[3], pt[4], pt[5], pt[6]);
    if (cur_rel >= 0) flush();
            set_base(rel);
            cur_rel = rel;
        }
        fetch_carry();
        // lay out this sub-tile's partitions (known from a1): carry + new tuples, group-rounded
        uint32_t cnt[PPT], seg[PPT], tsum = 0;
#pragma unroll
        for (int k = 0; k < PPT; ++k) {
            cnt[k] = cc[k] + ncnt[k];
            seg[k] = (cnt[k] + SG - 1) & ~(uint32_t)(SG - 1);
            tsum += seg[k];
        }
        load_counts(g + 1, ncnt);  // prefetch (consumed next iteration)
        uint32_t total;
        PT(0);  // carries fetched, counts: top of the sub-tile
        uint32_t o = SCAT_SCAN1 ? block_scan_reg1(tsum, tmp, total)   // its barrier: last write-out is done
                                : block_scan_reg(tsum, tmp, total);
        PT(1);  // layout scan (its barriers wait for the last write-out)
        uint32_t co[PPT], ccw[PPT];  // segment start and carried count (for the ALIAS carry write)
#pragma unroll
        for (int k = 0; k < PPT; ++k) ccw[k] = cc[k], co[k] = 0;
#pragma unroll
        for (int k = 0; k < PPT; ++k) {
            const int p = tid * PPT + k;
            if (p < P) {
                if (!ALIAS) {
#pragma unroll
                    for (int i = 0; i < CW; ++i)
                        if (i < (int)cc[k]) sput(o + i, carry[k][i]);
                }
                co[k] = o;
                off[p] = o + cc[k];
                const uint32_t full = cnt[k] & ~(uint32_t)(SG - 1);
                if constexpr (GD) {
                    const uint32_t ng = seg[k] / SG, nf = full / SG;
                    for (uint32_t j = 0; j < ng; ++j)  // a skipped partition's groups are never stored
                        gdst[o / SG + j] = (j < nf && !skp[k]) ? ((base[k] + (ull)j * GB) | (j == 0 ? hd[k] : 0u)) : 0ull;
                } else {
                    PInfo in;
                    in.wb = base[k] - (ull)o * TB;
                    in.lim = skp[k] ? o : o + cnt[k];  // a skipped partition's groups are never stored
                    in.head = (hd[k] && full) ? (o << 2 | hd[k]) : NONE;
                    pinfo[p] = in;
                }
                base[k] += (ull)full * TB;
                if (full) hd[k] = 0;
                cc[k] = cnt[k] - full;
                lim[k] = o + cnt[k];
            }
            o += seg[k];
        }
        pending = SG > 1;
        PT(2);  // layout: carries, descriptors
        K kk[V], pp[V];
        if constexpr (LDG) {
#pragma unroll
            for (int v = 0; v < V; ++v) kk[v] = kn[v], pp[v] = pn[v];
            if (g + 1 < ntot) fetch(g + 1);
        } else {
        mbar_wait(&bar, g & 1);
        PT(3);  // TMA wait
        const uint32_t body = len & ~(uint32_t)(LU - 1);
        const K *gk = static_cast<const K *>(c.in_key[rel]) + first;
        const K *gp = static_cast<const K *>(c.in_pay[rel]) + first;
        if (len == T) {  // full sub-tile: branch-free vector loads
#pragma unroll
            for (int u = 0; u < NU; ++u) {
                const uint32_t i0 = (uint32_t)(u * NT + tid) * LU;
                const uint4 a = *reinterpret_cast<const uint4 *>(skey + i0);
                const uint4 b = *reinterpret_cast<const uint4 *>(spay + i0);
                memcpy(&kk[u * LU], &a, 16);
                memcpy(&pp[u * LU], &b, 16);
            }
        } else {
#pragma unroll
            for (int u = 0; u < NU; ++u) {
#pragma unroll
                for (int e = 0; e < LU; ++e) {  // < LU trailing tuples of the relation come from global
                    const uint32_t i = (uint32_t)(u * NT + tid) * LU + e;
                    kk[u * LU + e] = i < body ? skey[i] : (i < len ? gk[i] : (K)0);
                    pp[u * LU + e] = i < body ? spay[i] : (i < len ? gp[i] : (K)0);
                }
            }
        }
        }
        __syncthreads();  // S1: offsets and carries in place, stage consumed
        PT(4);  // stage read + S1
        if (ALIAS) {  // the stage region is free now: carries to their segment heads
#pragma unroll
            for (int k = 0; k < PPT; ++k)
#pragma unroll
                for (int i = 0; i < CW; ++i)
                    if (i < (int)ccw[k]) sput(co[k] + i, carry[k][i]);
        } else if (!LDG && tid == 0 && g + 1 < ntot) {
            issue(g + 1);
        }
#if SCAT_ATOM_FIRST
        uint32_t pos[V];  // final slots: all atomics first, then the stores
#pragma unroll
        for (int v = 0; v < V; ++v) {
            const uint32_t i = (uint32_t)((v / LU) * NT + tid) * LU + (v % LU);
            pos[v] = (len == T || i < len) ? atomicAdd(&off[digit1(kk[v], P)], 1u) : NONE;
        }
#pragma unroll
        for (int v = 0; v < V; ++v) {
            if (pos[v] != NONE) {
                Tup t;
                t.x = kk[v];
                t.y = pp[v];
                sput(pos[v], t);
            }
        }
#else
#pragma unroll
        for (int v = 0; v < V; ++v) {
            const uint32_t i = (uint32_t)((v / LU) * NT + tid) * LU + (v % LU);
            if (i < len) {
                Tup t;
                t.x = kk[v];
                t.y = pp[v];
                sput(atomicAdd(&off[digit1(kk[v], P)], 1u), t);
            }
        }
#endif
        __syncthreads();  // S2
        PT(5);  // rank + scatter into sorted + S2
        if (ALIAS) fetch_carry();  // before the stage region is reloaded
        // write-out, two groups per thread per step (independent load chains)
        const uint32_t ngroups = total / SG;
        constexpr int WU = SCAT_WO_UNROLL;
        for (uint32_t u0 = tid; u0 < ngroups; u0 += WU * NT) {
            GV gv[WU];
            PInfo in[WU];
            uint32_t slot[WU];
            bool on[WU];
#pragma unroll
            for (int r = 0; r < WU; ++r) {
                slot[r] = (u0 + r * NT) * SG;
                on[r] = u0 + r * NT < ngroups;
                if (on[r]) {
                    if constexpr (SOA) {  // 4 keys + 4 payloads -> (k0,p0,k1,p1 | k2,p2,k3,p3)
                        const uint4 kv = *reinterpret_cast<const uint4 *>(ks + slot[r]);
                        const uint4 pv = *reinterpret_cast<const uint4 *>(ps + slot[r]);
                        gv[r].a = make_uint4(kv.x, pv.x, kv.y, pv.y);
                        gv[r].b = make_uint4(kv.z, pv.z, kv.w, pv.w);
                    } else if constexpr (GB == 32 && EAGER) {  // two conflict-free 16-byte halves (swizzled)
                        gv[r].a = lds128(sorted + swz(slot[r]));
                        gv[r].b = lds128(sorted + swz(slot[r] + SG / 2));
                    } else if constexpr (GB == 32) {
                        gv[r].a = *reinterpret_cast<const uint4 *>(sorted + swz(slot[r]));
                        gv[r].b = *reinterpret_cast<const uint4 *>(sorted + swz(slot[r] + SG / 2));
                    } else {
                        gv[r] = *reinterpret_cast<const GV *>(sorted + slot[r]);
                    }
                }
            }
            if constexpr (GD) {
#pragma unroll
                for (int r = 0; r < WU; ++r) {
                    const ull d = on[r] ? gdst[slot[r] / SG] : 0ull;
                    if (d) {
                        char *dst = reinterpret_cast<char *>(d & ~(ull)(GB - 1));
                        if (SCAT_RING) dst = c.arena[0] + c.lay.recv[0] + ((dst - c.arena[0] - c.lay.recv[0]) & (ull)(SCAT_RING - 1));
                        const uint32_t h = (uint32_t)(d & (GB - 1));
                        if (!h) {
                            st_group<GB>(dst, gv[r]);
                        } else {
                            for (uint32_t i = h; i < SG; ++i) reinterpret_cast<Tup *>(dst)[i] = sget(slot[r] + i);
                        }
                    }
                }
            } else {
#pragma unroll
            for (int r = 0; r < WU; ++r) {
                if (on[r]) {
                    const PInfo *pi = pinfo + (reinterpret_cast<const uint32_t *>(&gv[r])[0] & (uint32_t)(P - 1));
                    if constexpr (EAGER) {
                        const uint4 v = lds128(pi);
                        in[r].wb = (ull)v.x | ((ull)v.y << 32);
                        in[r].lim = v.z;
                        in[r].head = v.w;
                    } else {
                        in[r] = *pi;
                    }
                }
            }
#pragma unroll
            for (int r = 0; r < WU; ++r) {
                if (on[r] && slot[r] + SG <= in[r].lim) {
                    char *dst = reinterpret_cast<char *>(in[r].wb + (ull)slot[r] * TB);
                    if (SCAT_RING) dst = c.arena[0] + c.lay.recv[0] + ((dst - c.arena[0] - c.lay.recv[0]) & (ull)(SCAT_RING - 1));
                    if ((in[r].head >> 2) != slot[r]) {
                        st_group<GB>(dst, gv[r]);
                    } else {
                        for (uint32_t i = in[r].head & 3u; i < SG; ++i)
                            reinterpret_cast<Tup *>(dst)[i] = sget(slot[r] + i);
                    }
                }
            }
            }
        }
        PT(6);  // write-out
        if (ALIAS) {  // the sorted buffer is read: load the next sub-tile into its head
            __syncthreads();  // S3
            if (tid == 0 && g + 1 < ntot) issue(g + 1);
        }
    }
    if (cur_rel >= 0) flush();

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

template <typename K>
inline void (*scatter_kernel(int P))(Ctx) {
    if constexpr (sizeof(K) == 8) {
        if (P <= 1024) return k_scatter<K, 4096, 2, 1, 1024, false>;
        if (P == 2048) return k_scatter<K, 2048, 2, 2, 1024, false>;
        return k_scatter<K, 4096, 1, 4, 1024, false>;
    } else {
#if SCAT_ALIAS
        if (P <= 512) return k_scatter<K, 4096, 4, 1, 512, true>;
        if (P == 1024) return k_scatter<K, 4096, 4, 2, 512, true>;
#elif SCAT_2CTA
        if (P <= 512) return k_scatter<K, 4096, 2, 1, 512, false>;
        if (P == 1024) return k_scatter<K, 4096, 2, 2, 512, false>;
#else
        if (P <= 1024) return k_scatter<K, SCAT_T4, 4, 1, 1024, false>;
#endif
        if (P == 2048) return k_scatter<K, 4096, 4, 2, 1024, false>;
        return k_scatter<K, 8192, 1, 4, 1024, false>;
    }
}
inline int scatter_threads(int P, int key_bytes) { return scat_geom(P, key_bytes).NT; }

}  // namespace mgj
