// EXPERIMENT (round 2), not built: the a3 scatter with its write-out as one
// TMA bulk copy (shared -> global) per partition per sub-tile, issued by the
// partition's owner thread, the sorted sub-tiles in a shared-memory ring so
// that sub-tile g is laid out while the copies of g - 1 still read theirs.
// Correct (all GPU tests passed with it as the P <= 1024 scatter), but
// measured slower at M2: scatter 5.67 ms against 4.15 ms (M5: 5.36 vs 3.73).
// Why: a bulk copy instruction keeps its warp until the TMA unit has taken
// every lane's copy, and the unit takes about one copy per 4.4 cycles per SM
// (tools/tma_store_bench.cu); with 1024 partitions per 8192-tuple sub-tile
// that is ~4500 cycles per sub-tile in which every warp waits, so the copies
// serialise with the ranking instead of overlapping it.  Kept for reference
// (drop into csrc/scatter.cuh and dispatch P <= 1024 to k_scatter_tma).
// ---------------------------------------------------------------------------
// a3 for P <= 1024 (the configurations the bench times): the same layout
// (sub-tiles of T tuples, partitions group-aligned, < 32-byte tails carried
// in registers), but the write-out is one TMA bulk copy per partition per
// sub-tile (cp.async.bulk.global.shared::cta, issued by the partition's owner
// thread) instead of 32-byte stores by every thread.
//
// Why: the register/shared-memory write-out kept the SM's L1 data pipe 81%
// busy (ncu, round 2: 978 M wavefronts per M2 launch, of which ~320 M were
// the write-out's group loads, descriptor loads and 32-byte global stores
// touching ~16 lines per warp store).  Bulk copies leave that pipe to the
// ranking and run on the TMA unit (measured, tools/tma_store_bench.cu: one
// 64-byte copy per 4.4 cycles per SM with every warp issuing, the same DRAM
// rate as 32-byte stores).  They are asynchronous, so the sorted sub-tiles
// live in a ring: sub-tile g is laid out while the copies of g - 1 are still
// reading their region; the region of g - 2 is reused once its copies have
// read it (bulk wait_group.read 1 before the layout scan, whose barriers make
// it CTA-wide; a region that would overlap g - 1's waits for all copies).
// The ring needs the shared memory the input stage had: keys still arrive by
// TMA, payloads by 16-byte register loads one sub-tile ahead.
// ---------------------------------------------------------------------------
constexpr size_t SCAT_SMEM_BYTES = 226 * 1024;  // dynamic shared memory of k_scatter_tma
__host__ __device__ constexpr bool scat_uses_tma(int P) { return P <= 1024; }
// shared-memory layout: keys stage [T] | off [1024] u32 | ring (128-byte aligned)
__host__ __device__ inline size_t scat_ring_off(int P, int key_bytes) {
    return ((size_t)scat_geom(P, key_bytes).T * key_bytes + 1024 * 4 + 127) / 128 * 128;
}
__host__ __device__ inline uint32_t scat_ring_slots(int P, int key_bytes) {
    const ScatGeom g = scat_geom(P, key_bytes);
    const size_t TB = 2 * (size_t)key_bytes;
    return (uint32_t)((SCAT_SMEM_BYTES - scat_ring_off(P, key_bytes)) / TB) / g.SG * g.SG;
}

template <typename K, int T, int SG>
__global__ void __launch_bounds__(1024, 1) k_scatter_tma(Ctx c) {
    using Tup = typename TupT<K>::T;
    constexpr int NT = 1024;
    constexpr int TB = (int)sizeof(Tup);
    constexpr int V = T / NT;                  // tuples per thread per sub-tile
    constexpr int LU = 16 / (int)sizeof(K);    // tuples per 16-byte vector
    constexpr int NU = V / LU;                 // vectors per thread
    static_assert(NU * LU == V && NU >= 1 && SG >= 2, "sub-tile");
    constexpr int GB = SG * TB;                // group bytes (32)
    constexpr int CW = SG - 1;                 // carry capacity (tuples)
    typedef unsigned long long ull;
    extern __shared__ __align__(128) unsigned char smem[];
    const int P = c.P;
    K *const skey = reinterpret_cast<K *>(smem);                 // TMA stage: the sub-tile's keys
    uint32_t *const off = reinterpret_cast<uint32_t *>(skey + T);  // next free ring slot per partition
    Tup *const ring = reinterpret_cast<Tup *>(smem + scat_ring_off(P, sizeof(K)));
    const uint32_t RC = scat_ring_slots(P, sizeof(K));
    __shared__ __align__(8) uint64_t bar;
    __shared__ uint32_t tmp[32];
    const int tid = threadIdx.x;
    const int tile = blockIdx.x;
    const int ok = *(volatile int32_t *)&c.meta[MT_OK];
    const bool own = tid < P;  // thread tid owns partition tid

    uint64_t lo0, hi0, lo1, hi1;
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

    // the owned partition (registers): destination of its next group, carry
    ull base = 0;
    uint32_t cc = 0, hd = 0, lim = 0, seg_o = 0, full = 0;
    bool skp = false;
    Tup carry[CW];
    bool pending = false;  // the carry of the last sub-tile still sits in the ring
    uint32_t cur = 0, pa = 0, pb = 0;  // ring cursor and the region of the previous sub-tile (uniform)

    auto subtile = [&](uint32_t g, int &rel, uint64_t &first, uint32_t &len) {
        rel = g < nsub0 ? 0 : 1;
        const uint32_t j = rel ? g - nsub0 : g;
        first = (rel ? lo1 : lo0) + (uint64_t)j * T;
        len = (uint32_t)min((uint64_t)T, (rel ? hi1 : hi0) - first);
    };
    auto issue = [&](uint32_t g) {  // thread 0: TMA the 16-byte-aligned body of sub-tile g's keys
        int rel;
        uint64_t first;
        uint32_t len;
        subtile(g, rel, first, len);
        const uint32_t bytes = (len & ~(uint32_t)(LU - 1)) * (uint32_t)sizeof(K);
        mbar_arrive_expect_tx(&bar, bytes);
        if (bytes) tma_load_1d(skey, static_cast<const K *>(c.in_key[rel]) + first, bytes, &bar, pol);
    };
    K pn[V];  // payloads of the next sub-tile (16-byte register loads, one sub-tile ahead)
    auto fetch_pay = [&](uint32_t g) {
        int rel;
        uint64_t first;
        uint32_t len;
        subtile(g, rel, first, len);
        const K *gp = static_cast<const K *>(c.in_pay[rel]) + first;
        if (len == T) {
#pragma unroll
            for (int u = 0; u < NU; ++u) {
                const uint4 b = __ldcs(reinterpret_cast<const uint4 *>(gp + (uint32_t)(u * NT + tid) * LU));
                memcpy(&pn[u * LU], &b, 16);
            }
        } else {
#pragma unroll
            for (int u = 0; u < NU; ++u)
#pragma unroll
                for (int e = 0; e < LU; ++e) {
                    const uint32_t i = (uint32_t)(u * NT + tid) * LU + e;
                    pn[u * LU + e] = i < len ? __ldcs(gp + i) : (K)0;
                }
        }
    };
    auto fetch_carry = [&]() {  // the incomplete last group of the previous sub-tile -> registers
        if (pending) {
#pragma unroll
            for (int i = 0; i < CW; ++i)
                if (i < (int)cc) carry[i] = ring[lim - cc + i];
            pending = false;
        }
    };
    auto flush = [&]() {  // end of a relation: store the remaining tail tuple by tuple
        fetch_carry();
#pragma unroll
        for (int i = 0; i < CW; ++i)
            if (own && !skp && i >= (int)hd && i < (int)cc) reinterpret_cast<Tup *>(base)[i] = carry[i];
    };
    auto set_base = [&](int rel) {  // destination of this tile's first tuple of the owned partition
        cc = hd = 0;
        if (own) {
            const int p = tid;
            // destination: the owner, or this rank itself for the S side of a
            // selectively broadcast partition (a2, NEXT-2)
            const int dst = (rel && c.bcast[p]) ? c.rank : c.owner[p];
            skp = c.pskip[p] != 0;
            const uint32_t *tb = c.tile_base + ((size_t)rel * c.G + tile) * P;
            const ull a = (ull)(c.arena[dst] + c.lay.recv[rel]) +
                          (c.send_off[(size_t)rel * P + p] + tb[p]) * (uint64_t)TB;
            const uint32_t h = (uint32_t)((a & (GB - 1)) / TB);
            base = a - (ull)h * TB;
            cc = hd = h;
#pragma unroll
            for (int i = 0; i < CW; ++i) {  // placeholders: digit1 = p, never stored
                carry[i].x = (K)p;
                carry[i].y = 0;
            }
        }
    };
    auto load_count = [&](uint32_t g) -> uint32_t {  // a1's count of sub-tile g for the owned partition
        if (g >= ntot || !own) return 0;
        const int rel = g < nsub0 ? 0 : 1;
        const uint32_t j = rel ? g - nsub0 : g;
        return __ldg(c.sub_hist + (((size_t)rel * c.G + tile) * c.sub_ns + j) * P + tid);
    };
    uint32_t ncnt = load_count(0);
    if (ntot > 0) {
        if (tid == 0) issue(0);
        fetch_pay(0);
    }
    int cur_rel = -1;
    for (uint32_t g = 0; g < ntot; ++g) {
        int rel;
        uint64_t first;
        uint32_t len;
        subtile(g, rel, first, len);
        if (rel != cur_rel) {  // thread-private partition state: no barrier needed
            if (cur_rel >= 0) flush();
            set_base(rel);
            cur_rel = rel;
        }
        fetch_carry();
        const uint32_t cnt = cc + ncnt;
        const uint32_t seg = own ? (cnt + SG - 1) & ~(uint32_t)(SG - 1) : 0u;
        ncnt = load_count(g + 1);  // prefetch (consumed next iteration)
        bulk_wait_read<1>();       // the copies of sub-tile g - 2 have read their region
        uint32_t total;
        uint32_t o = block_scan_reg(seg, tmp, total);  // its barriers: every thread's wait above is done
        // ring region of this sub-tile (the same on every thread): contiguous,
        // and not overlapping the previous sub-tile's, whose copies may still read
        uint32_t reg = cur + total <= RC ? cur : 0u;
        if (reg < pb && pa < reg + total) {  // (rare) wait for every copy
            bulk_wait_read<0>();
            __syncthreads();
        }
        pa = reg;
        pb = reg + total;
        cur = pb;
        o += reg;
        if (own) {
#pragma unroll
            for (int i = 0; i < CW; ++i)
                if (i < (int)cc) ring[o + i] = carry[i];
            off[tid] = o + cc;
            seg_o = o;
            full = cnt & ~(uint32_t)(SG - 1);
            lim = o + cnt;
        }
        K kk[V], pp[V];
#pragma unroll
        for (int v = 0; v < V; ++v) pp[v] = pn[v];
        mbar_wait(&bar, g & 1);
        const uint32_t body = len & ~(uint32_t)(LU - 1);
        const K *gk = static_cast<const K *>(c.in_key[rel]) + first;
        if (len == T) {
#pragma unroll
            for (int u = 0; u < NU; ++u) {
                const uint4 a = *reinterpret_cast<const uint4 *>(skey + (uint32_t)(u * NT + tid) * LU);
                memcpy(&kk[u * LU], &a, 16);
            }
        } else {
#pragma unroll
            for (int u = 0; u < NU; ++u)
#pragma unroll
                for (int e = 0; e < LU; ++e) {  // < LU trailing tuples of the relation come from global
                    const uint32_t i = (uint32_t)(u * NT + tid) * LU + e;
                    kk[u * LU + e] = i < body ? skey[i] : (i < len ? gk[i] : (K)0);
                }
        }
        __syncthreads();  // S1: offsets and carries in place, stage consumed
        if (g + 1 < ntot) {
            if (tid == 0) issue(g + 1);
            fetch_pay(g + 1);
        }
#pragma unroll
        for (int v = 0; v < V; ++v) {
            const uint32_t i = (uint32_t)((v / LU) * NT + tid) * LU + (v % LU);
            if (i < len) {
                Tup t;
                t.x = kk[v];
                t.y = pp[v];
                ring[atomicAdd(&off[digit1(kk[v], P)], 1u)] = t;
            }
        }
        fence_proxy_async_smem();  // this thread's ring stores before the bulk copies read them
        __syncthreads();           // S2: the sub-tile is sorted
        // write-out: the owned partition's complete groups, one bulk copy
        if (own && full && !skp) {
            char *dst = reinterpret_cast<char *>(base);
            uint32_t so = seg_o, nb = full * TB;
            if (hd) {  // the tile's first group starts hd tuples before the destination: store its tail
#pragma unroll
                for (int i = 1; i < SG; ++i)
                    if (i >= (int)hd) reinterpret_cast<Tup *>(dst)[i] = ring[so + i];
                dst += GB;
                so += SG;
                nb -= GB;
            }
            if (nb) tma_store_1d(dst, ring + so, nb);
        }
        bulk_commit();  // one (possibly empty) bulk group per thread per sub-tile
        base += (ull)full * TB;
        if (full) hd = 0;
        cc = cnt - full;
        pending = true;
    }
    if (cur_rel >= 0) flush();

    // ---- every CTA: its bulk copies complete and visible, the last one signals ----
    bulk_wait0();
    fence_proxy_async_global();
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

