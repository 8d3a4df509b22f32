// hist_plan.cuh — phase a1 (radix histogram fused with its all-gather) and
// phase a2 (partition -> GPU assignment and exact receive offsets).
#pragma once

#include "common.cuh"

namespace mgj {

#ifndef HIST_MINB
#define HIST_MINB 1  // k_hist: minimum resident CTAs per SM (register cap)
#endif

// ---------------------------------------------------------------------------
// a1: per-GPU radix histogram (§3.2 "Histogram generation",
// P:356-370, built in shared memory after Rui et al. [38]; bin count from the
// Eq. 1 analogue).  H[rel][p] = #{t in rel_g : digit1(t.key) = p}.
// grid = (G, 2): CTA (c, rel) counts tile c of relation rel (the same tiles
// the scatter kernel processes) reading only the key column with 16-byte
// streaming loads, and stores its per-tile histogram (so the scatter knows
// its exact output offsets without atomics) and adds it into the rank
// histogram.  The last CTA stores the rank histogram into every peer's
// arena mailbox and raises SIG_HIST there (histogram exchange X4 fused).
// ---------------------------------------------------------------------------
template <typename K>
__global__ void __launch_bounds__(HIST_THREADS, HIST_MINB) k_hist(Ctx c) {
    extern __shared__ uint32_t sh[];  // sub[P] (current sub-tile), acc[P] (this CTA's share of the tile)
    const int P = c.P, T = c.scat_T;
    uint32_t *const sub = sh, *const acc = sh + P;
    const int rel = blockIdx.y, tile = blockIdx.x / HIST_SPLIT, part = blockIdx.x % HIST_SPLIT;
    const int tid = threadIdx.x;
    const K *keys = static_cast<const K *>(c.in_key[rel]);
    uint64_t tlo, thi;
    tile_range(c.n_in[rel], c.G, tile, tlo, thi);
    // HIST_SPLIT CTAs share a tile: contiguous runs of the scatter's sub-tiles
    const uint32_t nsub = (uint32_t)((thi - tlo + T - 1) / T);
    const uint32_t j0 = nsub * part / HIST_SPLIT, j1 = nsub * (part + 1) / HIST_SPLIT;
    for (int i = tid; i < 2 * P; i += blockDim.x) sh[i] = 0;
    __syncthreads();

    constexpr int VEC = 16 / sizeof(K);
    constexpr int NV = 4;  // 16-byte vectors per thread per sub-tile (T / VEC <= NV * HIST_THREADS)
    const uint32_t m = (uint32_t)(P - 1);
    auto count = [&](const uint4 &v) {
        if (sizeof(K) == 4) {
            atomicAdd(&sub[v.x & m], 1u);
            atomicAdd(&sub[v.y & m], 1u);
            atomicAdd(&sub[v.z & m], 1u);
            atomicAdd(&sub[v.w & m], 1u);
        } else {  // two 8-byte keys: low words are .x and .z
            atomicAdd(&sub[v.x & m], 1u);
            atomicAdd(&sub[v.z & m], 1u);
        }
    };
    auto load = [&](uint32_t j, uint4 (&v)[NV], uint32_t &nvec) {  // sub-tile j's key vectors
        nvec = 0;
        if (j >= j1) return;
        const uint64_t a = tlo + (uint64_t)j * T, b = min(thi, a + T);
        nvec = (uint32_t)((b - a) / VEC);
        const uint4 *kv = reinterpret_cast<const uint4 *>(keys + a);
#pragma unroll
        for (int q = 0; q < NV; ++q)
            if (tid + q * HIST_THREADS < nvec) v[q] = __ldcs(kv + tid + q * HIST_THREADS);
    };
    uint16_t *const out = c.sub_hist + ((size_t)rel * c.G + tile) * c.sub_ns * P;
    uint4 v[NV], vn[NV];
    uint32_t nv, nvn;
    load(j0, v, nv);
    for (uint32_t j = j0; j < j1; ++j) {
        load(j + 1, vn, nvn);  // next sub-tile's loads in flight while this one is counted
#pragma unroll
        for (int q = 0; q < NV; ++q)
            if (tid + q * HIST_THREADS < nv) count(v[q]);
        const uint64_t a = tlo + (uint64_t)j * T, b = min(thi, a + T);
        for (uint64_t t = a + (uint64_t)nv * VEC + tid; t < b; t += blockDim.x) atomicAdd(&sub[digit1(keys[t], P)], 1u);
        __syncthreads();
        // sub-tile histogram (u16 pairs) for the scatter's layout, then fold into acc
        uint32_t *o32 = reinterpret_cast<uint32_t *>(out + (size_t)j * P);
        for (int q = tid; q < P / 2; q += blockDim.x) {
            const uint32_t x0 = sub[2 * q], x1 = sub[2 * q + 1];
            o32[q] = x0 | x1 << 16;
            acc[2 * q] += x0;
            acc[2 * q + 1] += x1;
            sub[2 * q] = 0;
            sub[2 * q + 1] = 0;
        }
        __syncthreads();
#pragma unroll
        for (int q = 0; q < NV; ++q) v[q] = vn[q];
        nv = nvn;
    }
    uint32_t *th = c.tile_hist + ((size_t)rel * c.G + tile) * P;
    for (int p = tid; p < P; p += blockDim.x) {
        const uint32_t x = acc[p];
        if (x) {
            atomicAdd(&th[p], x);
            atomicAdd(&c.rank_hist[rel * P + p], x);
        }
    }

    // ---- fused exchange: the last CTA publishes the rank histogram ----
    __threadfence();
    __syncthreads();
    __shared__ int last;
    if (threadIdx.x == 0) last = (atomicAdd(&c.ticket[TK_HIST], 1u) == gridDim.x * gridDim.y - 1);
    __syncthreads();
    if (!last) return;
    __threadfence();
    for (int d = 0; d < c.world; ++d) {
        uint32_t *mb = reinterpret_cast<uint32_t *>(c.arena[d] + c.lay.mail) + (size_t)c.rank * 2 * P;
        for (int j = threadIdx.x; j < 2 * P; j += blockDim.x) mb[j] = __ldcg(&c.rank_hist[j]);
    }
    __threadfence_system();
    __syncthreads();
    if (threadIdx.x == 0) signal_all(c, SIG_HIST);
}

// Exclusive prefix of the per-tile histograms over tiles: tile c's tuples of
// partition p start at send_off[p] + tile_base[rel][c][p] in the owner's
// receive range (deterministic placement; one thread per (rel, p)).
__global__ void k_tilescan(Ctx c) {
    const int idx = blockIdx.x * blockDim.x + threadIdx.x;
    if (idx >= 2 * c.P) return;
    const int rel = idx / c.P, p = idx % c.P;
    const size_t stride = c.P;
    const uint32_t *src = c.tile_hist + (size_t)rel * c.G * c.P + p;
    uint32_t *dst = c.tile_base + (size_t)rel * c.G * c.P + p;
    uint32_t run = 0;
    int t = 0;
    for (; t + 4 <= c.G; t += 4) {
        const uint32_t v0 = src[(t + 0) * stride], v1 = src[(t + 1) * stride];
        const uint32_t v2 = src[(t + 2) * stride], v3 = src[(t + 3) * stride];
        dst[(t + 0) * stride] = run;
        run += v0;
        dst[(t + 1) * stride] = run;
        run += v1;
        dst[(t + 2) * stride] = run;
        run += v2;
        dst[(t + 3) * stride] = run;
        run += v3;
    }
    for (; t < c.G; ++t) {
        const uint32_t v = src[t * stride];
        dst[t * stride] = run;
        run += v;
    }
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

__host__ __device__ inline int ceil_log2_u64(uint64_t x) {
    int l = 0;
    while (l < 63 && (1ull << l) < x) ++l;
    return l;
}

// B2 from the largest owned R partition: co-partitions of ~target tuples
// (2/3 of the probe stage capacity, so they fit one shared-memory table).
__host__ __device__ inline int choose_b2(uint64_t max_r, int b2_cfg, int b2_max, uint64_t target) {
    if (b2_cfg > 0) return b2_cfg < b2_max ? b2_cfg : b2_max;
    const uint64_t need = (max_r + target - 1) / target;
    int b = ceil_log2_u64(need);
    if (b > b2_max) b = b2_max;
    return b;
}

// ---------------------------------------------------------------------------
// a2 device plan: one CTA of 1024 threads.  Every rank computes the same
// owner[] and receive sizes from the same all-gathered histograms, plus its
// own send offsets (u64 tuples into the owner's receive buffer, layout:
// owned p ascending, then source rank ascending), its owned segments, the
// local radix bits B2 and the chunk table of the local pass.
// ---------------------------------------------------------------------------
__global__ void __launch_bounds__(1024) k_plan(Ctx c) {
    extern __shared__ uint64_t sp[];
    const int P = c.P, N = c.world, tid = threadIdx.x;
    uint64_t *tot0 = sp, *tot1 = sp + P, *pre0 = sp + 2 * P, *pre1 = sp + 3 * P, *cum = sp + 4 * P;
    int32_t *own = reinterpret_cast<int32_t *>(sp + 5 * P);
    uint32_t *chn = reinterpret_cast<uint32_t *>(own + P);  // [P+1] chunk counts -> base (one rel at a time)
    __shared__ uint64_t tmp[33];
    __shared__ uint32_t tmp32[33];
    __shared__ int first[MAX_RANKS], endp[MAX_RANKS];
    __shared__ int ok, cap_bad;
    __shared__ unsigned long long maxr;
    if (tid == 0) {
        ok = wait_all_flags(c, SIG_HIST);
        cap_bad = 0;
        maxr = 0;
    }
    if (tid < MAX_RANKS) first[tid] = endp[tid] = P;
    __syncthreads();
    if (!ok) {
        if (tid == 0) c.meta[MT_OK] = 0;
        return;
    }
    const uint32_t *mail = reinterpret_cast<const uint32_t *>(c.arena[c.rank] + c.lay.mail);
    for (int p = tid; p < P; p += blockDim.x) {
        uint64_t t0 = 0, t1 = 0;
        for (int g = 0; g < N; ++g) {
            t0 += __ldcg(mail + (size_t)(g * 2 + 0) * P + p);
            t1 += __ldcg(mail + (size_t)(g * 2 + 1) * P + p);
        }
        tot0[p] = pre0[p] = t0;
        tot1[p] = pre1[p] = t1;
        cum[p] = t0 + t1;
    }
    __syncthreads();
    block_excl_scan_u64(pre0, P, tmp);
    block_excl_scan_u64(pre1, P, tmp);
    const uint64_t total = block_excl_scan_u64(cum, P, tmp);
    for (int p = tid; p < P; p += blockDim.x) {
        const int o = owner_of(cum[p], tot0[p] + tot1[p], total, N, p, P);
        own[p] = o;
        c.owner[p] = o;
    }
    __syncthreads();
    for (int p = tid; p < P; p += blockDim.x) {
        if (p == 0 || own[p - 1] != own[p]) first[own[p]] = p;
        if (p == P - 1 || own[p + 1] != own[p]) endp[own[p]] = p + 1;
    }
    __syncthreads();
    for (int p = tid; p < P; p += blockDim.x) {
        const int f = first[own[p]];
        uint64_t m0 = 0, m1 = 0;
        for (int g = 0; g < c.rank; ++g) {
            m0 += __ldcg(mail + (size_t)(g * 2 + 0) * P + p);
            m1 += __ldcg(mail + (size_t)(g * 2 + 1) * P + p);
        }
        const uint64_t b0 = pre0[p] - pre0[f], b1 = pre1[p] - pre1[f];
        if (!c.ext) {
            c.send_off[p] = b0 + m0;
            c.send_off[P + p] = b1 + m1;
        }
        c.seg_start[p] = b0;
        c.seg_start[P + p] = b1;
        c.seg_len[p] = tot0[p];
        c.seg_len[P + p] = tot1[p];
    }
    if (tid < 2 * MAX_RANKS) {
        const int d = tid >> 1, rel = tid & 1;
        uint64_t size = 0;
        if (d < N && first[d] < P) {
            const uint64_t *pre = rel ? pre1 : pre0;
            const uint64_t *tot = rel ? tot1 : tot0;
            size = pre[endp[d] - 1] + tot[endp[d] - 1] - pre[first[d]];
        }
        c.recv_size[rel * MAX_RANKS + d] = size;
        if (size > c.recv_cap[rel]) atomicOr(&cap_bad, 1);
    }
    const int plo = first[c.rank] < P ? first[c.rank] : 0;
    const int phi = first[c.rank] < P ? endp[c.rank] : 0;
    for (int p = plo + tid; p < phi; p += blockDim.x) atomicMax(&maxr, (unsigned long long)tot0[p]);
    __syncthreads();
    const int B2 = choose_b2(maxr, c.b2_cfg, c.b2_max, (uint64_t)c.probe_target);
    // received pieces of every owned partition pi: P2P — one piece (the whole
    // segment, sources ascending inside it); EXTERNAL — one piece per source
    // rank g, the receive area being [g0 | g1 | ...], each [owned p ascending]
    const int np = phi - plo;
    const uint64_t C = (uint64_t)c.chunk_tuples;
    const uint32_t *mine = mail + (size_t)c.rank * 2 * P;
    for (int rel = 0; rel < 2; ++rel) {
        uint64_t *ps = c.piece_start + (size_t)rel * P * MAX_RANKS;
        uint32_t *pl = c.piece_len + (size_t)rel * P * MAX_RANKS;
        if (!c.ext) {
            for (int i = tid; i < np; i += blockDim.x)
                for (int g = 0; g < MAX_RANKS; ++g) {
                    ps[(size_t)i * MAX_RANKS + g] = g == 0 ? c.seg_start[rel * P + plo + i] : 0;
                    pl[(size_t)i * MAX_RANKS + g] = g == 0 ? (uint32_t)(rel ? tot1 : tot0)[plo + i] : 0;
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
                ps[(size_t)i * MAX_RANKS + g] = displ + chn[i];
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
    // chunk table of the local pass: chunk_base[rel][pi] = first chunk of owned partition plo+pi,
    // piece_chunk[rel][pi][g] = first chunk of piece g inside pi
    uint32_t nch[2];
    for (int rel = 0; rel < 2; ++rel) {
        const uint32_t *pl = c.piece_len + (size_t)rel * P * MAX_RANKS;
        uint32_t *pc = c.piece_chunk + (size_t)rel * P * (MAX_RANKS + 1);
        for (int i = tid; i <= np; i += blockDim.x) {
            uint32_t t = 0;
            if (i < np)
                for (int g = 0; g < MAX_RANKS; ++g) {
                    pc[(size_t)i * (MAX_RANKS + 1) + g] = t;
                    t += (uint32_t)((pl[(size_t)i * MAX_RANKS + g] + C - 1) / C);
                }
            if (i < np) pc[(size_t)i * (MAX_RANKS + 1) + MAX_RANKS] = t;
            chn[i] = t;
        }
        __syncthreads();
        nch[rel] = block_excl_scan_u32(chn, np + 1, tmp32);
        for (int i = tid; i <= np; i += blockDim.x) c.chunk_base[(size_t)rel * c.cb_stride + i] = chn[i];
        __syncthreads();
    }
    if (tid == 0) {
        const bool fits = nch[0] <= c.max_chunks && nch[1] <= c.max_chunks;
        if (cap_bad || !fits) set_err(c, MGJ_ECAPACITY);
        c.meta[MT_PLO] = plo;
        c.meta[MT_PHI] = phi;
        c.meta[MT_B2] = B2;
        c.meta[MT_NCH_R] = (int)nch[0];
        c.meta[MT_NCH_S] = (int)nch[1];
        c.meta[MT_CHUNK] = c.chunk_tuples;
        // two-level local partitioning: when the owned
        // partitions span more than LOCAL2_NCH chunks on average, a first
        // histogram-based pass splits every owned partition into 2^BA
        // contiguous sub-partitions of ~48 chunks, and the chunked pass then
        // uses the remaining B2 - BA bits.  The mean, not the maximum: a few
        // heavy-hitter partitions (Zipf) are not helped by splitting the rest
        const uint32_t meannch = np ? (max(nch[0], nch[1]) + np - 1) / np : 0;
        int BA = 0;
        if (c.split_cfg > 0) {
            BA = c.split_cfg;
        } else if (c.split_cfg == 0 && meannch > (uint32_t)LOCAL2_NCH) {
            BA = ceil_log2_u64((meannch + 47) / 48);
            while (BA > 0 && (np << BA) > c.vcap) --BA;
        }
        if (BA > B2) BA = B2;
        if (BA > MAX_BA) BA = MAX_BA;
        if (!c.mid[0] || (np << BA) > c.vcap) BA = 0;
        c.meta[MT_BA] = BA;
        c.meta[MT_QB] = B2 - BA;
        c.meta[MT_NLP] = np;
        c.meta[MT_OK] = (cap_bad || !fits) ? 0 : 1;
    }
}

__global__ void k_wait(Ctx c, int kind) {
    if (threadIdx.x == 0 && blockIdx.x == 0) wait_all_flags(c, kind);
}

}  // namespace mgj
