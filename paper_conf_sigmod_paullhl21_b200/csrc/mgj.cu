// mgj.cu — C ABI of libmgj.so (include/mgj.h, include/mgj_aux.h): handle,
// workspace and arena management, phase launches, result read-back.
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <new>

#include "common.cuh"
#include "gen.cuh"
#include "hist_plan.cuh"
#include "local_probe.cuh"
#include "mgj.h"
#include "mgj_aux.h"
#include "scatter.cuh"

using namespace mgj;

namespace {

enum State { ST_PLANNED = 1, ST_PARTITIONED = 2, ST_SHUFFLED = 3, ST_JOINED = 4, ST_DONE = 5 };

uint64_t align_up(uint64_t x, uint64_t a) { return (x + a - 1) / a * a; }
constexpr int COMP_MAX_TILES = 1024;  // compressed shuffle: scatter tiles per relation and rank at most

struct Norm {  // validated config with the automatic fields filled in
    mgj_config c;
    int B1, P, b2_max, tuple_bytes, chunk_tuples, chunk_region, probe_slots, probe_target;
    int chunk_tuples2, chunk_region2, qm2_bits, chunk_tuples1s;
    uint64_t recv_cap[2], max_chunks, max_items, out_cap, mid_cap;
    uint64_t recv_cap_u[2];  // compressed shuffle: 32-byte units each receive buffer holds
    bool split;  // first local pass possible (mid buffers allocated)
    Arena lay;
};

int ceil_log2(uint64_t x) {
    int l = 0;
    while (l < 63 && (1ull << l) < x) ++l;
    return l;
}

mgj_status normalize(const mgj_config *in, Norm *o) {
    if (!in) return MGJ_EINVAL;
    mgj_config c = *in;
    for (int i = 0; i < 1; ++i)
        if (c.reserved[i]) return MGJ_EINVAL;
    if (c.assign != 0 && c.assign != 1) return MGJ_EINVAL;
    if (c.assign && c.shuffle_mode != MGJ_SHUFFLE_P2P) return MGJ_EINVAL;  // EXTERNAL needs contiguous owners
    if (c.peer_timeout_ms < 0) return MGJ_EINVAL;
    if (c.shuffle_overlap < -1 || c.shuffle_overlap > 2 || c.overlap_local_sms < 0) return MGJ_EINVAL;
    // chunk streaming (NEXT-3) needs the in-kernel shuffle's completion counts
    if (c.shuffle_overlap == 2 && c.shuffle_mode != MGJ_SHUFFLE_P2P) return MGJ_EINVAL;
    if (c.trace != 0 && c.trace != 1) return MGJ_EINVAL;
    if (c.compress != 0 && c.compress != 1) return MGJ_EINVAL;
    // the compressed shuffle (NEXT-1): 4-byte keys and payloads, in-kernel peer stores
    if (c.compress && (c.key_bytes != 4 || c.shuffle_mode != MGJ_SHUFFLE_P2P)) return MGJ_EINVAL;
    if (c.compress && c.radix_bits_global > 10) return MGJ_EINVAL;  // the compressed instance: P <= 1024
    if (c.skew_bcast < -1 || c.skew_bcast > 1) return MGJ_EINVAL;
    if (c.local_split_bits < -1 || c.local_split_bits > MAX_BA) return MGJ_EINVAL;
    if (c.shuffle_mode != MGJ_SHUFFLE_P2P && c.shuffle_mode != MGJ_SHUFFLE_EXTERNAL) return MGJ_EINVAL;
    if (c.world_size < 1 || c.world_size > MAX_RANKS || c.rank < 0 || c.rank >= c.world_size) return MGJ_EINVAL;
    if (!((c.key_bytes == 4 && c.payload_bytes == 4) || (c.key_bytes == 8 && c.payload_bytes == 8)))
        return MGJ_EINVAL;
    if (c.radix_bits_global == 0) c.radix_bits_global = 10;
    if (c.radix_bits_global < 1 || c.radix_bits_global > MAX_B1) return MGJ_EINVAL;
    if (c.radix_bits_local < 0 || c.radix_bits_local > MAX_B2) return MGJ_EINVAL;
    if (c.materialize != 0 && c.materialize != 1) return MGJ_EINVAL;
    if (c.num_sms < 0) return MGJ_EINVAL;
    if (c.r_capacity > (1ull << 32) - 1 || c.s_capacity > (1ull << 32) - 1) return MGJ_EINVAL;
    const uint64_t slack = c.world_size > 1 ? 4 : 0;  // N>1: +25% for imbalance
    if (c.recv_capacity_r == 0) c.recv_capacity_r = c.r_capacity + (slack ? c.r_capacity / slack + 65536 : 0);
    if (c.recv_capacity_s == 0) c.recv_capacity_s = c.s_capacity + (slack ? c.s_capacity / slack + 65536 : 0);
    if (c.recv_capacity_r > (1ull << 32) - 1 || c.recv_capacity_s > (1ull << 32) - 1) return MGJ_EINVAL;
    o->B1 = c.radix_bits_global;
    o->P = 1 << o->B1;
    o->tuple_bytes = 2 * c.key_bytes;
    o->recv_cap[0] = c.recv_capacity_r;
    o->recv_cap[1] = c.recv_capacity_s;
    o->probe_slots = PROBE_SLOTS8 * 8 / o->tuple_bytes;
    o->probe_target = (PROBE_SLOTS8 - PROBE_HEAD8) * 8 / o->tuple_bytes;
    const uint64_t target = (uint64_t)o->probe_target;
    // B2 upper bound: the largest R segment this rank could own is recv_cap_r.
    if (c.radix_bits_local > 0) {
        o->b2_max = c.radix_bits_local;
    } else {
        // expected largest owned R partition ~ recv_cap / P; +2 bits of headroom for skew
        const uint64_t per_p = (c.recv_capacity_r + o->P - 1) / o->P;
        const uint64_t per_rs = (c.recv_capacity_r + c.recv_capacity_s + o->P - 1) / o->P;
        const int b = std::max(ceil_log2((per_p + target - 1) / target), ceil_log2((per_rs + 2 * target - 1) / (2 * target)));
        o->b2_max = std::min(MAX_B2, std::max(1, b + 2));
    }
    const int Qm = 1 << o->b2_max;
    int C = 0;  // largest chunk (multiple of LOCAL_THREADS) whose buffers fit shared memory
    for (int v = local_vmax(o->tuple_bytes); v >= 1 && !C; --v)
        if (local_smem_bytes(v * LOCAL_THREADS, Qm, o->tuple_bytes) <= 225 * 1024) C = v * LOCAL_THREADS;
    if (!C) return MGJ_EINVAL;
    o->chunk_tuples = C;
    o->chunk_region = C + Qm;  // worst-case padding: one slot per run
    // the chunked pass after a first pass (BA >= 1) has fan-out <= 2^(b2_max - 1)
    o->qm2_bits = std::max(1, o->b2_max - 1);
    int C2 = 0;
    for (int v = local_vmax(o->tuple_bytes); v >= 1 && !C2; --v)
        if (local_smem_bytes(v * LOCAL_THREADS, 1 << o->qm2_bits, o->tuple_bytes) <= 225 * 1024) C2 = v * LOCAL_THREADS;
    if (C2 < C) C2 = C;
    o->chunk_tuples2 = C2;
    int C1s = 0;  // the first (split) pass: fan-out <= 2^MAX_BA
    for (int v = local_vmax(o->tuple_bytes); v >= 1 && !C1s; --v)
        if (local_smem_bytes(v * LOCAL_THREADS, 1 << MAX_BA, o->tuple_bytes) <= 225 * 1024) C1s = v * LOCAL_THREADS;
    o->chunk_tuples1s = std::max(C1s, C);
    o->chunk_region2 = C2 + (1 << o->qm2_bits);
    const uint64_t rmax = std::max(o->recv_cap[0], o->recv_cap[1]);
    // chunks of the chunked pass: sum over (sub-)partitions of ceil(size / C); at most
    // local2_vcap(P) sub-partitions after a first pass
    o->max_chunks = rmax / C + (uint64_t)local2_vcap(o->P) + 2;
    if (c.compress)  // chunks of CHUNK_UNITS units: >= rmax / CU_N units plus one partial unit per (rank, tile, p)
        o->max_chunks = (rmax / CU_N + (uint64_t)MAX_RANKS * 1024 * o->P) / CHUNK_UNITS + o->P + 2;
    // the first local pass exists if forced, or (auto) if one owned partition could
    // span more than LOCAL2_NCH chunks; its output pads each (chunk, run) once
    o->split = c.local_split_bits > 0 || (c.local_split_bits == 0 && rmax > (uint64_t)LOCAL2_NCH * C);
    // the first pass stores every chunk in place: a region of C1s + 2^MAX_BA slots per chunk
    o->mid_cap = o->split ? o->max_chunks * (uint64_t)(o->chunk_tuples1s + (1 << MAX_BA)) : 0;
    o->max_items = (uint64_t)o->P * Qm + o->recv_cap[1] / (o->probe_slots / 2) * 2 +
                   o->recv_cap[0] / (o->probe_slots / 2) * 2 + 4096;
    if (o->max_items > 0x7fffffffull) o->max_items = 0x7fffffffull;
    o->out_cap = c.out_capacity ? c.out_capacity : (c.materialize ? std::max(o->recv_cap[0], o->recv_cap[1]) : 0);
    Arena &L = o->lay;
    uint64_t off = 0;
    L.sig = off;
    off = align_up(off + SIG_COUNT * MAX_RANKS * 8, 4096);
    L.mail = off;
    off = align_up(off + (uint64_t)MAX_RANKS * 2 * o->P * 4, 4096);
    L.resmail = off;
    off = align_up(off + MAX_RANKS * RES_W * 8, 4096);
    L.umail = off;
    off = align_up(off + (uint64_t)MAX_RANKS * 2 * o->P * 4, 4096);
    L.cfgmail = off;
    off = align_up(off + MAX_RANKS * 4 * 8, 4096);
    L.rbmail = off;
    off = align_up(off + (uint64_t)STREAM_RMAX * (o->P + 1) * 4, 4096);
    L.rdone = off;
    off = align_up(off + STREAM_RMAX * 8, 4096);
    // compressed: a (source rank, tile, partition) run ends in a partial unit, so
    // short runs take more room than their tuples (at most one unit per tuple);
    // the bound counts <= 8 ranks x COMP_MAX_TILES tiles x P partial units (mgj_plan
    // rejects a plan with more tiles per relation: chunk streaming uses 4 per SM)
    for (int r = 0; r < 2; ++r)
        o->recv_cap_u[r] = c.compress ? std::min<uint64_t>(o->recv_cap[r], o->recv_cap[r] / CU_N + 1 +
                                                                               (uint64_t)MAX_RANKS * COMP_MAX_TILES * o->P)
                                      : 0;
    auto recv_bytes = [&](int r) {
        return std::max<uint64_t>(o->recv_cap[r] * o->tuple_bytes, o->recv_cap_u[r] * 32);
    };
    L.recv[0] = off;
    off = align_up(off + recv_bytes(0), 4096);
    L.recv[1] = off;
    off = align_up(off + recv_bytes(1), 4096);
    L.total = off;
    o->c = c;
    return MGJ_OK;
}

}  // namespace

struct mgj_plan_s {
    Norm n;
    int dev = 0, nsm = 0;
    char *own_arena = nullptr;
    char *arena[MAX_RANKS] = {};
    void *zero_block = nullptr;
    size_t zero_bytes = 0;
    void *allocs[64] = {};
    int nalloc = 0;
    Ctx ctx{};
    ChunkDesc *cdesc = nullptr;   // chunks of the (first) local pass, written by k_chunkmap
    ChunkDescB *cdescB = nullptr;  // chunks of the chunked pass after a first pass (k_emit2)
    char *send_arena = nullptr;  // EXTERNAL shuffle
    uint64_t epoch = 0;
    int state = 0;
    int launches = 0;  // kernels launched for the current run
    cudaStream_t stream = nullptr;
    cudaEvent_t ev[7] = {};
    void *stage = nullptr;
    size_t stage_bytes = 0;
    unsigned long long *h_res = nullptr;  // pinned result [8] + meta [MT_COUNT ints]
    int32_t *h_meta = nullptr;
    uint64_t recv_r = 0, recv_s = 0;
    int32_t host_err = 0;
    // §8(e) overlap: R's local pass on a second stream beside S's scatter
    bool overlap = false;
    int local_sms = 0, scatter_sms = 0;
    cudaStream_t aux = nullptr;
    cudaEvent_t ev_fork = nullptr, ev_join = nullptr;
};

namespace {

mgj_status cuda_ok(cudaError_t e) {
    if (e == cudaSuccess) return MGJ_OK;
    return e == cudaErrorMemoryAllocation ? MGJ_ENOMEM : MGJ_ECUDA;
}

void *dalloc(mgj_plan_s *h, size_t bytes, mgj_status *st) {
    void *p = nullptr;
    if (*st != MGJ_OK) return nullptr;
    cudaError_t e = cudaMalloc(&p, std::max<size_t>(bytes, 256));
    if (e != cudaSuccess) {
        (void)cudaGetLastError();
        *st = MGJ_ENOMEM;
        return nullptr;
    }
    h->allocs[h->nalloc++] = p;
    return p;
}

// sub-tile of the scatter (a1 counts per sub-tile of the same size)
int scat_T_of(const Norm &n) { return n.c.compress ? scat_geom_comp().T : scat_geom(n.P, n.c.key_bytes).T; }

size_t hist_smem(const Norm &n) {
    const int T = scat_T_of(n);
    const int TB = T / hist_halves(T, n.c.key_bytes);  // k_hist's ring blocks
    return (size_t)hist_nb(TB, n.c.key_bytes) * TB * n.c.key_bytes + (size_t)n.P * 8;
}
size_t plan_smem(const Norm &n) {
    // totals, prefixes, owners, scan scratch, broadcast flags, then the unit
    // totals (compression only) and the preferred ranks (assignment only)
    return (size_t)n.P * 5 * 8 + (size_t)n.P * 4 + (size_t)(n.P + 1) * 4 + (size_t)n.P + 8 +
           (n.c.compress ? (size_t)n.P * 2 * 8 : 0) + (n.c.assign ? (size_t)n.P : 0);
}
size_t scatter_smem(const Norm &n) { return scatter_smem_bytes(n.P, n.c.key_bytes); }
size_t planA_smem(const Norm &n) { return ((size_t)local2_vcap(n.P) + 1) * 12; }
size_t local_smem(const Norm &n) { return local_smem_bytes(n.chunk_tuples, 1 << n.b2_max, n.tuple_bytes); }
size_t local_smem2(const Norm &n) { return local_smem_bytes(n.chunk_tuples2, 1 << n.qm2_bits, n.tuple_bytes); }
size_t local_smem1s(const Norm &n) { return local_smem_bytes(n.chunk_tuples1s, 1 << MAX_BA, n.tuple_bytes); }
size_t probe_smem(const Norm &n) { return probe_smem_bytes(n.probe_slots, n.tuple_bytes); }

template <typename K>
cudaError_t set_attrs(const Norm &n) {
    cudaError_t e;
    const auto A = cudaFuncAttributeMaxDynamicSharedMemorySize;
    if ((e = cudaFuncSetAttribute(k_hist<K>, A, (int)hist_smem(n)))) return e;
    if ((e = cudaFuncSetAttribute(k_plan, A, (int)plan_smem(n)))) return e;
    if ((e = cudaFuncSetAttribute(scatter_kernel<K>(n.P), A, (int)scatter_smem(n)))) return e;
    if (n.c.compress && n.P <= 1024) {
        if ((e = cudaFuncSetAttribute(scatter_kernel_comp(), A, (int)scat_smem_bytes_comp(n.P)))) return e;
        if ((e = cudaFuncSetAttribute(k_local<uint32_t, 0, true>, A, (int)local_smem(n)))) return e;
        if ((e = cudaFuncSetAttribute(k_local<uint32_t, 1, true>, A, (int)local_smem(n)))) return e;
        if ((e = cudaFuncSetAttribute(k_local<uint32_t, 2, true>, A, (int)local_smem(n)))) return e;
        if ((e = cudaFuncSetAttribute(k_local<uint32_t, 1, true, true>, A, (int)local_smem(n)))) return e;
    }
    if ((e = cudaFuncSetAttribute(k_local<K, 0>, A, (int)local_smem(n)))) return e;
    if ((e = cudaFuncSetAttribute(k_local<K, 1>, A, (int)local_smem(n)))) return e;
    if ((e = cudaFuncSetAttribute(k_local<K, 2>, A, (int)local_smem(n)))) return e;
    if ((e = cudaFuncSetAttribute(k_local<K, 1, false, true>, A, (int)local_smem(n)))) return e;
    if ((e = cudaFuncSetAttribute(k_local_second<K>, A, (int)local_smem2(n)))) return e;
    if ((e = cudaFuncSetAttribute(k_local_split<K>, A, (int)local_smem1s(n)))) return e;
    if ((e = cudaFuncSetAttribute(k_planA, A, (int)planA_smem(n)))) return e;
    if ((e = cudaFuncSetAttribute(k_probe<K, false>, A, (int)probe_smem(n)))) return e;
    return cudaFuncSetAttribute(k_probe<K, true>, A, (int)probe_smem(n));
}

// Load every kernel of the plan now.  With lazy module loading (the CUDA
// default) a kernel's first launch loads its module, and the loader waits for
// the device: a launch issued while another rank's kernel on this GPU spins on
// a peer signal (virtual ranks; k_plan waiting for a histogram that the
// blocked host thread has yet to launch) would stall until that wait times out.
template <typename K>
cudaError_t preload_kernels(const Norm &n) {
    cudaFuncAttributes a;
    const void *f[] = {(const void *)k_hist<K>, (const void *)k_tilescan, (const void *)k_plan,
                       (const void *)k_chunkmap, (const void *)k_chunkorder, (const void *)scatter_kernel<K>(n.P),
                       (const void *)k_wait, (const void *)k_local<K, 0>, (const void *)k_local<K, 1>,
                       (const void *)k_local<K, 2>, (const void *)k_local<K, 1, false, true>,
                       (const void *)k_emit2<K>, (const void *)k_planA, (const void *)k_local_split<K>,
                       (const void *)k_local_second<K>, (const void *)k_itemize<K>, (const void *)k_probe<K, false>,
                       (const void *)k_probe<K, true>, (const void *)k_reduce};
    for (const void *fn : f)
        if (cudaError_t e = cudaFuncGetAttributes(&a, fn)) return e;
    if (n.c.compress && n.P <= 1024) {
        const void *fc[] = {(const void *)scatter_kernel_comp(), (const void *)k_local<uint32_t, 0, true>,
                            (const void *)k_local<uint32_t, 1, true>, (const void *)k_local<uint32_t, 2, true>,
                            (const void *)k_local<uint32_t, 1, true, true>};
        for (const void *fn : fc)
            if (cudaError_t e = cudaFuncGetAttributes(&a, fn)) return e;
    }
    return cudaSuccess;
}

bool is_device_ptr(const void *p) {
    cudaPointerAttributes a;
    if (cudaPointerGetAttributes(&a, p) != cudaSuccess) {
        (void)cudaGetLastError();
        return false;
    }
    return a.type == cudaMemoryTypeDevice || a.type == cudaMemoryTypeManaged;
}

template <typename K>
void launch_partition(mgj_plan_s *h, cudaStream_t s) {
    const Norm &n = h->n;
    k_hist<K><<<h->ctx.G * h->ctx.hist_split, HIST_THREADS, hist_smem(n), s>>>(h->ctx);
    h->launches = 1;
}

template <typename K>
void launch_shuffle(mgj_plan_s *h, cudaStream_t s) {
    const Norm &n = h->n;
    if (h->ctx.stream)
        k_tilescan<<<(2 * n.P + 127) / 128, 128, 0, s>>>(h->ctx);  // a thread per (rel, p): round boundaries
    else
        k_tilescan<<<(2 * n.P * 32 + 255) / 256, 256, 0, s>>>(h->ctx);  // a warp per (rel, p)
    k_plan<<<1, 1024, plan_smem(n), s>>>(h->ctx);
    k_chunkmap<<<h->nsm * 2, 256, 0, s>>>(h->ctx, h->cdesc);
    if (h->ctx.stream) k_chunkorder<<<h->nsm, 256, 0, s>>>(h->ctx);
    cudaEventRecord(h->ev[2], s);
    Ctx cs = h->ctx;
    if (cs.ext)
        for (int g = 0; g < MAX_RANKS; ++g) cs.arena[g] = h->send_arena;
    const bool comp = h->ctx.comp;
    const auto scat = comp ? scatter_kernel_comp() : scatter_kernel<K>(n.P);
    const size_t ssm = comp ? scat_smem_bytes_comp(n.P) : scatter_smem(n);
    const int nt = scatter_threads(n.P, n.c.key_bytes);
    const int sg = std::min(h->ctx.G, h->nsm);  // persistent scatter CTAs (tiles blockIdx + k * grid)
    if (h->overlap) {
        scat<<<sg, nt, ssm, s>>>(cs, 0, 0);  // a3, R
        // §8(e) ("data distribution and local partitioning start
        // together"; Rationale 2): once every rank's R tuples have
        // landed, R is partitioned locally on local_sms SMs of a second stream
        // while S is scattered on the others
        cudaEventRecord(h->ev_fork, s);
        cudaStreamWaitEvent(h->aux, h->ev_fork, 0);
        k_wait<<<1, 32, 0, h->aux>>>(h->ctx, SIG_DATA_R, -1);
        if (comp)
            k_local<uint32_t, 0, true><<<h->local_sms, LOCAL_THREADS, local_smem(n), h->aux>>>(h->ctx, h->cdesc);
        else
            k_local<K, 0><<<h->local_sms, LOCAL_THREADS, local_smem(n), h->aux>>>(h->ctx, h->cdesc);
        if (h->ctx.stream) {
            // NEXT-3 ("packets" as they arrive): S's local pass right
            // after R's, each chunk once the S scatter rounds it needs are done
            if (comp)
                k_local<uint32_t, 1, true, true><<<h->local_sms, LOCAL_THREADS, local_smem(n), h->aux>>>(h->ctx, h->cdesc);
            else
                k_local<K, 1, false, true><<<h->local_sms, LOCAL_THREADS, local_smem(n), h->aux>>>(h->ctx, h->cdesc);
            h->launches += 2;  // chunk order, S's local pass
        }
        cudaEventRecord(h->ev_join, h->aux);
        scat<<<h->scatter_sms, nt, ssm, s>>>(cs, 1, 1);  // a3, S
        h->launches += 7;
    } else {
        scat<<<sg, nt, ssm, s>>>(cs, 0, 1);  // a3, R then S in one launch
        h->launches += 4;
    }
}

template <typename K>
void launch_join(mgj_plan_s *h, cudaStream_t s) {
    const Norm &n = h->n;
    if (h->overlap) {
        cudaStreamWaitEvent(s, h->ev_join, 0);  // R's local pass (second stream) is done
        k_wait<<<1, 32, 0, s>>>(h->ctx, SIG_DATA_S, -1);
        h->launches += 1;
    } else if (!h->ctx.ext && h->ctx.world > 1) {  // EXTERNAL: the caller's exchange is stream-ordered;
        k_wait<<<1, 32, 0, s>>>(h->ctx, SIG_DATA_R, SIG_DATA_S);  // one rank: its own scatter precedes
        h->launches += 1;                                           // in stream order
    }
    // two-level local partitioning: k_plan decides on the device (MT_BA); when
    // it chooses one pass these four kernels return at once.  (Measured, not
    // kept: a guard kernel that tail-launches the chosen kernels from the
    // device costs 18 us; one kernel for both chunked passes spills, +0.1 ms at
    // M2; k_planA run by k_countA's last CTA, +0.28 ms at B1 = 7.)  Round 2: the
    // first pass stores its chunks in place and counts the sub-partitions
    // itself, so no counting pass reads the received data first.
    if (n.split) {
        k_local_split<K><<<h->nsm, LOCAL_THREADS, local_smem1s(n), s>>>(h->ctx, h->cdesc);
        k_planA<<<1, 1024, planA_smem(n), s>>>(h->ctx);
        k_emit2<K><<<h->nsm * 4, 256, 0, s>>>(h->ctx, h->cdescB);
        k_local_second<K><<<h->nsm, LOCAL_THREADS, local_smem2(n), s>>>(h->ctx, h->cdescB);
        h->launches += 4;
    }
    if (h->ctx.stream)
        h->launches -= 1;  // S's local pass already ran, streamed beside the scatter
    else if (h->overlap)
        if (h->ctx.comp)
            k_local<uint32_t, 1, true><<<h->nsm, LOCAL_THREADS, local_smem(n), s>>>(h->ctx, h->cdesc);
        else
            k_local<K, 1><<<h->nsm, LOCAL_THREADS, local_smem(n), s>>>(h->ctx, h->cdesc);
    else
        if (h->ctx.comp)
            k_local<uint32_t, 2, true><<<h->nsm, LOCAL_THREADS, local_smem(n), s>>>(h->ctx, h->cdesc);
        else
            k_local<K, 2><<<h->nsm, LOCAL_THREADS, local_smem(n), s>>>(h->ctx, h->cdesc);
    cudaEventRecord(h->ev[4], s);
    k_itemize<K><<<h->nsm * 4, 256, 0, s>>>(h->ctx);
    if (n.c.materialize)
        k_probe<K, true><<<h->nsm, PROBE_THREADS, probe_smem(n), s>>>(h->ctx);
    else
        k_probe<K, false><<<h->nsm, PROBE_THREADS, probe_smem(n), s>>>(h->ctx);
    cudaEventRecord(h->ev[5], s);
    k_reduce<<<1, 32, 0, s>>>(h->ctx);  // a6: cross-rank sums (inside the step)
    h->launches += 4;  // local, itemize, probe, reduce
}

}  // namespace

extern "C" {

const char *mgj_strerror(mgj_status s) {
    switch (s) {
        case MGJ_OK: return "ok";
        case MGJ_EINVAL: return "invalid argument or configuration";
        case MGJ_EALIGN: return "device pointer not 16-byte aligned";
        case MGJ_ENOMEM: return "device allocation failed";
        case MGJ_ECUDA: return "CUDA error";
        case MGJ_ESTATE: return "call out of order";
        case MGJ_ECAPACITY: return "capacity exceeded";
        case MGJ_EPEER: return "peer signal timeout";
    }
    return "unknown status";
}

uint64_t mgj_arena_bytes(const mgj_config *cfg) {
    Norm n;
    if (normalize(cfg, &n) != MGJ_OK) return 0;
    return n.lay.total;
}

mgj_status mgj_plan(const mgj_config *cfg, const mgj_peers *peers, mgj_handle *out) {
    if (!out) return MGJ_EINVAL;
    *out = nullptr;
    Norm n;
    mgj_status st = normalize(cfg, &n);
    if (st != MGJ_OK) return st;
    const int W = n.c.world_size;
    if (W > 1) {
        if (!peers || !peers->arena_ptrs || peers->arena_bytes < n.lay.total) return MGJ_EINVAL;
        for (int g = 0; g < W; ++g)
            if (!peers->arena_ptrs[g] || ((uintptr_t)peers->arena_ptrs[g] & 15)) return MGJ_EALIGN;
    } else if (peers && peers->arena_ptrs) {
        if (peers->arena_bytes < n.lay.total || !peers->arena_ptrs[0]) return MGJ_EINVAL;
        if ((uintptr_t)peers->arena_ptrs[0] & 15) return MGJ_EALIGN;  // TMA reads the receive buffers
    }
    mgj_plan_s *h = new (std::nothrow) mgj_plan_s();
    if (!h) return MGJ_ENOMEM;
    h->n = n;
    if ((st = cuda_ok(cudaGetDevice(&h->dev))) != MGJ_OK) { delete h; return st; }
    int nsm = 0;
    cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, h->dev);
    h->nsm = n.c.num_sms ? std::min(n.c.num_sms, nsm) : nsm;
    if (h->nsm <= 0) { delete h; return MGJ_ECUDA; }

    if (peers && peers->arena_ptrs) {
        for (int g = 0; g < W; ++g) h->arena[g] = static_cast<char *>(peers->arena_ptrs[g]);
    } else {
        h->own_arena = static_cast<char *>(dalloc(h, n.lay.total, &st));
        if (st == MGJ_OK) st = cuda_ok(cudaMemset(h->own_arena, 0, n.lay.total));
        h->arena[0] = h->own_arena;
    }
    const int P = n.P;
    const uint64_t Qm = 1ull << n.b2_max;
    // §8(e) overlap: R's local pass on a second stream beside S's scatter;
    // NEXT-3 streaming adds S's local pass there, chunk by chunk
    const bool ext = n.c.shuffle_mode == MGJ_SHUFFLE_EXTERNAL;
    h->overlap = !ext && (n.c.shuffle_overlap > 0 || (n.c.shuffle_overlap == 0 && W > 1));
    const bool stream = !ext && n.c.shuffle_overlap == 2;
    if (h->overlap) {
        h->local_sms = n.c.overlap_local_sms ? std::min(n.c.overlap_local_sms, h->nsm - 1) : h->nsm / 2;
        if (stream && W > 1) {
            // ranks sharing this GPU (virtual ranks): their streaming local
            // passes wait inside the kernel for the others' scatter, so they
            // may hold at most half the SMs together
            bool colocated = false;
            for (int g = 0; g < W; ++g) {
                cudaPointerAttributes a;
                if (g != n.c.rank && cudaPointerGetAttributes(&a, h->arena[g]) == cudaSuccess && a.device == h->dev)
                    colocated = true;
            }
            (void)cudaGetLastError();
            if (colocated) h->local_sms = std::min(h->local_sms, h->nsm / (2 * W));
        }
        h->local_sms = std::max(h->local_sms, 1);
        h->scatter_sms = std::max(h->nsm - h->local_sms, 1);
    }
    // scatter tiles per relation: one per SM, or (streaming) STREAM_TPC per
    // S scatter CTA, in at most STREAM_RMAX rounds
    const int G = stream ? std::min(h->nsm * STREAM_TPC, STREAM_RMAX * h->scatter_sms) : h->nsm;
    if (n.c.compress && G > COMP_MAX_TILES) {  // the receive capacity in units assumes at most this many
        mgj_destroy(h);
        return MGJ_EINVAL;
    }
    // per-run zero block: rank_hist, ticket, meta, acc, err, cop_slots
    size_t zo = 0;
    const size_t z_hist = zo; zo += align_up(2ull * P * 4, 256);
    const size_t z_tick = zo; zo += 256;
    const size_t z_meta = zo; zo += 256;
    const size_t z_acc = zo; zo += 256;
    const size_t z_err = zo; zo += 256;
    const size_t z_cop = zo; zo += align_up(2ull * P * Qm * 4, 256);
    const size_t z_th = zo; zo += align_up(2ull * G * P * 4, 256);
    const size_t z_rc = zo; zo += 256;  // streaming: chunks per round + cursors
    const size_t z_ha = zo; zo += align_up(2ull * local2_vcap(P) * 4, 256);
    h->zero_bytes = zo;
    char *zb = static_cast<char *>(dalloc(h, zo, &st));
    h->zero_block = zb;
    Ctx &c = h->ctx;
    c.rank = n.c.rank;
    c.world = W;
    c.B1 = n.B1;
    c.P = P;
    c.b2_cfg = n.c.radix_bits_local;
    c.b2_max = n.b2_max;
    c.G = G;
    c.hist_split = G > h->nsm ? 1 : 2;  // k_hist: two CTAs per SM
    c.stream = stream;
    c.sgrid = stream ? h->scatter_sms : 0;
    c.nrounds = stream ? (G + c.sgrid - 1) / c.sgrid : 0;
    c.chunk_tuples = n.chunk_tuples;
    c.chunk_region = n.chunk_region;
    c.chunk_tuples2 = n.chunk_tuples2;
    c.chunk_region2 = n.chunk_region2;
    c.qm2_bits = n.qm2_bits;
    c.chunk_tuples1s = n.chunk_tuples1s;
    c.probe_slots = n.probe_slots;
    c.probe_target = n.probe_target;
    c.materialize = n.c.materialize;
    c.timeout_ns = (n.c.peer_timeout_ms ? (uint64_t)n.c.peer_timeout_ms : 20000ull) * 1000000ull;
    c.ext = n.c.shuffle_mode == MGJ_SHUFFLE_EXTERNAL;
    c.comp = n.c.compress;
    c.assign = n.c.assign;
    c.chunk_units = CHUNK_UNITS;
    c.max_items = (uint32_t)n.max_items;
    c.recv_cap[0] = n.recv_cap[0];
    c.recv_cap_u[0] = n.recv_cap_u[0];
    c.recv_cap_u[1] = n.recv_cap_u[1];
    c.recv_cap[1] = n.recv_cap[1];
    c.max_chunks = n.max_chunks;
    c.out_cap = n.out_cap;
    c.lay = n.lay;
    for (int g = 0; g < MAX_RANKS; ++g) c.arena[g] = h->arena[g];
    if (zb) {
        c.rank_hist = reinterpret_cast<uint32_t *>(zb + z_hist);
        c.ticket = reinterpret_cast<uint32_t *>(zb + z_tick);
        c.meta = reinterpret_cast<int32_t *>(zb + z_meta);
        c.acc = reinterpret_cast<unsigned long long *>(zb + z_acc);
        c.err = reinterpret_cast<int32_t *>(zb + z_err);
        c.cop_slots = reinterpret_cast<uint32_t *>(zb + z_cop);
        c.tile_hist = reinterpret_cast<uint32_t *>(zb + z_th);
        c.hA = reinterpret_cast<uint32_t *>(zb + z_ha);
        c.rcount = reinterpret_cast<uint32_t *>(zb + z_rc);
    }
    c.tile_base = static_cast<uint32_t *>(dalloc(h, 2ull * c.G * P * 4, &st));
    if (c.comp) {
        c.rowbase = static_cast<uint32_t *>(dalloc(h, 2ull * MAX_RANKS * c.G * 4, &st));
        c.rank_units = static_cast<uint32_t *>(dalloc(h, 2ull * P * 4, &st));
    }
    c.scat_T = scat_T_of(n);
    c.sub_ns = (int32_t)((std::max(n.c.r_capacity, n.c.s_capacity) / c.G + 8) / c.scat_T + 2);
    c.sub_hist = static_cast<uint16_t *>(dalloc(h, 2ull * c.G * c.sub_ns * P * 2, &st));
    h->cdesc = static_cast<ChunkDesc *>(dalloc(h, 2 * n.max_chunks * sizeof(ChunkDesc), &st));
    if (stream) {
        c.cwait = static_cast<uint32_t *>(dalloc(h, n.max_chunks * 4, &st));
        c.corder = static_cast<uint32_t *>(dalloc(h, n.max_chunks * 4, &st));
    }
    if (n.split) h->cdescB = static_cast<ChunkDescB *>(dalloc(h, 2 * n.max_chunks * sizeof(ChunkDescB), &st));
    c.owner = static_cast<int32_t *>(dalloc(h, P * 4, &st));
    c.bcast = static_cast<uint8_t *>(dalloc(h, P, &st));
    c.pskip = static_cast<uint8_t *>(dalloc(h, P, &st));
    c.plist = static_cast<int32_t *>(dalloc(h, P * 4, &st));
    c.bcast_cfg = n.c.skew_bcast;
    c.send_off = static_cast<uint64_t *>(dalloc(h, 2ull * P * 8, &st));
    c.seg_start = static_cast<uint64_t *>(dalloc(h, 2ull * P * 8, &st));
    c.seg_len = static_cast<uint64_t *>(dalloc(h, 2ull * P * 8, &st));
    c.recv_size = static_cast<uint64_t *>(dalloc(h, 2ull * MAX_RANKS * 8, &st));
    c.piece_start = static_cast<uint64_t *>(dalloc(h, 2ull * P * MAX_RANKS * 8, &st));
    c.piece_len = static_cast<uint32_t *>(dalloc(h, 2ull * P * MAX_RANKS * 4, &st));
    c.piece_chunk = static_cast<uint32_t *>(dalloc(h, 2ull * P * (MAX_RANKS + 1) * 4, &st));
    c.ext_counts = static_cast<uint64_t *>(dalloc(h, 2ull * 2 * MAX_RANKS * 8, &st));
    // EXTERNAL shuffle: a send arena with the receive layout; the scatter is
    // launched with every peer pointer aimed at it (tuples land ordered by
    // destination rank, see k_plan)
    if (c.ext) h->send_arena = static_cast<char *>(dalloc(h, n.lay.total, &st));
    c.vcap = local2_vcap(P);
    c.cb_stride = c.vcap + 1;
    c.split_cfg = n.c.local_split_bits;
    c.mid_cap = n.mid_cap;
    c.chunk_base = static_cast<uint32_t *>(dalloc(h, 2ull * c.cb_stride * 4, &st));
    c.chunk_base1 = static_cast<uint32_t *>(dalloc(h, 2ull * c.cb_stride * 4, &st));
    c.chunk_region1 = n.chunk_tuples1s + (1 << MAX_BA);
    for (int r = 0; r < 2 && n.split; ++r) {
        c.mid[r] = dalloc(h, n.mid_cap * n.tuple_bytes, &st);
        c.eoffA[r] = static_cast<uint16_t *>(dalloc(h, n.max_chunks * EA_STRIDE * 2, &st));
    }
    for (int r = 0; r < 2; ++r)
        c.eoff[r] = static_cast<uint16_t *>(dalloc(h, n.max_chunks * (Qm + 1) * 2, &st));
    c.items = static_cast<Item *>(dalloc(h, n.max_items * sizeof(ItemX), &st));
    for (int r = 0; r < 2; ++r)
        c.local[r] = dalloc(h, n.max_chunks * std::max(n.chunk_region, n.chunk_region2) * n.tuple_bytes, &st);
    c.result = static_cast<unsigned long long *>(dalloc(h, 64, &st));
    if (n.c.materialize) {
        c.out_key = dalloc(h, n.out_cap * n.c.key_bytes, &st);
        c.out_a = dalloc(h, n.out_cap * n.c.key_bytes, &st);
        c.out_b = dalloc(h, n.out_cap * n.c.key_bytes, &st);
    }
    if (n.c.trace) c.trace = static_cast<unsigned long long *>(dalloc(h, MGJ_TRACE_COUNT * 2 * 8, &st));
    if (h->overlap) {
        if (st == MGJ_OK) st = cuda_ok(cudaStreamCreateWithFlags(&h->aux, cudaStreamNonBlocking));
        if (st == MGJ_OK) st = cuda_ok(cudaEventCreateWithFlags(&h->ev_fork, cudaEventDisableTiming));
        if (st == MGJ_OK) st = cuda_ok(cudaEventCreateWithFlags(&h->ev_join, cudaEventDisableTiming));
    }
    if (st == MGJ_OK) st = cuda_ok(cudaMallocHost(&h->h_res, 8 * 8 + MT_COUNT * 4));
    if (st == MGJ_OK) h->h_meta = reinterpret_cast<int32_t *>(h->h_res + 8);
    for (int i = 0; i < 7 && st == MGJ_OK; ++i) st = cuda_ok(cudaEventCreate(&h->ev[i]));
    if (st == MGJ_OK) st = cuda_ok(n.c.key_bytes == 4 ? set_attrs<uint32_t>(n) : set_attrs<uint64_t>(n));
    if (st == MGJ_OK) st = cuda_ok(n.c.key_bytes == 4 ? preload_kernels<uint32_t>(n) : preload_kernels<uint64_t>(n));
    if (st != MGJ_OK) {
        mgj_destroy(h);
        return st;
    }
    h->state = ST_PLANNED;
    *out = h;
    return MGJ_OK;
}

mgj_status mgj_partition(mgj_handle h, const void *r_keys, const void *r_payloads, uint64_t n_r,
                         const void *s_keys, const void *s_payloads, uint64_t n_s, void *stream) {
    if (!h) return MGJ_EINVAL;
    if (h->state != ST_PLANNED && h->state != ST_JOINED && h->state != ST_DONE) return MGJ_ESTATE;
    cudaStream_t s = static_cast<cudaStream_t>(stream);
    if (h->state == ST_JOINED && h->stream != s) {  // previous run on another stream: let it finish
        if (cudaStreamSynchronize(h->stream) != cudaSuccess) return MGJ_ECUDA;
    }
    const Norm &n = h->n;
    if (n_r > n.c.r_capacity || n_s > n.c.s_capacity) return MGJ_EINVAL;
    if ((n_r && (!r_keys || !r_payloads)) || (n_s && (!s_keys || !s_payloads))) return MGJ_EINVAL;
    const void *ptr[4] = {r_keys, r_payloads, s_keys, s_payloads};
    const uint64_t cnt[4] = {n_r, n_r, n_s, n_s};
    const size_t w = n.c.key_bytes;
    bool host[4];
    size_t need = 0;
    for (int i = 0; i < 4; ++i) {
        host[i] = cnt[i] && !is_device_ptr(ptr[i]);
        if (host[i]) need += align_up(cnt[i] * w, 256);
        else if (cnt[i] && ((uintptr_t)ptr[i] & 15)) return MGJ_EALIGN;
    }
    if (need > h->stage_bytes) {
        if (h->stage) cudaFree(h->stage);
        h->stage = nullptr;
        h->stage_bytes = 0;
        const size_t cap = align_up(n.c.r_capacity * w, 256) * 2 + align_up(n.c.s_capacity * w, 256) * 2;
        if (cudaMalloc(&h->stage, cap) != cudaSuccess) {
            (void)cudaGetLastError();
            return MGJ_ENOMEM;
        }
        h->stage_bytes = cap;
    }
    const void *dptr[4];
    size_t so = 0;
    for (int i = 0; i < 4; ++i) {
        dptr[i] = ptr[i];
        if (host[i]) {
            char *d = static_cast<char *>(h->stage) + so;
            if (cudaMemcpyAsync(d, ptr[i], cnt[i] * w, cudaMemcpyHostToDevice, s) != cudaSuccess) return MGJ_ECUDA;
            dptr[i] = d;
            so += align_up(cnt[i] * w, 256);
        }
    }
    h->epoch += 1;
    Ctx &c = h->ctx;
    c.epoch = h->epoch;
    c.in_key[0] = dptr[0];
    c.in_pay[0] = dptr[1];
    c.in_key[1] = dptr[2];
    c.in_pay[1] = dptr[3];
    c.n_in[0] = n_r;
    c.n_in[1] = n_s;
    h->stream = s;
    if (cudaMemsetAsync(h->zero_block, 0, h->zero_bytes, s) != cudaSuccess) return MGJ_ECUDA;
    if (c.trace && cudaMemsetAsync(c.trace, 0, MGJ_TRACE_COUNT * 2 * 8, s) != cudaSuccess) return MGJ_ECUDA;
    cudaEventRecord(h->ev[0], s);
    if (n.c.key_bytes == 4) launch_partition<uint32_t>(h, s);
    else launch_partition<uint64_t>(h, s);
    cudaEventRecord(h->ev[1], s);
    if (cudaGetLastError() != cudaSuccess) return MGJ_ECUDA;
    h->state = ST_PARTITIONED;
    return MGJ_OK;
}

mgj_status mgj_shuffle(mgj_handle h, void *stream) {
    if (!h) return MGJ_EINVAL;
    if (h->state != ST_PARTITIONED) return MGJ_ESTATE;
    cudaStream_t s = static_cast<cudaStream_t>(stream);
    h->stream = s;
    if (h->n.c.key_bytes == 4) launch_shuffle<uint32_t>(h, s);
    else launch_shuffle<uint64_t>(h, s);
    cudaEventRecord(h->ev[3], s);
    if (cudaGetLastError() != cudaSuccess) return MGJ_ECUDA;
    h->state = ST_SHUFFLED;
    return MGJ_OK;
}

mgj_status mgj_join(mgj_handle h, void *stream) {
    if (!h) return MGJ_EINVAL;
    if (h->state != ST_SHUFFLED) return MGJ_ESTATE;
    cudaStream_t s = static_cast<cudaStream_t>(stream);
    h->stream = s;
    if (h->n.c.key_bytes == 4) launch_join<uint32_t>(h, s);
    else launch_join<uint64_t>(h, s);
    cudaEventRecord(h->ev[6], s);
    if (cudaGetLastError() != cudaSuccess) return MGJ_ECUDA;
    h->state = ST_JOINED;
    return MGJ_OK;
}

mgj_status mgj_result(mgj_handle h, mgj_result_t *out) {
    if (!h || !out) return MGJ_EINVAL;
    if (h->state != ST_JOINED && h->state != ST_DONE) return MGJ_ESTATE;
    if (h->state == ST_JOINED) {  // read back the sums k_reduce (end of mgj_join) left
        cudaMemcpyAsync(h->h_res, h->ctx.result, 8 * 8, cudaMemcpyDeviceToHost, h->stream);
        cudaMemcpyAsync(h->h_meta, h->ctx.meta, MT_COUNT * 4, cudaMemcpyDeviceToHost, h->stream);
    }
    if (cudaStreamSynchronize(h->stream) != cudaSuccess) return MGJ_ECUDA;
    memset(out, 0, sizeof(*out));
    const Ctx &c = h->ctx;
    uint64_t rs[2 * MAX_RANKS] = {};
    if (cudaMemcpy(rs, c.recv_size, sizeof(rs), cudaMemcpyDeviceToHost) != cudaSuccess) return MGJ_ECUDA;
    unsigned long long acc[4] = {};
    if (cudaMemcpy(acc, c.acc, sizeof(acc), cudaMemcpyDeviceToHost) != cudaSuccess) return MGJ_ECUDA;
    out->match_count = h->h_res[0];
    out->checksum = h->h_res[1];
    out->local_count = acc[0];
    out->local_checksum = acc[1];
    out->pair_digest = h->h_res[4];
    out->local_pair_digest = acc[3];
    out->n_materialized = std::min<uint64_t>(h->h_res[2], h->n.out_cap);
    out->out_key = c.out_key;
    out->out_payload_r = c.out_a;
    out->out_payload_s = c.out_b;
    out->recv_r = rs[c.rank];
    out->recv_s = rs[MAX_RANKS + c.rank];
    for (int i = 0; i < 6; ++i) {
        float ms = 0.f;
        cudaEventElapsedTime(&ms, h->ev[i], h->ev[i + 1]);
        out->phase_ms[i] = ms;
    }
    out->status = (int32_t)(uint32_t)h->h_res[3];
    out->radix_bits_global = h->n.B1;
    out->radix_bits_local = h->h_meta[MT_B2];
    out->n_items = (int32_t)std::min<uint64_t>(h->h_meta[MT_NITEMS] ? h->h_meta[MT_NITEMS] : 0, h->n.max_items);
    unsigned int ni = 0;
    cudaMemcpy(&ni, c.ticket + TK_ITEMS, 4, cudaMemcpyDeviceToHost);
    out->n_items = (int32_t)std::min<uint64_t>(ni, h->n.max_items);
    out->n_launches = h->launches;
    h->state = ST_DONE;
    return (mgj_status)out->status;
}

mgj_status mgj_exchange_layout(mgj_handle h, mgj_exchange_t *out) {
    if (!h || !out) return MGJ_EINVAL;
    if (!h->ctx.ext) return MGJ_EINVAL;
    if (h->state != ST_SHUFFLED) return MGJ_ESTATE;
    if (cudaStreamSynchronize(h->stream) != cudaSuccess) return MGJ_ECUDA;
    memset(out, 0, sizeof(*out));
    uint64_t cnt[2 * 2 * MAX_RANKS];
    if (cudaMemcpy(cnt, h->ctx.ext_counts, sizeof(cnt), cudaMemcpyDeviceToHost) != cudaSuccess) return MGJ_ECUDA;
    for (int rel = 0; rel < 2; ++rel) {
        out->send[rel] = h->send_arena + h->n.lay.recv[rel];
        out->recv[rel] = h->arena[h->ctx.rank] + h->n.lay.recv[rel];
        for (int g = 0; g < MAX_RANKS; ++g) {
            out->send_count[rel][g] = g < h->ctx.world ? cnt[(0 * 2 + rel) * MAX_RANKS + g] : 0;
            out->recv_count[rel][g] = g < h->ctx.world ? cnt[(1 * 2 + rel) * MAX_RANKS + g] : 0;
        }
    }
    out->tuple_bytes = h->n.tuple_bytes;
    out->world_size = h->ctx.world;
    return MGJ_OK;
}

void mgj_destroy(mgj_handle h) {
    if (!h) return;
    if (h->stream) cudaStreamSynchronize(h->stream);
    for (int i = 0; i < h->nalloc; ++i) cudaFree(h->allocs[i]);
    if (h->stage) cudaFree(h->stage);
    if (h->h_res) cudaFreeHost(h->h_res);
    for (int i = 0; i < 7; ++i)
        if (h->ev[i]) cudaEventDestroy(h->ev[i]);
    if (h->aux) {
        cudaStreamSynchronize(h->aux);
        cudaStreamDestroy(h->aux);
    }
    if (h->ev_fork) cudaEventDestroy(h->ev_fork);
    if (h->ev_join) cudaEventDestroy(h->ev_join);
    delete h;
}

mgj_status mgj_plan_host(int32_t world_size, int32_t rank, int32_t bits, const uint32_t *hist, int32_t *owner,
                         uint64_t *send_off, uint64_t *recv_size, int32_t skew_bcast, uint8_t *bcast,
                         uint8_t *skip, int32_t assign) {
    if (world_size < 1 || world_size > MAX_RANKS || rank < 0 || rank >= world_size || bits < 1 || bits > MAX_B1 ||
        !hist || !owner || !send_off || !recv_size || skew_bcast < -1 || skew_bcast > 1 || assign < 0 || assign > 1)
        return MGJ_EINVAL;
    const int P = 1 << bits, N = world_size;
    auto H = [&](int g, int rel, int p) -> uint64_t { return hist[((size_t)g * 2 + rel) * P + p]; };
    uint64_t *tot = new (std::nothrow) uint64_t[2 * (size_t)P];
    uint64_t *pre = new (std::nothrow) uint64_t[2 * (size_t)P];  // R prefix; S prefix over non-broadcast partitions
    uint8_t *bc = new (std::nothrow) uint8_t[(size_t)P];
    if (!tot || !pre || !bc) {
        delete[] tot;
        delete[] pre;
        delete[] bc;
        return MGJ_ENOMEM;
    }
    uint64_t s_total = 0;
    for (int p = 0; p < P; ++p) {
        for (int rel = 0; rel < 2; ++rel) {
            uint64_t t = 0;
            for (int g = 0; g < N; ++g) t += H(g, rel, p);
            tot[rel * P + p] = t;
        }
        const bool sk = skip_of(tot[p], tot[P + p]);
        if (skip) skip[p] = sk;
        if (sk) tot[p] = tot[P + p] = 0;
        s_total += tot[P + p];
    }
    uint64_t total = 0, run[2] = {0, 0};
    for (int p = 0; p < P; ++p) {
        bc[p] = bcast_of(tot[p], tot[P + p], s_total, N, P, skew_bcast);
        if (bcast) bcast[p] = bc[p];
        total += owner_weight(tot[p], tot[P + p], bc[p], N);
        pre[p] = run[0];
        run[0] += tot[p];
        pre[P + p] = run[1];
        run[1] += bc[p] ? 0 : tot[P + p];
    }
    if (assign) {  // placement-aware (k_plan's assign branch, same formulas)
        assign_greedy(
            N, P, [&](int p) { return owner_weight(tot[p], tot[P + p], bc[p], N); },
            [&](int p) {
                int b = 0;
                uint64_t hb = 0;
                for (int g = 0; g < N; ++g) {
                    const uint64_t h = H(g, 0, p) + (bc[p] ? 0 : H(g, 1, p));
                    if (h > hb) hb = h, b = g;
                }
                return b;
            },
            owner);
        uint64_t run[2][MAX_RANKS] = {};
        for (int p = 0; p < P; ++p)
            for (int rel = 0; rel < 2; ++rel) {
                if (rel && bc[p]) continue;
                uint64_t m = 0;
                for (int g = 0; g < rank; ++g) m += H(g, rel, p);
                send_off[rel * P + p] = run[rel][owner[p]] + m;
                run[rel][owner[p]] += tot[rel * P + p];
            }
        uint64_t own_bc = 0;
        for (int p = 0; p < P; ++p)
            if (bc[p]) {
                send_off[P + p] = run[1][rank] + own_bc;
                own_bc += H(rank, 1, p);
            }
        for (int rel = 0; rel < 2; ++rel)
            for (int d = 0; d < N; ++d) {
                uint64_t sz = run[rel][d];
                if (rel)
                    for (int p = 0; p < P; ++p) sz += bc[p] ? H(d, 1, p) : 0;
                recv_size[rel * N + d] = sz;
            }
        delete[] tot;
        delete[] pre;
        delete[] bc;
        return MGJ_OK;
    }
    uint64_t cum = 0;
    int first[MAX_RANKS], endp[MAX_RANKS];
    for (int d = 0; d < MAX_RANKS; ++d) first[d] = endp[d] = P;
    for (int p = 0; p < P; ++p) {
        const uint64_t T = owner_weight(tot[p], tot[P + p], bc[p], N);
        owner[p] = owner_of(cum, T, total, N, p, P);
        cum += T;
    }
    for (int p = 0; p < P; ++p) {
        if (p == 0 || owner[p - 1] != owner[p]) first[owner[p]] = p;
        if (p == P - 1 || owner[p + 1] != owner[p]) endp[owner[p]] = p + 1;
    }
    auto range_size = [&](int rel, int d) -> uint64_t {  // non-broadcast part of d's receive layout
        if (first[d] >= P) return 0;
        const int l = endp[d] - 1;
        return pre[rel * P + l] + (rel && bc[l] ? 0 : tot[rel * P + l]) - pre[rel * P + first[d]];
    };
    uint64_t own_bc = 0;  // this rank's S tuples of broadcast partitions before p
    for (int p = 0; p < P; ++p) {
        uint64_t m0 = 0, m1 = 0;
        for (int g = 0; g < rank; ++g) m0 += H(g, 0, p), m1 += H(g, 1, p);
        send_off[p] = pre[p] - pre[first[owner[p]]] + m0;
        if (bc[p]) {
            send_off[P + p] = range_size(1, rank) + own_bc;
            own_bc += H(rank, 1, p);
        } else {
            send_off[P + p] = pre[P + p] - pre[P + first[owner[p]]] + m1;
        }
    }
    for (int rel = 0; rel < 2; ++rel)
        for (int d = 0; d < N; ++d) {
            uint64_t sz = range_size(rel, d);
            if (rel)
                for (int p = 0; p < P; ++p) sz += bc[p] ? H(d, 1, p) : 0;
            recv_size[rel * N + d] = sz;
        }
    delete[] tot;
    delete[] pre;
    delete[] bc;
    return MGJ_OK;
}

mgj_status mgj_gen_relation(int32_t kind, int32_t rel, uint64_t n_r, uint64_t n_s, double z, uint64_t row0,
                            uint64_t count, void *keys, void *payloads, void *stream) {
    if (kind < 0 || kind > 2 || rel < 0 || rel > 1) return MGJ_EINVAL;
    if (count && (!keys || !payloads)) return MGJ_EINVAL;
    const uint64_t n = rel == 0 ? n_r : n_s;
    if (n == 0 || n > (1ull << 32) || row0 + count > n) return MGJ_EINVAL;
    int zmode = 0;
    if (kind == 1) {
        if (n_r & (n_r - 1)) return MGJ_EINVAL;
        if (z == 0.0) zmode = 0;
        else if (z == 0.5) zmode = 1;
        else if (z == 1.0) zmode = 2;
        else return MGJ_EINVAL;
    }
    if (!count) return MGJ_OK;
    int dev = 0, nsm = 148;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
    const uint64_t blocks = std::min<uint64_t>((count + 255) / 256, (uint64_t)nsm * 16);
    mgj_gen::k_gen<<<(unsigned)blocks, 256, 0, static_cast<cudaStream_t>(stream)>>>(kind, rel, n_r, n_s, zmode, row0,
                                                                                    count, keys, payloads);
    return cudaGetLastError() == cudaSuccess ? MGJ_OK : MGJ_ECUDA;
}

mgj_status mgj_debug_copy(mgj_handle h, int32_t what, void *dst, uint64_t bytes, uint64_t *size_out) {
    if (!h) return MGJ_EINVAL;
    if (cudaDeviceSynchronize() != cudaSuccess) return MGJ_ECUDA;
    const Ctx &c = h->ctx;
    const Norm &n = h->n;
    const int P = n.P;
    int32_t meta[MT_COUNT];
    if (cudaMemcpy(meta, c.meta, sizeof(meta), cudaMemcpyDeviceToHost) != cudaSuccess) return MGJ_ECUDA;
    uint64_t rs[2 * MAX_RANKS];
    if (cudaMemcpy(rs, c.recv_size, sizeof(rs), cudaMemcpyDeviceToHost) != cudaSuccess) return MGJ_ECUDA;
    const int Q = 1 << meta[MT_QB];  // runs per chunk of the chunked pass
    const uint64_t nchl[2] = {(uint64_t)(uint32_t)meta[meta[MT_BA] ? MT_NCHB_R : MT_NCH_R],
                              (uint64_t)(uint32_t)meta[meta[MT_BA] ? MT_NCHB_S : MT_NCH_S]};
    const void *src = nullptr;
    uint64_t size = 0;
    switch (what) {
        case MGJ_DBG_RANK_HIST: src = c.rank_hist; size = 2ull * P * 4; break;
        case MGJ_DBG_MAIL_HIST: src = h->arena[c.rank] + n.lay.mail; size = (uint64_t)c.world * 2 * P * 4; break;
        case MGJ_DBG_OWNER: src = c.owner; size = (uint64_t)P * 4; break;
        case MGJ_DBG_BCAST: src = c.bcast; size = (uint64_t)P; break;
        case MGJ_DBG_SKIP: src = c.pskip; size = (uint64_t)P; break;
        case MGJ_DBG_PLIST: src = c.plist; size = (uint64_t)std::max(meta[MT_NP], 0) * 4; break;
        case MGJ_DBG_SEND_OFF: src = c.send_off; size = 2ull * P * 8; break;
        case MGJ_DBG_RECV_SIZE: src = c.recv_size; size = sizeof(rs); break;
        case MGJ_DBG_RECV_R: src = h->arena[c.rank] + n.lay.recv[0]; size = rs[c.rank] * n.tuple_bytes; break;
        case MGJ_DBG_RECV_S:
            src = h->arena[c.rank] + n.lay.recv[1];
            size = rs[MAX_RANKS + c.rank] * n.tuple_bytes;
            break;
        case MGJ_DBG_LOCAL_R:
            src = c.local[0];
            size = nchl[0] * (meta[MT_BA] ? n.chunk_region2 : n.chunk_region) * n.tuple_bytes;
            break;
        case MGJ_DBG_LOCAL_S:
            src = c.local[1];
            size = nchl[1] * (meta[MT_BA] ? n.chunk_region2 : n.chunk_region) * n.tuple_bytes;
            break;
        case MGJ_DBG_META: src = c.meta; size = sizeof(meta); break;
        case MGJ_DBG_CHUNK_OFF_R: src = c.eoff[0]; size = nchl[0] * (Q + 1) * 2; break;
        case MGJ_DBG_CHUNK_OFF_S: src = c.eoff[1]; size = nchl[1] * (Q + 1) * 2; break;
        case MGJ_DBG_CHUNK_BASE: src = c.chunk_base; size = 2ull * c.cb_stride * 4; break;
        case MGJ_DBG_MID_R:
        case MGJ_DBG_MID_S: {
            if (!meta[MT_BA]) return MGJ_EINVAL;
            const int r = what == MGJ_DBG_MID_S;
            src = c.mid[r];  // the first pass's chunks in place, chunk_region1 slots each
            size = (uint64_t)meta[MT_NCH_R + r] * c.chunk_region1 * n.tuple_bytes;
            break;
        }
        case MGJ_DBG_MID_OFF_R:
        case MGJ_DBG_MID_OFF_S: {
            if (!meta[MT_BA]) return MGJ_EINVAL;
            const int r = what == MGJ_DBG_MID_OFF_S;
            src = c.eoffA[r];
            size = (uint64_t)meta[MT_NCH_R + r] * EA_STRIDE * 2;
            break;
        }
        case MGJ_DBG_TRACE: {
            if (!c.trace) return MGJ_EINVAL;
            unsigned long long t[MGJ_TRACE_COUNT * 2];
            if (cudaMemcpy(t, c.trace, sizeof(t), cudaMemcpyDeviceToHost) != cudaSuccess) return MGJ_ECUDA;
            for (int i = 0; i < MGJ_TRACE_COUNT; ++i)
                if (t[2 * i]) t[2 * i] = ~t[2 * i];  // stored as UINT64_MAX - first start
            if (size_out) *size_out = sizeof(t);
            if (dst && bytes) memcpy(dst, t, std::min<uint64_t>(bytes, sizeof(t)));
            return MGJ_OK;
        }
        case MGJ_DBG_OUT_KEY:
        case MGJ_DBG_OUT_PAY_R:
        case MGJ_DBG_OUT_PAY_S: {
            if (!n.c.materialize) return MGJ_EINVAL;
            unsigned long long no = 0;
            if (cudaMemcpy(&no, c.acc + 2, 8, cudaMemcpyDeviceToHost) != cudaSuccess) return MGJ_ECUDA;
            src = what == MGJ_DBG_OUT_KEY ? c.out_key : (what == MGJ_DBG_OUT_PAY_R ? c.out_a : c.out_b);
            size = std::min<uint64_t>(no, n.out_cap) * n.c.key_bytes;
            break;
        }
        case MGJ_DBG_SEGMENTS: {
            if (size_out) *size_out = 4ull * P * 8;
            if (!dst) return MGJ_OK;
            uint64_t tmp[4 * 4096];
            if (cudaMemcpy(tmp, c.seg_start, 2ull * P * 8, cudaMemcpyDeviceToHost) != cudaSuccess) return MGJ_ECUDA;
            if (cudaMemcpy(tmp + 2 * P, c.seg_len, 2ull * P * 8, cudaMemcpyDeviceToHost) != cudaSuccess)
                return MGJ_ECUDA;
            memcpy(dst, tmp, std::min<uint64_t>(bytes, 4ull * P * 8));
            return MGJ_OK;
        }
        default: return MGJ_EINVAL;
    }
    if (size_out) *size_out = size;
    if (!dst || !bytes) return MGJ_OK;
    return cudaMemcpy(dst, src, std::min(bytes, size), cudaMemcpyDeviceToHost) == cudaSuccess ? MGJ_OK : MGJ_ECUDA;
}

}  // extern "C"
