/*
 * mgj.h — C ABI of libmgj.so, the B200-native hot path of MG-Join
 * (Paul, Lu, He, Lau, "MG-Join: A Scalable Join for Massively Parallel
 * Multi-GPU Architectures", SIGMOD '21; text in PAPER.md, cited P:line).
 *
 * The operation: an equi-join of two relations R and S of fixed-width
 * (key, payload) tuples, "distributed over multiple GPUs in the same
 * machine", inputs "evenly distributed" and resident on the
 * GPUs, 4-byte key + 4-byte id tuples;
 * the result must not depend on data placement.  The join runs
 * the paper's four phases: histogram generation,
 * global partitioning = partition + assignment + data distribution
 * (§4), local partitioning and probe.
 *
 * Result (readings C1-C3, C3b): match count, a 64-bit checksum
 *   checksum = sum over matches (k,a,b) of (a*C + b) mod 2^64,
 *   C = 2^32 for 4-byte payloads, 0x9E3779B97F4A7C15 for 8-byte payloads,
 * a 64-bit pair digest
 *   pair_digest = sum over matches (k,a,b) of a*b mod 2^64,
 * and optionally the materialised (key, payloadR, payloadS) triples (bag
 * semantics: every equal-key (R,S) pair once).
 *
 * Conventions
 *  - Every call returns mgj_status (0 = MGJ_OK, < 0 = error); nothing throws
 *    or aborts.  Argument/state errors (EINVAL, EALIGN, ESTATE) are returned
 *    synchronously.  Device-side errors (ECUDA, EPEER on a peer-signal
 *    timeout, ECAPACITY when a receive/output buffer would overflow) are
 *    sticky per run and returned by mgj_result.
 *  - Collective calls (mgj_plan, mgj_partition, mgj_shuffle, mgj_join) must
 *    be made by every rank in the same order, like NCCL.  They only enqueue
 *    work on the given CUDA stream (passed as void*, a cudaStream_t) and
 *    return.  Several ranks may live in ONE process on ONE GPU ("virtual
 *    ranks", each with its own handle and its own stream): then call each
 *    phase for all ranks before the next phase.
 *  - Ownership: input columns are borrowed (valid until mgj_join's work has
 *    completed).  The handle owns its workspace and the materialised output
 *    (valid until the next mgj_partition or mgj_destroy).  A caller-provided
 *    symmetric arena (mgj_peers) is owned by the caller and must outlive the
 *    handle.
 */
#ifndef MGJ_H
#define MGJ_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
    MGJ_OK = 0,
    MGJ_EINVAL = -1,     /* bad argument / config */
    MGJ_EALIGN = -2,     /* a device pointer is not 16-byte aligned */
    MGJ_ENOMEM = -3,     /* device allocation failed */
    MGJ_ECUDA = -4,      /* a CUDA runtime call or kernel failed */
    MGJ_ESTATE = -5,     /* call out of order (plan -> partition -> shuffle -> join -> result) */
    MGJ_ECAPACITY = -6,  /* receive / chunk / work-item / output capacity exceeded */
    MGJ_EPEER = -7       /* a peer did not signal within the timeout */
} mgj_status;

enum { MGJ_MAX_RANKS = 8 };

typedef struct {
    int32_t  rank, world_size;         /* 0 <= rank < world_size <= 8; one handle per rank */
    int32_t  key_bytes, payload_bytes; /* {4,4} (paper's tuples) or {8,8} */
    uint64_t r_capacity, s_capacity;   /* max local tuples this rank passes to mgj_partition */
    uint64_t recv_capacity_r;          /* tuples of R this rank can receive (0 = auto) */
    uint64_t recv_capacity_s;          /* tuples of S this rank can receive (0 = auto); identical on all ranks */
    int32_t  radix_bits_global;        /* B1: 2^B1 global partitions, Eq. 1 analogue (0 = auto = 10) */
    int32_t  radix_bits_local;         /* B2: local fan-out per pass (0 = auto from sizes, chosen on device) */
    int32_t  materialize;              /* 0/1: emit (key, payR, payS) triples */
    int32_t  num_sms;                  /* 0 = device attribute */
    uint64_t out_capacity;             /* max materialised triples on this rank (0 = auto) */
    int32_t  shuffle_mode;             /* MGJ_SHUFFLE_P2P (0, default) | MGJ_SHUFFLE_EXTERNAL (1) */
    int32_t  local_split_bits;         /* a4 first (histogram) pass: 0 = auto (only for owned partitions
                                          of more than 256 chunks), -1 = never, 1..6 = always, 2^k
                                          sub-partitions per owned partition */
    int32_t  skew_bcast;               /* a2 selective broadcast:
                                          0 = auto (heavy partitions with (N-1)|R_p| < |S_p|: R_p is read by
                                          every rank from its owner, S_p stays where it is), -1 = never,
                                          1 = every partition passing the traffic test.  Never with one
                                          rank or MGJ_SHUFFLE_EXTERNAL */
    int32_t  peer_timeout_ms;          /* bound on every wait for a peer's signal (0 = 20000 ms); a wait
                                          that times out makes the run fail with MGJ_EPEER */
    int32_t  shuffle_overlap;          /* SURVEY.md §8(e) / P:455-468: local-partition R (on a second
                                          stream, overlap_local_sms SMs) while S is still being shuffled
                                          (the rest of the SMs).  0 = auto (on for world_size > 1 with
                                          MGJ_SHUFFLE_P2P), 1 = on, -1 = off.  Never with EXTERNAL.
                                          2 = on, plus chunk streaming (NEXT-3): S's local
                                          pass also runs on the second stream, beside S's scatter, and
                                          starts each received chunk as soon as the scatter rounds that
                                          fill it are complete at every source rank (S tiles complete in
                                          rounds; each completed tile is counted at every owner, which
                                          waits in the kernel, bounded by peer_timeout_ms).  P2P only.
                                          Ranks sharing one GPU (virtual ranks) then hold at most half the
                                          SMs with their local passes together */
    int32_t  overlap_local_sms;        /* SMs of R's local pass during the overlap (0 = half the SMs) */
    int32_t  trace;                    /* 1: record the first start and last end (globaltimer, ns) of
                                          every kernel of the run (mgj_debug_copy MGJ_DBG_TRACE) */
    int32_t  compress;                 /* NEXT-1: 1 = compress the shuffle.  Needs 4-byte keys,
                                          MGJ_SHUFFLE_P2P and payloads that are global row ids (rank g's
                                          row i has payload sum_{g'<g} n_g' + i, the paper's id column;
                                          checked per tuple, a run that breaks it fails with MGJ_EINVAL).
                                          A tuple travels as its key without the B1 partition bits plus
                                          its row's offset in its source tile, five per 32-byte unit
                                          (+ source rank, tile, count): 6.4 instead of 8 bytes.  Forces a
                                          single local pass */
    int32_t  assign;                   /* a2 partition assignment: 0 = contiguous ranges balanced on counts
                                          (the optimum for random placement on a uniform one-hop fabric);
                                          1 = placement-aware (NEXT-2, the migration step of Track-Join
                                          the paper adopts): each partition goes to the rank
                                          holding most of its tuples unless that rank's load would pass
                                          9/8 of the mean.  MGJ_SHUFFLE_P2P only */
    int32_t  reserved[1];              /* must be zero */
} mgj_config;

/*
 * Shuffle modes.  P2P (the product path): k_scatter stores every tuple
 * straight into its owner's receive buffer through peer-mapped symmetric
 * memory (NVLink/NVSwitch).  EXTERNAL (the measured NCCL baseline): k_scatter
 * packs the tuples into a per-relation send buffer laid out by destination
 * rank, the caller exchanges it with its own collective (e.g. NCCL
 * all_to_all_single) into each rank's receive area between mgj_shuffle and
 * mgj_join, using the sizes from mgj_exchange_layout.
 */
enum { MGJ_SHUFFLE_P2P = 0, MGJ_SHUFFLE_EXTERNAL = 1 };

typedef struct mgj_plan_s *mgj_handle;

/*
 * Peer-mapped symmetric memory (e.g. torch.distributed._symmetric_memory
 * buffer_ptrs).  arena_ptrs[g] is rank g's arena as mapped in THIS process;
 * every arena has the same size >= mgj_arena_bytes(cfg) and must be
 * zero-filled on every rank before any rank calls mgj_partition (caller
 * barrier).  Pass NULL peers when world_size == 1: the handle then
 * allocates its own arena.
 */
typedef struct {
    void *const *arena_ptrs;   /* [world_size] */
    uint64_t     arena_bytes;
} mgj_peers;

typedef struct {
    uint64_t match_count;          /* global (summed over ranks, a6) */
    uint64_t checksum;             /* global, wrapping sum mod 2^64 */
    uint64_t local_count;          /* this rank's co-partitions */
    uint64_t local_checksum;
    uint64_t n_materialized;       /* triples in this rank's output shard */
    const void *out_key;           /* device SoA of n_materialized entries, */
    const void *out_payload_r;     /*   key_bytes wide each; owned by the handle */
    const void *out_payload_s;
    uint64_t recv_r, recv_s;       /* tuples this rank received in the shuffle */
    float    phase_ms[6];          /* device time of: hist, plan, shuffle, local_part, probe, reduce */
    int32_t  status;               /* sticky device status of the run (mgj_status) */
    int32_t  radix_bits_global;    /* B1 used */
    int32_t  radix_bits_local;     /* B2 chosen on device for this rank */
    int32_t  n_items;              /* probe work items (co-partition slices) on this rank */
    int32_t  n_launches;           /* kernels this handle launched for the run (partition .. join) */
    uint64_t pair_digest;          /* global sum over matches (k,a,b) of a*b mod 2^64 (DESIGN.md reading
                                      C3b): bilinear, so it detects a wrong pairing of R and S rows */
    uint64_t local_pair_digest;    /* this rank's co-partitions */
} mgj_result_t;

/* Bytes each rank's symmetric arena needs for cfg (0 if cfg is invalid). */
uint64_t mgj_arena_bytes(const mgj_config *cfg);

/* Validate cfg, allocate the workspace on the current CUDA device, bind peers.
 * Collective (every rank, same cfg except rank).  *out = NULL on error. */
mgj_status mgj_plan(const mgj_config *cfg, const mgj_peers *peers, mgj_handle *out);

/*
 * Phase a1: radix histogram of both key columns (2^B1 bins, key
 * low bits), fused with its all-gather: the rank histogram is stored into
 * every peer's arena and a release flag is raised.  Columns are SoA
 * (keys[n], payloads[n]), key_bytes/payload_bytes wide; device pointers must
 * be 16-byte aligned.  Host pointers are accepted too: they are copied into
 * handle-owned device staging on `stream` (the end-to-end path).
 */
mgj_status mgj_partition(mgj_handle h,
                         const void *r_keys, const void *r_payloads, uint64_t n_r,
                         const void *s_keys, const void *s_payloads, uint64_t n_s,
                         void *stream);

/*
 * Phases a2 + a3 (§4): waits for every rank's histogram, computes
 * the partition->GPU assignment (contiguous balanced owner ranges) and the
 * exact receive offsets, then scatters every tuple straight into its owner's
 * receive buffer (peer stores over NVLink/NVSwitch of shared-memory-sorted
 * sub-tiles, whole 32-byte sectors) and raises a data-done flag at every
 * peer.  With MGJ_SHUFFLE_EXTERNAL the tuples go to a send buffer ordered by
 * destination instead (see mgj_exchange_layout).
 */
mgj_status mgj_shuffle(mgj_handle h, void *stream);

/*
 * Phases a4 + a5 + a6: waits for every rank's data, radix
 * partitions the received segments by the next B2 key bits into
 * shared-memory-sized co-partitions, builds a shared-memory hash table per
 * R co-partition and probes it with S, then sums (count, checksum, pair
 * digest) over ranks (a6: each rank stores its partial sums into every
 * peer's arena, raises a flag, and waits for all N).  Materialised triples
 * stay on the owning rank.  Because a6 waits for every peer inside the
 * enqueued work, ranks that share one GPU ("virtual ranks") must each use
 * their own stream.
 */
mgj_status mgj_join(mgj_handle h, void *stream);

/* EXTERNAL shuffle: buffers and per-rank sizes (tuples) of the exchange the
 * caller performs between mgj_shuffle and mgj_join.  send[rel] holds the
 * tuples for rank 0, then rank 1, ...; recv[rel] (this rank's arena) must
 * receive the tuples from rank 0, then rank 1, ...  Synchronises the stream
 * of the last call (the sizes are computed on the device). */
typedef struct {
    void    *send[2];
    void    *recv[2];
    uint64_t send_count[2][MGJ_MAX_RANKS];
    uint64_t recv_count[2][MGJ_MAX_RANKS];
    int32_t  tuple_bytes;
    int32_t  world_size;
} mgj_exchange_t;

mgj_status mgj_exchange_layout(mgj_handle h, mgj_exchange_t *out);

/* Synchronise the last stream and fill *out (no device work is enqueued).
 * Returns the run's sticky status. */
mgj_status mgj_result(mgj_handle h, mgj_result_t *out);

void        mgj_destroy(mgj_handle h);
const char *mgj_strerror(mgj_status s);

/*
 * Host reference of the partition assignment of phase a2, used by the
 * multi-process CPU tests: from the all-gathered histograms
 * hist[world][2][2^bits] (u32) compute owner[2^bits], this rank's send
 * offsets send_off[2][2^bits] (tuples, into the owner's receive buffer) and
 * recv_size[2][world].  Same formulas as the device plan kernel
 * (csrc/plan.cuh).  Pure host code, no CUDA call.
 */
mgj_status mgj_plan_host(int32_t world_size, int32_t rank, int32_t bits,
                         const uint32_t *hist, int32_t *owner,
                         uint64_t *send_off, uint64_t *recv_size,
                         int32_t skew_bcast, uint8_t *bcast, uint8_t *skip,
                         int32_t assign);

#ifdef __cplusplus
}
#endif
#endif /* MGJ_H */
