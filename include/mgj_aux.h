/*
 * mgj_aux.h — auxiliary C ABI of libmgj.so: the seeded input generator and
 * debug read-back of intermediate state.  Neither is part of the join's hot
 * path; the generator writes synthetic inputs into HBM before the timed
 * region, the debug copies are for the per-phase unit tests.
 */
#ifndef MGJ_AUX_H
#define MGJ_AUX_H

#include <stdint.h>
#include "mgj.h"

#ifdef __cplusplus
extern "C" {
#endif

/*
 * Generator (identical to
 * paper_conf_sigmod_paullhl21_b200/datagen.py bit for bit).  Writes rows
 * [row0, row0+count) of relation `rel` (0 = R, 1 = S) of the workload
 * kind/n_r/n_s/z into device columns keys/payloads (4-byte for kinds
 * UNIQUE and ZIPF, 8-byte for WIDE).  The paper's workload: keys "generated
 * sequentially and then shuffled randomly", 4-byte key + 4-byte id
 * (P:867-870), plus a Zipf variant.  Enqueued on `stream`.
 */
typedef enum { MGJ_GEN_UNIQUE = 0, MGJ_GEN_ZIPF = 1, MGJ_GEN_WIDE = 2 } mgj_gen_kind;

mgj_status mgj_gen_relation(int32_t kind, int32_t rel, uint64_t n_r, uint64_t n_s,
                            double z, uint64_t row0, uint64_t count,
                            void *keys, void *payloads, void *stream);

/* Debug read-back (synchronises the device).  Copies min(bytes, size) bytes
 * of the selected internal array into host memory `dst`; *size_out (if not
 * NULL) receives the array's full size in bytes. */
typedef enum {
    MGJ_DBG_RANK_HIST = 1,   /* u32[2][P]            this rank's histogram (a1) */
    MGJ_DBG_MAIL_HIST = 2,   /* u32[world][2][P]     all-gathered histograms */
    MGJ_DBG_OWNER = 3,       /* i32[P]               owner rank of each global partition (a2) */
    MGJ_DBG_SEND_OFF = 4,    /* u64[2][P]            this rank's offsets in the owners' buffers */
    MGJ_DBG_RECV_SIZE = 5,   /* u64[2][8]            receive size per relation per rank */
    MGJ_DBG_RECV_R = 6,      /* tuples received (a3), R, packed (key, payload) */
    MGJ_DBG_RECV_S = 7,
    MGJ_DBG_LOCAL_R = 8,     /* tuples after local partitioning (a4) */
    MGJ_DBG_LOCAL_S = 9,
    MGJ_DBG_META = 10,       /* i32[16]: p_lo, p_hi, B2, plan_ok, chunks_r, chunks_s, n_items, C, BA, QB,
                                NLP, chunks_r / chunks_s of the chunked pass after a first pass,
                                np (owned partitions incl. broadcast), n_bcast */
    MGJ_DBG_CHUNK_OFF_R = 11,/* u16[chunks_r][2^B2+1]  sub-partition offsets per chunk */
    MGJ_DBG_CHUNK_OFF_S = 12,
    MGJ_DBG_CHUNK_BASE = 13, /* u32[2][4P+1]         first chunk of each (sub-)partition of the chunked pass */
    MGJ_DBG_SEGMENTS = 14,   /* u64[4][P]            seg_start_r, seg_start_s, seg_len_r, seg_len_s */
    MGJ_DBG_OUT_KEY = 15,    /* materialised triples (n_materialized entries, key_bytes wide) */
    MGJ_DBG_OUT_PAY_R = 16,
    MGJ_DBG_OUT_PAY_S = 17,
    MGJ_DBG_MID_R = 18,      /* tuples after the first local pass (two-level a4 only): first-pass chunk k
                                at slots [k * region, k * region + E[k][2^BA]), region = chunk_tuples1s + 64 */
    MGJ_DBG_MID_S = 19,
    MGJ_DBG_MID_OFF_R = 20,  /* u16[chunks][65] first-pass run offsets E[k][a] (start | odd count for 8-byte
                                tuples; E[k][2^BA] = the chunk's slots) of MID_R */
    MGJ_DBG_BCAST = 21,      /* u8[P]                selective-broadcast flag of each global partition (a2) */
    MGJ_DBG_PLIST = 22,      /* i32[np]              owned partitions: the range, then broadcast ones outside it */
    MGJ_DBG_SKIP = 23,       /* u8[P]                partition has no R or no S tuple anywhere: not shuffled (a2) */
    MGJ_DBG_TRACE = 24,      /* u64[MGJ_TRACE_COUNT][2] (first start, last end) in ns of each kernel of
                                the last run (globaltimer; 0 = not run); needs mgj_config.trace = 1 */
    MGJ_DBG_MID_OFF_S = 25   /* as MID_OFF_R, of MID_S */
} mgj_debug_what;

/* Trace slots (MGJ_DBG_TRACE), in pipeline order. */
enum {
    MGJ_TR_HIST = 0, MGJ_TR_PLAN = 1, MGJ_TR_SCATTER_R = 2, MGJ_TR_SCATTER_S = 3,
    MGJ_TR_LOCAL_R = 4, MGJ_TR_LOCAL_S = 5, MGJ_TR_LOCAL_RS = 6 /* not stamped (spill) */, MGJ_TR_LOCAL_SPLIT = 7,
    MGJ_TR_LOCAL_SECOND = 8, MGJ_TR_ITEMIZE = 9, MGJ_TR_PROBE = 10 /* not stamped: between itemize and reduce */,
    MGJ_TR_REDUCE = 11,
    MGJ_TRACE_COUNT = 12
};

mgj_status mgj_debug_copy(mgj_handle h, int32_t what, void *dst, uint64_t bytes, uint64_t *size_out);

#ifdef __cplusplus
}
#endif
#endif /* MGJ_AUX_H */
