/*
 * arbalest.h — C ABI of the B200-native ARBALEST replay library (libarbalest.so).
 *
 * Problem statement: given an execution trace
 * of host/device memory accesses and OpenMP device directives, replay it through
 * the per-location variable state machine (VSM) over 1 byte of shadow
 * per 8-byte word (Table II) and report every read that
 * fails to observe the latest write (Definition 1) — as a use of
 * uninitialized memory (UUM) or a use of stale data (USD) — and
 * every race between mapping-relevant operations of an unjoined nowait region
 * and another operation (Theorem 1) as a mapping-induced race (MIR).
 * The readings of the paper that fix every silent case are listed in
 * DESIGN.md §2 (Z1-Z18).
 *
 * Conventions
 *  - All integers little-endian.  No C++ exception crosses the ABI.
 *  - Every call returns an int: ARB_OK (0), a negative error, or a positive
 *    warning (ARB_TRUNCATED).
 *  - One host thread per context.  Work is ordered on the CUDA stream passed
 *    to the call (NULL = the legacy default stream); arb_flush synchronizes
 *    that stream before it returns (the report counts cross to the host).
 *  - Device pointers must be CUDA device (or managed) memory of the context's
 *    device; "host" pointers are ordinary (pageable or pinned) host memory.
 */
#ifndef ARBALEST_H
#define ARBALEST_H
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

/* ---- trace records ---------------------------------------- */
/* 16 B, 16-B aligned so that one 128-bit load reads one record.
 * w0: [0,48) byte address | [48,56) op | [56,64) arg (map-type / update dir)
 * w1: [0,48) length in bytes | [48,64) task id (TASK_BEGIN / TASK_END / SYNC) */
typedef struct { uint64_t w0, w1; } arb_event;

/* ops: accesses and device directives */
enum arb_op {
  ARB_RH = 0, ARB_WH = 1, ARB_RT = 2, ARB_WT = 3,       /* read/write host/target, 1..8 bytes */
  ARB_MAP_ENTER = 8, ARB_MAP_EXIT = 9,                  /* map clause on region entry / exit   */
  ARB_UPDATE = 10,                                      /* target update to/from       */
  ARB_TASK_BEGIN = 12, ARB_TASK_END = 13,               /* nowait region block (Z8)     */
  ARB_SYNC = 14,                                        /* taskwait: joins task k, 0xFFFF = all */
  ARB_TASK_DEPEND = 15, /* inside a block: the task depends on the last ended instance of task k
                           (a `depend` clause; Z22): their ops are ordered, and
                           joining the dependant joins the instance it depends on            */
  ARB_BASE = 11         /* pointer tag k (w1 [48,64), 1..0xFFFF) now has the base byte address
                           w0 [0,48) -- the base LLVM IR gives a pointer (Z25).  With
                           ARB_F_BO a target access whose w1 [48,64) holds tag k is also BO
                           when its word lies in another mapping entry than that base (an
                           overflow into another variable's CV); no word-ops          */
};
/* map-types (Table I) */
enum arb_map { ARB_TO = 0, ARB_FROM = 1, ARB_TOFROM = 2, ARB_ALLOC = 3,
               ARB_RELEASE = 4, ARB_DELETE = 5 };
/* map-type modifier, or-ed into the map-type (OpenMP 5.1 `always`; Z21):
 * MAP_ENTER to/tofrom copies OV->CV even when the entry is present, MAP_EXIT
 * from/tofrom copies CV->OV even when the reference count stays above 0 */
#define ARB_MAP_ALWAYS 0x10u
/* map-type modifier `present` (MAP_ENTER): the section must already be mapped,
 * else the flush fails with ARB_EMAP (OpenMP 5.1 runtime error; Z21) */
#define ARB_MAP_PRESENT 0x20u
/* target update direction */
enum arb_upd { ARB_UPD_TO = 0, ARB_UPD_FROM = 1 };
#define ARB_SYNC_ALL 0xFFFFu

/* ---- reports ---------------------------------------------------------------- */
enum arb_kind { ARB_UUM = 1, ARB_USD = 2, ARB_MIR = 3,
                ARB_BO = 4  /* buffer overflow, with ARB_F_BO only (Z20) */ };
/* w0: [0,48) absolute word index (= byte address / 8) | [48,56) kind
 * w1: global record index (0-based; see arb_submit_events)
 * Canonical order: word, then record, then kind, ascending; no duplicates. */
typedef struct { uint64_t w0, w1; } arb_report;

/* ---- status codes -------------------------------------------------------------- */
enum arb_status {
  ARB_OK = 0,
  ARB_TRUNCATED = 1,  /* warning: more reports than the buffer; the count is exact   */
  ARB_EINVAL = -1,    /* bad argument                                                 */
  ARB_ENOMEM = -2,    /* device or host allocation failed                             */
  ARB_ECUDA = -3,     /* CUDA / NCCL failure: destroy the context                     */
  ARB_EMAP = -4,      /* map clause partially overlaps a present entry (Z6)          */
  ARB_ETRACE = -5,    /* malformed trace (Z18)                              */
  ARB_ESTATE = -6,    /* call out of order (e.g. get_reports before any flush)        */
  ARB_EOPEN = -7,     /* reserved: open blocks are carried across flushes (Z19); the
                         oracle returns it for a whole trace that ends inside a block */
  ARB_EPEER = -8      /* communicator only: another rank's arb_flush failed (see below) */
};
/* After ARB_EMAP / ARB_ETRACE / ARB_EOPEN the pending batch is discarded, the
 * committed shadow is unchanged and the context stays usable.  After ARB_ECUDA
 * the context must be destroyed.
 * With a communicator (world > 1, or world == 1 with an NCCL id) arb_flush is a
 * collective: every rank calls it equally often, and the ranks exchange their
 * status twice per flush (ncclAllGather):
 *  - after validation (decode, Table I resolution): if any rank's batch is
 *    rejected, every rank discards its batch — the failing rank returns its own
 *    error, the others ARB_EPEER — and every context stays usable (shadow,
 *    mapping tables and carried tasks unchanged);
 *  - with the report counts at the end: a rank that failed after validation
 *    (ARB_ENOMEM / ARB_ECUDA) still takes part, and the others return ARB_EPEER;
 *    then every rank's context must be destroyed (their shadows differ in state).
 * So one malformed record on one shard fails every rank's flush, and none waits
 * in a collective a peer skipped. */

/* ---- configuration ------------------------------------------------------------- */
#define ARB_F_DEDUP_FIRST 0x1u  /* keep only the first report per (word, kind) (Z3) over the
                                   whole trace: a pair reported by an earlier flush is not
                                   reported again (a device set of the reported pairs
                                   persists across flushes).  With
                                   ARB_TRUNCATED the count is an upper bound and the stored
                                   set may miss firsts that were dropped                    */
#define ARB_F_TIMING      0x2u  /* record CUDA events around every kernel (arb_get_stats) */
#define ARB_F_SMALL_PARTS 0x4u  /* test knob: split every bucket with >= 2048 range-op words
                                   into word-range parts replayed by separate CTAs, and
                                   replay every small bucket with >= 64 events as 3 time
                                   slices (the mechanisms normally used for range-heavy
                                   and hot buckets only)                                  */
/* several accelerators (Z24): n = 1 + ARB_F_DEVICES(flags) devices,
 * n <= 3; the device of RT/WT is the record's arg, that of MAP_ENTER / MAP_EXIT /
 * UPDATE bits 6-7 of its arg; batches of at most 2^29 records; excludes ARB_F_BO
 * and ARB_F_UNIFIED */
#define ARB_F_DEVICES_SHIFT 8
#define ARB_F_DEVICES(n)  ((uint32_t)((n) - 1) << ARB_F_DEVICES_SHIFT)
#define ARB_F_UNIFIED     0x10u /* unified memory (Z23): OV and CV are one
                                   storage — map clauses and target update move no data
                                   (reference counts and ARB_EMAP only), a write of either side
                                   is visible to both, reads fault only on never-written words
                                   (UUM), races among the accesses are still MIR.  Excludes
                                   ARB_F_BO (ARB_EINVAL)                                   */
#define ARB_F_BO          0x8u  /* buffer-overflow extension (reading Z20): every
                                   word carries a 5th state bit "has a CV" (set by allocate,
                                   cleared by release); a target access (RT/WT) to a word
                                   without a CV is reported as ARB_BO and has no VSM effect.
                                   Hot buckets are then replayed whole (no time slices).
                                   Target accesses may carry a pointer tag (ARB_BASE, Z25):
                                   an access outside its base's entry is BO as well, and
                                   still acts on the CV it reached                         */

typedef struct {
  uint64_t addr_base;        /* tracked OV byte range [addr_base, addr_base+addr_bytes);   */
  uint64_t addr_bytes;       /*   both multiples of 8; shadow = addr_bytes/8 bytes of HBM. */
                             /*   Words outside the range are ignored (Z12): in sharded    */
                             /*   mode the range is this rank's shard.                     */
  int      device;           /* CUDA ordinal                                               */
  int      rank, world;      /* address shard of this process; world == 1: single GPU      */
  const void* nccl_unique_id;/* ncclUniqueId* (128 B): required when world > 1; with
                                world == 1 an id makes a 1-rank communicator (the count
                                exchange then runs on one GPU); NULL: no communicator      */
  uint64_t report_capacity;  /* device report-candidate capacity, 0 = default (2^24)       */
  uint32_t flags;            /* ARB_F_*                                                    */
  uint32_t bucket_bits;      /* log2 words per address bucket, 0 = automatic               */
} arb_config;

/* Statistics of the last flush (and totals since arb_init). */
typedef struct {
  uint64_t records;          /* records in the last flush                                  */
  uint64_t access_words;     /* word-events from access records (tracked words only)       */
  uint64_t range_words;      /* word-events from MAP / UPDATE data ops (tracked words)     */
  uint64_t control_records;  /* MAP / UPDATE / TASK / SYNC records                         */
  uint64_t range_ops;        /* resolved ALLOC/UPT/UPH/REL range ops                       */
  uint64_t tasks;            /* nowait task instances                                      */
  uint64_t reports;          /* reports of the last flush (exact)                          */
  uint64_t reports_by_kind[4];
  uint64_t ignored_words;    /* word-ops outside the tracked range                        */
  uint64_t buckets, bucket_bits, max_bucket_events;
  uint64_t total_records, total_word_events, total_reports, flushes;
  /* stream time of each phase of the last flush in milliseconds (ARB_F_TIMING):
     ms_partition = sampling + partition (+ the counter read-back), ms_control =
     segment sort on the GPU overlapped with host control resolution + op upload,
     ms_replay = the replay kernel, ms_mir, ms_reports = compaction, ms_total */
  double   ms_partition, ms_control, ms_replay, ms_mir, ms_reports, ms_total;
  uint64_t kernel_launches;  /* kernels launched by the last flush                         */
  double   ms_sample;        /* address sampling + bucket balancing (inside ms_partition)  */
  uint64_t steps_fast, steps_sort;  /* replay steps by kind                  */
  double   ms_segsort;       /* GPU: segment-entry sort (inside ms_control)                 */
  double   ms_host_control;  /* host wall time of the Table I / task resolution             */
  uint64_t work_items;       /* replay work items (buckets, word-range parts, hot slices)   */
  uint64_t hot_buckets;      /* buckets replayed as time slices (hot words, K5)             */
  uint64_t reports_bo;       /* reports of kind ARB_BO in the last flush (ARB_F_BO)         */
  uint64_t nccl_ranks;       /* ranks of the context's NCCL communicator (ncclCommCount), 0 =
                                no communicator                                              */
  uint64_t exchanges;        /* collectives (status / count ncclAllGather) of the last flush */
  uint64_t steps_run;        /* replay steps made only of run segments       */
  uint64_t segments;         /* (chunk, bucket) segment entries of the last flush (runs and
                                stored-event segments)                                        */
  uint64_t chunks, chunks_fast, chunks_run;  /* partition chunks (256 records) of the last flush:
                                all, on the fast path, written in run form                     */
  uint64_t run_merges;       /* runs continued from the previous chunk (one entry for both)    */
} arb_stats;

typedef struct arb_ctx_s* arb_ctx;

/* Create a context on cfg->device: allocates and zeroes the shadow (all words
 * start invalid), workspaces, and (if cfg->nccl_unique_id) the NCCL
 * communicator of cfg->world ranks.  Returns ARB_OK and *out, or an error
 * (*out = NULL): ARB_EINVAL for a bad range, rank, or an unknown flag bit.
 * Ownership: the context owns the shadow, workspaces and report buffer. */
int arb_init(const arb_config* cfg, arb_ctx* out);

/* Append n records to the pending batch.
 *  ev           device pointer (ev_on_device = 1): used zero-copy, must stay valid
 *               and unmodified until arb_flush returns; host pointer (0): copied
 *               (stream-ordered) before the call returns.
 *  global_index NULL: record i of the batch gets the index (records submitted
 *               since arb_init) + i; else an array of n u64 global indices in the
 *               same memory space as ev (sharded mode: the rank sees a subset of
 *               the global trace, in order).  Read only on the report path: a
 *               device array is read by the compaction kernel, a host array is
 *               NOT copied — it is read on the host for the reports only and must
 *               stay valid until arb_flush returns.  One batch's arrays are all
 *               host (host submits) or all device (a device submit with an index
 *               array after a host one is ARB_EINVAL).
 *  stream       cudaStream_t (NULL = legacy default stream).
 * Records of one batch keep their relative order; a batch holds at most 2^30
 * records.  Errors: ARB_EINVAL, ARB_ENOMEM, ARB_ECUDA. */
int arb_submit_events(arb_ctx ctx, const arb_event* ev, uint64_t n,
                      const uint64_t* global_index, int ev_on_device, void* stream);

/* Replay the pending batch: decode + partition, control resolution (Table I),
 * per-address segmented scan + classification, MIR join, canonical report
 * compaction, and (world > 1) the allgather of per-rank report counts.
 * Flush points may fall anywhere, also inside a TASK_BEGIN..TASK_END block:
 * nowait instances whose block is still open or that ended but are not joined
 * yet are carried into the next flush (their access summary stays on the
 * device) and keep racing until their SYNC (Z19), so the union of the
 * flushes' reports equals the replay of the whole trace.
 *  n_reports_local       this rank's report count (exact even if truncated)
 *  report_offset_global  exclusive prefix of the counts over ranks (0 if world 1)
 * Both may be NULL.  Synchronizes `stream`.  The batch is consumed.  Returns
 * ARB_OK, ARB_TRUNCATED (more candidates than report_capacity; the count is
 * exact, the stored set is the canonical order of the retained candidates),
 * ARB_EMAP / ARB_ETRACE (batch discarded, shadow, mapping tables and carried
 * tasks unchanged), ARB_ENOMEM (also: more than 2^20 - 2 racy or carried task
 * instances in one flush) or ARB_ECUDA. */
int arb_flush(arb_ctx ctx, void* stream, uint64_t* n_reports_local,
              uint64_t* report_offset_global);

/* Copy up to cap reports of the last flush, in canonical order, to out
 * (out_on_device = 1: device pointer, else host).  *n_written = copied count.
 * Returns ARB_OK, ARB_TRUNCATED if cap < count, ARB_ESTATE before any flush. */
int arb_get_reports(arb_ctx ctx, arb_report* out, uint64_t cap, uint64_t* n_written,
                    int out_on_device);

/* Copy the final shadow byte of words [word_lo, word_lo + n) (absolute word
 * indices inside the tracked range) to out (host or device).  Bits: 0 OVv,
 * 1 CVv, 2 OVi, 3 CVi (Table II); with ARB_F_BO bit 4 = CVp (the word
 * has a CV, Z20); with ARB_F_DEVICES(n) bits 1/3 are device 0's CV valid /
 * initialised and bits 4/5, 6/7 those of devices 1 and 2 (Z24).  Synchronous. */
int arb_get_shadow(arb_ctx ctx, uint64_t word_lo, uint64_t n, uint8_t* out, int out_on_device);

/* Statistics of the last flush and totals. */
int arb_get_stats(arb_ctx ctx, arb_stats* out);

/* Human-readable description of the last error of ctx (never NULL). */
const char* arb_last_error(arb_ctx ctx);

/* Release every resource of ctx (NULL is a no-op). */
int arb_destroy(arb_ctx ctx);

#ifdef __cplusplus
}
#endif
#endif
