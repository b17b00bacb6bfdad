/*
 * arb_oracle.h — plain, slow, sequential CPU oracle for the ARBALEST replay.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and
 * bench.py's cpu_baseline / --impl reference legs may load this library.
 * It shares no code, header, table or constant generator with the CUDA path
 * (paper_conf_ipps_yuphs21_b200/csrc); every constant below is restated here
 * from the paper and from the trace format in DESIGN.md §3.
 *
 * Paper: L. Yu, J. Protze, O. Hernandez, V. Sarkar, "ARBALEST: Dynamic
 * Detection of Data Mapping Issues in Heterogeneous OpenMP Applications",
 * IPDPS 2021.  Citations "P:n" are lines of /root/reference/PAPER.md.
 *
 * What it computes:
 *   for every record i in trace order, expand it into word-ops; for every
 *   (word x, op o): MIR check against the log of unjoined async ops on x,
 *   VSM check, VSM transition (bits of Table II),
 *   log the op if it runs inside a nowait task.  Output: the sorted unique
 *   (word, record, kind) triples and the final 4-bit state of every word.
 *
 * Parity status of each part:
 *   VSM edges / fault condition          pinned (prose edges + Definition-1 brute force)
 *   UUM-vs-USD split (init bits, Z2)      pinned to Definition 1 (value simulator);
 *                                         parity unpinned BY THE PAPER (Fig.1/Fig.2 do not split readings)
 *   Table I refcount resolution (Z5-Z7)   pinned (hand scenarios + brute force vs independent model)
 *   MIR predicate (Theorem 1, Z10)        pinned (schedule enumeration)
 *   MIR attribution to later event (Z11)  pinned (brute-force pair search: a record is reported
 *                                         iff it is the later op of a race, tests/test_theorem1.py)
 *   dedup-first mode (Z3)                 parity unpinned (definition only)
 *   sub-word semantics (Z4)               pinned (metamorphic: sub-word invariance and straddling
 *                                         access = two word accesses, tests/test_oracle_metamorphic.py)
 *   several accelerators (Z24)            pinned (brute force vs the value simulator with one CV per device)
 *   map modifiers always/present (Z21)    pinned (brute force vs the value simulator's own refcount model)
 *   unified memory (Z23)                  pinned (brute force vs the value simulator with OV and CV aliased)
 *   depend (Z22)                          pinned (schedule enumeration with dependencies + witness search)
 *   buffer overflow, present-bit form (Z20) pinned (P:279 worked example + brute force vs the
 *                                         value simulator's CV existence)
 *   buffer overflow, base-interval form (Z25) pinned (the P:279 adjacent-CV example + brute force vs
 *                                         the value simulator's per-entry CV identities)
 */
#ifndef ARB_ORACLE_H
#define ARB_ORACLE_H
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

/* Trace record: two little-endian 64-bit words.
 * (CV translation, Z26: parity pinned by brute force vs the value simulator's own
 * CV-address table, tests/test_oracle_bruteforce.py.)
 * w0: [0,48) byte address | [48,56) op | [56,64) arg (map-type or update dir)
 * w1: [0,48) length in bytes          | [48,64) task id (TASK_BEGIN/END, SYNC) */
typedef struct { uint64_t w0, w1; } orc_record;

/* ops (P:242-245 read/write host/target; P:106-123 device directives) */
enum { ORC_RH = 0, ORC_WH = 1, ORC_RT = 2, ORC_WT = 3,
       ORC_MAP_ENTER = 8, ORC_MAP_EXIT = 9, ORC_UPDATE = 10,
       ORC_TASK_BEGIN = 12, ORC_TASK_END = 13, ORC_SYNC = 14,
       ORC_TASK_DEPEND = 15 /* inside a block: the task depends on the last ended
                               instance of task id k (N4, reading Z22) */,
       ORC_BASE = 11,       /* pointer tag k (task-id field, 1..0xFFFF) now has the base
                               byte address of this record (LLVM IR base; N1,
                               reading Z25); no word-ops */
       ORC_CV_BASE = 16     /* the mapping entry holding OV byte address w0[0,48) has its CV
                               at device address w1[0,48) for that byte (N1, reading Z26);
                               no word-ops */ };
/* arg bit of RT / WT (reading Z26): the record's address is a CV (device) address,
 * translated to the OV address through the mapping entries' CV intervals (the
 * interval tree of P:269); a CV address in no entry's CV is not tracked */
#define ORC_CV_ADDR 0x80u
/* map-types (Table I) */
enum { ORC_TO = 0, ORC_FROM = 1, ORC_TOFROM = 2, ORC_ALLOC = 3,
       ORC_RELEASE = 4, ORC_DELETE = 5 };
/* map-type modifier bit in arg (OpenMP 5.1 `always`, reading Z21):
 * on entry with to/tofrom the OV->CV copy happens even if the entry is present;
 * on exit with from/tofrom the CV->OV copy happens even if the reference count
 * stays above 0 */
#define ORC_ALWAYS 0x10u
/* `present` modifier (OpenMP 5.1; N4, reading Z21): a MAP_ENTER whose section is
 * not present is a mapping error (ORC_EMAP) */
#define ORC_PRESENT 0x20u
/* update direction */
enum { ORC_UPD_TO = 0, ORC_UPD_FROM = 1 };
#define ORC_SYNC_ALL 0xFFFFu
/* report kinds (BO: P:277-281) */
enum { ORC_UUM = 1, ORC_USD = 2, ORC_MIR = 3, ORC_BO = 4 };
/* status codes (same values as the library's, restated) */
enum { ORC_OK = 0, ORC_EINVAL = -1, ORC_ENOMEM = -2, ORC_EMAP = -4,
       ORC_ETRACE = -5, ORC_EOPEN = -7 };

typedef struct {
  uint64_t word;    /* absolute word index = byte address / 8 */
  uint64_t record;  /* record index (global_index[i] if given, else i) */
  uint32_t kind;    /* ORC_UUM / ORC_USD / ORC_MIR */
  uint32_t pad;
} orc_report;

typedef struct {
  uint64_t addr_base;    /* tracked byte range [addr_base, addr_base+addr_bytes), 8-B aligned */
  uint64_t addr_bytes;
  int      dedup_first;  /* Z3: keep only the first report per (word, kind) */
  /* Sparse mode: if tracked_words != NULL only these absolute word indices
   * (sorted ascending, unique, inside the range) carry state and reports.
   * Words of the range that are not listed are ignored.  Dense mode
   * (tracked_words == NULL) tracks every word of the range (Z12). */
  const uint64_t* tracked_words;
  uint64_t        n_tracked;
  /* Buffer-overflow extension (reading Z20 of DESIGN.md): a 5th
   * state bit CVp ("the word has a CV") is set by allocate and cleared by
   * release; a target access (RT/WT) to a word without a CV is reported as
   * ORC_BO and has no VSM effect (no UUM/USD check, no transition: the access
   * did not touch this word's CV).  0 = off (the 4-bit VSM of P:255-263). */
  int             detect_bo;
  /* ... and (reading Z25) a target access whose record carries a pointer
   * tag t != 0 in w1[48,64) with a base defined by an ORC_BASE record is also
   * reported as ORC_BO when its word and the base lie in different mapping
   * entries (or the base in none) -- an overflow into ANOTHER variable's CV; the
   * access then still acts on the CV it reached (VSM effect as usual). */
  /* Unified-memory mode (reading Z23): OV and CV are
   * one storage, so map clauses and target update move no data (refcount
   * bookkeeping and ORC_EMAP only, no word-ops), a write by either side is
   * visible to both (all four bits set), reads fault only on never-written
   * words (UUM), and races among the accesses remain (MIR).  Excludes detect_bo. */
  int             unified;
  /* Several accelerators (reading Z24): n_devices > 1
   * gives every word an (n+1)-tuple — OV plus one CV per device d < n_devices
   * (n <= 3), each with its valid and initialised bit — and one mapping table
   * per device.  The device is arg of RT/WT records and bits 6-7 of the arg of
   * MAP_ENTER / MAP_EXIT / UPDATE.  Single-device traces are unchanged.
   * Excludes detect_bo and unified. */
  int             n_devices;
  /* Continuation: if non-NULL, the state of every tracked word before the first
   * record (one byte per slot, as shadow_out) — the final shadow of a replay of
   * the records that precede this trace, cut where no task is open or unjoined
   * and no section is mapped (a quiescent point).  NULL: every word starts
   * invalid. */
  const uint8_t*  shadow_in;
} orc_config;

typedef struct {
  uint64_t records;        /* records replayed */
  uint64_t word_events;    /* (tracked word, data-op) pairs */
  uint64_t transitions;    /* VSM transitions applied; invariant: == word_events */
  uint64_t control_records;
  uint64_t ignored_word_events; /* word-ops on untracked words */
  uint64_t tasks;          /* task instances */
  uint64_t error_record;   /* index of the offending record when rc < 0 */
} orc_stats;

/* Replay n records.  global_index may be NULL (record index = position).
 * On success *out / *n_out receive a malloc'ed array of reports in canonical
 * order (word, record, kind ascending) that the caller frees with
 * orc_free(); shadow_out (dense: addr_bytes/8 bytes, sparse: n_tracked
 * bytes, may be NULL) receives the final states (bit0 OVv, bit1 CVv,
 * bit2 OVi, bit3 CVi — Table II; bit4 CVp with detect_bo; with
 * n_devices > 1 bits 4/5 and 6/7 are CV valid/initialised of devices 1 and 2).
 * Returns ORC_OK or an error. */
int  orc_replay(const orc_config* cfg, const orc_record* rec, uint64_t n,
                const uint64_t* global_index, orc_report** out, uint64_t* n_out,
                uint8_t* shadow_out, orc_stats* stats);
/* Address-sharded mode (the oracle "on all host cores"): the
 * same sequential replay run by `threads` POSIX threads, each over a contiguous
 * range of the tracked words (each thread walks every record and resolves the
 * replicated control stream itself; the task pre-pass is shared).  Results —
 * reports, shadow, stats — are identical to orc_replay's. */
int  orc_replay_sharded(const orc_config* cfg, const orc_record* rec, uint64_t n,
                        const uint64_t* global_index, int threads, orc_report** out, uint64_t* n_out,
                        uint8_t* shadow_out, orc_stats* stats);
void orc_free(void* p);

#ifdef __cplusplus
}
#endif
#endif
