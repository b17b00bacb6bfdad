// arb_internal.h — internal declarations of libarbalest (product path).
// Nothing here is shared with oracle/ (DESIGN.md §4 keeps the two independent).
#pragma once
#include <cstdint>
#include <cstddef>
#include <cuda_runtime.h>

namespace arb {

// ---- trace format ------------------------------------------
constexpr uint64_t kMask48 = (1ull << 48) - 1;
enum Op : uint32_t { OP_RH = 0, OP_WH = 1, OP_RT = 2, OP_WT = 3,
                     OP_MAP_ENTER = 8, OP_MAP_EXIT = 9, OP_UPDATE = 10,
                     OP_TASK_BEGIN = 12, OP_TASK_END = 13, OP_SYNC = 14,
                     OP_TASK_DEPEND = 15,     // N4, Z22
                     OP_BASE = 11,            // pointer tag -> base address (N1, Z25)
                     OP_CV_BASE = 16 };       // an entry's CV placement (N1, Z26)
constexpr uint32_t kCvAddrBit = 1u << 31;     // q.y bit 31 = arg bit 7 of RT / WT: a CV address (Z26)
enum MapType : uint32_t { MT_TO = 0, MT_FROM = 1, MT_TOFROM = 2, MT_ALLOC = 3,
                          MT_RELEASE = 4, MT_DELETE = 5 };
constexpr uint32_t kMapAlways = 0x10;   // `always` map-type modifier bit (N4, Z21)
constexpr uint32_t kMapPresent = 0x20;  // `present`: an unmapped section is a mapping error (Z21)
constexpr uint32_t kSyncAll = 0xFFFFu;

// ---- VSM bits (Table II) ----------------------------------------
constexpr uint32_t kOVv = 1, kCVv = 2, kOVi = 4, kCVi = 8;
// buffer-overflow extension (ARB_F_BO, Z20): the word has a CV
constexpr uint32_t kCVp = 16;

// A transition function of the VSM in "selector" form: output bit j of the
// 4-bit state is taken from source sel_j (0..3 = input bit, 4 = constant 0,
// 5 = constant 1); 3 bits per output bit.  Every transition of P:255-261 is
// a set-constant or copy-a-bit map, so the form is closed under composition.
using Sel = uint32_t;
__host__ __device__ constexpr Sel sel_make(uint32_t s0, uint32_t s1, uint32_t s2, uint32_t s3) {
  return s0 | (s1 << 3) | (s2 << 6) | (s3 << 9);
}
// Bits 12-13 act on the 5th state bit (kCVp, ARB_F_BO only): 0 keep, 2 clear,
// 3 set; composition keeps the later non-keep action.
constexpr Sel kPopClr = 2u << 12, kPopSet = 3u << 12;
constexpr Sel kSelId    = sel_make(0, 1, 2, 3);
constexpr Sel kSelUPT   = sel_make(0, 0, 2, 2);   // CV takes OV's validity and init (update_target)
constexpr Sel kSelUPH   = sel_make(1, 1, 3, 3);   // OV takes CV's (update_host)
constexpr Sel kSelALLOC = sel_make(0, 4, 2, 4);   // fresh CV: not valid, not initialised
constexpr Sel kSelREL   = sel_make(0, 4, 2, 4);   // released CV: same bits as allocate

// ---- several accelerators (Z24) ---------------------------
// 8-bit state: bit0 OVv, bit1 CV0v, bit2 OVi, bit3 CV0i, bits 4/5 CV1 valid /
// initialised, bits 6/7 CV2.  Range ops use an 8-output selector ("Sel8"):
// 4 bits per output bit j = its source (0-7 an input bit, 8 constant 0, 9 constant 1).
__host__ __device__ constexpr uint32_t md_cvv(uint32_t d) { return d == 0 ? 1u : 4u + 2u * (d - 1u); }
__host__ __device__ constexpr uint32_t md_cvi(uint32_t d) { return d == 0 ? 3u : 5u + 2u * (d - 1u); }
constexpr uint32_t kSel8Id = 0x76543210u;
__host__ __device__ constexpr uint32_t sel8_set(uint32_t s, uint32_t out_bit, uint32_t src) {
  return (s & ~(15u << (4 * out_bit))) | (src << (4 * out_bit));
}
__host__ __device__ constexpr uint32_t sel8_upt(uint32_t d) { return sel8_set(sel8_set(kSel8Id, md_cvv(d), 0), md_cvi(d), 2); }
__host__ __device__ constexpr uint32_t sel8_uph(uint32_t d) { return sel8_set(sel8_set(kSel8Id, 0, md_cvv(d)), 2, md_cvi(d)); }
__host__ __device__ constexpr uint32_t sel8_clear(uint32_t d) { return sel8_set(sel8_set(kSel8Id, md_cvv(d), 8), md_cvi(d), 8); }

// ---- compact event (partition output, 8 B) ---------------------------------
// x: [0,30) word offset inside the address bucket | [30,32) access op (RH/WH/RT/WT)
// y: record position inside the batch (< 2^30)
constexpr int kMaxBucketSpanBits = 30;               // buckets span <= 2^30 words
constexpr uint32_t kMaxBatchRecords = 1u << 30;
constexpr int kSegChunkBits = 21;                    // chunk id bits in the entry key (bit 21 in y)
// Run segments: a segment entry whose start has kRunFlag holds a run —
// event j of the segment is {key + j, position + j}, where {key, position} is the
// run's descriptor stored at the start slot of the chunk's output (no other events
// are written).  A fast chunk of at most kMaxChunkRuns runs is written in this form;
// a run that continues into the warp's next chunk extends its entry (len < 2^15).
constexpr uint32_t kRunFlag = 0x8000u;
constexpr int kMaxChunkRuns = 16;
#ifndef ARB_CHUNK_BLOCK
#define ARB_CHUNK_BLOCK 64
#endif
constexpr uint32_t kChunkBlock = ARB_CHUNK_BLOCK;   // partition work unit: consecutive chunks per ticket

// ---- partition geometry ----------------------------------------------------
constexpr int kPartThreads = 512;
constexpr int kPartStages = 2;
constexpr int kPartWarps = kPartThreads / 32;
constexpr int kChunkRecords = 256;                  // records per chunk (one warp, independently)
constexpr int kChunkCap = 2 * kChunkRecords;        // events per chunk (<= 2 words per access)
constexpr int kBucketBits = 11;                    // bucket ids are 11-bit
constexpr int kMaxBuckets = 1 << kBucketBits;
constexpr uint32_t kBucketMask = kMaxBuckets - 1;

// ---- replay geometry -------------------------------------------------------
constexpr int kReplayThreads = 256;
constexpr int kReplayItems = 4;
constexpr int kStep = kReplayThreads * kReplayItems;  // events per step
#ifndef ARB_REPLAY_CTAS_PER_SM
#define ARB_REPLAY_CTAS_PER_SM 4
#endif
constexpr int kReplayCtasPerSm = ARB_REPLAY_CTAS_PER_SM;
constexpr int kReplayHashBits = 12;                  // fast-step hash: 2^12 slots
#ifndef ARB_RUN_GROUPS_IN_FLIGHT
#define ARB_RUN_GROUPS_IN_FLIGHT 1
#endif
constexpr uint32_t kRunGroupsInFlight = ARB_RUN_GROUPS_IN_FLIGHT;   // run step: shadow loads per thread issued together

// replay work items {bucket, y, z, kind}
constexpr uint32_t kItemWhole = 0;      // the whole bucket
constexpr uint32_t kItemPart = 1;       // words [y, z) of the bucket (range-heavy buckets)
constexpr uint32_t kItemSlice = 2;      // hot bucket (K5), phase 3: events of time slice y of z,
                                        //   replayed on a private copy of the carried-in states
constexpr uint32_t kItemSummary = 3;    // hot bucket (K5), phase 1: transition functions of slice y of z
constexpr uint32_t kHotSpan = 1u << 20; // hot buckets span at most this many words

// device-side counters and error flags of one flush
struct DevStats {
  unsigned long long access_words;    // tracked access word-events
  unsigned long long ignored_words;   // access word-ops outside the tracked range
  unsigned long long n_ctl;           // control records seen
  unsigned long long err_pos;         // first malformed record (UINT64_MAX = none)
  unsigned long long n_cand;          // report candidates produced (may exceed capacity)
  unsigned long long work;            // replay work counter
  unsigned long long max_bucket_events;
  unsigned long long range_words_applied;
  unsigned long long n_mir_cand;
  unsigned long long steps_fast, steps_sort;
  unsigned long long n_segs;          // (chunk, bucket) segment entries written by k_partition
  unsigned long long n_carry_out;     // N2: access summaries of instances carried into the next flush
  unsigned long long n_bo_cand;       // N1 (Z25): base-tag overflow candidates
  unsigned long long n_cv_acc;        // N1 (Z26): target accesses by CV address (left untracked)
  unsigned long long steps_run;      // replay steps made only of run segments
  unsigned long long chunks_run, chunks_fast;   // partition chunks written in run form / fast event form
  unsigned long long part_ticket;       // partition work distribution (blocks of kChunkBlock chunks)
  unsigned long long run_merges;        // runs continued from a warp's previous chunk (entry extended)
};

// control record extracted by the partition kernel
struct CtlRec { uint64_t pos, w0, w1; };

// a resolved range op restricted to one address bucket
struct BucketOp {
  uint32_t pos;      // record position in the batch
  uint32_t sel;      // transition function (selector form)
  uint64_t lo, hi;   // word range [lo, hi) relative to the tracked base
};

// N1 (Z25): from batch position `pos` on, the mapping entry holding pointer tag t's
// base spans the absolute words [lo, hi) (lo == hi: the base is not mapped)
struct TagSeg { uint32_t pos; uint32_t pad; uint64_t lo, hi; };

// N1 (Z26): a live CV placement: device bytes [cv_lo, cv_hi) hold OV bytes from ov_lo on
struct CvPlace { uint64_t cv_lo, cv_hi, ov_lo; };

// a range op for the MIR join (absolute relative words, instance of its block)
struct RangeRef { uint64_t lo, hi; uint32_t pos; uint32_t inst; };

// Address buckets are contiguous word ranges made of whole "coarse bins" of
// 2^coarse_bits words.  bin_map[bin] = bucket | (bin - first bin of bucket) << kBucketBits,
// so one lookup gives both the bucket and the word offset inside it.  The map
// is balanced on a sampled histogram of the batch's access addresses.
#ifndef ARB_COARSE_BINS_LOG2
#define ARB_COARSE_BINS_LOG2 19
#endif
constexpr int kMaxCoarseBins = 1 << ARB_COARSE_BINS_LOG2;
constexpr uint32_t kSampleCap = 1u << 20;

struct SampleParams {
  const uint4* ev; uint64_t n; uint64_t stride;   // sample records 0, stride, 2*stride, ...
  uint64_t base_word, n_words; uint32_t coarse_bits;
  uint32_t* hist;                                 // [n_bins]
};

struct PartParams {
  const uint4* ev; uint64_t n;            // batch records
  uint64_t base_word, n_words;            // tracked words [base_word, base_word + n_words)
  uint32_t coarse_bits; const uint32_t* bin_map;
  uint32_t bucket_bits, n_buckets;
  uint32_t n_chunks;
  uint2* part_ev;                         // [n_chunks][kChunkCap]
  uint2* seg_out; uint64_t seg_cap;       // {bucket << 21 | chunk bits 0-20, start | len << 16 | chunk
                                          // bit 21 << 31} per touched bucket of a chunk
  CtlRec* ctl; uint64_t ctl_cap;
  DevStats* st;
  uint32_t n_dev;                         // accelerators (Z24): > 1 puts the device of RT/WT in pos bits 30-31
  uint32_t no_runs;                       // debug (ARB_NO_RUNS): never write the run form
  uint32_t grid;                          // CTAs (persistent, <= one per SM)
};

struct ReplayParams {
  const uint2* part_ev;
  const uint4* segs;                      // segment entries sorted by (bucket, chunk); .w = exclusive
                                          // prefix of the event counts over the sorted array
  const uint32_t* seg_first;              // [n_buckets + 1] first entry of each bucket
  uint32_t n_buckets, bucket_bits;
  const uint64_t* bucket_start;           // [n_buckets + 1] first relative word of each bucket
  const uint4* items; uint32_t n_items;   // work items in scheduling order (largest first):
                                          // {bucket, y, z, kItem*}
  // hot buckets (K5): bucket b's scratch starts at entry hot_off[b] of hot_F
  // (slice functions, 32 bits: see kfun_* in replay.cu) and hot_P (carried-in states, u8);
  // slice k uses [hot_off[b] + k * span16, + span16), span16 = span rounded to 16
  const uint64_t* hot_off; uint32_t* hot_F; uint8_t* hot_P;
  uint64_t n_words;
  uint8_t* shadow;                        // n_words bytes
  uint32_t bo;                            // ARB_F_BO: target accesses to words without kCVp are BO
  uint32_t um;                            // ARB_F_UNIFIED: OV and CV are one storage (Z23)
  uint32_t md;                            // several accelerators (Z24): 8-bit states, device in pos bits 30-31
  uint32_t no_run_steps;                  // debug (ARB_NO_RUN_STEPS): run segments only as synthesised events
  uint32_t no_run_prep;                   // debug (ARB_NO_RUN_PREP): no run-step table built during the previous step
  uint32_t run_step_max;                  // events per run step (ARB_RUN_STEP_MAX, default 16384)
  const uint32_t* ops_start;              // [n_buckets + 1]
  const BucketOp* ops;
  uint4* cand; uint64_t cand_cap;         // report candidates {word lo, word hi, pos, kind}
  DevStats* st;
};

struct MirParams {
  const uint4* ev;                         // batch records
  uint64_t base_word, n_words;
  // position ranges to insert (racy task blocks) / query (windows)
  const uint64_t* ins_lo; const uint64_t* ins_cum; const uint32_t* ins_inst; uint32_t n_ins;
  const uint64_t* qry_lo; const uint64_t* qry_cum; const uint32_t* qry_open_start; uint32_t n_qry;
  const uint32_t* open_list;                // instances open in each query segment
  // per racy instance (dense index): own range ops and window range ops
  const uint32_t* own_start; const RangeRef* own_ops;
  const uint32_t* win_start; const RangeRef* win_ops;
  const uint32_t* inst_dense;               // instance -> dense index (or 0xFFFFFFFF)
  // hash table (word, instance) -> write flag
  unsigned long long* hkeys; uint32_t* hvals; uint64_t hmask;
  // (ii) range-vs-range emission list
  const RangeRef* rr; const uint64_t* rr_cum; uint32_t n_rr;
  // N2: access summaries of instances carried in from earlier flushes
  // {word lo, word hi, carried index, write flag}; cmap: carried index -> dense index
  const uint4* carry; uint64_t n_carry; const uint32_t* cmap;
  uint4* cand; uint64_t cand_cap;
  DevStats* st;
};

// ---- kernel launchers (kernels.cu) -----------------------------------------
cudaError_t launch_sample(const SampleParams& p, uint64_t n_samples, cudaStream_t s);
// scratch: 2 * ceil(n_bins / 1024) + 4 + n_bins u32.  Writes the bucket count
// (*nb_out), bucket starts and the sampled event weight of every bucket.
cudaError_t launch_cut(uint32_t* hist_map, uint32_t n_bins, uint32_t coarse_bits, uint64_t n_words,
                       uint32_t max_buckets, uint64_t* bucket_start, uint32_t* weight, uint32_t* first_bin,
                       uint32_t* nb_out, uint32_t* scratch, cudaStream_t s, int* launches);
cudaError_t launch_partition(const PartParams& p, cudaStream_t s);
// Sorts the 8-B segment entries {bucket << 21 | chunk, start | len << 16 | chunk bit 21 << 31}
// by (bucket, chunk) (a, b: ping-pong buffers), writes the replay form
// {chunk, bucket, start | len << 16, exclusive event prefix} to out and each
// bucket's first entry; cnt: (n / 4096 + 1) * 256 + 4096 u32
// The entries of one partition block (kChunkBlock consecutive chunks, one warp) are in
// chunk order in the input, so a stable sort by (bucket, chunk / kChunkBlock) orders
// them by (bucket, chunk); n_chunks: chunks of the batch
cudaError_t launch_sort_segments(uint2* a, uint2* b, uint64_t n, uint64_t n_chunks, uint32_t n_buckets, uint32_t* cnt,
                                 uint32_t* first, uint4* out, cudaStream_t s, int* launches);
cudaError_t launch_replay(const ReplayParams& p, int n_ctas, cudaStream_t s);
// K5 phase 2: for every hot bucket {bucket, slices, span, 0} carry the states
// across its slices: P_0 = shadow, P_{k+1} = F_k(P_k); shadow = F_last(P_last)
cudaError_t launch_carry(const uint4* hot, uint32_t n_hot, uint32_t max_span, const uint64_t* bucket_start,
                         const uint64_t* hot_off, const uint32_t* hot_F, uint8_t* hot_P, uint8_t* shadow,
                         int bo, int md, cudaStream_t s);
cudaError_t launch_mir(const MirParams& p, uint64_t n_ins_pos, uint64_t n_qry_pos, uint64_t n_rr_words,
                       cudaStream_t s, int* launches);
// N1 (Z26): copy the batch, translating CV-addressed target accesses to OV addresses
// through the placements live at their position (epoch e covers positions from
// epoch_pos[e], its placements are place[epoch_first[e], epoch_first[e+1]), sorted
// by cv_lo and disjoint); an access in no placement keeps its CV flag (untracked)
cudaError_t launch_cv_translate(const uint4* in, uint4* out, uint64_t n, const uint32_t* epoch_pos,
                                const uint32_t* epoch_first, uint32_t n_epochs, const CvPlace* place,
                                cudaStream_t s);
// N1 (Z25): target accesses through pointer tag t (w1[48,64)) whose word lies outside
// the entry of t's base at that position -> BO candidates {word lo, word hi, pos, 4}
// (tag_first: [65537] CSR into segs, by tag; words relative to base_word in the output)
cudaError_t launch_bo_tags(const uint4* ev, uint64_t n, uint64_t base_word, uint64_t n_words,
                           const uint32_t* tag_first, const TagSeg* segs, uint4* cand, uint64_t cand_cap,
                           unsigned long long* count, cudaStream_t s);
// N2: the hash entries of the instances still unjoined at the end of the flush
// (dense index d with co_of[d] != 0xFFFFFFFF) -> out {word lo, word hi, co_of[d], flag};
// *n_out counts them (out holds hcap entries)
cudaError_t launch_carry_extract(const unsigned long long* hkeys, const uint32_t* hvals, uint64_t hcap,
                                 const uint32_t* co_of, uint4* out, unsigned long long* n_out, cudaStream_t s);
// report compaction: sorts candidates, removes duplicates, optional dedup-first,
// maps positions to global indices and writes arb_report records.
struct CompactParams {
  uint4* cand; uint64_t n_cand;           // in/out scratch
  uint4* tmp;                             // same size scratch
  uint32_t* blk; uint64_t blk_cap;        // block counters scratch
  uint64_t base_word;
  int word_bits, pos_bits;
  int dedup_first;
  const uint64_t* gidx;                   // device global index per batch position, or null
  uint64_t index_base;                    // used when gidx is null
  uint4* out;                             // arb_report output (w0 lo/hi, w1 lo/hi)
  unsigned long long* n_out;              // device count
  // dedup_first across flushes: persistent set of reported (word, kind) keys, or null
  unsigned long long* dset; uint64_t dset_mask; unsigned long long* dset_count;
};
cudaError_t launch_compact(const CompactParams& p, cudaStream_t s, int* launches);
// grow the cross-flush dedup set: reinsert the n_old slots of `old` into `set` (mask + 1 slots, zeroed)
cudaError_t launch_dedup_rehash(const unsigned long long* old, uint64_t n_old, unsigned long long* set, uint64_t mask,
                                cudaStream_t s);

}  // namespace arb
