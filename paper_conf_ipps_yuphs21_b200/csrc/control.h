// control.h — host control plane of libarbalest.
//
// Input: the control records of one batch (MAP_ENTER / MAP_EXIT / UPDATE /
// TASK_BEGIN / TASK_END / SYNC) with their positions, extracted on the device
// by k_partition.  Output: resolved range ops (Table I),
// task instances with their joins (Theorem 1, reading Z8),
// the per-bucket range-op lists consumed by k_replay and the MIR join plan
// consumed by k_mir_*.  O(C log C) for C control records.  Also: TASK_DEPEND
// edges (Z22), the `always` / `present` modifiers (Z21), unified memory (Z23),
// one mapping table per accelerator (Z24) and the instances carried across
// flushes (N2, Z19).
#pragma once
#include <cstdint>
#include <map>
#include <string>
#include <unordered_map>
#include <vector>
#include "arb_internal.h"
#include "arbalest.h"

namespace arb {

struct MapEntry { uint64_t hi; uint64_t rc; uint64_t cv = UINT64_MAX; };   // keyed by lo (bytes), [lo, hi);
                                                      // cv: CV address of byte lo (Z26), MAX unknown
using MapTable = std::map<uint64_t, MapEntry>;

struct RangeOpH { uint32_t pos; uint32_t sel; uint64_t lo, hi; uint32_t inst; };  // rel words [lo, hi)

struct MirPlanH {
  std::vector<uint64_t> ins_lo, ins_cum; std::vector<uint32_t> ins_inst;
  std::vector<uint64_t> qry_lo, qry_cum; std::vector<uint32_t> qry_open_start, open_list;
  std::vector<uint32_t> own_start, win_start;
  std::vector<RangeRef> own_ops, win_ops;
  std::vector<RangeRef> rr; std::vector<uint64_t> rr_cum;
  uint64_t n_ins_pos = 0, n_qry_pos = 0, n_rr_words = 0;
  uint32_t n_racy = 0;
  bool empty() const { return n_ins_pos == 0 && n_qry_pos == 0 && n_rr_words == 0; }
};

// A nowait task instance that ended in an earlier flush and is not joined yet
// (SURVEY §8(f) N2): its own range ops (relative words; pos unused) travel on the
// host, its (word, write-class) access summary on the device (ctx->carry_ent).
// open: its TASK_BEGIN..TASK_END block is still open (its next records belong to it).
// deps: carried indices of the (unjoined) instances it depends on (Z22).
struct CarriedInst { uint32_t task_id; std::vector<RangeRef> own; bool open; std::vector<uint32_t> deps; };

// For every task id, the last instance that ended in an earlier flush (Z22: a
// TASK_DEPEND(k) binds to the last ended instance of task id k, joined or not):
// its carried index if that instance is still carried, else -1 (it is joined, so a
// dependency on it adds no constraint).  Ids that never ended have no entry.
using LastEnded = std::unordered_map<uint32_t, int32_t>;

// N1 (Z25): the base byte address of every pointer tag defined so far (ARB_BASE records)
using TagBases = std::map<uint32_t, uint64_t>;

struct FlushPlan {
  std::vector<RangeOpH> range_ops;       // in trace order
  std::vector<uint32_t> ops_start;       // per bucket CSR
  std::vector<BucketOp> ops;
  MirPlanH mir;
  std::vector<uint32_t> carry_in_dense;  // per carried-in instance: its MIR dense index, or 0xFFFFFFFF
  std::vector<uint32_t> dense_carry_out; // per MIR dense index: its carried-out index, or 0xFFFFFFFF
  std::vector<CarriedInst> carry_out;    // instances still unjoined at the end of this flush
  LastEnded last_ended_out;              // LastEnded after this flush (committed with carry_out)
  TagBases tags_out;                     // tag bases after this flush (committed likewise)
  std::vector<uint32_t> tag_first;       // N1 with bo: [65537] CSR of tag_segs by tag (empty: no tag)
  std::vector<TagSeg> tag_segs;
  // N1 (Z26, with want_cv): CV placements by epoch: epoch e starts at batch position
  // cv_epoch_pos[e]; its live placements are cv_place[cv_epoch_first[e], [e + 1]), sorted
  std::vector<uint32_t> cv_epoch_pos, cv_epoch_first;
  std::vector<CvPlace> cv_place;
  uint64_t range_words = 0, ignored_words = 0, tasks = 0;
  int rc = 0; uint64_t err_pos = 0; std::string err;
};

// Resolve the control records `ctl` (sorted by position) of a batch of
// n_records records.  `map` is the persistent mapping table; it is modified in
// place only on success (the caller passes a copy and commits it).
// `bucket_start` holds the first relative word of every address bucket plus
// n_words at the end (ascending).
// bo (ARB_F_BO): allocate / release also set / clear the kCVp bit (Z20).
// carried_in: instances unjoined at the end of the previous flush (their window
// in this flush starts at position 0); instances unjoined at the end of this one
// are returned in out.carry_out instead of being treated as joined (Z19).
// last_ended_in: the LastEnded table after the previous flush (indices into
// carried_in); the updated table is returned in out.last_ended_out.
// tags_in: pointer tag bases defined by earlier flushes (ARB_BASE, Z25); the updated
// set is returned in out.tags_out; with bo, out.tag_first / tag_segs give every
// defined tag's base entry over the batch (the k_bo_tags timeline).
void resolve_control(const std::vector<CtlRec>& ctl, uint64_t n_records, uint64_t base_word,
                     uint64_t n_words, const std::vector<uint64_t>& bucket_start, MapTable& map,
                     FlushPlan& out, bool bo = false, const std::vector<CarriedInst>* carried_in = nullptr,
                     bool unified = false, uint32_t n_dev = 1, const LastEnded* last_ended_in = nullptr,
                     const TagBases* tags_in = nullptr, bool want_cv = false);
// n_dev > 1 (Z24): device bits 6-7 of MAP / UPDATE args select the device; its
// entries live in the same table under keys offset by device << 56, and range
// ops are 8-output selectors (Sel8).
// unified (ARB_F_UNIFIED, Z23): map clauses and target update keep the reference
// counts (and their errors) but emit no range ops: nothing moves between OV and CV.

}  // namespace arb
