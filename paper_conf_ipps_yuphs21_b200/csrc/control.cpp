// control.cpp — host control plane (see control.h).
#include "control.h"
#include <algorithm>
#include <set>

namespace arb {

namespace {

// 1 = [lo,hi) contained in an entry (it = entry), 0 = disjoint from every
// entry, -1 = partial overlap (reading Z6).
int map_find(MapTable& m, uint64_t lo, uint64_t hi, MapTable::iterator& it) {
  auto nx = m.upper_bound(lo);
  if (nx != m.begin()) {
    auto pv = std::prev(nx);
    if (lo < pv->second.hi) {
      if (hi <= pv->second.hi) { it = pv; return 1; }
      return -1;
    }
  }
  if (nx != m.end() && nx->first < hi) return -1;
  return 0;
}

struct Emitter {
  uint64_t base_word, n_words;
  FlushPlan* out;
  bool none;                              // unified memory: no data op exists (Z23)
  void emit(uint32_t pos, Sel sel, uint64_t byte_lo, uint64_t byte_hi, uint32_t inst) {
    if (none) return;
    uint64_t w0 = byte_lo >> 3, w1 = ((byte_hi - 1) >> 3) + 1;    // [w0, w1) absolute
    uint64_t total = w1 - w0;
    uint64_t lo = std::max(w0, base_word), hi = std::min(w1, base_word + n_words);
    if (lo >= hi) { out->ignored_words += total; return; }
    out->ignored_words += total - (hi - lo);
    out->range_words += hi - lo;
    out->range_ops.push_back(RangeOpH{pos, sel, lo - base_word, hi - base_word, inst});
  }
};

}  // namespace

void resolve_control(const std::vector<CtlRec>& ctl, uint64_t n_records, uint64_t base_word,
                     uint64_t n_words, const std::vector<uint64_t>& bucket_start, MapTable& map,
                     FlushPlan& out, bool bo, const std::vector<CarriedInst>* carried_in, bool unified,
                     uint32_t n_dev, const LastEnded* last_ended_in, const TagBases* tags_in, bool want_cv) {
  const uint32_t n_buckets = (uint32_t)bucket_start.size() - 1;
  out = FlushPlan();
  Emitter em{base_word, n_words, &out, unified};
  // task instances (1-based; 0 = host); instances 1..nc are the carried-in ones:
  // they began before this flush (t_begin = kBefore) and either ended before it
  // (t_end = kBefore) or are still open (t_end = kOpen until their TASK_END)
  constexpr uint64_t kBefore = UINT64_MAX - 1, kOpen = UINT64_MAX - 2;
  const uint32_t nc = carried_in ? (uint32_t)carried_in->size() : 0u;
  std::vector<uint64_t> t_begin{0}, t_end{0}, t_join{0};
  std::vector<uint32_t> t_id{0};
  std::vector<uint32_t> unjoined;
  uint32_t open = 0;
  // depend edges {child, parent} in order of the child's creation (Z22)
  std::vector<std::pair<uint32_t, uint32_t>> edges;
  for (uint32_t c = 0; c < nc; ++c) {
    const bool op_ = (*carried_in)[c].open;
    t_begin.push_back(kBefore); t_end.push_back(op_ ? kOpen : kBefore); t_join.push_back(UINT64_MAX);
    t_id.push_back((*carried_in)[c].task_id);
    if (op_) open = c + 1; else unjoined.push_back(c + 1);
    for (uint32_t pc : (*carried_in)[c].deps) edges.push_back({c + 1, pc + 1});
  }
  auto fail = [&](int rc, uint64_t pos, const char* why) {
    out.rc = rc; out.err_pos = pos; out.err = why;
  };
  const bool md = n_dev > 1;
  // selectors of the data ops on device d (Z24) — the 4-bit forms for one device
  auto s_upt = [&](uint32_t d) { return md ? sel8_upt(d) : kSelUPT; };
  auto s_uph = [&](uint32_t d) { return md ? sel8_uph(d) : kSelUPH; };
  auto s_alloc = [&](uint32_t d) { return md ? sel8_clear(d) : (kSelALLOC | (bo ? kPopSet : 0u)); };
  auto s_rel = [&](uint32_t d) { return md ? sel8_clear(d) : (kSelREL | (bo ? kPopClr : 0u)); };
  constexpr uint64_t kAddrMask = (1ull << 56) - 1;
  // N1 (Z25): pointer tags and the entry holding each tag's base, as a timeline
  if (tags_in) out.tags_out = *tags_in;
  std::vector<std::vector<TagSeg>> tseg;        // per tag (index into tag_ids)
  std::map<uint32_t, uint32_t> tag_ix;          // tag -> index
  auto entry_words = [&](uint64_t byte, uint64_t& lo, uint64_t& hi) {   // the entry holding `byte`
    lo = hi = 0;
    auto nx = map.upper_bound(byte);
    if (nx == map.begin()) return;
    auto pv = std::prev(nx);
    // the words whose first byte lies in the entry (the oracle's containment test)
    if (byte < pv->second.hi) { lo = ((pv->first & kAddrMask) + 7) >> 3; hi = ((pv->second.hi & kAddrMask) + 7) >> 3; }
  };
  auto tag_note = [&](uint32_t t, uint32_t pos) {   // tag t's base entry from pos on
    auto it = tag_ix.find(t);
    if (it == tag_ix.end()) { it = tag_ix.emplace(t, (uint32_t)tseg.size()).first; tseg.emplace_back(); }
    TagSeg g{pos, 0, 0, 0};
    entry_words(out.tags_out[t], g.lo, g.hi);
    auto& v = tseg[it->second];
    if (!v.empty() && v.back().pos == pos) v.back() = g; else v.push_back(g);
  };
  auto tags_in_range = [&](uint64_t lo, uint64_t hi, uint32_t pos) {   // an entry [lo, hi) changed
    for (const auto& kv : out.tags_out)
      if (kv.second >= lo && kv.second < hi) tag_note(kv.first, pos);
  };
  if (bo && n_dev == 1)
    for (const auto& kv : out.tags_out) tag_note(kv.first, 0);
  // N1 (Z26): snapshot of the live CV placements from position pos on
  auto cv_epoch = [&](uint32_t pos) {
    if (!want_cv) return;
    if (!out.cv_epoch_pos.empty() && out.cv_epoch_pos.back() == pos) {   // replace the same position's
      out.cv_place.resize(out.cv_epoch_first.back());
      out.cv_epoch_pos.pop_back(); out.cv_epoch_first.pop_back();
    }
    out.cv_epoch_pos.push_back(pos);
    out.cv_epoch_first.push_back((uint32_t)out.cv_place.size());
    const size_t a = out.cv_place.size();
    for (const auto& kv : map)
      if (kv.second.cv != UINT64_MAX && (kv.first >> 56) == 0)       // device 0 (single device)
        out.cv_place.push_back(CvPlace{kv.second.cv, kv.second.cv + (kv.second.hi - kv.first), kv.first});
    std::sort(out.cv_place.begin() + a, out.cv_place.end(), [](const CvPlace& x, const CvPlace& y) { return x.cv_lo < y.cv_lo; });
  };
  cv_epoch(0);
  for (const CtlRec& c : ctl) {
    uint32_t op = (uint32_t)(c.w0 >> 48) & 0xFFu, arg = (uint32_t)(c.w0 >> 56);
    uint32_t dev = 0;                               // Z24: device of a MAP / UPDATE record
    if (md && (op == OP_MAP_ENTER || op == OP_MAP_EXIT || op == OP_UPDATE || op == OP_CV_BASE)) {
      dev = arg >> 6;
      arg &= 0x3Fu;
      if (dev >= n_dev) return fail(ARB_ETRACE, c.pos, "device id of a map / update record out of range");
    }
    const uint64_t dkey = (uint64_t)dev << 56;     // the device's entries: keys offset by dev << 56
    uint64_t addr = c.w0 & kMask48, len = c.w1 & kMask48;
    uint32_t tid = (uint32_t)(c.w1 >> 48);
    uint32_t pos = (uint32_t)c.pos;
    switch (op) {
      case OP_TASK_BEGIN:
        if (open) return fail(ARB_ETRACE, c.pos, "TASK_BEGIN inside an open task block");
        if (tid == 0 || tid == kSyncAll) return fail(ARB_ETRACE, c.pos, "TASK_BEGIN with task id 0 or 0xFFFF");
        t_begin.push_back(c.pos); t_end.push_back(kOpen); t_join.push_back(UINT64_MAX); t_id.push_back(tid);
        open = (uint32_t)(t_begin.size() - 1);
        break;
      case OP_TASK_END:
        if (!open || t_id[open] != tid) return fail(ARB_ETRACE, c.pos, "TASK_END does not match the open block");
        t_end[open] = c.pos;
        unjoined.push_back(open);
        open = 0;
        break;
      case OP_SYNC: {
        if (open) return fail(ARB_ETRACE, c.pos, "SYNC inside a task block");
        size_t k = 0;
        for (size_t j = 0; j < unjoined.size(); ++j) {
          uint32_t q = unjoined[j];
          if (tid == kSyncAll || t_id[q] == tid) t_join[q] = c.pos;
          else unjoined[k++] = q;
        }
        unjoined.resize(k);
        break;
      }
      case OP_MAP_ENTER: {                          // Table I, entry
        const bool always = arg & kMapAlways;       // Z21
        const bool present = arg & kMapPresent;
        arg &= ~(kMapAlways | kMapPresent);
        if (arg > MT_ALLOC || len == 0 || addr + len > (1ull << 48))
          return fail(ARB_ETRACE, c.pos, "bad MAP_ENTER record");
        MapTable::iterator it;
        int f = map_find(map, dkey | addr, dkey | (addr + len), it);
        if (f < 0) return fail(ARB_EMAP, c.pos, "map clause partially overlaps a present entry");
        if (f == 0 && present) return fail(ARB_EMAP, c.pos, "map(present) of a section that is not mapped");
        if (f == 1) {                               // exist(CV): ref_count += 1, no transfer ...
          it->second.rc += 1;
          if (always && (arg == MT_TO || arg == MT_TOFROM)) em.emit(pos, s_upt(dev), addr, addr + len, open);
          break;                                    // ... unless `always`
        }
        map.emplace(dkey | addr, MapEntry{dkey | (addr + len), 1});  // new CV, ref_count = 1
        if (bo && n_dev == 1 && !out.tags_out.empty()) tags_in_range(addr, addr + len, pos);
        em.emit(pos, s_alloc(dev), addr, addr + len, open);
        if (arg == MT_TO || arg == MT_TOFROM) em.emit(pos, s_upt(dev), addr, addr + len, open);
        break;
      }
      case OP_MAP_EXIT: {                           // Table I, exit (reading Z5)
        const bool always = arg & kMapAlways;       // Z21
        arg &= ~kMapAlways;
        if (arg > MT_DELETE || len == 0 || addr + len > (1ull << 48))
          return fail(ARB_ETRACE, c.pos, "bad MAP_EXIT record");
        MapTable::iterator it;
        int f = map_find(map, dkey | addr, dkey | (addr + len), it);
        if (f < 0) return fail(ARB_EMAP, c.pos, "map clause partially overlaps a present entry");
        if (f == 0) break;                          // not present: no-op (Z7)
        if (arg == MT_DELETE) it->second.rc = 0; else it->second.rc -= 1;
        if (it->second.rc != 0 && always && (arg == MT_FROM || arg == MT_TOFROM))
          em.emit(pos, s_uph(dev), addr, addr + len, open);   // `always`: copy back at rc > 0
        if (it->second.rc == 0) {
          if (arg == MT_FROM || arg == MT_TOFROM) em.emit(pos, s_uph(dev), addr, addr + len, open);
          em.emit(pos, s_rel(dev), it->first & kAddrMask, it->second.hi & kAddrMask, open);
          const uint64_t elo = it->first & kAddrMask, ehi = it->second.hi & kAddrMask;
          const bool had_cv = it->second.cv != UINT64_MAX;
          map.erase(it);
          if (bo && n_dev == 1 && !out.tags_out.empty()) tags_in_range(elo, ehi, pos);
          if (had_cv) cv_epoch(pos);
        }
        break;
      }
      case OP_UPDATE: {
        if (arg > 1 || len == 0 || addr + len > (1ull << 48))
          return fail(ARB_ETRACE, c.pos, "bad UPDATE record");
        MapTable::iterator it;
        int f = map_find(map, dkey | addr, dkey | (addr + len), it);
        if (f < 0) return fail(ARB_EMAP, c.pos, "target update partially overlaps a present entry");
        if (f == 0) break;                          // not present: no-op (Z7)
        em.emit(pos, arg == 0 ? s_upt(dev) : s_uph(dev), addr, addr + len, open);
        break;
      }
      case OP_CV_BASE: {                            // Z26: the runtime placed an entry's CV
        MapTable::iterator it;
        if (map_find(map, dkey | addr, dkey | (addr + 1), it) == 1) {
          const uint64_t c = len - (addr - (it->first & kAddrMask)), sz = it->second.hi - it->first;
          for (auto& kv : map)                      // one CV per device address: older overlaps go
            if (&kv.second != &it->second && (kv.first >> 56) == (dkey >> 56) && kv.second.cv != UINT64_MAX &&
                kv.second.cv < c + sz && c < kv.second.cv + (kv.second.hi - kv.first))
              kv.second.cv = UINT64_MAX;
          it->second.cv = c;
          cv_epoch(pos);
        }
        break;
      }
      case OP_BASE: {                               // Z25: pointer tag -> base address
        if (tid == 0) return fail(ARB_ETRACE, c.pos, "ARB_BASE with pointer tag 0");
        out.tags_out[tid] = addr;
        if (bo && n_dev == 1) tag_note(tid, pos);
        break;
      }
      case OP_TASK_DEPEND: {                        // Z22: the open task runs after the last
        if (!open || tid == 0 || tid == kSyncAll)   // ended instance of task `tid`
          return fail(ARB_ETRACE, c.pos, "TASK_DEPEND outside a task block or with task id 0 / 0xFFFF");
        // instances of this flush (and a carried block that ended in it), latest first;
        // blocks do not nest, so creation order is end order
        bool found = false;
        for (uint32_t q = open - 1; q >= 1 && !found; --q) {
          if (t_end[q] == kBefore) break;              // carried, ended in an earlier flush
          if (t_id[q] == tid && t_end[q] != kOpen) { edges.push_back({open, q}); found = true; }
        }
        if (!found && last_ended_in) {                 // ended in an earlier flush: joined or carried
          auto it = last_ended_in->find(tid);
          if (it != last_ended_in->end() && it->second >= 0 && (uint32_t)it->second < nc)
            edges.push_back({open, (uint32_t)it->second + 1});
        }
        break;
      }
      default:
        return fail(ARB_ETRACE, c.pos, "unknown control op");
    }
  }
  if (want_cv) out.cv_epoch_first.push_back((uint32_t)out.cv_place.size());
  if (!tseg.empty()) {                          // N1: CSR by tag id for k_bo_tags
    out.tag_first.assign(65537, 0);
    for (const auto& kv : tag_ix) out.tag_first[kv.first + 1] = (uint32_t)tseg[kv.second].size();
    for (uint32_t t = 0; t < 65536; ++t) out.tag_first[t + 1] += out.tag_first[t];
    out.tag_segs.resize(out.tag_first[65536]);
    for (const auto& kv : tag_ix)
      std::copy(tseg[kv.second].begin(), tseg[kv.second].end(), out.tag_segs.begin() + out.tag_first[kv.first]);
  }
  // Z22: joining a dependant joins its ancestors (children come after parents)
  for (size_t k = edges.size(); k-- > 0;)
    t_join[edges[k].second] = std::min(t_join[edges[k].second], t_join[edges[k].first]);
  auto is_anc = [&](uint32_t a, uint32_t c) {   // a is an ancestor of c through depend edges
    std::vector<uint32_t> st{c};
    while (!st.empty()) {
      const uint32_t x = st.back(); st.pop_back();
      for (const auto& e : edges)
        if (e.first == x) { if (e.second == a) return true; st.push_back(e.second); }
    }
    return false;
  };
  // a block still open at the end of the flush is carried (N2): its records so
  // far are its own ops, its window starts after its TASK_END in a later flush
  const uint32_t ninst = (uint32_t)t_begin.size() - 1;
  out.tasks = ninst - nc;
  // instances not joined in this flush race with everything up to its end and
  // are carried into the next flush (N2)
  std::vector<uint8_t> carry(ninst + 1, 0);
  for (uint32_t q = 1; q <= ninst; ++q)
    if (t_join[q] == UINT64_MAX) { t_join[q] = n_records; carry[q] = 1; }
  // LastEnded after this flush; carried indices are filled in once carry_out is built
  // (set_last_ended below), joined instances map to -1
  std::vector<uint32_t> last_q;                  // instances that ended in this flush, in end order
  for (uint32_t q = 1; q <= ninst; ++q)
    if (t_end[q] != kBefore && t_end[q] != kOpen) last_q.push_back(q);
  auto set_last_ended = [&](const std::vector<uint32_t>& carry_idx) {   // carry_idx[q]: carried-out index or ~0
    out.last_ended_out.clear();
    if (last_ended_in)
      for (const auto& kv : *last_ended_in) {
        int32_t v = -1;
        if (kv.second >= 0 && (uint32_t)kv.second < nc && carry_idx[kv.second + 1] != ~0u) v = (int32_t)carry_idx[kv.second + 1];
        out.last_ended_out[kv.first] = v;
      }
    for (uint32_t q : last_q) out.last_ended_out[t_id[q]] = carry_idx[q] != ~0u ? (int32_t)carry_idx[q] : -1;
  };
  auto wstart = [&](uint32_t q) { return t_end[q] == kBefore ? 0 : t_end[q] + 1; };   // window [wstart, join)
  auto has_window = [&](uint32_t q) { return t_end[q] != kOpen && t_join[q] > wstart(q); };

  // ---- per-bucket CSR of range ops (trace order kept inside each bucket) ----
  auto first_bucket = [&](uint64_t w) {   // bucket holding relative word w
    return (uint32_t)(std::upper_bound(bucket_start.begin(), bucket_start.end() - 1, w) - bucket_start.begin() - 1);
  };
  out.ops_start.assign(n_buckets + 1, 0);
  for (const RangeOpH& r : out.range_ops)
    for (uint32_t b = first_bucket(r.lo); b < n_buckets && bucket_start[b] < r.hi; ++b) out.ops_start[b + 1]++;
  for (uint32_t b = 0; b < n_buckets; ++b) out.ops_start[b + 1] += out.ops_start[b];
  out.ops.resize(out.ops_start[n_buckets]);
  {
    std::vector<uint32_t> fill(out.ops_start.begin(), out.ops_start.end() - 1);
    for (const RangeOpH& r : out.range_ops)
      for (uint32_t b = first_bucket(r.lo); b < n_buckets && bucket_start[b] < r.hi; ++b)
        out.ops[fill[b]++] = BucketOp{r.pos, r.sel, std::max(r.lo, bucket_start[b]),
                                      std::min(r.hi, bucket_start[b + 1])};
  }

  // ---- MIR join plan (Theorem 1) -------------------------------
  // An instance q is racy if its window (end_q, join_q) holds at least one
  // record; carried-out instances are listed too (their access summary is
  // extracted from the join's hash after the MIR kernels).
  MirPlanH& M = out.mir;
  std::vector<uint32_t> dense(ninst + 1, 0xFFFFFFFFu);
  std::vector<uint32_t> racy;
  for (uint32_t q = 1; q <= ninst; ++q)
    if (has_window(q) || carry[q]) { dense[q] = (uint32_t)racy.size(); racy.push_back(q); }
  M.n_racy = (uint32_t)racy.size();
  if (racy.size() >= (1u << 20) - 1)          // the MIR join keys hold the dense index in 20 bits
    return fail(ARB_ENOMEM, n_records, "more than 2^20 - 2 racy or unjoined task instances in one flush");
  out.carry_in_dense.resize(nc);
  for (uint32_t c = 0; c < nc; ++c) out.carry_in_dense[c] = dense[c + 1];
  out.dense_carry_out.assign(racy.size(), 0xFFFFFFFFu);
  if (racy.empty()) {                         // nothing is carried
    set_last_ended(std::vector<uint32_t>(ninst + 1, ~0u));
    return;
  }
  // insert ranges: the records of each listed block that lie in this flush
  M.ins_cum.push_back(0);
  for (uint32_t q : racy) {
    if (t_end[q] == kBefore) continue;                       // ended in an earlier flush
    const uint64_t lo = t_begin[q] == kBefore ? 0 : t_begin[q] + 1;
    const uint64_t hi = t_end[q] == kOpen ? n_records : t_end[q];
    if (hi > lo) {
      M.ins_lo.push_back(lo);
      M.ins_inst.push_back(dense[q]);
      M.ins_cum.push_back(M.ins_cum.back() + (hi - lo));
    }
  }
  M.n_ins_pos = M.ins_cum.back();
  M.ins_cum.pop_back();
  // own and window range ops per racy instance
  M.own_start.assign(racy.size() + 1, 0);
  M.win_start.assign(racy.size() + 1, 0);
  std::vector<std::vector<RangeRef>> own(racy.size()), win(racy.size());
  for (const RangeOpH& r : out.range_ops) {
    if (r.inst && dense[r.inst] != 0xFFFFFFFFu)
      own[dense[r.inst]].push_back(RangeRef{r.lo, r.hi, r.pos, r.inst});
  }
  for (uint32_t c = 0; c < nc; ++c)          // a carried instance's range ops from earlier flushes
    if (dense[c + 1] != 0xFFFFFFFFu)
      own[dense[c + 1]].insert(own[dense[c + 1]].end(), (*carried_in)[c].own.begin(), (*carried_in)[c].own.end());
  for (size_t d = 0; d < racy.size(); ++d) {
    uint32_t q = racy[d];
    if (!carry[q]) continue;
    out.dense_carry_out[d] = (uint32_t)out.carry_out.size();
    out.carry_out.push_back(CarriedInst{t_id[q], own[d], t_end[q] == kOpen, {}});
  }
  {
    std::vector<uint32_t> carry_idx(ninst + 1, ~0u);
    for (size_t d = 0; d < racy.size(); ++d) carry_idx[racy[d]] = out.dense_carry_out[d];
    set_last_ended(carry_idx);
  }
  for (const auto& e : edges) {              // depend edges between carried-out instances (Z22)
    const uint32_t dc = dense[e.first], dp = dense[e.second];
    if (dc == 0xFFFFFFFFu || dp == 0xFFFFFFFFu) continue;
    const uint32_t cc = out.dense_carry_out[dc], cp = out.dense_carry_out[dp];
    if (cc != 0xFFFFFFFFu && cp != 0xFFFFFFFFu) out.carry_out[cc].deps.push_back(cp);
  }
  for (size_t d = 0; d < racy.size(); ++d) {
    uint32_t q = racy[d];
    if (!has_window(q)) continue;
    // range ops are in trace order: binary search the window
    auto first = t_end[q] == kBefore ? out.range_ops.begin()
                 : std::upper_bound(out.range_ops.begin(), out.range_ops.end(), (uint32_t)t_end[q],
                                    [](uint32_t p, const RangeOpH& r) { return p < r.pos; });
    for (auto it = first; it != out.range_ops.end() && it->pos < t_join[q]; ++it)
      if (edges.empty() || !it->inst || !is_anc(q, it->inst))   // a dependant's ops come after q's (Z22)
        win[d].push_back(RangeRef{it->lo, it->hi, it->pos, it->inst});
  }
  for (size_t d = 0; d < racy.size(); ++d) {
    M.own_start[d + 1] = M.own_start[d] + (uint32_t)own[d].size();
    M.win_start[d + 1] = M.win_start[d] + (uint32_t)win[d].size();
    M.own_ops.insert(M.own_ops.end(), own[d].begin(), own[d].end());
    M.win_ops.insert(M.win_ops.end(), win[d].begin(), win[d].end());
    // (ii) a window range op against the instance's own range ops
    for (const RangeRef& r : win[d])
      for (const RangeRef& a : own[d]) {
        uint64_t lo = std::max(r.lo, a.lo), hi = std::min(r.hi, a.hi);
        if (lo < hi) M.rr.push_back(RangeRef{lo, hi, r.pos, 0});
      }
  }
  M.rr_cum.push_back(0);
  for (const RangeRef& r : M.rr) M.rr_cum.push_back(M.rr_cum.back() + (r.hi - r.lo));
  M.n_rr_words = M.rr_cum.back();
  M.rr_cum.pop_back();
  // query segments: positions covered by at least one window, with the open set
  std::vector<std::pair<uint64_t, int64_t>> evs;   // (position, +/-(dense+1))
  for (size_t d = 0; d < racy.size(); ++d) {
    uint32_t q = racy[d];
    if (!has_window(q)) continue;             // a carried-out instance with no window here
    evs.push_back({wstart(q), (int64_t)d + 1});
    evs.push_back({t_join[q], -((int64_t)d + 1)});
  }
  // Z22: inside the block of an instance c, the windows of c's ancestors are not
  // open (their ops precede c's): with depend edges, block boundaries split the
  // query segments too (code 0; `blk` maps the position to the block's owner)
  std::map<uint64_t, uint32_t> blk;          // position -> instance whose block starts (0: block ends)
  if (!edges.empty()) {
    for (uint32_t q = 1; q <= ninst; ++q) {
      if (t_end[q] == kBefore) continue;
      const uint64_t lo = t_begin[q] == kBefore ? 0 : t_begin[q] + 1;
      const uint64_t hi = t_end[q] == kOpen ? n_records : t_end[q];
      if (hi <= lo) continue;
      blk[lo] = q;
      if (!blk.count(hi)) blk[hi] = 0;
      evs.push_back({lo, 0});
      evs.push_back({hi, 0});
    }
  }
  std::sort(evs.begin(), evs.end());
  std::set<uint32_t> active;
  uint32_t cur_blk = 0;
  M.qry_cum.push_back(0);
  M.qry_open_start.push_back(0);
  for (size_t k = 0; k < evs.size();) {
    uint64_t p = evs[k].first;
    while (k < evs.size() && evs[k].first == p) {
      if (evs[k].second > 0) active.insert((uint32_t)(evs[k].second - 1));
      else if (evs[k].second < 0) active.erase((uint32_t)(-evs[k].second - 1));
      ++k;
    }
    if (!edges.empty()) {
      auto b = blk.find(p);
      if (b != blk.end()) cur_blk = b->second;
    }
    if (k < evs.size() && !active.empty() && evs[k].first > p) {
      const size_t before = M.open_list.size();
      for (uint32_t d : active)
        if (!cur_blk || !is_anc(racy[d], cur_blk)) M.open_list.push_back(d);
      if (M.open_list.size() == before) continue;
      uint64_t len = evs[k].first - p;
      M.qry_lo.push_back(p);
      M.qry_cum.push_back(M.qry_cum.back() + len);
      M.qry_open_start.push_back((uint32_t)M.open_list.size());
    }
  }
  M.n_qry_pos = M.qry_cum.back();
  M.qry_cum.pop_back();
}

}  // namespace arb
