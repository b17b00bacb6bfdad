// replay.cu — A3b + A4 + A5: per-address replay of each bucket.
//
// One CTA per address bucket at a time (persistent; buckets in largest-first
// order).  The bucket's events are the segments of its sorted segment entries
// (chunk order = trace order); the CTA gathers them step by step through a
// staged window of entries (cp.async, double-buffered), applies the resolved range ops
// (Table I transfers / allocate / release; target update P:121) to
// the bucket's shadow at their trace positions, and processes the events in
// steps of <= 1024 that never straddle a range op:
//
//   fast step  (every word has at most one write in the step): a shared-memory
//              hash of the written words, word -> write position.  A read's
//              state-before is the initial state, or the image of the one
//              write when that write precedes it; the word's final state is
//              the image of the write (reads do not change the state).
//   sort step  (otherwise): stable LSD radix sort of the step by word, then a
//              segmented scan of the access monoid seeded with the shadow
//              state.
//
// Both classify reads as in P:263 (read_host needs OV valid, read_target CV
// valid) and split UUM / USD with the init bits (Table II).  The shadow
// (1 byte per word) carries each word's state across steps.
//
// k_replay<BO, UM, MD> instances: the default one, the buffer-overflow extension
// (ARB_F_BO, Z20), unified memory (ARB_F_UNIFIED, Z23) and several accelerators
// (ARB_F_DEVICES, 8-bit states, Z24); the mode checks compile away in the others.
#include "kcommon.cuh"
#include <algorithm>
#include <type_traits>

namespace arb {

constexpr int RT = kReplayThreads;           // threads per CTA (>= 256)
constexpr int RI = kReplayItems;             // events per thread per step
constexpr int STEP = RT * RI;                // events per step (1024)
static_assert(RT >= 256 && STEP <= 4096, "sort_pass digit loop and u16 offsets");
constexpr int kWin = 2 * RT;                 // segment descriptors staged per step
constexpr int kHBits = kReplayHashBits;
constexpr int kHSlots = 1 << kHBits;         // hash slots (load <= 1/2)
constexpr uint32_t kEmpty = 0xFFFFFFFFu;
constexpr uint32_t kWordMask = 0x3FFFFFFFu;
constexpr int ilog2c(int x) { return x <= 1 ? 0 : 1 + ilog2c(x >> 1); }
constexpr int kZBits = ilog2c(2 * STEP);
constexpr int kZSlots = 1 << kZBits;         // summary-step hash slots (2 x the events of a step)
static_assert(kZSlots == 2 * STEP, "summary hash: twice the step");

// Run steps: a step made only of run segments never materialises
// its events; the gather stages the runs' descriptors in the step's event buffer.
constexpr int kMaxStepRuns = 32;             // run segments per run step
struct RunStage {
  uint4 info[kMaxStepRuns];                  // {first event's offset in the run, events, step-relative start, 0}
  uint2 desc[kMaxStepRuns];                  // the runs' descriptors {key, position} (cp.async)
  uint4 run[kMaxStepRuns];                   // {A, B, op, position of word A} (A, B: words from the
                                             //   4-aligned word below the bucket's first word)
  uint4 cmp[kMaxStepRuns];                   // compounds: adjacent runs on identical words {A, B, first
                                             //   run | runs << 5, their ops (2 bits each, trace order)}
  uint2 mi[kMaxStepRuns];                    // merged group intervals {first group, first unit}
  uint32_t mm[kMaxStepRuns];                 // the runs overlapping merged interval j
  uint32_t nm, G;                            // merged intervals, groups
};
static_assert(sizeof(RunStage) <= sizeof(uint2) * STEP, "a run stage fits in one step buffer");

struct ReplaySmem {
  uint2 ev[2][STEP];              // double-buffered step events {key, pos} (cp.async), or a RunStage
  union {
    struct { uint32_t keyA[STEP], posA[STEP], keyB[STEP], posB[STEP]; uint16_t hist[RT / 32][256]; } s;
    struct { uint2 slot[kHSlots]; } h;      // fast step: written words {word, pos << 2 | op}
    struct { uint32_t key[kZSlots], lastw[kZSlots], anyw[kZSlots / 4]; } z;  // hot-slice summary step (K5);
                                                                            // anyw: one byte per slot
  } u;
  uint32_t wstart[kWin];          // staged segment list window: global event index
  uint32_t wcum[kWin + 1];        //   and bucket-relative first event of each segment
  uint32_t pref[256];             // radix digit scratch
  uint32_t red[RT / 32], red2[RT / 32], wscan[RT / 32];
  uint32_t wcnt[RT / 32], wev[RT / 32];
  uint32_t bucket, op_cur, op_end, next_op;
  uint32_t part_lo, part_hi;      // the work item's word range inside the bucket
  bool partial;                   //   (partial: not the whole bucket)
  uint32_t mode;                  // kItem* of the work item
  uint8_t* shrel;                 // state of bucket-relative word w: shrel[w]
  uint32_t* fsum;                 // summary slice: composed transition of word w: fsum[w] (kfun_*)
  uint32_t slice, n_slices;       // hot bucket slice (kItemSlice / kItemSummary)
  uint32_t seg0, cum0, n_segs, n_events, wsc, nwin;
  uint32_t span;                  // words of the bucket
  uint64_t bucket_base;
};

// ---- block-level helpers ----------------------------------------------------
__device__ __forceinline__ uint32_t block_sum(uint32_t v, uint32_t* red) {
  const uint32_t lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
#pragma unroll
  for (int d = 16; d; d >>= 1) v += __shfl_xor_sync(FULL, v, d);
  __syncthreads();
  if (lane == 0) red[warp] = v;
  __syncthreads();
  uint32_t t = 0;
#pragma unroll
  for (int w = 0; w < RT / 32; ++w) t += red[w];
  return t;
}
__device__ __forceinline__ void block_minmax(uint32_t& lo, uint32_t& hi, uint32_t* r1, uint32_t* r2) {
  const uint32_t lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
#pragma unroll
  for (int d = 16; d; d >>= 1) {
    lo = min(lo, __shfl_xor_sync(FULL, lo, d));
    hi = max(hi, __shfl_xor_sync(FULL, hi, d));
  }
  __syncthreads();
  if (lane == 0) { r1[warp] = lo; r2[warp] = hi; }
  __syncthreads();
  lo = 0xFFFFFFFFu; hi = 0;
#pragma unroll
  for (int w = 0; w < RT / 32; ++w) { lo = min(lo, r1[w]); hi = max(hi, r2[w]); }
}

// ---- K5 slice functions (32 bits per word) -------------------------------------------------
// default / UM: a 4-bit selector (low 16 bits); ARB_F_BO (Z20): a pair of selectors
// with CVp actions, the low half for a word entering the slice without a CV, the
// high half with one (a target write is the identity on a word without a CV, so
// the function depends on CVp); several accelerators (Z24): an 8-output selector.
template <bool BO, bool MD>
__device__ __forceinline__ uint32_t kfun_id() { return MD ? kSel8Id : BO ? (kSelId | (kSelId << 16)) : kSelId; }
// an unconditional transition g (range op) after f
template <bool BO, bool MD>
__device__ __forceinline__ uint32_t kfun_then(uint32_t g, uint32_t f) {
  if (MD) return sel8_compose(g, f);
  if (BO) return sel_compose(g, f & 0xFFFFu) | (sel_compose(g, f >> 16) << 16);
  return sel_compose(g, f);
}
// CVp after selector half h for a word entering with CVp = c (bits 12-13: 0 keep, 2 clear, 3 set)
__device__ __forceinline__ uint32_t half_cvp(uint32_t h, uint32_t c) {
  const uint32_t pop = (h >> 12) & 3u;
  return pop == 0 ? c : (pop == 3 ? 1u : 0u);
}
template <bool BO, bool MD>
__device__ __forceinline__ uint32_t kfun_apply(uint32_t f, uint32_t s) {
  if (MD) return sel8_apply4(f, s) & 255u;
  if (BO) return sel_apply5((s & kCVp) ? f >> 16 : f & 0xFFFFu, s) & 31u;
  return sel_apply4(f, s) & 15u;
}

// ---- range ops ----------------------------------------------------------------
// Apply transition `sel` to the state bytes base[lo, hi) (BO: 5-bit states, ARB_F_BO).
template <bool BO, bool MD>
__device__ __forceinline__ uint32_t apply_sel(Sel s, uint32_t x) {
  return MD ? sel8_apply4(s, x) : BO ? sel_apply5(s, x) : sel_apply4(s, x);
}
// A 4-bit selector as SWAR masks over 4 states: out = (x & K) | C | ((x << 1) & U) |
// ((x >> 1) & D) — every output bit kept, constant, or copied from the other bit of
// its pair (OV/CV valid bits 0-1, init bits 2-3), which covers the transitions of
// Table I and their compositions.  Returns false for any other selector.
__device__ __forceinline__ bool sel_swar(Sel s, uint32_t& K, uint32_t& C, uint32_t& U, uint32_t& D) {
  K = C = U = D = 0;
#pragma unroll
  for (uint32_t j = 0; j < 4; ++j) {
    const uint32_t src = (s >> (3 * j)) & 7u, b = 0x01010101u << j;
    if (src == j) K |= b;
    else if (src == 5) C |= b;
    else if (src == 4) {}
    else if ((j & 1u) && src == j - 1) U |= b;
    else if (!(j & 1u) && src == j + 1) D |= b;
    else return false;
  }
  return true;
}

template <bool BO, bool MD>
__device__ void stream_apply(uint8_t* base, uint64_t lo, uint64_t hi, Sel sel) {
  if (lo >= hi) return;
  // 16-B aligned middle [a, b) of [lo, hi), by address
  const uintptr_t p0 = reinterpret_cast<uintptr_t>(base + lo), p1 = reinterpret_cast<uintptr_t>(base + hi);
  const uintptr_t pa = (p0 + 15) & ~(uintptr_t)15, pb = p1 & ~(uintptr_t)15;
  uint64_t a = hi, b = hi;                       // no aligned middle: all bytes in the head loop
  if (pa < pb) { a = lo + (pa - p0); b = hi - (p1 - pb); }
  for (uint64_t j = lo + threadIdx.x; j < a; j += RT) __stcg(base + j, (uint8_t)apply_sel<BO, MD>(sel, __ldcg(base + j)));
  for (uint64_t j = b + threadIdx.x; j < hi; j += RT) __stcg(base + j, (uint8_t)apply_sel<BO, MD>(sel, __ldcg(base + j)));
  uint4* v = reinterpret_cast<uint4*>(base + a);
  const uint64_t nv = (b - a) >> 4;
  constexpr int U = 4;   // 4 x 16 B loads in flight per thread
  uint64_t j = threadIdx.x;
  uint32_t mK, mC, mU, mD;
  if (!BO && !MD && sel_swar(sel, mK, mC, mU, mD)) {
    auto f = [&](uint32_t x) { return (x & mK) | mC | ((x << 1) & mU) | ((x >> 1) & mD); };
    for (; j + (U - 1) * RT < nv; j += U * RT) {
      uint4 x[U];
#pragma unroll
      for (int u = 0; u < U; ++u) x[u] = __ldcg(v + j + u * RT);
#pragma unroll
      for (int u = 0; u < U; ++u) {
        x[u].x = f(x[u].x); x[u].y = f(x[u].y); x[u].z = f(x[u].z); x[u].w = f(x[u].w);
        __stcg(v + j + u * RT, x[u]);
      }
    }
    for (; j < nv; j += RT) {
      uint4 x = __ldcg(v + j);
      x.x = f(x.x); x.y = f(x.y); x.z = f(x.z); x.w = f(x.w);
      __stcg(v + j, x);
    }
    return;
  }
  for (; j + (U - 1) * RT < nv; j += U * RT) {
    uint4 x[U];
#pragma unroll
    for (int u = 0; u < U; ++u) x[u] = __ldcg(v + j + u * RT);
#pragma unroll
    for (int u = 0; u < U; ++u) {
      x[u].x = apply_sel<BO, MD>(sel, x[u].x); x[u].y = apply_sel<BO, MD>(sel, x[u].y);
      x[u].z = apply_sel<BO, MD>(sel, x[u].z); x[u].w = apply_sel<BO, MD>(sel, x[u].w);
      __stcg(v + j + u * RT, x[u]);
    }
  }
  for (; j < nv; j += RT) {
    uint4 x = __ldcg(v + j);
    x.x = apply_sel<BO, MD>(sel, x.x); x.y = apply_sel<BO, MD>(sel, x.y);
    x.z = apply_sel<BO, MD>(sel, x.z); x.w = apply_sel<BO, MD>(sel, x.w);
    __stcg(v + j, x);
  }
}

// Apply every pending range op of the bucket with position < limit; runs of
// ops on the identical range with no event in between are composed first.
// S.next_op caches the position of the first pending op.
template <bool BO, bool MD>
__device__ void apply_ops_before(ReplaySmem& S, const ReplayParams& p, uint32_t limit) {
  while (S.next_op < limit) {
    const uint32_t k = S.op_cur;
    const BucketOp o = p.ops[k];
    Sel sel = o.sel;
    uint32_t k2 = k + 1;
    while (k2 < S.op_end) {
      const BucketOp o2 = p.ops[k2];
      if (o2.pos >= limit || o2.lo != o.lo || o2.hi != o.hi) break;
      sel = MD ? sel8_compose(o2.sel, sel) : sel_compose(o2.sel, sel);
      ++k2;
    }
    const uint64_t lo = max(o.lo, S.bucket_base + S.part_lo), hi = min(o.hi, S.bucket_base + S.part_hi);
    if (S.mode == kItemSummary) {
      // hot slice, phase 1: compose the op into the words' slice functions
      for (uint64_t j = lo + threadIdx.x; j < hi; j += RT) {
        const uint32_t w = (uint32_t)(j - S.bucket_base);
        S.fsum[w] = kfun_then<BO, MD>(sel, S.fsum[w]);
      }
    } else if (hi > lo) {
      stream_apply<BO, MD>(S.shrel, lo - S.bucket_base, hi - S.bucket_base, sel);
    }
    __syncthreads();
    if (threadIdx.x == 0) {
      S.op_cur = k2;
      S.next_op = k2 < S.op_end ? p.ops[k2].pos : 0xFFFFFFFFu;
      if (hi > lo) atomicAdd(&p.st->range_words_applied, (unsigned long long)(hi - lo));
    }
    __syncthreads();
  }
}

// ---- report candidates (warp-aggregated append) ----------------------------------
__device__ __forceinline__ void emit_faults(const ReplayParams& p, const uint32_t* fk, const uint32_t* word,
                                            const uint32_t* pos, uint64_t bucket_base) {
  const uint32_t lane = threadIdx.x & 31;
  uint32_t nf = 0;
#pragma unroll
  for (int j = 0; j < RI; ++j) nf += fk[j] != 0;
  if (!__any_sync(FULL, nf != 0)) return;
  uint32_t wf = nf;
#pragma unroll
  for (int d = 1; d < 32; d <<= 1) {
    const uint32_t o = __shfl_up_sync(FULL, wf, d);
    if (lane >= (uint32_t)d) wf += o;
  }
  const uint32_t wtot = __shfl_sync(FULL, wf, 31);
  unsigned long long base = 0;
  if (lane == 31) base = atomicAdd(&p.st->n_cand, (unsigned long long)wtot);
  base = __shfl_sync(FULL, base, 31);
  uint64_t slot = base + wf - nf;
#pragma unroll
  for (int j = 0; j < RI; ++j) {
    if (!fk[j]) continue;
    if (slot < p.cand_cap) {
      const uint64_t wr = bucket_base + word[j];
      p.cand[slot] = make_uint4((uint32_t)wr, (uint32_t)(wr >> 32), pos[j], fk[j]);
    }
    ++slot;
  }
}

__device__ __forceinline__ uint32_t classify(uint32_t op, uint32_t before) {
  if (op == OP_RH && !(before & kOVv)) return (before & kOVi) ? 2u : 1u;   // USD : UUM
  if (op == OP_RT && !(before & kCVv)) return (before & kCVi) ? 2u : 1u;
  return 0u;
}

__device__ __forceinline__ void hash_clear(ReplaySmem& S) {
  for (uint32_t i = threadIdx.x; i < kHSlots; i += RT) S.u.h.slot[i] = make_uint2(kEmpty, kEmpty);
}

// VSM write by access op (WH = 1, WT = 3) on a 4-bit state, branch-free
__device__ __forceinline__ uint32_t vsm_write_op(uint32_t op, uint32_t s) {
  return op == OP_WH ? ((s & kCVi) | kOVv | kOVi) : ((s & kOVi) | kCVv | kCVi);
}
// fault kind of an access with state-before `before`: a read
// (RH = 0, RT = 2) whose side (bit op/2) is not valid: UUM (1) if that side was
// never initialised, else USD (2); 0 for writes and valid reads
__device__ __forceinline__ uint32_t classify_bits(uint32_t op, uint32_t before) {
  const uint32_t v = before >> (op >> 1);
  return (op & 1u) || (v & 1u) || op > 3 ? 0u : 1u + ((v >> 2) & 1u);
}

// ---- several accelerators (Z24): 8-bit states ---------------------------------------------
constexpr uint32_t kMdPos = 0x3FFFFFFFu;        // event position without the device bits
constexpr uint32_t kMdAllCvv = 0x52u;           // CV0v | CV1v | CV2v
// the state after a write: code bit 0 = target, bits 1-2 = its device
__device__ __forceinline__ uint32_t md_write(uint32_t code, uint32_t s) {
  if (!(code & 1u)) return (s & ~kMdAllCvv) | kOVv | kOVi;
  const uint32_t d = code >> 1;
  return (s & ~(kMdAllCvv | kOVv)) | (1u << md_cvv(d)) | (1u << md_cvi(d));
}
__device__ __forceinline__ uint32_t md_classify(uint32_t op, uint32_t dev, uint32_t s) {
  if (op == OP_RH) return (s & kOVv) ? 0u : ((s & kOVi) ? 2u : 1u);
  if (op == OP_RT) return ((s >> md_cvv(dev)) & 1u) ? 0u : (((s >> md_cvi(dev)) & 1u) ? 2u : 1u);
  return 0u;
}

// hash slot of a word (Fibonacci hashing: consecutive words land far apart, so
// the linear probe chains of a run's words stay short)
__device__ __forceinline__ uint32_t hslot(uint32_t w) { return (w * 2654435761u) >> (32 - kHBits); }

// ---- fast step: at most one write per word -------------------------------------------
// Returns false (and leaves the shadow untouched) if some word has two writes.
//
// Only writes enter the hash (word -> first write position | kind): reads do
// not change the state, so a read's state-before is the state loaded
// at the start of the step, or — if its word's single write precedes it — the
// image of that write; the write event itself commits the word's final state.
//
// BO (ARB_F_BO) is a template parameter: deciding that a target access is a
// buffer overflow needs its word's state before the inserts, which would put
// the shadow-load latency in front of the hashing for every replay.
// UM (ARB_F_UNIFIED, Z23): OV and CV are one storage — a write of either side
// makes the word's state 0xF (both valid, both initialised).
// MD (several accelerators, Z24): 8-bit states; the device of a target access is in
// bits 30-31 of its position, and a hash slot holds pos << 3 | device << 1 | target.
template <bool PARTIAL, bool BO, bool UM, bool MD>
__device__ __forceinline__ bool step_fast(ReplaySmem& S, const ReplayParams& p, const uint2* ev, uint32_t m) {
  uint32_t slot[RI], word[RI], pos[RI], op[RI], s_pre[RI];
  uint32_t bom = 0;                // bit j: event j is a buffer overflow (ARB_F_BO, Z20)
  uint32_t devs = 0;               // MD: 2 bits per event
  bool multi = false;
  const uint8_t* sh = S.shrel;
  uint2* hs = S.u.h.slot;
  uint32_t plo = 0, pw = 0;
  if (PARTIAL) { plo = S.part_lo; pw = S.part_hi - S.part_lo; }
#pragma unroll
  for (int j = 0; j < RI; ++j) {   // shadow loads first: their latency overlaps the hashing
    const uint32_t i = threadIdx.x + j * RT;
    slot[j] = 0; word[j] = 0; pos[j] = 0; op[j] = 4; s_pre[j] = 0;
    if (i < m) {
      const uint2 e = ev[i];
      word[j] = e.x & kWordMask; op[j] = e.x >> 30; pos[j] = MD ? (e.y & kMdPos) : e.y;
      if (MD) devs |= (e.y >> 30) << (2 * j);
      if (!PARTIAL || word[j] - plo < pw) s_pre[j] = __ldcg(sh + word[j]);
      else op[j] = 4;                                       // another work item's word
      // a target access (RT = 2, WT = 3) to a word without a CV: BO, no VSM effect
      if (BO && (op[j] & 2u) && !(s_pre[j] & kCVp)) { bom |= 1u << j; op[j] = 4; }
    }
  }
  // writes (WH = 1, WT = 3: odd ops) enter the table: slot {word, pos << 2 | op}
  bool any_w = false;
#pragma unroll
  for (int j = 0; j < RI; ++j) {
    if (op[j] & 1u) {
      any_w = true;
      uint32_t h = hslot(word[j]);
      bool won = false;
      for (;;) {
        const uint32_t old = atomicCAS(&hs[h].x, kEmpty, word[j]);
        if (old == kEmpty) { won = true; break; }
        if (old == word[j]) { multi = true; break; }        // a second write of the word
        h = (h + 1) & (kHSlots - 1);
      }
      slot[j] = h;
      if (won)   // the slot's owner; a second writer only flags the fallback
        hs[h].y = MD ? ((pos[j] << 3) | (((devs >> (2 * j)) & 3u) << 1) | (op[j] >> 1)) : ((pos[j] << 2) | op[j]);
    }
  }
  any_w = __syncthreads_or(any_w);
  if (any_w && __syncthreads_or(multi)) {
#pragma unroll
    for (int j = 0; j < RI; ++j)
      if (op[j] & 1u) hs[slot[j]] = make_uint2(kEmpty, kEmpty);
    __syncthreads();
    return false;
  }
  uint32_t fk[RI];
#pragma unroll
  for (int j = 0; j < RI; ++j) {
    const uint32_t s0 = s_pre[j] & (MD ? 255u : 15u);
    uint32_t before = s0;
    if (op[j] == OP_RH || op[j] == OP_RT) {
      if (any_w) {
        uint32_t h = hslot(word[j]);
        for (;;) {                                          // probe for the word's write
          const uint2 k = hs[h];
          if (k.x == word[j]) {
            if (MD) { if ((k.y >> 3) < pos[j]) before = md_write(k.y & 7u, s0); }
            else if ((k.y >> 2) < pos[j]) before = UM ? 15u : vsm_write_op(k.y & 3u, s0);
            break;
          }
          if (k.x == kEmpty) break;
          h = (h + 1) & (kHSlots - 1);
        }
      }
    } else if (op[j] & 1u) {
      __stcg(const_cast<uint8_t*>(sh) + word[j],
             (uint8_t)(MD ? md_write((op[j] >> 1) | (((devs >> (2 * j)) & 3u) << 1), s0)
                       : UM ? 15u : vsm_write_op(op[j], s0) | (BO ? (s_pre[j] & kCVp) : 0u)));
    }
    fk[j] = ((bom >> j) & 1u) ? 4u : MD ? md_classify(op[j], (devs >> (2 * j)) & 3u, before)
                                        : classify_bits(op[j], before);
  }
  emit_faults(p, fk, word, pos, S.bucket_base);
  if (any_w) {
    __syncthreads();
#pragma unroll
    for (int j = 0; j < RI; ++j)
      if (op[j] & 1u) hs[slot[j]] = make_uint2(kEmpty, kEmpty);
  }
  // the caller's next barrier orders this reset before the next step's inserts
  return true;
}

// the fast step of a word-range part (rare: range-heavy buckets), out of line
template <bool BO, bool UM, bool MD>
__device__ bool step_fast_partial(ReplaySmem& S, const ReplayParams& p, const uint2* ev, uint32_t m) {
  return step_fast<true, BO, UM, MD>(S, p, ev, m);
}

// ---- sort step -------------------------------------------------------------------------
// One stable LSD pass on the word offset (low 30 bits of the key) of m elements.
__device__ void sort_pass(ReplaySmem& S, const uint32_t* kin, const uint32_t* pin, uint32_t* kout,
                          uint32_t* pout, uint32_t m, uint32_t minw, uint32_t shift, uint32_t dmask) {
  const uint32_t tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  uint32_t* h32 = reinterpret_cast<uint32_t*>(&S.u.s.hist[0][0]);
  for (uint32_t i = tid; i < (RT / 32) * 256 / 2; i += RT) h32[i] = 0;
  __syncthreads();
  uint16_t* row = S.u.s.hist[warp];
  uint32_t kk[RI], pp[RI], rk[RI], dg[RI];
  const uint32_t lt = lanemask_lt();
#pragma unroll
  for (int r = 0; r < RI; ++r) {
    const uint32_t i = warp * (32 * RI) + r * 32 + lane;
    const bool valid = i < m;
    const uint32_t k = valid ? kin[i] : 0, pv = valid ? pin[i] : 0;
    const uint32_t d = valid ? ((((k & kWordMask) - minw) >> shift) & dmask) : 0xFFFFu;
    const uint32_t grp = __match_any_sync(FULL, d);
    const uint32_t base = valid ? row[d] : 0;
    __syncwarp();
    if (valid && lane == 31u - __clz(grp)) row[d] = (uint16_t)(base + __popc(grp));
    __syncwarp();
    kk[r] = k; pp[r] = pv; dg[r] = d; rk[r] = base + __popc(grp & lt);
  }
  __syncthreads();
  if (tid < 256) {   // digit tid: per-warp offsets and total
    uint32_t s = 0;
#pragma unroll
    for (int w = 0; w < RT / 32; ++w) {
      const uint32_t c = S.u.s.hist[w][tid];
      S.u.s.hist[w][tid] = (uint16_t)s;
      s += c;
    }
    S.pref[tid] = s;
  }
  __syncthreads();
  if (tid < 32) {   // exclusive scan of the 256 digit totals by one warp
    uint32_t v[8], t = 0;
#pragma unroll
    for (int j = 0; j < 8; ++j) { v[j] = S.pref[tid * 8 + j]; t += v[j]; }
    uint32_t incl = t;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
      const uint32_t o = __shfl_up_sync(FULL, incl, d);
      if (tid >= (uint32_t)d) incl += o;
    }
    uint32_t run = incl - t;
#pragma unroll
    for (int j = 0; j < 8; ++j) { S.pref[tid * 8 + j] = run; run += v[j]; }
  }
  __syncthreads();
  if (tid < 256) {
    const uint32_t b = S.pref[tid];
#pragma unroll
    for (int w = 0; w < RT / 32; ++w) S.u.s.hist[w][tid] = (uint16_t)(S.u.s.hist[w][tid] + b);
  }
  __syncthreads();
#pragma unroll
  for (int r = 0; r < RI; ++r) {
    const uint32_t i = warp * (32 * RI) + r * 32 + lane;
    if (i < m) {
      const uint32_t o = S.u.s.hist[warp][dg[r]] + rk[r];
      kout[o] = kk[r];
      pout[o] = pp[r];
    }
  }
  __syncthreads();
}

// access transition monoid for the segmented scan:
//   bit7 HEAD, bit6 CONST; const: bits0-3 = state; summary: bits0-1 last
//   write (1 WH, 2 WT), bit2 any WH, bit3 any WT.  0 is the identity.
constexpr uint32_t kHead = 0x80, kConst = 0x40;
__device__ __forceinline__ uint32_t acc_apply(uint32_t v, uint32_t s) {
  const uint32_t lw = v & 3u;
  if (lw) s = (s & ~3u) | lw;     // WH: OVv=1,CVv=0 ; WT: OVv=0,CVv=1
  return s | (v & 12u);           // any WH sets OVi, any WT sets CVi
}
__device__ __forceinline__ uint32_t acc_combine(uint32_t a, uint32_t b) {  // a before b
  if (b & kHead) return b;
  if (a & kConst) return (a & kHead) | kConst | acc_apply(b, a & 15u);
  const uint32_t lw = (b & 3u) ? (b & 3u) : (a & 3u);
  return (a & kHead) | lw | ((a | b) & 12u);
}
__device__ __forceinline__ uint32_t acc_summary(uint32_t op) {
  return op == OP_WH ? (1u | 4u) : (op == OP_WT ? (2u | 8u) : 0u);
}
// MD (Z24): bit 31 HEAD, bit 30 CONST; const: bits 0-7 = state; summary: bits 0-2
// last write (1 host, 2 + d target on device d), bits 3-6 "some write initialised"
// OV, CV0, CV1, CV2.
constexpr uint32_t kHeadMd = 1u << 31, kConstMd = 1u << 30;
__device__ __forceinline__ uint32_t acc_apply_md(uint32_t v, uint32_t s) {
  const uint32_t lw = v & 7u;
  if (lw == 1u) s = (s & ~kMdAllCvv) | kOVv;
  else if (lw >= 2u) s = (s & ~(kMdAllCvv | kOVv)) | (1u << md_cvv(lw - 2u));
  if (v & 8u) s |= kOVi;
#pragma unroll
  for (uint32_t d = 0; d < 3; ++d)
    if (v & (16u << d)) s |= 1u << md_cvi(d);
  return s;
}
__device__ __forceinline__ uint32_t acc_combine_md(uint32_t a, uint32_t b) {  // a before b
  if (b & kHeadMd) return b;
  if (a & kConstMd) return (a & kHeadMd) | kConstMd | acc_apply_md(b, a & 255u);
  const uint32_t lw = (b & 7u) ? (b & 7u) : (a & 7u);
  return (a & kHeadMd) | lw | ((a | b) & 0x78u);
}
__device__ __forceinline__ uint32_t acc_summary_md(uint32_t op, uint32_t dev) {
  return op == OP_WH ? (1u | 8u) : (op == OP_WT ? ((2u + dev) | (16u << dev)) : 0u);
}
template <bool MD>
__device__ __forceinline__ uint32_t acc_comb(uint32_t a, uint32_t b) { return MD ? acc_combine_md(a, b) : acc_combine(a, b); }

template <bool BO, bool UM, bool MD>
__device__ void step_sort(ReplaySmem& S, const ReplayParams& p, const uint2* ev, uint32_t m) {
  const uint32_t tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  uint32_t lo = 0xFFFFFFFFu, hi = 0;
  if (S.partial) {
    // keep only the events of the work item's words (stable block compaction)
    uint32_t keep[RI], c = 0;
#pragma unroll
    for (int j = 0; j < RI; ++j) {
      const uint32_t i = tid * RI + j;
      const uint32_t w = i < m ? (ev[i].x & kWordMask) : 0;
      keep[j] = i < m && w >= S.part_lo && w < S.part_hi;
      c += keep[j];
    }
    uint32_t incl = c;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
      const uint32_t o = __shfl_up_sync(FULL, incl, d);
      if (lane >= (uint32_t)d) incl += o;
    }
    __syncthreads();
    if (lane == 31) S.wscan[warp] = incl;
    __syncthreads();
    uint32_t o = incl - c, tot = 0;
    for (uint32_t w = 0; w < RT / 32; ++w) { if (w < warp) o += S.wscan[w]; tot += S.wscan[w]; }
#pragma unroll
    for (int j = 0; j < RI; ++j) {
      if (keep[j]) {
        const uint2 e = ev[tid * RI + j];
        S.u.s.keyA[o] = e.x; S.u.s.posA[o] = e.y;
        const uint32_t w = e.x & kWordMask;
        lo = min(lo, w); hi = max(hi, w);
        ++o;
      }
    }
    m = tot;
    if (m == 0) {
      __syncthreads();
      hash_clear(S);
      __syncthreads();
      return;
    }
  } else {
    for (uint32_t i = tid; i < m; i += RT) {
      const uint2 e = ev[i];
      S.u.s.keyA[i] = e.x; S.u.s.posA[i] = e.y;
      const uint32_t w = e.x & kWordMask;
      lo = min(lo, w); hi = max(hi, w);
    }
  }
  block_minmax(lo, hi, S.red, S.red2);
  const uint32_t span = hi - lo;
  const uint32_t bits = span ? 32 - __clz(span) : 0;
  uint32_t* kin = S.u.s.keyA; uint32_t* pin = S.u.s.posA; uint32_t* kout = S.u.s.keyB; uint32_t* pout = S.u.s.posB;
  for (uint32_t sh = 0; sh < bits; sh += 8) {
    sort_pass(S, kin, pin, kout, pout, m, lo, sh, (1u << min(8u, bits - sh)) - 1u);
    uint32_t* t = kin; kin = kout; kout = t;
    t = pin; pin = pout; pout = t;
  }
  // blocked arrangement: thread t owns sorted elements [RI*t, RI*t + RI)
  const uint64_t bb = S.bucket_base;
  uint8_t* const sh = S.shrel;
  uint32_t val[RI], s0[RI], key[RI], wd[RI], ps[RI], pf[RI];
  bool head[RI], isb[RI];
  uint32_t agg = 0;
  constexpr bool bo = BO;
#pragma unroll
  for (int j = 0; j < RI; ++j) {
    const uint32_t i = tid * RI + j;
    key[j] = 0; head[j] = false; s0[j] = 0; val[j] = 0; wd[j] = 0; ps[j] = 0; pf[j] = 0; isb[j] = false;
    if (i < m) {
      const uint32_t k = kin[i];
      const uint32_t w = k & kWordMask;
      const bool h = (i == 0) || ((kin[i - 1] & kWordMask) != w);
      // ARB_F_BO: kCVp is constant within a step (range ops cut steps); a target
      // access to a word without a CV is BO and the identity (Z20)
      const uint32_t full = (h || bo) ? __ldcg(sh + w) : 0u;
      const bool b = bo && ((k >> 30) & 2u) && !(full & kCVp);
      // UM: every write is {both valid, both initialised} (last write 3, any-WH and any-WT)
      const uint32_t dev = MD ? pin[i] >> 30 : 0u;
      uint32_t v = b ? 0u : MD ? acc_summary_md(k >> 30, dev) : UM ? (((k >> 30) & 1u) ? 15u : 0u)
                                                                  : acc_summary(k >> 30);
      uint32_t st = 0;
      if (h) {
        st = full & (MD ? 255u : 15u);
        v = MD ? (kHeadMd | kConstMd | acc_apply_md(v, st)) : (kHead | kConst | acc_apply(v, st));
      }
      key[j] = k; head[j] = h; s0[j] = st; val[j] = v; wd[j] = w;
      ps[j] = MD ? (pin[i] & kMdPos) : pin[i];
      pf[j] = MD ? dev : (full & kCVp);          // MD: the event's device (no kCVp bit then)
      isb[j] = b;
    }
    agg = acc_comb<MD>(agg, val[j]);
  }
  uint32_t incl = agg;
#pragma unroll
  for (int d = 1; d < 32; d <<= 1) {
    const uint32_t o = __shfl_up_sync(FULL, incl, d);
    if (lane >= (uint32_t)d) incl = acc_comb<MD>(o, incl);
  }
  uint32_t excl_lane = __shfl_up_sync(FULL, incl, 1);
  if (lane == 0) excl_lane = 0;
  __syncthreads();
  if (lane == 31) S.wscan[warp] = incl;
  __syncthreads();
  uint32_t wpre = 0;
  for (uint32_t w = 0; w < warp; ++w) wpre = acc_comb<MD>(wpre, S.wscan[w]);
  uint32_t run = acc_comb<MD>(wpre, excl_lane);
  uint32_t fk[RI];
#pragma unroll
  for (int j = 0; j < RI; ++j) {
    const uint32_t i = tid * RI + j;
    fk[j] = 0;
    if (i < m) {
      const uint32_t before = head[j] ? s0[j] : (run & (MD ? 255u : 15u));
      run = acc_comb<MD>(run, val[j]);
      fk[j] = isb[j] ? 4u : MD ? md_classify(key[j] >> 30, pf[j], before) : classify(key[j] >> 30, before);
      const bool tail = (i + 1 == m) || ((kin[i + 1] & kWordMask) != wd[j]);
      if (tail) __stcg(sh + wd[j], (uint8_t)(MD ? (run & 255u) : ((run & 15u) | pf[j])));
    }
  }
  emit_faults(p, fk, wd, ps, bb);
  __syncthreads();
  hash_clear(S);      // the sort arrays overlap the hash table
  __syncthreads();
}

// ---- hot bucket slices (K5) ---------------------------------------------------------
// Phase 1: compose, for every word of the bucket, the transition function of the
// slice (selector form; reads are identity).  Within a step a word's
// writes compose to: valid bits of the last write, OVi set if any WH, CVi set if
// any WT (Table II init bits); the last write of each word (by step
// index) folds that function into fsum.  ARB_F_BO: CVp is constant inside a step
// (range ops cut steps), so for each half of the pair the word's CVp after the
// slice so far decides whether its target writes count (Z20).  Several
// accelerators: the last write's device and the devices any WT initialised (Z24).
template <bool BO, bool UM, bool MD>
__device__ void step_summary(ReplaySmem& S, const uint2* ev, uint32_t m) {
  uint32_t* key = S.u.z.key;
  uint32_t* lastw = S.u.z.lastw;
  uint32_t* anyw = S.u.z.anyw;
  uint32_t word[RI], op[RI], idx[RI], slot[RI];
  bool last[RI];
  uint32_t ab[RI], lw[RI];
#pragma unroll
  for (int j = 0; j < RI; ++j) {
    const uint32_t i = threadIdx.x + j * RT;
    op[j] = 4; word[j] = 0; idx[j] = i + 1; slot[j] = 0;
    if (i < m) {
      const uint2 e = ev[i];
      word[j] = e.x & kWordMask; op[j] = e.x >> 30;
      const uint32_t dev = MD ? e.y >> 30 : 0u;
      if (op[j] & 1u) {                // a write: find or insert the word's slot
        uint32_t h = (word[j] * 2654435761u) >> (32 - kZBits);
        for (;;) {
          const uint32_t old = atomicCAS(&key[h], kEmpty, word[j]);
          if (old == kEmpty || old == word[j]) break;
          h = (h + 1) & (kZSlots - 1);
        }
        slot[j] = h;
        atomicMax(&lastw[h], (idx[j] << 4) | (dev << 2) | op[j]);
        atomicOr(&anyw[h >> 2], (op[j] == OP_WH ? 1u : (2u << dev)) << (8 * (h & 3)));   // bit 0 WH, bit 1 + d WT on d
      }
    }
  }
  __syncthreads();
#pragma unroll
  for (int j = 0; j < RI; ++j) {
    const uint32_t l = (op[j] & 1u) ? lastw[slot[j]] : 0u;
    last[j] = (op[j] & 1u) && (l >> 4) == idx[j];
    ab[j] = last[j] ? (anyw[slot[j] >> 2] >> (8 * (slot[j] & 3))) & 0xFFu : 0u;
    lw[j] = l & 15u;
  }
  __syncthreads();
#pragma unroll
  for (int j = 0; j < RI; ++j) {
    if (last[j]) {
      const uint32_t f = S.fsum[word[j]];
      uint32_t nf;
      if (MD) {
        const uint32_t ldev = (lw[j] >> 2) & 3u;
        const bool host = (lw[j] & 3u) == OP_WH;
        uint32_t g = kSel8Id;
        g = sel8_set(g, 0, host ? 9u : 8u);                             // OVv: the last write was the host's
        for (uint32_t d = 0; d < 3; ++d) {
          g = sel8_set(g, md_cvv(d), (!host && ldev == d) ? 9u : 8u);   // only the writing device's CV valid
          if (ab[j] & (2u << d)) g = sel8_set(g, md_cvi(d), 9u);       // initialised by a WT on d
        }
        if (ab[j] & 1u) g = sel8_set(g, 2, 9u);                        // OVi: some WH
        nf = sel8_compose(g, f);
      } else {
        const Sel g = UM ? sel_make(5, 5, 5, 5)                                      // Z23: one shared value
                    : op[j] == OP_WH ? sel_make(5, 4, 5, (ab[j] & 2u) ? 5 : 3)     // OV latest; CVi kept unless a WT
                                     : sel_make(4, 5, (ab[j] & 1u) ? 5 : 2, 5);    // CV latest; OVi kept unless a WH
        if (BO) {
          // without a CV the step's target writes do nothing: only its host writes count
          const Sel gh = (ab[j] & 1u) ? sel_make(5, 4, 5, 3) : kSelId;
          const uint32_t lo = f & 0xFFFFu, hi = f >> 16;
          nf = sel_compose(half_cvp(lo, 0u) ? g : gh, lo) | (sel_compose(half_cvp(hi, 1u) ? g : gh, hi) << 16);
        } else {
          nf = sel_compose(g, f);
        }
      }
      S.fsum[word[j]] = nf;
      key[slot[j]] = kEmpty;           // the word's only slot: reset by its last writer
      lastw[slot[j]] = 0;
      atomicAnd(&anyw[slot[j] >> 2], ~(0xFFu << (8 * (slot[j] & 3))));
    }
  }
  __syncthreads();
}

// Position of event e of the bucket (one thread; several accelerators: device bits stripped).
__device__ uint32_t event_pos(const ReplaySmem& S, const ReplayParams& p, uint32_t e) {
  uint32_t lo = 0, z = S.n_segs;
  while (z - lo > 1) {
    const uint32_t mid = (lo + z) >> 1;
    if (p.segs[S.seg0 + mid].w - S.cum0 <= e) lo = mid; else z = mid;
  }
  const uint4 sg = p.segs[S.seg0 + lo];
  const uint32_t st = sg.z & 0xFFFFu, off = e - (sg.w - S.cum0);
  const uint32_t pos = (st & kRunFlag) ? p.part_ev[(uint64_t)sg.x * kChunkCap + (st & ~kRunFlag)].y + off
                                       : p.part_ev[(uint64_t)sg.x * kChunkCap + st + off].y;
  return p.md ? (pos & kMdPos) : pos;
}
// first op of the bucket (ops [a, z), trace order) at or after position q
__device__ uint32_t ops_lower_bound(const ReplayParams& p, uint32_t a, uint32_t z, uint32_t q) {
  while (a < z) {
    const uint32_t mid = (a + z) >> 1;
    if (p.ops[mid].pos < q) a = mid + 1; else z = mid;
  }
  return a;
}

// Phase 2: carry the word states across the slices (grid: words x hot buckets).
template <bool BO, bool MD>
__global__ void k_carry(const uint4* hot, const uint64_t* bucket_start, const uint64_t* hot_off,
                        const uint32_t* hot_F, uint8_t* hot_P, uint8_t* shadow) {
  const uint4 h = hot[blockIdx.y];
  const uint32_t b = h.x, slices = h.y, span = h.z, span16 = (span + 15) & ~15u;
  const uint64_t off = hot_off[b];
  uint8_t* sh = shadow + bucket_start[b];
  for (uint32_t w = blockIdx.x * blockDim.x + threadIdx.x; w < span; w += gridDim.x * blockDim.x) {
    uint32_t st = sh[w];
    for (uint32_t k = 0; k < slices; ++k) {
      hot_P[off + (uint64_t)k * span16 + w] = (uint8_t)st;
      st = kfun_apply<BO, MD>(hot_F[off + (uint64_t)k * span16 + w], st);
    }
    sh[w] = (uint8_t)st;
  }
}

cudaError_t launch_carry(const uint4* hot, uint32_t n_hot, uint32_t max_span, const uint64_t* bucket_start,
                         const uint64_t* hot_off, const uint32_t* hot_F, uint8_t* hot_P, uint8_t* shadow,
                         int bo, int md, cudaStream_t s) {
  if (!n_hot) return cudaSuccess;
  const uint32_t gx = std::min<uint32_t>((max_span + 255) / 256, 1024);
  auto kern = md ? k_carry<false, true> : bo ? k_carry<true, false> : k_carry<false, false>;
  kern<<<dim3(gx, n_hot), 256, 0, s>>>(hot, bucket_start, hot_off, hot_F, hot_P, shadow);
  return cudaGetLastError();
}

// ---- the bucket's segments -------------------------------------------------------------
// The sorted entries of bucket b are p.segs[f0, f1) in chunk order (= trace
// order); entry i covers bucket-relative events [segs[i].w - segs[f0].w, + len)
// stored at part_ev[chunk * kChunkCap + start].
__device__ void bucket_setup(ReplaySmem& S, const ReplayParams& p, uint32_t b) {
  if (threadIdx.x == 0) {
    const uint32_t f0 = p.seg_first[b], f1 = p.seg_first[b + 1];
    S.seg0 = f0; S.n_segs = f1 - f0;
    S.cum0 = 0; S.n_events = 0;
    if (f1 > f0) {
      const uint4 first = p.segs[f0], last = p.segs[f1 - 1];
      S.cum0 = first.w;
      S.n_events = last.w + (last.z >> 16) - first.w;
    }
    S.wsc = 0; S.nwin = 0; S.wcum[0] = 1;      // empty window: forces a load
  }
  __syncthreads();
}

// Make the staged window of segment descriptors contain event e0 (reloads
// about every kWin segments; sequential progress needs no search).
__device__ void ensure_window(ReplaySmem& S, const ReplayParams& p, uint32_t e0, uint32_t& hint) {
  if (e0 >= S.wcum[0] && e0 < S.wcum[S.nwin]) return;
  hint = 0;
  __syncthreads();
  if (threadIdx.x == 0) {
    uint32_t a;
    if (S.nwin && e0 == S.wcum[S.nwin]) {
      a = S.wsc + S.nwin;                       // the window's successor
    } else {                                    // last segment starting at or before e0
      uint32_t lo = 0, z = S.n_segs;
      while (z - lo > 1) {
        const uint32_t mid = (lo + z) >> 1;
        if (p.segs[S.seg0 + mid].w - S.cum0 <= e0) lo = mid; else z = mid;
      }
      a = lo;
    }
    S.wsc = a;
    S.nwin = min((uint32_t)kWin, S.n_segs - a);
  }
  __syncthreads();
  const uint32_t sc = S.wsc, nwin = S.nwin;
  const uint4* segs = p.segs + S.seg0 + sc;
  for (uint32_t k = threadIdx.x; k < nwin; k += RT) {
    const uint4 e = segs[k];
    const uint32_t st = e.z & 0xFFFFu;         // bit 31 of wstart: a run segment
    S.wstart[k] = (e.x * (uint32_t)kChunkCap + (st & ~kRunFlag)) | ((st & kRunFlag) << 16);
    S.wcum[k] = e.w - S.cum0;
  }
  if (threadIdx.x == 0) S.wcum[nwin] = sc + nwin < S.n_segs ? segs[nwin].w - S.cum0 : S.n_events;
  __syncthreads();
}

// Event j of window segment `seg` into shared memory: a cp.async of the stored
// event, or (a run segment, bit 31 of wstart) the run's descriptor + j.
__device__ __forceinline__ void gather_ev(uint2* d, const ReplayParams& p, uint32_t ws, uint32_t j) {
  if (ws >> 31) {
    const uint2 r = p.part_ev[ws & 0x7FFFFFFFu];
    *d = make_uint2(r.x + j, r.y + j);
  } else {
    cp_async8(d, p.part_ev + (ws + j));
  }
}

// Stage the step that starts at event e0 of the bucket into buffer buf; the
// window must contain e0.  Returns the step's event count m.
// `hint` (per thread, block-uniform) is a window segment index with
// wcum[hint] <= e0; it is advanced to the last segment gathered.
//
// Run step (runs_ok: a whole-bucket item of a single-device context): when the
// segment holding e0 is a run segment, the step is the following run segments (at
// most kMaxStepRuns, p.run_step_max events, the window's end): warp 0 stages one
// {offset, count, start} entry per segment and cp.async-copies its descriptor;
// nrun = the number of segments.  Otherwise an event step of <= STEP events
// (nrun = 0): cp.async copies of the stored events, runs synthesised.
__device__ uint32_t issue_gather(ReplaySmem& S, const ReplayParams& p, uint32_t e0, uint32_t total, uint32_t buf,
                                 uint32_t& hint, bool runs_ok, uint32_t& nrun) {
  nrun = 0;
  const uint32_t lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const uint32_t nwin = S.nwin;
  uint2* dst = S.ev[buf];
  const uint32_t base0 = hint & ~31u;
  if (runs_ok) {
    // the segment holding e0: usually the hint or the next one (steps end at segment ends)
    uint32_t sa = hint;
    if (sa + 1 < nwin && S.wcum[sa + 1] <= e0) {
      ++sa;
      if (sa + 1 < nwin && S.wcum[sa + 1] <= e0) {
        uint32_t c0 = 0;                   // segments of the window starting at or before e0
        for (uint32_t base = base0; base < nwin; base += 32) {
          const uint32_t j = base + lane;
          const uint32_t bl = __ballot_sync(FULL, (j < nwin ? S.wcum[j] : 0xFFFFFFFFu) <= e0);
          c0 += __popc(bl);
          if (bl != FULL) break;
        }
        sa = base0 + c0 - 1;
      }
    }
    if (S.wstart[sa] >> 31) {
      const uint32_t j = sa + lane;
      const uint32_t msk = __ballot_sync(FULL, j < nwin && (S.wstart[j] >> 31));
      const uint32_t nr = msk == FULL ? 32u : (uint32_t)__ffs(~msk) - 1u;   // consecutive run segments
      const uint32_t e_end = min(min(total, S.wcum[sa + nr]), e0 + p.run_step_max);
      const bool in = lane < nr && S.wcum[j] < e_end;
      const uint32_t nseg = __popc(__ballot_sync(FULL, in));
      if (warp == 0 && in) {
        RunStage& R = *reinterpret_cast<RunStage*>(dst);
        const uint32_t a = max(S.wcum[j], e0), z = min(S.wcum[j + 1], e_end);
        R.info[lane] = make_uint4(a - S.wcum[j], z - a, a - e0, 0u);
        cp_async8(&R.desc[lane], p.part_ev + (S.wstart[j] & 0x7FFFFFFFu));
      }
      cp_async_commit();
      nrun = nseg;
      hint = sa + nseg - 1;
      return e_end - e0;
    }
  }
  const uint32_t m = min(min((uint32_t)STEP, total - e0), S.wcum[nwin] - e0);
  // Warp w gathers the slice [e0 + 32*RI*w, +32*RI) of the step.  Segment j holds
  // event e iff wcum[j] <= e < wcum[j+1]; every warp counts, from the hint, the
  // segments starting at or before its slice start and before the step's last
  // event (ballots, no barrier), then each lane walks forward to the segment of
  // each of its events (segments are usually longer than the slice).
  const uint32_t s0 = e0 + warp * (32 * RI), last = e0 + m - 1;
  uint32_t c0 = 0, c1 = 0;
  for (uint32_t base = base0; base < nwin; base += 32) {
    const uint32_t j = base + lane;
    const uint32_t w = j < nwin ? S.wcum[j] : 0xFFFFFFFFu;
    c0 += __popc(__ballot_sync(FULL, w <= s0));
    const uint32_t b1 = __ballot_sync(FULL, w <= last);
    c1 += __popc(b1);
    if (b1 != FULL) break;
  }
  hint = base0 + c1 - 1;                 // segment of the step's last event
  if (s0 < e0 + m) {
    uint32_t seg = base0 + c0 - 1, seg_end = S.wcum[seg + 1];
    const uint32_t s_end = min(s0 + 32 * RI, e0 + m);
    uint2* d = dst + (s0 - e0);
    if (s_end <= seg_end) {
      // the whole slice lies in one segment (warp-uniform; the common case):
      // a contiguous copy, 16 B per lane when both sides are 16-B aligned
      const uint32_t ws = S.wstart[seg], c = S.wcum[seg];
      const uint32_t cnt = s_end - s0;
      if (ws >> 31) {
        const uint2 r = p.part_ev[ws & 0x7FFFFFFFu];
#pragma unroll
        for (int k = 0; k < RI; ++k)
          if (lane + 32 * k < cnt) d[lane + 32 * k] = make_uint2(r.x + (s0 - c) + lane + 32 * k, r.y + (s0 - c) + lane + 32 * k);
      } else {
        const uint2* src = p.part_ev + (ws + (s0 - c));
        if (cnt == 32 * RI && ((reinterpret_cast<uintptr_t>(src) & 15u) == 0)) {
#pragma unroll
          for (int k = 0; k < RI / 2; ++k) cp_async16(d + 2 * (lane + 32 * k), src + 2 * (lane + 32 * k));
        } else {
#pragma unroll
          for (int k = 0; k < RI; ++k)
            if (lane + 32 * k < cnt) cp_async8(d + lane + 32 * k, src + lane + 32 * k);
        }
      }
      cp_async_commit();
      return m;
    }
    d += lane;
    if (seg + 2 <= nwin && s_end <= S.wcum[seg + 2]) {
      // two segments: select the segment per event
#pragma unroll
      for (int k = 0; k < RI; ++k) {
        const uint32_t e = s0 + k * 32 + lane;
        if (e < s_end) {
          const uint32_t sg = e < seg_end ? seg : seg + 1;
          gather_ev(d + k * 32, p, S.wstart[sg], e - S.wcum[sg]);
        }
      }
      cp_async_commit();
      return m;
    }
#pragma unroll
    for (int k = 0; k < RI; ++k) {
      const uint32_t e = s0 + k * 32 + lane;
      if (e < e0 + m) {
        if (e >= seg_end) {
          do { ++seg; seg_end = S.wcum[seg + 1]; } while (e >= seg_end);
        }
        gather_ev(d + k * 32, p, S.wstart[seg], e - S.wcum[seg]);
      }
    }
  }
  cp_async_commit();
  return m;
}

// ---- run step -------------------------------------------------------------------------
// Byte mask of bytes [a, a + n) of a 32-bit group (n = 1..4)
// Run steps process the shadow in aligned groups of kGW words (kGW states in one
// GWord, SWAR form): 4 words / 32 bits, 8 words / 64 bits or 16 words / 2 x 64
// bits (ARB_RUN_GROUP_WORDS).  The SWAR code only shifts right by < 8 bits before
// masking one bit per byte, so the 128-bit form needs no carries between halves.
#ifndef ARB_RUN_GROUP_WORDS
#define ARB_RUN_GROUP_WORDS 16
#endif
constexpr uint32_t kGW = ARB_RUN_GROUP_WORDS;
constexpr uint32_t kGWLog = kGW == 16 ? 4 : kGW == 8 ? 3 : 2;
static_assert(kGW == 4 || kGW == 8 || kGW == 16, "4-, 8- or 16-word groups");
struct W16 {
  unsigned long long x, y;
  __host__ __device__ constexpr W16(unsigned long long a = 0) : x(a), y(a) {}     // both halves
  __host__ __device__ constexpr W16(unsigned long long a, unsigned long long b) : x(a), y(b) {}
};
__device__ __forceinline__ W16 operator&(W16 a, W16 b) { return W16(a.x & b.x, a.y & b.y); }
__device__ __forceinline__ W16 operator|(W16 a, W16 b) { return W16(a.x | b.x, a.y | b.y); }
__device__ __forceinline__ W16 operator~(W16 a) { return W16(~a.x, ~a.y); }
__device__ __forceinline__ W16& operator|=(W16& a, W16 b) { a.x |= b.x; a.y |= b.y; return a; }
__device__ __forceinline__ W16 operator>>(W16 a, uint32_t sh) { return W16(a.x >> sh, a.y >> sh); }  // sh < 8
__device__ __forceinline__ W16 operator*(W16 a, uint32_t c) { return W16(a.x * c, a.y * c); }       // per byte
using GWord = std::conditional<kGW == 16, W16, std::conditional<kGW == 8, unsigned long long, uint32_t>::type>::type;
using Slot = std::conditional<kGW == 16, unsigned long long, uint32_t>::type;   // a report slot (below)
constexpr GWord kRep = GWord(kGW == 4 ? 0x01010101ull : 0x0101010101010101ull);  // one bit per state byte
constexpr uint32_t kBytesM = (1u << kGW) - 1u;     // faulting-byte bits of a report slot
__device__ __forceinline__ bool any(uint32_t v) { return v != 0; }
__device__ __forceinline__ bool any(unsigned long long v) { return v != 0; }
__device__ __forceinline__ bool any(W16 v) { return (v.x | v.y) != 0; }
__device__ __forceinline__ uint32_t byte_of(uint32_t v, uint32_t b) { return (v >> (8 * b)) & 0xFFu; }
__device__ __forceinline__ uint32_t byte_of(unsigned long long v, uint32_t b) { return (uint32_t)(v >> (8 * b)) & 0xFFu; }
__device__ __forceinline__ uint32_t byte_of(W16 v, uint32_t b) { return byte_of(b < 8 ? v.x : v.y, b & 7u); }
// Byte mask of bytes [a, a + n) of a group (n = 1..kGW)
__device__ __forceinline__ unsigned long long mask64(uint32_t a, uint32_t n) {   // a + n <= 8
  return n == 0 ? 0ull : (~0ull >> (8 * (8 - n))) << (8 * a);
}
__device__ __forceinline__ uint32_t byte_mask_t(const uint32_t*, uint32_t a, uint32_t n) {
  return (0xFFFFFFFFu >> (8 * (4 - n))) << (8 * a);
}
__device__ __forceinline__ unsigned long long byte_mask_t(const unsigned long long*, uint32_t a, uint32_t n) {
  return mask64(a, n);
}
__device__ __forceinline__ W16 byte_mask_t(const W16*, uint32_t a, uint32_t n) {
  const uint32_t e = a + n;
  return W16(a < 8 ? mask64(a, min(e, 8u) - a) : 0ull, e > 8 ? mask64(a > 8 ? a - 8 : 0u, e - max(a, 8u)) : 0ull);
}
__device__ __forceinline__ GWord byte_mask(uint32_t a, uint32_t n) { return byte_mask_t((const GWord*)nullptr, a, n); }
__device__ __forceinline__ uint32_t ld_group(const uint32_t* p) { return __ldcg(p); }
__device__ __forceinline__ unsigned long long ld_group(const unsigned long long* p) { return __ldcg(p); }
__device__ __forceinline__ W16 ld_group(const W16* p) {
  const ulonglong2 v = __ldcg(reinterpret_cast<const ulonglong2*>(p));
  return W16(v.x, v.y);
}
__device__ __forceinline__ void st_group(uint32_t* p, uint32_t v) { __stcg(p, v); }
__device__ __forceinline__ void st_group(unsigned long long* p, unsigned long long v) { __stcg(p, v); }
__device__ __forceinline__ void st_group(W16* p, W16 v) { __stcg(reinterpret_cast<ulonglong2*>(p), make_ulonglong2(v.x, v.y)); }

// One warp: the step's run table (segments that continue one another joined,
// adjacent runs on identical words grouped into compounds) and the merged
// kGW-word-group intervals, for the step's first `cut` events.
__device__ void run_setup(RunStage& R, uint32_t nseg, uint32_t cut, uint32_t a3, uint32_t plo, uint32_t phi) {
  const uint32_t lane = threadIdx.x & 31;
  constexpr uint32_t kNone = 0xFFFFFFFFu;
  uint32_t A = 0, B = 0, ga = kNone, gb = 0, op = 0, pos = 0;
  uint32_t len = 0;
  if (lane < nseg) {
    const uint4 inf = R.info[lane];
    const uint2 ds = R.desc[lane];
    len = inf.z >= cut ? 0u : min(inf.y, cut - inf.z);
    const uint32_t key = ds.x + inf.x;
    op = key >> 30; pos = ds.y + inf.x;
    A = a3 + (key & kWordMask); B = A + len;
  }
  // a segment that continues the previous one (a run cut at a chunk boundary: same
  // op, next word, next position) joins it: runs = chains of segments
  const uint32_t pA = __shfl_up_sync(FULL, B, 1), pop = __shfl_up_sync(FULL, op, 1);
  const uint32_t ppe = __shfl_up_sync(FULL, pos + (B - A), 1);
  const uint32_t lens = __ballot_sync(FULL, len != 0);
  const bool cont = lane > 0 && len && ((lens >> (lane - 1)) & 1u) && pA == A && pop == op && ppe == pos;
  const uint32_t heads = __ballot_sync(FULL, len && !cont);
  // chain end: the lane before the next head or the next empty segment
  const uint32_t after = (heads | ~lens) & (lane == 31 ? 0u : 0xFFFFFFFEu << lane);
  const uint32_t endl = after ? __ffs(after) - 2 : 31u;
  const uint32_t Bc = __shfl_sync(FULL, B, endl);
  const uint32_t nr = __popc(heads);
  if ((heads >> lane) & 1u) {                        // clipped to the work item's words [plo, phi)
    const uint32_t Ac = max(A, plo), Be = min(Bc, phi);
    R.run[__popc(heads & lanemask_lt())] = Ac < Be ? make_uint4(Ac, Be, op, pos + (Ac - A)) : make_uint4(0, 0, 0, 0);
  }
  R.mm[lane] = 0;
  __syncwarp();
  // compounds: adjacent runs on identical words (config 5's WT, RT, RT of one run of
  // words) — the group pass computes their overlap once and applies their ops in order
  uint4 r = make_uint4(0, 0, 0, 0);
  if (lane < nr) r = R.run[lane];
  const bool ne = lane < nr && r.y > r.x;
  const uint32_t pX = __shfl_up_sync(FULL, r.x, 1), pY = __shfl_up_sync(FULL, r.y, 1);
  const bool same = lane > 0 && ne && pX == r.x && pY == r.y;
  const uint32_t le = 0xFFFFFFFFu >> (31 - lane);
  uint32_t cst = __ballot_sync(FULL, ne && !same);
  uint32_t t = ne ? lane - (31 - __clz(cst & le)) : 0u;
  cst |= __ballot_sync(FULL, ne && t >= 16 && (t & 15u) == 0);        // at most 16 ops per compound
  const uint32_t cs = ne ? 31 - __clz(cst & le) : lane;
  t = lane - cs;
  uint32_t opsv = ne ? r.z << (2 * t) : 0u;                            // OR over the compound's members so far
#pragma unroll
  for (uint32_t d = 1; d < 32; d <<= 1) {
    const uint32_t o = __shfl_up_sync(FULL, opsv, d);
    if (lane >= d && lane - d >= cs) opsv |= o;
  }
  const uint32_t nxs = __shfl_down_sync(FULL, (uint32_t)same, 1);      // does the next lane continue the compound?
  const bool tail = ne && (lane == 31 || !nxs || ((cst >> (lane + 1)) & 1u));
  const uint32_t nc = __popc(cst);
  if (tail) R.cmp[__popc(cst & le) - 1] = make_uint4(r.x, r.y, cs | ((t + 1) << 5), opsv);
  __syncwarp();
  if (lane < nc) {
    const uint4 c = R.cmp[lane];
    ga = c.x >> kGWLog; gb = (c.y + kGW - 1) >> kGWLog;
  }
  // sort the group intervals by first group (bitonic over the lanes; empty ones last)
  uint32_t sga = ga, sgb = gb, sr = lane;
  const uint32_t kmax = nc <= 1 ? 1u : 1u << (32 - __clz(nc - 1));       // sorting network width
#pragma unroll
  for (uint32_t k = 2; k <= 32; k <<= 1) {
    if (k > kmax) break;
#pragma unroll
    for (uint32_t j = k >> 1; j > 0; j >>= 1) {
      const uint32_t oga = __shfl_xor_sync(FULL, sga, j), ogb = __shfl_xor_sync(FULL, sgb, j);
      const uint32_t orr = __shfl_xor_sync(FULL, sr, j);
      const bool keep_min = ((lane & j) == 0) == ((lane & k) == 0 || k == kmax);
      if (keep_min ? oga < sga : oga > sga) { sga = oga; sgb = ogb; sr = orr; }
    }
  }
  const bool valid = sga != kNone;
  uint32_t incl = valid ? sgb : 0u;                  // inclusive prefix max of the interval ends
#pragma unroll
  for (uint32_t d = 1; d < 32; d <<= 1) {
    const uint32_t o = __shfl_up_sync(FULL, incl, d);
    if (lane >= d) incl = max(incl, o);
  }
  uint32_t excl = __shfl_up_sync(FULL, incl, 1);
  if (lane == 0) excl = 0;
  const bool start = valid && (lane == 0 || sga >= excl);
  const uint32_t smask = __ballot_sync(FULL, start), vmask = __ballot_sync(FULL, valid);
  const uint32_t nm = __popc(smask);
  const uint32_t idx = __popc(smask & (0xFFFFFFFFu >> (31 - lane))) - 1u;   // merged interval of this lane
  const bool lastl = valid && (lane == 31 || !((vmask >> (lane + 1)) & 1u) || ((smask >> (lane + 1)) & 1u));
  __syncwarp();
  if (valid) atomicOr(&R.mm[idx], 1u << sr);
  if (start) R.mi[idx].x = sga;
  if (lastl) R.mi[idx].y = incl;                     // the interval's end (exclusive group)
  __syncwarp();
  uint32_t n = 0, gs = 0;
  if (lane < nm) { const uint2 v = R.mi[lane]; gs = v.x; n = v.y - v.x; }
  uint32_t sc = n;
#pragma unroll
  for (uint32_t d = 1; d < 32; d <<= 1) {
    const uint32_t o = __shfl_up_sync(FULL, sc, d);
    if (lane >= d) sc += o;
  }
  __syncwarp();
  if (lane < nm) R.mi[lane] = make_uint2(gs, sc - n);
  if (lane == 31) { R.nm = nm; R.G = sc; }
  __syncwarp();
}

// A step made only of runs (each: word A + j, op, position + j for j < count).  No
// event is materialised: the shadow is processed in aligned groups of kGW words (one
// load per group, kGW states in SWAR form), and each group applies, in trace
// order, every run that overlaps it — reads classify the covered bytes (P:263:
// read_host needs OVv, read_target CVv; UUM / USD by the init bits), writes
// take the VSM write image (WH: OVv, OVi set, CVv clear; WT: CVv, CVi set, OVv
// clear).  Groups are the union of the runs' group intervals, merged so
// that each group has one owner thread.  BO (Z20): a target access to a word
// without kCVp is a BO report and no transition; UM (Z23): a write makes 0xF.
// The table is built by run_setup (warp 0, usually during the previous step:
// `prepared`, a block-uniform register — not a shared flag, which warp 0 would set
// while other warps still test it); warps 1.. process the groups while warp 0
// builds the next run step's table (Rn, nsn segments of mn events; nsn = 0: the
// next step is not a run step).
template <bool BO, bool UM>
__device__ void step_runs(ReplaySmem& S, const ReplayParams& p, RunStage& R, uint32_t nseg, uint32_t cut,
                          bool prepared, RunStage& Rn, uint32_t nsn, uint32_t mn) {
  const uint32_t lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const uint64_t bb = S.bucket_base;
  const uint32_t a3 = (uint32_t)bb & (kGW - 1);
  GWord* const gbase = reinterpret_cast<GWord*>(p.shadow + (bb - a3));
  // the work item's words in A-coordinates: the bucket, or a part of it (kItemPart)
  const uint32_t wlo = a3 + (S.partial ? S.part_lo : 0u), whi = a3 + (S.partial ? S.part_hi : S.span);
  if (!prepared) {                                  // first run step of a stretch, or cut by a range op
    if (warp == 0) run_setup(R, nseg, cut, a3, wlo, whi);
    __syncthreads();
  }
  if (warp == 0) {
    if (nsn) {                                      // the next step's table, overlapped with this step
      cp_async_wait_all();                          // its descriptors (copied by warp 0)
      __syncwarp();
      run_setup(Rn, nsn, mn, a3, wlo, whi);
    }
    return;
  }
  const uint32_t nm = R.nm, G = R.G;
  const uint64_t wbase = bb - a3;                    // relative word of A = 0
  // a run's reports in one group, packed: run index (bits 0-4), faulting bytes
  // (kGW bits from bit 5), 2 bits of kind per byte above them (0 UUM, 1 USD, 2 BO)
  auto emit_one = [&](Slot slot, uint32_t w0, unsigned long long base) {
    const uint4 r = R.run[(uint32_t)slot & 31u];
#pragma unroll
    for (uint32_t b = 0; b < kGW; ++b) {
      if (!((slot >> (5 + b)) & 1u)) continue;
      const uint32_t kc = (uint32_t)(slot >> (5 + kGW + 2 * b)) & 3u;
      if (base < p.cand_cap) {
        const uint64_t wd = wbase + w0 + b;
        p.cand[base] = make_uint4((uint32_t)wd, (uint32_t)(wd >> 32), r.w + (w0 + b - r.x), kc == 2 ? 4u : kc + 1u);
      }
      ++base;
    }
  };
  const uint32_t st0 = nm <= 1 ? 0u : 1u << (31 - __clz(nm - 1));   // search span (nm is uniform)
  constexpr uint32_t GU = kRunGroupsInFlight;      // groups per thread whose loads are issued together
  constexpr uint32_t GT = RT - 32;                  // group threads (warps 1..)
  for (uint32_t u00 = 0; u00 < G; u00 += GU * GT) {
  uint32_t gq[GU], jq[GU];
  GWord sq[GU];
#pragma unroll
  for (uint32_t q = 0; q < GU; ++q) {
    const uint32_t u = u00 + q * GT + threadIdx.x - 32;
    gq[q] = 0; jq[q] = 0; sq[q] = 0;
    if (u < G) {
      uint32_t j = 0;                                 // merged interval: the last with first unit <= u
      for (uint32_t st = st0; st; st >>= 1)
        if (j + st < nm && R.mi[j + st].y <= u) j += st;
      const uint2 mv = R.mi[j];
      gq[q] = mv.x + (u - mv.y);
      jq[q] = j;
      sq[q] = ld_group(gbase + gq[q]);
    }
  }
#pragma unroll
  for (uint32_t q = 0; q < GU; ++q) {
    const uint32_t u = u00 + q * GT + threadIdx.x - 32;
    uint32_t ns = 0;
    Slot fs0 = 0, fs1 = 0;
    uint32_t w0 = 0;
    if (u < G) {
      const uint32_t j = jq[q], g = gq[q];
      w0 = kGW * g;
      GWord s = sq[q];
      GWord wr = 0;
      for (uint32_t mm = R.mm[j]; mm; mm &= mm - 1) {
        const uint4 cp = R.cmp[__ffs(mm) - 1];
        const uint32_t lo = max(cp.x, w0), hi = min(cp.y, w0 + kGW);
        if (lo >= hi) continue;
        const GWord M = byte_mask(lo - w0, hi - lo);
        const uint32_t r0 = cp.z & 31u, kn = cp.z >> 5;
        for (uint32_t t = 0; t < kn; ++t) {
        const uint32_t ri = r0 + t;
        const uint32_t o = (cp.w >> (2 * t)) & 3u;
        GWord Me = M, bof = 0;
        if (BO && (o & 2u)) {                         // no CV: buffer overflow, no transition (Z20)
          bof = (~s >> 4) & kRep & M;
          Me = M & ~(bof * 0xFFu);
        }
        GWord fv = 0;
        if (!(o & 1u)) {
          fv = (~s >> (o >> 1)) & kRep & Me;        // RH: OVv (bit 0), RT: CVv (bit 1)
        } else {
          const GWord img = UM ? kRep * 0x0Fu
                       : o == OP_WH ? ((s & (kRep * (BO ? 0x18u : 0x08u))) | (kRep * 0x05u))
                                    : ((s & (kRep * (BO ? 0x14u : 0x04u))) | (kRep * 0x0Au));
          s = (s & ~Me) | (img & Me);
          wr |= Me;
        }
        if (any(fv | bof)) {                          // reports (rare)
          const GWord usd = (s >> (2 + (o >> 1))) & kRep;   // the read side's init bit
          Slot slot = ri;
#pragma unroll
          for (uint32_t b = 0; b < kGW; ++b) {
            if (!(byte_of(fv | bof, b) & 1u)) continue;
            const uint32_t kc = (byte_of(bof, b) & 1u) ? 2u : byte_of(usd, b) & 1u;
            slot |= ((Slot)1 << (5 + b)) | ((Slot)kc << (5 + kGW + 2 * b));
          }
          if (ns == 0) fs0 = slot;
          else if (ns == 1) fs1 = slot;
          else emit_one(slot, w0, atomicAdd(&p.st->n_cand, (unsigned long long)__popc((uint32_t)(slot >> 5) & kBytesM)));
          ++ns;
        }
        }
      }
      if (any(wr)) {
        if (w0 >= wlo && w0 + kGW <= whi) {
          st_group(gbase + g, s);
        } else {                                      // a group shared with a neighbouring bucket
          uint8_t* gb8 = reinterpret_cast<uint8_t*>(gbase + g);
#pragma unroll
          for (uint32_t b = 0; b < kGW; ++b)
            if (byte_of(wr, b)) __stcg(gb8 + b, (uint8_t)byte_of(s, b));
        }
      }
    }
    // the reports of each lane's first two faulting runs: one warp-aggregated append
    const uint32_t k = (ns > 0 ? __popc((uint32_t)(fs0 >> 5) & kBytesM) : 0u) +
                       (ns > 1 ? __popc((uint32_t)(fs1 >> 5) & kBytesM) : 0u);
    if (__any_sync(FULL, k != 0)) {
      uint32_t sk = k;
#pragma unroll
      for (uint32_t d = 1; d < 32; d <<= 1) {
        const uint32_t o = __shfl_up_sync(FULL, sk, d);
        if (lane >= d) sk += o;
      }
      unsigned long long base = 0;
      if (lane == 31) base = atomicAdd(&p.st->n_cand, (unsigned long long)sk);
      base = __shfl_sync(FULL, base, 31) + (sk - k);
      if (ns > 0) emit_one(fs0, w0, base);
      if (ns > 1) emit_one(fs1, w0, base + __popc((uint32_t)(fs0 >> 5) & kBytesM));
    }
  }
  }
}

// BO: ARB_F_BO contexts (the buffer-overflow extension, Z20) get their own
// instance, so the default replay carries none of its checks.
template <bool BO, bool UM, bool MD>
__global__ void __launch_bounds__(RT, kReplayCtasPerSm) k_replay(ReplayParams p) {
  extern __shared__ __align__(16) uint8_t smem_raw[];
  ReplaySmem& S = *reinterpret_cast<ReplaySmem*>(smem_raw);
  const uint32_t tid = threadIdx.x;
  hash_clear(S);
  for (;;) {
    if (tid == 0) {
      const unsigned long long w = atomicAdd(&p.st->work, 1ull);
      if (w < p.n_items) {
        const uint4 it = p.items[w];
        S.bucket = it.x; S.mode = it.w;
        S.part_lo = it.w == kItemPart ? it.y : 0;
        S.part_hi = it.w == kItemPart ? it.z : 0xFFFFFFFFu;
        S.partial = it.w == kItemPart;
        S.slice = it.y; S.n_slices = it.z;
      } else {
        S.bucket = 0xFFFFFFFFu;
      }
    }
    __syncthreads();
    const uint32_t b = S.bucket;
    if (b >= p.n_buckets) return;
    const uint32_t mode = S.mode;
    if (tid == 0) {
      S.op_cur = p.ops_start[b];
      S.op_end = p.ops_start[b + 1];
      S.bucket_base = p.bucket_start[b];
      S.span = (uint32_t)(p.bucket_start[b + 1] - S.bucket_base);
      S.shrel = p.shadow + S.bucket_base;
    }
    bucket_setup(S, p, b);
    uint32_t first = 0, total = S.n_events;
    if (mode >= kItemSlice) {
      // hot bucket slice k of n: events [k E / n, (k+1) E / n) and the range ops
      // from the slice's first event (slice 0: the bucket's first op) up to the
      // next slice's first event (last slice: the bucket's last op)
      const uint32_t k = S.slice, ns = S.n_slices, E = S.n_events;
      const uint32_t span = (uint32_t)(p.bucket_start[b + 1] - p.bucket_start[b]), span16 = (span + 15) & ~15u;
      first = (uint32_t)((uint64_t)k * E / ns);
      total = (uint32_t)((uint64_t)(k + 1) * E / ns);
      if (tid == 0) {
        const uint32_t a0 = S.op_cur, a1 = S.op_end;
        if (E == 0) {
          if (k != 0) S.op_end = a0;
        } else {
          if (k > 0) S.op_cur = ops_lower_bound(p, a0, a1, event_pos(S, p, first));
          if (k + 1 < ns) S.op_end = ops_lower_bound(p, a0, a1, event_pos(S, p, total));
        }
        const uint64_t off = p.hot_off[b] + (uint64_t)k * span16;
        S.shrel = p.hot_P + off;
        S.fsum = p.hot_F + off;
        S.part_hi = span;
      }
      __syncthreads();
      if (mode == kItemSummary) {
        for (uint32_t w = tid; w < span; w += RT) S.fsum[w] = kfun_id<BO, MD>();
        for (uint32_t w = tid; w < kZSlots; w += RT) { S.u.z.key[w] = kEmpty; S.u.z.lastw[w] = 0; }
        for (uint32_t w = tid; w < kZSlots / 4; w += RT) S.u.z.anyw[w] = 0;
        __syncthreads();
      }
    }
    if (tid == 0) S.next_op = S.op_cur < S.op_end ? p.ops[S.op_cur].pos : 0xFFFFFFFFu;
    __syncthreads();
    uint32_t e0 = first, cur = 0, m_cur = 0, hint = 0, nr_cur = 0;
    bool prep_cur = false;                   // the current run step's table was built during the last step
    // run steps: whole buckets or word-range parts, one device
    const bool runs_ok = !MD && (mode == kItemWhole || mode == kItemPart) && !p.no_run_steps;
    if (e0 < total) {
      ensure_window(S, p, e0, hint);
      m_cur = issue_gather(S, p, e0, total, 0, hint, runs_ok, nr_cur);
    }
    while (e0 < total) {
      cp_async_wait_all();
      __syncthreads();
      const uint2* ev = S.ev[cur];
      const uint32_t m = m_cur;
      // ---- prefetch the next step's events (assumes the step is not cut) ---------
      const uint32_t nxt = e0 + m;
      uint32_t m_nxt = 0, nr_nxt = 0;
      if (nxt < total) {
        ensure_window(S, p, nxt, hint);
        m_nxt = issue_gather(S, p, nxt, total, cur ^ 1, hint, runs_ok, nr_nxt);
      }
      // ---- range ops before the first event, then cut at the next one -------------
      constexpr uint32_t pm = MD ? kMdPos : 0xFFFFFFFFu;   // MD: strip the device bits (Z24)
      const uint32_t nrs = MD ? 0u : nr_cur;
      RunStage& R = *reinterpret_cast<RunStage*>(S.ev[cur]);
      uint32_t cut = m;
      if (nrs) {                                   // run step: positions from the descriptors
        apply_ops_before<BO, MD>(S, p, R.desc[0].y + R.info[0].x);
        const uint4 li = R.info[nrs - 1];
        const uint32_t nx = S.next_op;
        if (nx != 0xFFFFFFFFu && R.desc[nrs - 1].y + li.x + li.y - 1 > nx) {
          const uint32_t lane = tid & 31;
          uint32_t c = 0;
          if (!MD && lane < nrs) {
            const uint4 in = R.info[lane];
            const uint32_t p0 = R.desc[lane].y + in.x;
            c = p0 + in.y <= nx ? in.y : (p0 < nx ? nx - p0 : 0u);
          }
          cut = __reduce_add_sync(FULL, c);
        }
      } else {
        apply_ops_before<BO, MD>(S, p, ev[0].y & pm);
        if (S.next_op != 0xFFFFFFFFu && (ev[m - 1].y & pm) > S.next_op) {
          uint32_t cnt = 0;
          for (uint32_t e = tid; e < m; e += RT) cnt += (ev[e].y & pm) < S.next_op;
          cut = block_sum(cnt, S.red);
        }
      }
      if (nrs) {
        const bool nx_run = nr_nxt != 0 && cut == m && !p.no_run_prep;
        step_runs<BO, UM>(S, p, R, nrs, cut, prep_cur && cut == m, *reinterpret_cast<RunStage*>(S.ev[cur ^ 1]),
                          nx_run ? nr_nxt : 0u, m_nxt);
        prep_cur = nx_run;
        if (tid == 0) atomicAdd(&p.st->steps_run, 1ull);
      } else if (mode == kItemSummary) {
        prep_cur = false;
        step_summary<BO, UM, MD>(S, ev, cut);
      } else {
        prep_cur = false;
        const bool fast = S.partial ? step_fast_partial<BO, UM, MD>(S, p, ev, cut)
                                    : step_fast<false, BO, UM, MD>(S, p, ev, cut);
        if (!fast) step_sort<BO, UM, MD>(S, p, ev, cut);
        if (tid == 0) atomicAdd(fast ? &p.st->steps_fast : &p.st->steps_sort, 1ull);
      }
      e0 += cut;
      if (cut == m) {
        cur ^= 1;
        m_cur = m_nxt;
        nr_cur = nr_nxt;
      } else {
        // the prefetch started at e0_old + m: drain it and gather from e0
        cp_async_wait_all();
        __syncthreads();
        hint = 0;
        prep_cur = false;
        ensure_window(S, p, e0, hint);
        m_cur = issue_gather(S, p, e0, total, cur, hint, runs_ok, nr_cur);
      }
    }
    // the ops after the last event (a slice replay's private states are not kept);
    // the last step's shadow stores (a run step ends without a barrier) come first
    __syncthreads();
    if (mode != kItemSlice) apply_ops_before<BO, MD>(S, p, 0xFFFFFFFFu);
    if (tid == 0 && total > first) atomicMax(&p.st->max_bucket_events, (unsigned long long)(total - first));
    __syncthreads();
    if (mode == kItemSummary) {
      hash_clear(S);                   // the summary arrays share the hash area
      __syncthreads();
    }
  }
}

cudaError_t launch_replay(const ReplayParams& p, int n_ctas, cudaStream_t s) {
  const size_t smem = sizeof(ReplaySmem);
  // ARB_F_BO and ARB_F_UNIFIED exclude each other (arb_init)
  auto kern = p.md ? k_replay<false, false, true> : p.um ? k_replay<false, true, false>
            : p.bo ? k_replay<true, false, false> : k_replay<false, false, false>;
  cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  kern<<<n_ctas, RT, smem, s>>>(p);
  return cudaGetLastError();
}

}  // namespace arb
