// replay.cu — A3b + A4 + A5: per-address replay of each bucket.
//
// One CTA per address bucket at a time (persistent; buckets in largest-first
// order).  For its bucket the CTA gathers the word-events in trace order from
// the chunk-major partition output (segment queue), applies the resolved range
// ops (Table I transfers / allocate / release; target update P:121)
// to the bucket's shadow at their trace positions, and processes the events in
// steps of <= 2048 that never straddle a range op:
//
//   fast step  (every word has at most one write in the step): a shared-memory
//              hash word -> (first write, state before the step).  A read's
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
#include "kcommon.cuh"

namespace arb {

constexpr int RT = kReplayThreads;           // 512 threads
constexpr int RI = 4;                        // events per thread per step
constexpr int STEP = RT * RI;                // 2048 events per step
constexpr int kQCap = 1024;                  // segment queue (circular)
constexpr int kScanChunks = 512;             // chunks examined per refill round
constexpr int kHSlots = 4096;                // hash slots (load <= 1/2)
constexpr uint32_t kEmpty = 0xFFFFFFFFu;
constexpr uint32_t kWordMask = 0x3FFFFFFFu;

struct ReplaySmem {
  uint32_t keyA[STEP], posA[STEP];
  union {
    struct { uint32_t keyB[STEP], posB[STEP]; uint16_t hist[RT / 32][256]; } s;   // sort step
    struct { uint32_t key[kHSlots], wpos[kHSlots]; uint8_t st[kHSlots]; } h;      // fast step
  } u;
  uint32_t q_start[kQCap];        // global event index of a segment
  uint32_t q_len[kQCap];
  uint32_t pref[kQCap];           // prefix of queue lengths (also radix scratch)
  uint32_t red[RT / 32], red2[RT / 32], wscan[RT / 32];
  uint32_t bucket;
  uint32_t q_head, q_tail, q_head_off;
  uint64_t q_events;
  uint32_t chunk_cur, n_gather, op_cur, op_end;
  uint64_t bucket_events, bucket_base;
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
// exclusive block scan (sum); *total = sum
__device__ __forceinline__ uint32_t block_excl_scan(uint32_t v, uint32_t* wscan, uint32_t* total) {
  const uint32_t lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  uint32_t incl = v;
#pragma unroll
  for (int d = 1; d < 32; d <<= 1) {
    const uint32_t o = __shfl_up_sync(FULL, incl, d);
    if (lane >= (uint32_t)d) incl += o;
  }
  __syncthreads();
  if (lane == 31) wscan[warp] = incl;
  __syncthreads();
  uint32_t wpre = 0, tot = 0;
#pragma unroll
  for (int w = 0; w < RT / 32; ++w) {
    const uint32_t x = wscan[w];
    if ((uint32_t)w < warp) wpre += x;
    tot += x;
  }
  *total = tot;
  return wpre + incl - v;
}

// ---- range ops ----------------------------------------------------------------
// Apply transition `sel` to shadow bytes [lo, hi) (relative word indices).
__device__ void stream_apply(uint8_t* shadow, uint64_t lo, uint64_t hi, Sel sel) {
  if (lo >= hi) return;
  uint64_t a = (lo + 15) & ~15ull, b = hi & ~15ull;
  if (a > b) { a = hi; b = hi; }
  for (uint64_t j = lo + threadIdx.x; j < a; j += RT) __stcg(shadow + j, (uint8_t)sel_apply4(sel, __ldcg(shadow + j)));
  for (uint64_t j = b + threadIdx.x; j < hi; j += RT) __stcg(shadow + j, (uint8_t)sel_apply4(sel, __ldcg(shadow + j)));
  uint4* v = reinterpret_cast<uint4*>(shadow + a);
  const uint64_t nv = (b - a) >> 4;
  constexpr int U = 4;   // 4 x 16 B loads in flight per thread
  uint64_t j = threadIdx.x;
  for (; j + (U - 1) * RT < nv; j += U * RT) {
    uint4 x[U];
#pragma unroll
    for (int u = 0; u < U; ++u) x[u] = __ldcg(v + j + u * RT);
#pragma unroll
    for (int u = 0; u < U; ++u) {
      x[u].x = sel_apply4(sel, x[u].x); x[u].y = sel_apply4(sel, x[u].y);
      x[u].z = sel_apply4(sel, x[u].z); x[u].w = sel_apply4(sel, x[u].w);
      __stcg(v + j + u * RT, x[u]);
    }
  }
  for (; j < nv; j += RT) {
    uint4 x = __ldcg(v + j);
    x.x = sel_apply4(sel, x.x); x.y = sel_apply4(sel, x.y);
    x.z = sel_apply4(sel, x.z); x.w = sel_apply4(sel, x.w);
    __stcg(v + j, x);
  }
}

// Apply every pending range op of the bucket with position < limit; runs of
// ops on the identical range with no event in between are composed first.
__device__ void apply_ops_before(ReplaySmem& S, const ReplayParams& p, uint32_t limit) {
  while (S.op_cur < S.op_end && p.ops[S.op_cur].pos < limit) {
    const uint32_t k = S.op_cur;
    const BucketOp o = p.ops[k];
    Sel sel = o.sel;
    uint32_t k2 = k + 1;
    while (k2 < S.op_end) {
      const BucketOp o2 = p.ops[k2];
      if (o2.pos >= limit || o2.lo != o.lo || o2.hi != o.hi) break;
      sel = sel_compose(o2.sel, sel);
      ++k2;
    }
    stream_apply(p.shadow, o.lo, o.hi, sel);
    __syncthreads();
    if (threadIdx.x == 0) {
      S.op_cur = k2;
      atomicAdd(&p.st->range_words_applied, (unsigned long long)(o.hi - o.lo));
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
  uint32_t wf = nf;
#pragma unroll
  for (int d = 1; d < 32; d <<= 1) {
    const uint32_t o = __shfl_up_sync(FULL, wf, d);
    if (lane >= (uint32_t)d) wf += o;
  }
  const uint32_t wtot = __shfl_sync(FULL, wf, 31);
  if (!wtot) return;
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
  for (uint32_t i = threadIdx.x; i < kHSlots; i += RT) { S.u.h.key[i] = kEmpty; S.u.h.wpos[i] = kEmpty; }
}

// ---- fast step: at most one write per word -------------------------------------------
// Returns false (and leaves the shadow untouched) if some word has two writes.
__device__ bool step_fast(ReplaySmem& S, const ReplayParams& p, uint32_t m) {
  uint32_t slot[RI], word[RI], pos[RI], op[RI];
  bool own[RI];
  bool multi = false;
#pragma unroll
  for (int j = 0; j < RI; ++j) {
    const uint32_t i = threadIdx.x + j * RT;
    own[j] = false; slot[j] = 0; word[j] = 0; pos[j] = 0; op[j] = 0xFFu;
    if (i < m) {
      const uint32_t k = S.keyA[i];
      word[j] = k & kWordMask; op[j] = k >> 30; pos[j] = S.posA[i];
      uint32_t h = (word[j] * 2654435761u) >> 20;          // 12 bits
      for (;;) {
        const uint32_t old = atomicCAS(&S.u.h.key[h], kEmpty, word[j]);
        if (old == kEmpty) { own[j] = true; break; }
        if (old == word[j]) break;
        h = (h + 1) & (kHSlots - 1);
      }
      slot[j] = h;
      if (op[j] == OP_WH || op[j] == OP_WT) {
        const uint32_t o = atomicMin(&S.u.h.wpos[h], (pos[j] << 2) | (op[j] == OP_WH ? 1u : 2u));
        if (o != kEmpty) multi = true;
      }
    }
  }
  if (__syncthreads_or(multi)) {
#pragma unroll
    for (int j = 0; j < RI; ++j)
      if (own[j]) { S.u.h.key[slot[j]] = kEmpty; S.u.h.wpos[slot[j]] = kEmpty; }
    __syncthreads();
    return false;
  }
  const uint64_t bb = S.bucket_base;
#pragma unroll
  for (int j = 0; j < RI; ++j)
    if (own[j]) S.u.h.st[slot[j]] = __ldcg(p.shadow + bb + word[j]) & 15u;
  __syncthreads();
  uint32_t fk[RI];
#pragma unroll
  for (int j = 0; j < RI; ++j) {
    fk[j] = 0;
    if (op[j] == 0xFFu) continue;
    const uint32_t s0 = S.u.h.st[slot[j]], wp = S.u.h.wpos[slot[j]];
    const bool hasw = wp != kEmpty;
    const uint32_t after = hasw ? vsm_write(wp & 3u, s0) : s0;
    const uint32_t before = (hasw && (wp >> 2) < pos[j]) ? after : s0;
    fk[j] = classify(op[j], before);
    if (own[j]) __stcg(p.shadow + bb + word[j], (uint8_t)after);
  }
  emit_faults(p, fk, word, pos, bb);
  __syncthreads();
#pragma unroll
  for (int j = 0; j < RI; ++j)
    if (own[j]) { S.u.h.key[slot[j]] = kEmpty; S.u.h.wpos[slot[j]] = kEmpty; }
  __syncthreads();
  return true;
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
  if (tid < 256) {
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

__device__ void step_sort(ReplaySmem& S, const ReplayParams& p, uint32_t m) {
  const uint32_t tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  uint32_t lo = 0xFFFFFFFFu, hi = 0;
  for (uint32_t i = tid; i < m; i += RT) {
    const uint32_t w = S.keyA[i] & kWordMask;
    lo = min(lo, w); hi = max(hi, w);
  }
  block_minmax(lo, hi, S.red, S.red2);
  const uint32_t span = hi - lo;
  const uint32_t bits = span ? 32 - __clz(span) : 0;
  uint32_t* kin = S.keyA; uint32_t* pin = S.posA; uint32_t* kout = S.u.s.keyB; uint32_t* pout = S.u.s.posB;
  for (uint32_t sh = 0; sh < bits; sh += 8) {
    sort_pass(S, kin, pin, kout, pout, m, lo, sh, (1u << min(8u, bits - sh)) - 1u);
    uint32_t* t = kin; kin = kout; kout = t;
    t = pin; pin = pout; pout = t;
  }
  // blocked arrangement: thread t owns sorted elements [RI*t, RI*t + RI)
  const uint64_t bb = S.bucket_base;
  uint32_t val[RI], s0[RI], key[RI], wd[RI], ps[RI];
  bool head[RI];
  uint32_t agg = 0;
#pragma unroll
  for (int j = 0; j < RI; ++j) {
    const uint32_t i = tid * RI + j;
    key[j] = 0; head[j] = false; s0[j] = 0; val[j] = 0; wd[j] = 0; ps[j] = 0;
    if (i < m) {
      const uint32_t k = kin[i];
      const uint32_t w = k & kWordMask;
      const bool h = (i == 0) || ((kin[i - 1] & kWordMask) != w);
      uint32_t v = acc_summary(k >> 30);
      uint32_t st = 0;
      if (h) {
        st = __ldcg(p.shadow + bb + w) & 15u;
        v = kHead | kConst | acc_apply(v, st);
      }
      key[j] = k; head[j] = h; s0[j] = st; val[j] = v; wd[j] = w; ps[j] = pin[i];
    }
    agg = acc_combine(agg, val[j]);
  }
  uint32_t incl = agg;
#pragma unroll
  for (int d = 1; d < 32; d <<= 1) {
    const uint32_t o = __shfl_up_sync(FULL, incl, d);
    if (lane >= (uint32_t)d) incl = acc_combine(o, incl);
  }
  uint32_t excl_lane = __shfl_up_sync(FULL, incl, 1);
  if (lane == 0) excl_lane = 0;
  __syncthreads();
  if (lane == 31) S.wscan[warp] = incl;
  __syncthreads();
  uint32_t wpre = 0;
  for (uint32_t w = 0; w < warp; ++w) wpre = acc_combine(wpre, S.wscan[w]);
  uint32_t run = acc_combine(wpre, excl_lane);
  uint32_t fk[RI];
#pragma unroll
  for (int j = 0; j < RI; ++j) {
    const uint32_t i = tid * RI + j;
    fk[j] = 0;
    if (i < m) {
      const uint32_t before = head[j] ? s0[j] : (run & 15u);
      run = acc_combine(run, val[j]);
      fk[j] = classify(key[j] >> 30, before);
      const bool tail = (i + 1 == m) || ((kin[i + 1] & kWordMask) != wd[j]);
      if (tail) __stcg(p.shadow + bb + wd[j], (uint8_t)(run & 15u));
    }
  }
  emit_faults(p, fk, wd, ps, bb);
  __syncthreads();
  hash_clear(S);      // the sort arrays overlap the hash table
  __syncthreads();
}

// ---- the kernel ------------------------------------------------------------------------
__global__ void __launch_bounds__(RT, 2) k_replay(ReplayParams p) {
  extern __shared__ __align__(16) uint8_t smem_raw[];
  ReplaySmem& S = *reinterpret_cast<ReplaySmem*>(smem_raw);
  const uint32_t tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  hash_clear(S);
  for (;;) {
    if (tid == 0) {
      const unsigned long long w = atomicAdd(&p.st->work, 1ull);
      S.bucket = w < p.n_buckets ? p.order[w] : 0xFFFFFFFFu;
    }
    __syncthreads();
    const uint32_t b = S.bucket;
    if (b >= p.n_buckets) return;
    if (tid == 0) {
      S.q_head = S.q_tail = S.q_head_off = 0;
      S.q_events = 0;
      S.chunk_cur = 0;
      S.op_cur = p.ops_start[b];
      S.op_end = p.ops_start[b + 1];
      S.bucket_events = 0;
      S.bucket_base = p.bucket_start[b];
    }
    __syncthreads();
    const uint16_t* row0 = p.part_off + (uint64_t)b * p.n_chunks;
    const uint16_t* row1 = row0 + p.n_chunks;
    for (;;) {
      // ---- refill the segment queue ----------------------------------------
      while (S.q_events < STEP && S.chunk_cur < p.n_chunks && (S.q_tail - S.q_head) + kScanChunks <= kQCap) {
        const uint32_t c = S.chunk_cur + tid;
        uint32_t len = 0, st = 0;
        if (c < p.n_chunks) { st = row0[c]; len = (uint32_t)row1[c] - st; }
        uint32_t tot;
        const uint32_t rank = block_excl_scan(len ? 1u : 0u, S.wscan, &tot);
        const uint32_t evs = block_sum(len, S.red);
        if (len) {
          const uint32_t q = (S.q_tail + rank) % kQCap;
          S.q_start[q] = c * (uint32_t)kChunkCap + st;
          S.q_len[q] = len;
        }
        __syncthreads();
        if (tid == 0) {
          S.q_tail += tot;
          S.q_events += evs;
          S.chunk_cur += kScanChunks;
          S.bucket_events += evs;
        }
        __syncthreads();
      }
      if (S.q_events == 0) {
        apply_ops_before(S, p, 0xFFFFFFFFu);
        break;
      }
      // ---- gather up to STEP events in trace order ---------------------------
      const uint32_t nseg = min(S.q_tail - S.q_head, (uint32_t)kQCap);
      {
        uint32_t v[2];
#pragma unroll
        for (int k = 0; k < 2; ++k) {
          const uint32_t e = 2 * tid + k;
          v[k] = 0;
          if (e < nseg) v[k] = S.q_len[(S.q_head + e) % kQCap] - (e == 0 ? S.q_head_off : 0);
        }
        uint32_t tot;
        const uint32_t ex = block_excl_scan(v[0] + v[1], S.wscan, &tot);
        if (2 * tid < nseg) S.pref[2 * tid] = ex;
        if (2 * tid + 1 < nseg) S.pref[2 * tid + 1] = ex + v[0];
        if (tid == 0) S.n_gather = min(tot, (uint32_t)STEP);
        __syncthreads();
      }
      const uint32_t m = S.n_gather;
      // number of segments that hold the first m events
      uint32_t nseg_m;
      {
        uint32_t a = 0, z = nseg;
        while (z - a > 1) { const uint32_t mid = (a + z) >> 1; if (S.pref[mid] < m) a = mid; else z = mid; }
        nseg_m = a + 1;
      }
      if (nseg_m * 8 <= m) {
        // long segments: one warp copies one segment at a time, coalesced
        for (uint32_t sgi = warp; sgi < nseg_m; sgi += RT / 32) {
          const uint32_t q = (S.q_head + sgi) % kQCap;
          const uint32_t dst = S.pref[sgi];
          const uint32_t len = min((sgi + 1 < nseg ? S.pref[sgi + 1] : m), m) - dst;
          const uint2* src = p.part_ev + (uint64_t)S.q_start[q] + (sgi == 0 ? S.q_head_off : 0);
          for (uint32_t k = lane; k < len; k += 64) {
            const uint2 e0 = ld_stream2(src + k);
            uint2 e1 = make_uint2(0, 0);
            if (k + 32 < len) e1 = ld_stream2(src + k + 32);
            S.keyA[dst + k] = e0.x; S.posA[dst + k] = e0.y;
            if (k + 32 < len) { S.keyA[dst + k + 32] = e1.x; S.posA[dst + k + 32] = e1.y; }
          }
        }
      } else {
        // short segments: every thread finds its events' segments
        uint2 evv[RI];
#pragma unroll
        for (int k = 0; k < RI; ++k) {
          const uint32_t e = tid + k * RT;
          evv[k] = make_uint2(0, 0);
          if (e < m) {
            uint32_t a = 0, z = nseg_m;
            while (z - a > 1) { const uint32_t mid = (a + z) >> 1; if (S.pref[mid] <= e) a = mid; else z = mid; }
            const uint32_t q = (S.q_head + a) % kQCap;
            const uint32_t off = e - S.pref[a] + (a == 0 ? S.q_head_off : 0);
            evv[k] = ld_stream2(p.part_ev + (uint64_t)S.q_start[q] + off);
          }
        }
#pragma unroll
        for (int k = 0; k < RI; ++k) {
          const uint32_t e = tid + k * RT;
          if (e < m) { S.keyA[e] = evv[k].x; S.posA[e] = evv[k].y; }
        }
      }
      __syncthreads();
      // ---- range ops before the first gathered event ---------------------------
      apply_ops_before(S, p, S.posA[0]);
      // ---- cut the step at the next pending range op -----------------------------
      const uint32_t next_op = S.op_cur < S.op_end ? p.ops[S.op_cur].pos : 0xFFFFFFFFu;
      uint32_t cnt = 0;
      for (uint32_t e = tid; e < m; e += RT) cnt += S.posA[e] < next_op;
      const uint32_t cut = block_sum(cnt, S.red);
      // ---- consume `cut` events from the queue (before pref is reused) -----------
      if (tid == 0) {
        uint32_t a = 0, z = nseg;
        while (z - a > 1) { const uint32_t mid = (a + z) >> 1; if (S.pref[mid] <= cut) a = mid; else z = mid; }
        const uint32_t q = (S.q_head + a) % kQCap;
        const uint32_t consumed = cut - S.pref[a] + (a == 0 ? S.q_head_off : 0);
        if (consumed >= S.q_len[q]) { S.q_head += a + 1; S.q_head_off = 0; }
        else { S.q_head += a; S.q_head_off = consumed; }
        S.q_events -= cut;
      }
      __syncthreads();
      if (!step_fast(S, p, cut)) step_sort(S, p, cut);
    }
    if (tid == 0 && S.bucket_events) atomicMax(&p.st->max_bucket_events, (unsigned long long)S.bucket_events);
    __syncthreads();
  }
}

cudaError_t launch_replay(const ReplayParams& p, int n_ctas, cudaStream_t s) {
  const size_t smem = sizeof(ReplaySmem);
  cudaError_t e = cudaFuncSetAttribute(k_replay, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  k_replay<<<n_ctas, RT, smem, s>>>(p);
  return cudaGetLastError();
}

}  // namespace arb
