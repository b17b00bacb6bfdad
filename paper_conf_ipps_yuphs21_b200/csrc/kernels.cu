// kernels.cu — sm_100a kernels of the ARBALEST replay hot path.
//
//   k_partition  (A1 + A3a) decode 16-B records with one 128-bit load each,
//                split access vs control records, map byte ranges to 8-B words
//                (P:267), stable-partition the word-events of each 4096-record
//                chunk by address bucket (chunk-major output + offset table).
//   k_replay     (A3b + A4 + A5) one CTA per address bucket (persistent work
//                queue): gathers the bucket's events in trace order, applies
//                the resolved range ops (Table I transfers / allocate /
//                release) at their trace positions, stable-sorts
//                each step of <= 4096 events by word in shared memory, runs a
//                segmented scan of the access transition monoid seeded with the
//                shadow state (VSM), classifies faulting reads as
//                UUM / USD and commits the shadow.
//   k_mir_*      (A6) mapping-induced races (Theorem 1, reading Z10)
//                as a join between the ops of nowait task instances and the ops
//                inside their race windows.
//   k_rs_* / k_compact_*  canonical report order (word, record, kind) + unique.
#include "arb_internal.h"
#include <cstdio>

namespace arb {

#define FULL 0xFFFFFFFFu

__device__ __forceinline__ uint32_t lanemask_lt() {
  uint32_t m;
  asm("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
  return m;
}

__device__ __forceinline__ uint4 ld_stream(const uint4* p) {
  uint4 r;
  asm volatile("ld.global.cs.v4.u32 {%0,%1,%2,%3}, [%4];"
               : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p));
  return r;
}
__device__ __forceinline__ uint2 ld_stream2(const uint2* p) {
  uint2 r;
  asm volatile("ld.global.cs.v2.u32 {%0,%1}, [%2];" : "=r"(r.x), "=r"(r.y) : "l"(p));
  return r;
}

// ---- selector-form transition functions (see arb_internal.h) -------------
__device__ __forceinline__ uint32_t sel_apply4(Sel s, uint32_t x) {
  // x holds 4 states, one per byte (low nibble); returns the 4 images.
  uint32_t out = 0;
#pragma unroll
  for (int j = 0; j < 4; ++j) {
    uint32_t src = (s >> (3 * j)) & 7u;
    uint32_t v = src < 4 ? (x >> src) & 0x01010101u : (src == 5 ? 0x01010101u : 0u);
    out |= v << j;
  }
  return out;
}
__device__ __forceinline__ Sel sel_compose(Sel g, Sel f) {  // g after f
  Sel r = 0;
#pragma unroll
  for (int j = 0; j < 4; ++j) {
    uint32_t gj = (g >> (3 * j)) & 7u;
    uint32_t v = gj < 4 ? (f >> (3 * gj)) & 7u : gj;
    r |= v << (3 * j);
  }
  return r;
}

// ===========================================================================
// k_partition
// ===========================================================================
struct Decoded {
  uint32_t cnt;        // tracked events of this record (0..2)
  uint32_t b0, b1;     // buckets
  uint32_t k0, k1;     // compact keys: op << 30 | word offset in bucket
  uint32_t ignored;    // word-ops outside the tracked range
  bool ctl, bad;
};

__device__ __forceinline__ Decoded decode(uint4 r, bool valid, const PartParams& p) {
  Decoded d;
  d.cnt = 0; d.b0 = d.b1 = 0xFFFFFFFFu; d.k0 = d.k1 = 0; d.ignored = 0; d.ctl = false; d.bad = false;
  if (!valid) return d;
  uint64_t w0 = (uint64_t)r.x | ((uint64_t)r.y << 32);
  uint64_t w1 = (uint64_t)r.z | ((uint64_t)r.w << 32);
  uint32_t op = (uint32_t)(w0 >> 48) & 0xFFu;
  if (op < 4) {
    uint64_t addr = w0 & kMask48, len = w1 & kMask48;
    if (len < 1 || len > 8 || addr + len > (1ull << 48)) { d.bad = true; return d; }
    uint64_t x0 = addr >> 3, x1 = (addr + len - 1) >> 3;
    const uint32_t cmask = (1u << p.coarse_bits) - 1u;
    for (uint64_t x = x0; x <= x1; ++x) {
      uint64_t rel = x - p.base_word;
      if (x >= p.base_word && rel < p.n_words) {
        uint32_t m = __ldg(p.bin_map + (rel >> p.coarse_bits));
        uint32_t b = m & 1023u;
        uint32_t off = ((m >> 10) << p.coarse_bits) | ((uint32_t)rel & cmask);
        uint32_t k = (op << 30) | off;
        if (d.cnt == 0) { d.b0 = b; d.k0 = k; } else { d.b1 = b; d.k1 = k; }
        d.cnt++;
      } else {
        d.ignored++;
      }
    }
  } else if (op == OP_MAP_ENTER || op == OP_MAP_EXIT || op == OP_UPDATE ||
             op == OP_TASK_BEGIN || op == OP_TASK_END || op == OP_SYNC) {
    d.ctl = true;
  } else {
    d.bad = true;
  }
  return d;
}

// Rank this round's events of one warp into the warp's per-bucket running
// counters `row` (u16, one row per warp).  Order = record order, and for a
// record with two words word0 before word1.  If `offs` is non-null the
// returned ranks are final positions (row holds running offsets).
__device__ __forceinline__ void warp_rank_round(const Decoded& d, uint16_t* row, uint32_t lane,
                                                uint32_t& r0, uint32_t& r1) {
  bool straddle = d.cnt == 2 && d.b0 != d.b1;
  if (__any_sync(FULL, straddle)) {
    // rare: a record crossing a bucket boundary somewhere in the warp; serial
    for (uint32_t L = 0; L < 32; ++L) {
      if (lane == L) {
        if (d.cnt >= 1) { r0 = row[d.b0]; row[d.b0] = (uint16_t)(r0 + 1); }
        if (d.cnt == 2) { r1 = row[d.b1]; row[d.b1] = (uint16_t)(r1 + 1); }
      }
      __syncwarp();
    }
    return;
  }
  uint32_t key = d.cnt ? d.b0 : 0xFFFFFFFFu;
  uint32_t grp = __match_any_sync(FULL, key);
  uint32_t two = __ballot_sync(FULL, d.cnt == 2);
  uint32_t lt = lanemask_lt();
  uint32_t before = __popc(grp & lt) + __popc(grp & lt & two);
  uint32_t total = __popc(grp) + __popc(grp & two);
  uint32_t base = 0;
  if (d.cnt) base = row[d.b0];
  __syncwarp();
  if (d.cnt && lane == 31u - __clz(grp)) row[d.b0] = (uint16_t)(base + total);
  __syncwarp();
  r0 = base + before;
  r1 = r0 + 1;
}

__global__ void __launch_bounds__(kPartThreads, 2) k_partition(PartParams p) {
  extern __shared__ __align__(16) uint8_t smem[];
  const uint32_t NB = p.n_buckets;
  uint16_t* hist = reinterpret_cast<uint16_t*>(smem);                      // [warps][NB]
  uint2* sorted = reinterpret_cast<uint2*>(smem + ((kPartWarps * NB * 2 + 15) & ~15u));
  __shared__ uint32_t s_wsum[kPartWarps];
  __shared__ uint32_t s_total;

  const uint32_t tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const uint64_t chunk = blockIdx.x;
  const uint64_t rec0 = chunk * kChunkRecords;
  constexpr int kRounds = kChunkRecords / kPartThreads;  // 8
  const uint64_t wrec0 = rec0 + (uint64_t)warp * (kChunkRecords / kPartWarps);

  for (uint32_t i = tid; i < kPartWarps * NB; i += kPartThreads) hist[i] = 0;
  __syncthreads();

  uint16_t* row = hist + warp * NB;
  uint4 rec[kRounds];
  uint32_t n_acc = 0, n_ign = 0;
  // ---- pass A: load, decode, count per (warp, bucket) ------------------------
#pragma unroll
  for (int r = 0; r < kRounds; ++r) {
    uint64_t i = wrec0 + (uint64_t)r * 32 + lane;
    bool valid = i < p.n;
    rec[r] = valid ? ld_stream(p.ev + i) : make_uint4(0, 0, 0, 0);
  }
#pragma unroll
  for (int r = 0; r < kRounds; ++r) {
    uint64_t i = wrec0 + (uint64_t)r * 32 + lane;
    bool valid = i < p.n;
    Decoded d = decode(rec[r], valid, p);
    n_acc += d.cnt; n_ign += d.ignored;
    if (d.bad) atomicMin(&p.st->err_pos, (unsigned long long)i);
    uint32_t cm = __ballot_sync(FULL, d.ctl);
    if (cm) {
      unsigned long long base = 0;
      if (lane == 0) base = atomicAdd(&p.st->n_ctl, (unsigned long long)__popc(cm));
      base = __shfl_sync(FULL, base, 0);
      if (d.ctl) {
        uint64_t slot = base + __popc(cm & lanemask_lt());
        if (slot < p.ctl_cap) {
          CtlRec c;
          c.pos = i;
          c.w0 = (uint64_t)rec[r].x | ((uint64_t)rec[r].y << 32);
          c.w1 = (uint64_t)rec[r].z | ((uint64_t)rec[r].w << 32);
          p.ctl[slot] = c;
        }
      }
    }
    uint32_t r0, r1;
    warp_rank_round(d, row, lane, r0, r1);
  }
  __syncthreads();

  // ---- scan: per bucket over warps, then over buckets ----------------------
  // thread t owns buckets 2t and 2t+1
  uint32_t bt[2] = {0, 0};
#pragma unroll
  for (int k = 0; k < 2; ++k) {
    uint32_t b = 2 * tid + k;
    if (b < NB) {
      uint32_t s = 0;
      for (int w = 0; w < kPartWarps; ++w) {
        uint32_t c = hist[w * NB + b];
        hist[w * NB + b] = (uint16_t)s;
        s += c;
      }
      bt[k] = s;
    }
  }
  uint32_t mine = bt[0] + bt[1], incl = mine;
#pragma unroll
  for (int d = 1; d < 32; d <<= 1) {
    uint32_t o = __shfl_up_sync(FULL, incl, d);
    if (lane >= (uint32_t)d) incl += o;
  }
  if (lane == 31) s_wsum[warp] = incl;
  __syncthreads();
  if (warp == 0) {
    uint32_t v = lane < kPartWarps ? s_wsum[lane] : 0, vi = v;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
      uint32_t o = __shfl_up_sync(FULL, vi, d);
      if (lane >= (uint32_t)d) vi += o;
    }
    if (lane < kPartWarps) s_wsum[lane] = vi - v;
    if (lane == kPartWarps - 1) s_total = vi;
  }
  __syncthreads();
  uint32_t excl = s_wsum[warp] + incl - mine;
  uint32_t bb[2] = {excl, excl + bt[0]};
#pragma unroll
  for (int k = 0; k < 2; ++k) {
    uint32_t b = 2 * tid + k;
    if (b < NB) {
      for (int w = 0; w < kPartWarps; ++w) hist[w * NB + b] = (uint16_t)(hist[w * NB + b] + bb[k]);
      p.part_off[(uint64_t)b * p.n_chunks + chunk] = (uint16_t)bb[k];
    }
  }
  if (tid == 0) p.part_off[(uint64_t)NB * p.n_chunks + chunk] = (uint16_t)s_total;
  __syncthreads();

  // ---- pass B: stable scatter into shared memory ---------------------------
#pragma unroll
  for (int r = 0; r < kRounds; ++r) {
    uint64_t i = wrec0 + (uint64_t)r * 32 + lane;
    bool valid = i < p.n;
    Decoded d = decode(rec[r], valid, p);
    uint32_t r0 = 0, r1 = 0;
    warp_rank_round(d, row, lane, r0, r1);
    if (d.cnt >= 1) sorted[r0] = make_uint2(d.k0, (uint32_t)i);
    if (d.cnt == 2) sorted[r1] = make_uint2(d.k1, (uint32_t)i);
  }
  __syncthreads();
  const uint32_t total = s_total;
  uint2* out = p.part_ev + chunk * kChunkCap;
  for (uint32_t j = tid; j < total; j += kPartThreads) out[j] = sorted[j];

  // ---- counters --------------------------------------------------------------
#pragma unroll
  for (int d = 16; d; d >>= 1) {
    n_acc += __shfl_xor_sync(FULL, n_acc, d);
    n_ign += __shfl_xor_sync(FULL, n_ign, d);
  }
  if (lane == 0) {
    if (n_acc) atomicAdd(&p.st->access_words, (unsigned long long)n_acc);
    if (n_ign) atomicAdd(&p.st->ignored_words, (unsigned long long)n_ign);
  }
}

// Sampled histogram of access addresses over coarse bins (bucket balancing).
__global__ void k_sample(SampleParams p, uint64_t n_samples) {
  for (uint64_t k = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; k < n_samples;
       k += (uint64_t)gridDim.x * blockDim.x) {
    uint4 r = ld_stream(p.ev + k * p.stride);
    uint64_t w0 = (uint64_t)r.x | ((uint64_t)r.y << 32);
    if (((w0 >> 48) & 0xFFu) >= 4) continue;
    uint64_t rel = ((w0 & kMask48) >> 3) - p.base_word;
    if ((w0 & kMask48) >> 3 >= p.base_word && rel < p.n_words) atomicAdd(&p.hist[rel >> p.coarse_bits], 1u);
  }
}

cudaError_t launch_sample(const SampleParams& p, uint64_t n_samples, cudaStream_t s) {
  if (!n_samples) return cudaSuccess;
  uint64_t g = (n_samples + 255) / 256;
  k_sample<<<(unsigned)(g > 148 * 16 ? 148 * 16 : g), 256, 0, s>>>(p, n_samples);
  return cudaGetLastError();
}

cudaError_t launch_partition(const PartParams& p, cudaStream_t s) {
  if (p.n_chunks == 0) return cudaSuccess;
  size_t smem = ((kPartWarps * p.n_buckets * 2 + 15) & ~15u) + (size_t)kChunkCap * sizeof(uint2);
  cudaError_t e = cudaFuncSetAttribute(k_partition, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  k_partition<<<p.n_chunks, kPartThreads, smem, s>>>(p);
  return cudaGetLastError();
}

// ===========================================================================
// k_replay
// ===========================================================================
constexpr int kQCap = 2048;       // segment queue (circular)
constexpr int kScanChunks = 512;  // chunks examined per refill round

struct ReplaySmem {
  uint32_t keyA[kStep], posA[kStep], keyB[kStep], posB[kStep];
  uint16_t hist[kReplayThreads / 32][256];
  uint32_t q_start[kQCap];        // global event index of a segment
  uint32_t q_len[kQCap];
  uint32_t pref[1024];            // prefix of queue lengths for gathering
  uint32_t red[kReplayThreads / 32];
  uint32_t red2[kReplayThreads / 32];
  uint32_t wscan[kReplayThreads / 32];
  // scalar state
  uint32_t bucket;
  uint32_t q_head, q_tail, q_head_off;
  uint64_t q_events;
  uint32_t chunk_cur;
  uint32_t n_gather;
  uint32_t m_valid;
  uint32_t op_cur, op_end;
  uint64_t bucket_events;
};

__device__ __forceinline__ uint32_t block_sum(uint32_t v, uint32_t* red) {
  const uint32_t lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
#pragma unroll
  for (int d = 16; d; d >>= 1) v += __shfl_xor_sync(FULL, v, d);
  __syncthreads();
  if (lane == 0) red[warp] = v;
  __syncthreads();
  uint32_t t = 0;
  for (int w = 0; w < kReplayThreads / 32; ++w) t += red[w];
  return t;
}
__device__ __forceinline__ uint32_t block_min(uint32_t v, uint32_t* red) {
  const uint32_t lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
#pragma unroll
  for (int d = 16; d; d >>= 1) v = min(v, __shfl_xor_sync(FULL, v, d));
  __syncthreads();
  if (lane == 0) red[warp] = v;
  __syncthreads();
  uint32_t t = 0xFFFFFFFFu;
  for (int w = 0; w < kReplayThreads / 32; ++w) t = min(t, red[w]);
  return t;
}
__device__ __forceinline__ uint32_t block_max(uint32_t v, uint32_t* red) {
  const uint32_t lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
#pragma unroll
  for (int d = 16; d; d >>= 1) v = max(v, __shfl_xor_sync(FULL, v, d));
  __syncthreads();
  if (lane == 0) red[warp] = v;
  __syncthreads();
  uint32_t t = 0;
  for (int w = 0; w < kReplayThreads / 32; ++w) t = max(t, red[w]);
  return t;
}
// exclusive block scan (sum); returns the exclusive prefix of v, *total = sum
__device__ __forceinline__ uint32_t block_excl_scan(uint32_t v, uint32_t* wscan, uint32_t* total) {
  const uint32_t lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  uint32_t incl = v;
#pragma unroll
  for (int d = 1; d < 32; d <<= 1) {
    uint32_t o = __shfl_up_sync(FULL, incl, d);
    if (lane >= (uint32_t)d) incl += o;
  }
  __syncthreads();
  if (lane == 31) wscan[warp] = incl;
  __syncthreads();
  uint32_t wpre = 0, tot = 0;
  for (int w = 0; w < kReplayThreads / 32; ++w) {
    uint32_t x = wscan[w];
    if ((uint32_t)w < warp) wpre += x;
    tot += x;
  }
  *total = tot;
  return wpre + incl - v;
}

// Apply transition `sel` to shadow bytes [lo, hi) (relative word indices).
__device__ void stream_apply(uint8_t* shadow, uint64_t lo, uint64_t hi, Sel sel) {
  if (lo >= hi) return;
  uint64_t a = (lo + 15) & ~15ull, b = hi & ~15ull;
  if (a > b) { a = hi; b = hi; }
  // head and tail bytes
  for (uint64_t j = lo + threadIdx.x; j < a; j += kReplayThreads) {
    uint32_t x = __ldcg(shadow + j);
    __stcg(shadow + j, (uint8_t)sel_apply4(sel, x));
  }
  for (uint64_t j = b + threadIdx.x; j < hi; j += kReplayThreads) {
    uint32_t x = __ldcg(shadow + j);
    __stcg(shadow + j, (uint8_t)sel_apply4(sel, x));
  }
  uint4* v = reinterpret_cast<uint4*>(shadow + a);
  uint64_t nv = (b - a) >> 4;
  for (uint64_t j = threadIdx.x; j < nv; j += kReplayThreads) {
    uint4 x = __ldcg(v + j);
    x.x = sel_apply4(sel, x.x); x.y = sel_apply4(sel, x.y);
    x.z = sel_apply4(sel, x.z); x.w = sel_apply4(sel, x.w);
    __stcg(v + j, x);
  }
}

// Apply every pending range op of the bucket with position < limit.
__device__ void apply_ops_before(ReplaySmem& S, const ReplayParams& p, uint32_t limit) {
  while (S.op_cur < S.op_end && p.ops[S.op_cur].pos < limit) {
    uint32_t k = S.op_cur;
    BucketOp o = p.ops[k];
    Sel sel = o.sel;
    uint32_t k2 = k + 1;
    // compose consecutive ops on the identical range with no event in between
    while (k2 < S.op_end) {
      BucketOp o2 = p.ops[k2];
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

// One stable LSD pass on keys (word offset in the low 30 bits) of m elements.
__device__ void sort_pass(ReplaySmem& S, const uint32_t* kin, const uint32_t* pin, uint32_t* kout,
                          uint32_t* pout, uint32_t m, uint32_t minw, uint32_t shift, uint32_t dmask) {
  const uint32_t tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  uint32_t* h32 = reinterpret_cast<uint32_t*>(&S.hist[0][0]);
  for (uint32_t i = tid; i < (kReplayThreads / 32) * 256 / 2; i += kReplayThreads) h32[i] = 0;
  __syncthreads();
  uint16_t* row = S.hist[warp];
  uint32_t kk[kReplayItems], pp[kReplayItems], rk[kReplayItems], dg[kReplayItems];
  const uint32_t lt = lanemask_lt();
#pragma unroll
  for (int r = 0; r < kReplayItems; ++r) {
    uint32_t i = warp * (32 * kReplayItems) + r * 32 + lane;
    bool valid = i < m;
    uint32_t k = valid ? kin[i] : 0, pv = valid ? pin[i] : 0;
    uint32_t d = valid ? ((((k & 0x3FFFFFFFu) - minw) >> shift) & dmask) : 0xFFFFu;
    uint32_t grp = __match_any_sync(FULL, d);
    uint32_t base = valid ? row[d] : 0;
    __syncwarp();
    if (valid && lane == 31u - __clz(grp)) row[d] = (uint16_t)(base + __popc(grp));
    __syncwarp();
    kk[r] = k; pp[r] = pv; dg[r] = d; rk[r] = base + __popc(grp & lt);
  }
  __syncthreads();
  if (tid < 256) {
    uint32_t s = 0;
#pragma unroll
    for (int w = 0; w < kReplayThreads / 32; ++w) {
      uint32_t c = S.hist[w][tid];
      S.hist[w][tid] = (uint16_t)s;
      s += c;
    }
    S.pref[tid] = s;  // digit totals (pref is free during a sort)
  }
  __syncthreads();
  if (tid < 32) {   // exclusive scan of 256 digit totals by one warp
    uint32_t v[8], t = 0;
#pragma unroll
    for (int j = 0; j < 8; ++j) { v[j] = S.pref[tid * 8 + j]; t += v[j]; }
    uint32_t incl = t;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
      uint32_t o = __shfl_up_sync(FULL, incl, d);
      if (tid >= (uint32_t)d) incl += o;
    }
    uint32_t run = incl - t;
#pragma unroll
    for (int j = 0; j < 8; ++j) { S.pref[tid * 8 + j] = run; run += v[j]; }
  }
  __syncthreads();
  if (tid < 256) {
    uint32_t b = S.pref[tid];
#pragma unroll
    for (int w = 0; w < kReplayThreads / 32; ++w) S.hist[w][tid] = (uint16_t)(S.hist[w][tid] + b);
  }
  __syncthreads();
#pragma unroll
  for (int r = 0; r < kReplayItems; ++r) {
    uint32_t i = warp * (32 * kReplayItems) + r * 32 + lane;
    if (i < m) {
      uint32_t o = S.hist[warp][dg[r]] + rk[r];
      kout[o] = kk[r];
      pout[o] = pp[r];
    }
  }
  __syncthreads();
}

// access transition monoid:
//   bit7 HEAD, bit6 CONST, const: bits0-3 = state; summary: bits0-1 last write
//   (1 WH, 2 WT), bit2 any WH, bit3 any WT.  0 is the identity.
constexpr uint32_t kHead = 0x80, kConst = 0x40;
__device__ __forceinline__ uint32_t acc_apply(uint32_t v, uint32_t s) {
  uint32_t lw = v & 3u;
  if (lw) s = (s & ~3u) | lw;     // WH: OVv=1,CVv=0 ; WT: OVv=0,CVv=1
  return s | (v & 12u);           // any WH sets OVi, any WT sets CVi
}
__device__ __forceinline__ uint32_t acc_combine(uint32_t a, uint32_t b) {  // a before b
  if (b & kHead) return b;
  if (a & kConst) return (a & kHead) | kConst | acc_apply(b, a & 15u);
  uint32_t lw = (b & 3u) ? (b & 3u) : (a & 3u);
  return (a & kHead) | lw | ((a | b) & 12u);
}
__device__ __forceinline__ uint32_t acc_summary(uint32_t op) {
  return op == OP_WH ? (1u | 4u) : (op == OP_WT ? (2u | 8u) : 0u);
}

__device__ void process_step(ReplaySmem& S, const ReplayParams& p, uint32_t m) {
  const uint32_t tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  // key range of the step -> number of radix passes
  uint32_t lo = 0xFFFFFFFFu, hi = 0;
  for (uint32_t i = tid; i < m; i += kReplayThreads) {
    uint32_t w = S.keyA[i] & 0x3FFFFFFFu;
    lo = min(lo, w); hi = max(hi, w);
  }
  uint32_t minw = block_min(lo, S.red);
  uint32_t maxw = block_max(hi, S.red2);
  uint32_t span = maxw - minw;
  uint32_t bits = span ? 32 - __clz(span) : 0;
  uint32_t* kin = S.keyA; uint32_t* pin = S.posA; uint32_t* kout = S.keyB; uint32_t* pout = S.posB;
  for (uint32_t sh = 0; sh < bits; sh += 8) {
    uint32_t nb = min(8u, bits - sh);
    sort_pass(S, kin, pin, kout, pout, m, minw, sh, (1u << nb) - 1u);
    uint32_t* t = kin; kin = kout; kout = t;
    t = pin; pin = pout; pout = t;
  }
  // blocked arrangement: thread t owns sorted elements [8t, 8t+8)
  const uint64_t bucket_base = p.bucket_start[S.bucket];
  uint32_t val[kReplayItems], s0[kReplayItems], key[kReplayItems];
  bool head[kReplayItems];
  uint32_t agg = 0;
#pragma unroll
  for (int j = 0; j < kReplayItems; ++j) {
    uint32_t i = tid * kReplayItems + j;
    if (i < m) {
      uint32_t k = kin[i];
      uint32_t w = k & 0x3FFFFFFFu;
      bool h = (i == 0) || ((kin[i - 1] & 0x3FFFFFFFu) != w);
      uint32_t op = k >> 30;
      uint32_t v = acc_summary(op);
      uint32_t st = 0;
      if (h) {
        st = __ldcg(p.shadow + bucket_base + w) & 15u;
        v = kHead | kConst | acc_apply(v, st);
      }
      key[j] = k; head[j] = h; s0[j] = st; val[j] = v;
    } else {
      key[j] = 0; head[j] = false; s0[j] = 0; val[j] = 0;
    }
    agg = acc_combine(agg, val[j]);
  }
  // warp inclusive scan of thread aggregates
  uint32_t incl = agg;
#pragma unroll
  for (int d = 1; d < 32; d <<= 1) {
    uint32_t o = __shfl_up_sync(FULL, incl, d);
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
  // per element: state before, classification, commit
  uint32_t n_fault = 0;
  uint32_t fk[kReplayItems];
#pragma unroll
  for (int j = 0; j < kReplayItems; ++j) {
    uint32_t i = tid * kReplayItems + j;
    fk[j] = 0;
    if (i < m) {
      uint32_t before = head[j] ? s0[j] : (run & 15u);
      run = acc_combine(run, val[j]);
      uint32_t op = key[j] >> 30;
      if (op == OP_RH && !(before & kOVv)) fk[j] = (before & kOVi) ? 2u : 1u;   // USD : UUM
      if (op == OP_RT && !(before & kCVv)) fk[j] = (before & kCVi) ? 2u : 1u;
      n_fault += fk[j] != 0;
      bool tail = (i + 1 == m) || ((kin[i + 1] & 0x3FFFFFFFu) != (key[j] & 0x3FFFFFFFu));
      if (tail) __stcg(p.shadow + bucket_base + (key[j] & 0x3FFFFFFFu), (uint8_t)(run & 15u));
    }
  }
  // report candidates
  uint32_t wf = n_fault;
#pragma unroll
  for (int d = 1; d < 32; d <<= 1) {
    uint32_t o = __shfl_up_sync(FULL, wf, d);
    if (lane >= (uint32_t)d) wf += o;
  }
  uint32_t wtot = __shfl_sync(FULL, wf, 31);
  if (wtot) {
    unsigned long long base = 0;
    if (lane == 31) base = atomicAdd(&p.st->n_cand, (unsigned long long)wtot);
    base = __shfl_sync(FULL, base, 31);
    uint64_t slot = base + wf - n_fault;
#pragma unroll
    for (int j = 0; j < kReplayItems; ++j) {
      if (fk[j]) {
        if (slot < p.cand_cap) {
          uint64_t wr = bucket_base + (key[j] & 0x3FFFFFFFu);
          uint32_t i = tid * kReplayItems + j;
          p.cand[slot] = make_uint4((uint32_t)wr, (uint32_t)(wr >> 32), pin[i], fk[j]);
        }
        ++slot;
      }
    }
  }
  __syncthreads();
}

__global__ void __launch_bounds__(kReplayThreads, 1) k_replay(ReplayParams p) {
  extern __shared__ __align__(16) uint8_t smem_raw[];
  ReplaySmem& S = *reinterpret_cast<ReplaySmem*>(smem_raw);
  const uint32_t tid = threadIdx.x;
  for (;;) {
    if (tid == 0) {
      unsigned long long w = atomicAdd(&p.st->work, 1ull);
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
    }
    __syncthreads();
    const uint16_t* row0 = p.part_off + (uint64_t)b * p.n_chunks;
    const uint16_t* row1 = row0 + p.n_chunks;
    for (;;) {
      // ---- refill the segment queue ----------------------------------------
      while (S.q_events < kStep && S.chunk_cur < p.n_chunks &&
             (S.q_tail - S.q_head) + kScanChunks <= kQCap) {
        uint32_t c = S.chunk_cur + tid;
        uint32_t len = 0, st = 0;
        if (c < p.n_chunks) { st = row0[c]; len = (uint32_t)row1[c] - st; }
        uint32_t tot;
        uint32_t rank = block_excl_scan(len ? 1u : 0u, S.wscan, &tot);
        uint32_t evs = block_sum(len, S.red);
        if (len) {
          uint32_t q = (S.q_tail + rank) % kQCap;
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
      // ---- gather up to kStep events in trace order -------------------------
      uint32_t nseg = min(S.q_tail - S.q_head, 1024u);
      {
        // prefix of queue segment lengths (first segment minus consumed offset)
        uint32_t v[2];
#pragma unroll
        for (int k = 0; k < 2; ++k) {
          uint32_t e = 2 * tid + k;
          v[k] = 0;
          if (e < nseg) {
            uint32_t q = (S.q_head + e) % kQCap;
            v[k] = S.q_len[q] - (e == 0 ? S.q_head_off : 0);
          }
        }
        uint32_t tot;
        uint32_t ex = block_excl_scan(v[0] + v[1], S.wscan, &tot);
        if (2 * tid < nseg) S.pref[2 * tid] = ex;
        if (2 * tid + 1 < nseg) S.pref[2 * tid + 1] = ex + v[0];
        if (tid == 0) S.n_gather = min(tot, (uint32_t)kStep);
        __syncthreads();
      }
      const uint32_t m = S.n_gather;
      for (uint32_t e = tid; e < m; e += kReplayThreads) {
        uint32_t a = 0, z = nseg;            // last prefix <= e
        while (z - a > 1) { uint32_t mid = (a + z) >> 1; if (S.pref[mid] <= e) a = mid; else z = mid; }
        uint32_t q = (S.q_head + a) % kQCap;
        uint32_t off = e - S.pref[a] + (a == 0 ? S.q_head_off : 0);
        uint2 ev = ld_stream2(p.part_ev + (uint64_t)S.q_start[q] + off);
        S.keyA[e] = ev.x;
        S.posA[e] = ev.y;
      }
      __syncthreads();
      // ---- range ops that come before the first gathered event ---------------
      apply_ops_before(S, p, S.posA[0]);
      // ---- cut the step at the next pending range op -------------------------
      uint32_t next_op = S.op_cur < S.op_end ? p.ops[S.op_cur].pos : 0xFFFFFFFFu;
      uint32_t cnt = 0;
      for (uint32_t e = tid; e < m; e += kReplayThreads) cnt += S.posA[e] < next_op;
      uint32_t cut = block_sum(cnt, S.red);
      // ---- consume `cut` events from the queue (before the sort reuses pref) --
      if (tid == 0) {
        uint32_t a = 0, z = nseg;
        while (z - a > 1) { uint32_t mid = (a + z) >> 1; if (S.pref[mid] <= cut) a = mid; else z = mid; }
        // segment a holds event `cut` (or ends exactly there)
        uint32_t q = (S.q_head + a) % kQCap;
        uint32_t consumed_in_a = cut - S.pref[a] + (a == 0 ? S.q_head_off : 0);
        if (consumed_in_a >= S.q_len[q]) { S.q_head += a + 1; S.q_head_off = 0; }
        else { S.q_head += a; S.q_head_off = consumed_in_a; }
        S.q_events -= cut;
      }
      __syncthreads();
      process_step(S, p, cut);
    }
    if (tid == 0 && S.bucket_events) atomicMax(&p.st->max_bucket_events, (unsigned long long)S.bucket_events);
    __syncthreads();
  }
}

cudaError_t launch_replay(const ReplayParams& p, int n_ctas, cudaStream_t s) {
  size_t smem = sizeof(ReplaySmem);
  cudaError_t e = cudaFuncSetAttribute(k_replay, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  k_replay<<<n_ctas, kReplayThreads, smem, s>>>(p);
  return cudaGetLastError();
}

// ===========================================================================
// MIR join kernels (Theorem 1; reading Z10 of DESIGN.md)
// ===========================================================================
__device__ __forceinline__ uint32_t seg_of(const uint64_t* cum, uint32_t n, uint64_t g) {
  uint32_t a = 0, z = n;          // last cum[a] <= g
  while (z - a > 1) { uint32_t mid = (a + z) >> 1; if (cum[mid] <= g) a = mid; else z = mid; }
  return a;
}
__device__ __forceinline__ uint64_t hslot(unsigned long long key, uint64_t mask) {
  unsigned long long h = key * 0x9E3779B97F4A7C15ull;
  return (h ^ (h >> 29)) & mask;
}
__device__ __forceinline__ void emit_mir(const MirParams& p, uint64_t word_rel, uint32_t pos) {
  unsigned long long slot = atomicAdd(&p.st->n_mir_cand, 1ull);
  if (slot < p.cand_cap) p.cand[slot] = make_uint4((uint32_t)word_rel, (uint32_t)(word_rel >> 32), pos, 3u);
}
// words of an access record inside the tracked range: returns count (0..2)
__device__ __forceinline__ int access_words(const MirParams& p, uint4 r, uint64_t* w, uint32_t* op) {
  uint64_t w0 = (uint64_t)r.x | ((uint64_t)r.y << 32), w1 = (uint64_t)r.z | ((uint64_t)r.w << 32);
  *op = (uint32_t)(w0 >> 48) & 0xFFu;
  if (*op >= 4) return 0;
  uint64_t addr = w0 & kMask48, len = w1 & kMask48;
  int n = 0;
  for (uint64_t x = addr >> 3; x <= (addr + len - 1) >> 3; ++x) {
    if (x >= p.base_word && x - p.base_word < p.n_words) w[n++] = x - p.base_word;
  }
  return n;
}

// (iv) insert the access word-ops of racy task blocks; (iii) range ops in the
// instance's window that cover an inserted word race with it.
__global__ void k_mir_insert(MirParams p, uint64_t n_pos) {
  for (uint64_t g = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; g < n_pos;
       g += (uint64_t)gridDim.x * blockDim.x) {
    uint32_t s = seg_of(p.ins_cum, p.n_ins, g);
    uint64_t pos = p.ins_lo[s] + (g - p.ins_cum[s]);
    uint32_t qd = p.ins_inst[s];
    uint4 r = p.ev[pos];
    uint64_t w[2]; uint32_t op;
    int n = access_words(p, r, w, &op);
    for (int k = 0; k < n; ++k) {
      unsigned long long key = ((unsigned long long)w[k] << 20) | (qd + 1);
      uint64_t h = hslot(key, p.hmask);
      for (;;) {
        unsigned long long old = atomicCAS(&p.hkeys[h], 0ull, key);
        if (old == 0ull || old == key) break;
        h = (h + 1) & p.hmask;
      }
      if (op == OP_WH || op == OP_WT) atomicOr(&p.hvals[h], 1u);
      for (uint32_t j = p.win_start[qd]; j < p.win_start[qd + 1]; ++j) {
        RangeRef rr = p.win_ops[j];
        if (w[k] >= rr.lo && w[k] < rr.hi) emit_mir(p, w[k], rr.pos);
      }
    }
  }
}

// (iv) + (i): access ops inside race windows against the open instances'
// access ops (hash) and range ops (lists).
__global__ void k_mir_query(MirParams p, uint64_t n_pos) {
  for (uint64_t g = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; g < n_pos;
       g += (uint64_t)gridDim.x * blockDim.x) {
    uint32_t s = seg_of(p.qry_cum, p.n_qry, g);
    uint64_t pos = p.qry_lo[s] + (g - p.qry_cum[s]);
    uint4 r = p.ev[pos];
    uint64_t w[2]; uint32_t op;
    int n = access_words(p, r, w, &op);
    bool is_write = op == OP_WH || op == OP_WT;
    for (int k = 0; k < n; ++k) {
      bool mir = false;
      for (uint32_t j = p.qry_open_start[s]; j < p.qry_open_start[s + 1] && !mir; ++j) {
        uint32_t qd = p.open_list[j];
        unsigned long long key = ((unsigned long long)w[k] << 20) | (qd + 1);
        uint64_t h = hslot(key, p.hmask);
        for (;;) {
          unsigned long long kk = p.hkeys[h];
          if (kk == 0ull) break;
          if (kk == key) { if (is_write || (p.hvals[h] & 1u)) mir = true; break; }
          h = (h + 1) & p.hmask;
        }
        for (uint32_t t = p.own_start[qd]; t < p.own_start[qd + 1] && !mir; ++t) {
          RangeRef rr = p.own_ops[t];
          if (w[k] >= rr.lo && w[k] < rr.hi) mir = true;   // range ops are write-class
        }
      }
      if (mir) emit_mir(p, w[k], (uint32_t)pos);
    }
  }
}

// (ii) range op in a window vs the instance's own range ops: every word of
// the overlap (precomputed on the host) races.
__global__ void k_mir_ranges(MirParams p, uint64_t n_words) {
  for (uint64_t g = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; g < n_words;
       g += (uint64_t)gridDim.x * blockDim.x) {
    uint32_t s = seg_of(p.rr_cum, p.n_rr, g);
    RangeRef rr = p.rr[s];
    emit_mir(p, rr.lo + (g - p.rr_cum[s]), rr.pos);
  }
}

cudaError_t launch_mir(const MirParams& p, uint64_t n_ins_pos, uint64_t n_qry_pos, uint64_t n_rr_words,
                       cudaStream_t s, int* launches) {
  auto grid = [](uint64_t n) { uint64_t g = (n + 255) / 256; return (unsigned)(g > 148 * 64 ? 148 * 64 : (g ? g : 1)); };
  if (n_ins_pos) { k_mir_insert<<<grid(n_ins_pos), 256, 0, s>>>(p, n_ins_pos); ++*launches; }
  if (n_qry_pos) { k_mir_query<<<grid(n_qry_pos), 256, 0, s>>>(p, n_qry_pos); ++*launches; }
  if (n_rr_words) { k_mir_ranges<<<grid(n_rr_words), 256, 0, s>>>(p, n_rr_words); ++*launches; }
  return cudaGetLastError();
}

// ===========================================================================
// Report compaction: LSD radix sort of candidates + unique
// candidate = {word lo, word hi, pos, kind}
// ===========================================================================
constexpr int kRsThreads = 512, kRsItems = 8, kRsTile = kRsThreads * kRsItems;

struct RsPass { int field; int shift; int bits; };
__device__ __forceinline__ uint32_t rs_digit(uint4 c, RsPass ps) {
  uint32_t f = ps.field == 0 ? c.w : ps.field == 1 ? c.z : ps.field == 2 ? c.x : c.y;
  return (f >> ps.shift) & ((1u << ps.bits) - 1u);
}

__global__ void __launch_bounds__(kRsThreads) k_rs_hist(const uint4* in, uint64_t n, RsPass ps, uint32_t* cnt,
                                                        uint32_t nblk) {
  __shared__ uint32_t h[256];
  for (int i = threadIdx.x; i < 256; i += kRsThreads) h[i] = 0;
  __syncthreads();
  uint64_t base = (uint64_t)blockIdx.x * kRsTile;
  for (int j = 0; j < kRsItems; ++j) {
    uint64_t i = base + (uint64_t)j * kRsThreads + threadIdx.x;
    if (i < n) atomicAdd(&h[rs_digit(in[i], ps)], 1u);
  }
  __syncthreads();
  for (int d = threadIdx.x; d < 256; d += kRsThreads) cnt[(uint64_t)d * nblk + blockIdx.x] = h[d];
}

// exclusive scan of n u32 values in place (single CTA)
__global__ void __launch_bounds__(1024) k_scan_inplace(uint32_t* a, uint64_t n) {
  __shared__ uint32_t ws[32];
  __shared__ uint32_t carry;
  if (threadIdx.x == 0) carry = 0;
  __syncthreads();
  const uint32_t lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  for (uint64_t base = 0; base < n; base += 1024) {
    uint64_t i = base + threadIdx.x;
    uint32_t v = i < n ? a[i] : 0, incl = v;
    for (int d = 1; d < 32; d <<= 1) {
      uint32_t o = __shfl_up_sync(FULL, incl, d);
      if (lane >= (uint32_t)d) incl += o;
    }
    if (lane == 31) ws[warp] = incl;
    __syncthreads();
    if (warp == 0) {
      uint32_t x = ws[lane], xi = x;
      for (int d = 1; d < 32; d <<= 1) {
        uint32_t o = __shfl_up_sync(FULL, xi, d);
        if (lane >= (uint32_t)d) xi += o;
      }
      ws[lane] = xi - x;
    }
    __syncthreads();
    uint32_t c = carry;
    if (i < n) a[i] = c + ws[warp] + incl - v;
    __syncthreads();
    if (threadIdx.x == 1023) carry = c + ws[warp] + incl;
    __syncthreads();
  }
}

__global__ void __launch_bounds__(kRsThreads) k_rs_scatter(const uint4* in, uint4* out, uint64_t n, RsPass ps,
                                                           const uint32_t* cnt, uint32_t nblk) {
  __shared__ uint16_t hist[kRsThreads / 32][256];
  __shared__ uint32_t dbase[256];
  const uint32_t tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  uint32_t* h32 = reinterpret_cast<uint32_t*>(&hist[0][0]);
  for (uint32_t i = tid; i < (kRsThreads / 32) * 128; i += kRsThreads) h32[i] = 0;
  __syncthreads();
  uint64_t base = (uint64_t)blockIdx.x * kRsTile;
  uint4 c[kRsItems]; uint32_t rk[kRsItems], dg[kRsItems];
  const uint32_t lt = lanemask_lt();
  for (int r = 0; r < kRsItems; ++r) {
    uint64_t i = base + warp * (32 * kRsItems) + r * 32 + lane;
    bool valid = i < n;
    c[r] = valid ? in[i] : make_uint4(0, 0, 0, 0);
    uint32_t d = valid ? rs_digit(c[r], ps) : 0xFFFFu;
    uint32_t grp = __match_any_sync(FULL, d);
    uint32_t b = valid ? hist[warp][d] : 0;
    __syncwarp();
    if (valid && lane == 31u - __clz(grp)) hist[warp][d] = (uint16_t)(b + __popc(grp));
    __syncwarp();
    dg[r] = d; rk[r] = b + __popc(grp & lt);
  }
  __syncthreads();
  if (tid < 256) {
    uint32_t s = 0;
    for (int w = 0; w < kRsThreads / 32; ++w) { uint32_t x = hist[w][tid]; hist[w][tid] = (uint16_t)s; s += x; }
    dbase[tid] = cnt[(uint64_t)tid * nblk + blockIdx.x];
  }
  __syncthreads();
  for (int r = 0; r < kRsItems; ++r) {
    uint64_t i = base + warp * (32 * kRsItems) + r * 32 + lane;
    if (i < n) out[dbase[dg[r]] + hist[warp][dg[r]] + rk[r]] = c[r];
  }
}

// keep flags: unique (all fields differ from the predecessor), or dedup-first
// (word, kind differ from the predecessor) for the (word, kind, pos) order.
__device__ __forceinline__ bool keep_elem(const uint4* a, uint64_t i, int mode) {
  if (i == 0) return true;
  uint4 x = a[i], y = a[i - 1];
  if (mode == 0) return x.x != y.x || x.y != y.y || x.z != y.z || x.w != y.w;
  return x.x != y.x || x.y != y.y || x.w != y.w;
}
__global__ void __launch_bounds__(kRsThreads) k_keep_count(const uint4* a, uint64_t n, int mode, uint32_t* blk) {
  __shared__ uint32_t red[kRsThreads / 32];
  uint32_t c = 0;
  uint64_t base = (uint64_t)blockIdx.x * kRsTile;
  for (int j = 0; j < kRsItems; ++j) {
    uint64_t i = base + (uint64_t)threadIdx.x * kRsItems + j;
    if (i < n) c += keep_elem(a, i, mode);
  }
  for (int d = 16; d; d >>= 1) c += __shfl_xor_sync(FULL, c, d);
  if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = c;
  __syncthreads();
  if (threadIdx.x == 0) {
    uint32_t t = 0;
    for (int w = 0; w < kRsThreads / 32; ++w) t += red[w];
    blk[blockIdx.x] = t;
  }
}
// write kept elements; final != 0: convert to arb_report records
__global__ void __launch_bounds__(kRsThreads) k_keep_write(const uint4* a, uint64_t n, int mode, const uint32_t* blk,
                                                           uint4* out, int final_out, uint64_t base_word,
                                                           const uint64_t* gidx, uint64_t index_base,
                                                           unsigned long long* n_out, uint32_t nblk) {
  __shared__ uint32_t ws[kRsThreads / 32];
  const uint32_t lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  uint64_t base = (uint64_t)blockIdx.x * kRsTile;
  bool kp[kRsItems];
  uint32_t c = 0;
  for (int j = 0; j < kRsItems; ++j) {
    uint64_t i = base + (uint64_t)threadIdx.x * kRsItems + j;
    kp[j] = i < n && keep_elem(a, i, mode);
    c += kp[j];
  }
  uint32_t incl = c;
  for (int d = 1; d < 32; d <<= 1) {
    uint32_t o = __shfl_up_sync(FULL, incl, d);
    if (lane >= (uint32_t)d) incl += o;
  }
  if (lane == 31) ws[warp] = incl;
  __syncthreads();
  uint32_t wpre = 0;
  for (uint32_t w = 0; w < warp; ++w) wpre += ws[w];
  uint64_t o = blk[blockIdx.x] + wpre + incl - c;
  for (int j = 0; j < kRsItems; ++j) {
    uint64_t i = base + (uint64_t)threadIdx.x * kRsItems + j;
    if (!kp[j]) continue;
    uint4 x = a[i];
    if (final_out) {
      uint64_t word = ((uint64_t)x.x | ((uint64_t)x.y << 32)) + base_word;
      uint64_t w0 = (word & kMask48) | ((uint64_t)x.w << 48);
      uint64_t w1 = gidx ? gidx[x.z] : index_base + x.z;
      out[o] = make_uint4((uint32_t)w0, (uint32_t)(w0 >> 32), (uint32_t)w1, (uint32_t)(w1 >> 32));
      atomicAdd(&n_out[x.w & 3u], 1ull);   // per-kind counts in n_out[1..3]
    } else {
      out[o] = x;
    }
    ++o;
  }
  if (blockIdx.x == nblk - 1 && threadIdx.x == kRsThreads - 1) *n_out = o;
}

static cudaError_t radix_sort(uint4*& a, uint4*& b, uint64_t n, const RsPass* passes, int np, uint32_t* cnt,
                              cudaStream_t s, int* launches) {
  uint32_t nblk = (uint32_t)((n + kRsTile - 1) / kRsTile);
  for (int k = 0; k < np; ++k) {
    k_rs_hist<<<nblk, kRsThreads, 0, s>>>(a, n, passes[k], cnt, nblk);
    k_scan_inplace<<<1, 1024, 0, s>>>(cnt, (uint64_t)nblk * 256);
    k_rs_scatter<<<nblk, kRsThreads, 0, s>>>(a, b, n, passes[k], cnt, nblk);
    *launches += 3;
    uint4* t = a; a = b; b = t;
  }
  return cudaGetLastError();
}

static int add_field_passes(RsPass* ps, int np, int field, int bits) {
  for (int sh = 0; sh < bits; sh += 8) ps[np++] = RsPass{field, sh, bits - sh < 8 ? bits - sh : 8};
  return np;
}

cudaError_t launch_compact(const CompactParams& p, cudaStream_t s, int* launches) {
  cudaMemsetAsync(p.n_out, 0, 4 * sizeof(unsigned long long), s);
  if (p.n_cand == 0) return cudaGetLastError();
  uint4* a = p.cand;
  uint4* b = p.tmp;
  uint64_t n = p.n_cand;
  RsPass ps[24];
  int np = 0;
  int wb_lo = p.word_bits > 32 ? 32 : p.word_bits, wb_hi = p.word_bits > 32 ? p.word_bits - 32 : 0;
  cudaError_t e;
  if (p.dedup_first) {
    // (word, kind, pos): keep the first of each (word, kind)
    np = add_field_passes(ps, np, 1, p.pos_bits);
    np = add_field_passes(ps, np, 0, 2);
    np = add_field_passes(ps, np, 2, wb_lo);
    np = add_field_passes(ps, np, 3, wb_hi);
    if ((e = radix_sort(a, b, n, ps, np, p.blk, s, launches)) != cudaSuccess) return e;
    uint32_t nblk = (uint32_t)((n + kRsTile - 1) / kRsTile);
    k_keep_count<<<nblk, kRsThreads, 0, s>>>(a, n, 1, p.blk);
    k_scan_inplace<<<1, 1024, 0, s>>>(p.blk, nblk);
    k_keep_write<<<nblk, kRsThreads, 0, s>>>(a, n, 1, p.blk, b, 0, 0, nullptr, 0, p.n_out, nblk);
    *launches += 3;
    // the number kept is needed on the host side to continue; read it back
    unsigned long long kept = 0;
    cudaMemcpyAsync(&kept, p.n_out, sizeof(kept), cudaMemcpyDeviceToHost, s);
    cudaStreamSynchronize(s);
    n = kept;
    uint4* t = a; a = b; b = t;
    np = 0;
  }
  np = add_field_passes(ps, np, 0, 2);
  np = add_field_passes(ps, np, 1, p.pos_bits);
  np = add_field_passes(ps, np, 2, wb_lo);
  np = add_field_passes(ps, np, 3, wb_hi);
  if ((e = radix_sort(a, b, n, ps, np, p.blk, s, launches)) != cudaSuccess) return e;
  uint32_t nblk = (uint32_t)((n + kRsTile - 1) / kRsTile);
  if (n == 0) {
    cudaMemsetAsync(p.n_out, 0, 4 * sizeof(unsigned long long), s);
    return cudaGetLastError();
  }
  k_keep_count<<<nblk, kRsThreads, 0, s>>>(a, n, 0, p.blk);
  k_scan_inplace<<<1, 1024, 0, s>>>(p.blk, nblk);
  k_keep_write<<<nblk, kRsThreads, 0, s>>>(a, n, 0, p.blk, p.out, 1, p.base_word, p.gidx, p.index_base,
                                           p.n_out, nblk);
  *launches += 3;
  return cudaGetLastError();
}

}  // namespace arb
