// partition.cu — A1 (ingest/decode) + A3a (stable partition by address bucket).
//
// k_partition  persistent CTAs, one 4096-record chunk at a time: 128-bit loads
//              of the 16-B records (the next chunk's loads are issued while the
//              current chunk is being ranked and written), split access vs
//              control records, map each access's byte range to its 8-byte
//              words (1 or 2 words) and stable-partition the word-events
//              by address bucket into the chunk's slot of the output
//              (chunk-major) plus one row of the bucket offset table.  Each
//              record is decoded and ranked once; per-chunk bookkeeping only
//              touches the buckets the chunk actually hits.
#include "kcommon.cuh"
#include <algorithm>

namespace arb {

constexpr int PT = kPartThreads;            // 512 threads
constexpr int PW = kPartWarps;              // 16 warps
constexpr int ROUNDS = kChunkRecords / PT;  // 8 rounds of 32 records per warp

struct PartSmem {
  uint32_t touched[kMaxBuckets / 32];       // bitmap of buckets hit by the chunk
  uint16_t tlist[kMaxBuckets];              // touched buckets, ascending
  uint32_t tstart[kMaxBuckets + 1];         // their first event in the chunk
  uint32_t wsum[PW];
  uint32_t n_touched, total;
  unsigned long long seg_base;
};

// Decoded access record: info = cnt | b0 << 2 | b1 << 12 (cnt = tracked words
// 0..2), keys k0/k1 = op << 30 | word offset inside the bucket.
struct Dec { uint32_t info, k0, k1; };

__device__ __forceinline__ uint32_t bucket_key(const PartParams& p, uint64_t rel, uint32_t op, uint32_t& b) {
  const uint32_t m = __ldg(p.bin_map + (rel >> p.coarse_bits));
  b = m & 1023u;
  return (op << 30) | (((m >> 10) << p.coarse_bits) | ((uint32_t)rel & ((1u << p.coarse_bits) - 1u)));
}

__device__ __forceinline__ Dec decode(uint4 q, const PartParams& p, uint32_t& ign, bool& ctl, bool& bad) {
  Dec d{0, 0, 0};
  const uint32_t op = (q.y >> 16) & 0xFFu;
  ctl = op >= 8 && op <= 14 && op != 11;
  bad = false;
  if (op >= 4) { bad = !ctl; return d; }
  const uint32_t ahi = q.y & 0xFFFFu;
  const uint32_t len = q.z;
  const uint64_t addr = ((uint64_t)ahi << 32) | q.x;
  if ((q.w & 0xFFFFu) || len - 1u > 7u || addr + len > (1ull << 48)) { bad = true; return d; }
  const uint64_t rel = (addr >> 3) - p.base_word;                 // wraps when below the range
  const bool two = (q.x & 7u) + len > 8u;                          // unaligned: 2 words (Z4)
  uint32_t cnt = 0, b0 = 0, b1 = 0;
  if (rel < p.n_words) { d.k0 = bucket_key(p, rel, op, b0); b1 = b0; cnt = 1; } else { ++ign; }
  if (two) {
    const uint64_t r1 = rel + 1;
    if (r1 < p.n_words) {
      uint32_t bb;
      const uint32_t k = bucket_key(p, r1, op, bb);
      if (cnt == 0) { d.k0 = k; b0 = bb; b1 = bb; } else { d.k1 = k; b1 = bb; }
      ++cnt;
    } else {
      ++ign;
    }
  }
  d.info = cnt | (b0 << 2) | (b1 << 12);
  return d;
}

// Stable rank of this round's events inside the warp's per-bucket counters
// (record order, word0 before word1); marks the touched buckets.
__device__ __forceinline__ void rank_round(uint32_t info, uint16_t* row, uint32_t* touched, uint32_t lane,
                                           uint32_t& r0, uint32_t& r1) {
  const uint32_t cnt = info & 3u, b0 = (info >> 2) & 1023u, b1 = (info >> 12) & 1023u;
  r0 = r1 = 0;
  const uint32_t vmask = __ballot_sync(FULL, cnt != 0);
  if (!vmask) return;
  const uint32_t lead = __ffs(vmask) - 1;
  const uint32_t bref = __shfl_sync(FULL, b0, lead);
  const uint32_t lt = lanemask_lt();
  if (__all_sync(FULL, cnt == 0 || (b0 == bref && b1 == bref))) {
    // the common case: the whole round lands in one bucket
    const uint32_t two = __ballot_sync(FULL, cnt == 2);
    const uint32_t base = row[bref];
    __syncwarp();
    if (lane == lead) {
      row[bref] = (uint16_t)(base + __popc(vmask) + __popc(two));
      atomicOr(&touched[bref >> 5], 1u << (bref & 31));
    }
    __syncwarp();
    r0 = base + __popc(vmask & lt) + __popc(two & lt);
    r1 = r0 + 1;
    return;
  }
  if (__any_sync(FULL, cnt == 2 && b0 != b1)) {
    // rare: a record crossing a bucket boundary; serial over lanes
    for (uint32_t L = 0; L < 32; ++L) {
      if (lane == L) {
        if (cnt >= 1) { r0 = row[b0]; row[b0] = (uint16_t)(r0 + 1); atomicOr(&touched[b0 >> 5], 1u << (b0 & 31)); }
        if (cnt == 2) { r1 = row[b1]; row[b1] = (uint16_t)(r1 + 1); atomicOr(&touched[b1 >> 5], 1u << (b1 & 31)); }
      }
      __syncwarp();
    }
    return;
  }
  const uint32_t two = __ballot_sync(FULL, cnt == 2);
  const uint32_t grp = __match_any_sync(FULL, cnt ? b0 : 0xFFFFFFFFu);
  const uint32_t base = cnt ? row[b0] : 0;
  __syncwarp();
  if (cnt && lane == 31u - __clz(grp)) {
    row[b0] = (uint16_t)(base + __popc(grp) + __popc(grp & two));
    atomicOr(&touched[b0 >> 5], 1u << (b0 & 31));
  }
  __syncwarp();
  r0 = base + __popc(grp & lt) + __popc(grp & lt & two);
  r1 = r0 + 1;
}

__global__ void __launch_bounds__(PT, 1) k_partition(PartParams p) {
  extern __shared__ __align__(16) uint8_t smem[];
  const uint32_t NB = p.n_buckets;
  uint16_t* cnt = reinterpret_cast<uint16_t*>(smem);                       // [PW][NB]
  uint2* sorted = reinterpret_cast<uint2*>(smem + ((PW * NB * 2 + 15) & ~15u));
  __shared__ PartSmem S;

  const uint32_t tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  for (uint32_t i = tid; i < PW * NB; i += PT) cnt[i] = 0;
  if (tid < kMaxBuckets / 32) S.touched[tid] = 0;
  uint16_t* row = cnt + warp * NB;
  uint32_t n_acc = 0, n_ign = 0;

  uint64_t chunk = blockIdx.x;
  uint4 rec[ROUNDS];
#pragma unroll
  for (int r = 0; r < ROUNDS; ++r) {
    const uint64_t i = chunk * kChunkRecords + warp * (kChunkRecords / PW) + r * 32 + lane;
    rec[r] = (chunk < p.n_chunks && i < p.n) ? ld_stream(p.ev + i) : make_uint4(0, 0, 0, 0);
  }
  __syncthreads();

  for (; chunk < p.n_chunks; chunk += gridDim.x) {
    const uint64_t wrec0 = chunk * kChunkRecords + warp * (kChunkRecords / PW);
    // ---- pass A: decode + rank ---------------------------------------------------
    Dec dec[ROUNDS];
    uint32_t rk[ROUNDS];
#pragma unroll
    for (int r = 0; r < ROUNDS; ++r) {
      const uint64_t i = wrec0 + r * 32 + lane;
      bool ctl = false, bad = false;
      dec[r] = Dec{0, 0, 0};
      if (i < p.n) dec[r] = decode(rec[r], p, n_ign, ctl, bad);
      n_acc += dec[r].info & 3u;
      if (bad) atomicMin(&p.st->err_pos, (unsigned long long)i);
      const uint32_t cm = __ballot_sync(FULL, ctl);
      if (cm) {
        unsigned long long base = 0;
        if (lane == 0) base = atomicAdd(&p.st->n_ctl, (unsigned long long)__popc(cm));
        base = __shfl_sync(FULL, base, 0);
        if (ctl) {
          const uint64_t slot = base + __popc(cm & lanemask_lt());
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
      rank_round(dec[r].info, row, S.touched, lane, r0, r1);
      rk[r] = r0 | (r1 << 16);
    }
    // ---- prefetch the next chunk while this one is finished -----------------------
    {
      const uint64_t nchunk = chunk + gridDim.x;
#pragma unroll
      for (int r = 0; r < ROUNDS; ++r) {
        const uint64_t i = nchunk * kChunkRecords + warp * (kChunkRecords / PW) + r * 32 + lane;
        rec[r] = (nchunk < p.n_chunks && i < p.n) ? ld_stream(p.ev + i) : make_uint4(0, 0, 0, 0);
      }
    }
    __syncthreads();
    // ---- touched buckets, their totals and starts -----------------------------------
    if (warp == 0) {
      uint32_t base = 0;
      for (uint32_t w0 = 0; w0 < (NB + 31) / 32; w0 += 32) {
        const uint32_t wi = w0 + lane;
        const uint32_t bits = wi < (NB + 31) / 32 ? S.touched[wi] : 0;
        if (wi < (NB + 31) / 32) S.touched[wi] = 0;
        const uint32_t pc = __popc(bits);
        uint32_t incl = pc;
#pragma unroll
        for (int d = 1; d < 32; d <<= 1) {
          const uint32_t o = __shfl_up_sync(FULL, incl, d);
          if (lane >= (uint32_t)d) incl += o;
        }
        uint32_t k = base + incl - pc;
        for (uint32_t b = bits; b; b &= b - 1) S.tlist[k++] = (uint16_t)(wi * 32 + __ffs(b) - 1);
        base += __shfl_sync(FULL, incl, 31);
      }
      if (lane == 0) S.n_touched = base;
    }
    __syncthreads();
    const uint32_t T = S.n_touched;
    // per touched bucket: total over the warps, then per-warp offsets
    uint32_t mytot[2] = {0, 0};
#pragma unroll
    for (int k = 0; k < 2; ++k) {
      const uint32_t t = tid + k * PT;
      if (t < T) {
        const uint32_t b = S.tlist[t];
        uint32_t s = 0;
#pragma unroll
        for (int w = 0; w < PW; ++w) s += cnt[w * NB + b];
        mytot[k] = s;
      }
    }
    {
      // exclusive scan of the totals in touched order (thread t holds t and t + PT)
      uint32_t v = mytot[0], incl = v;
#pragma unroll
      for (int d = 1; d < 32; d <<= 1) {
        const uint32_t o = __shfl_up_sync(FULL, incl, d);
        if (lane >= (uint32_t)d) incl += o;
      }
      if (lane == 31) S.wsum[warp] = incl;
      __syncthreads();
      uint32_t wpre = 0, all0 = 0;
#pragma unroll
      for (int w = 0; w < PW; ++w) { const uint32_t x = S.wsum[w]; if ((uint32_t)w < warp) wpre += x; all0 += x; }
      const uint32_t s0 = wpre + incl - v;
      __syncthreads();
      uint32_t v1 = mytot[1], incl1 = v1;
#pragma unroll
      for (int d = 1; d < 32; d <<= 1) {
        const uint32_t o = __shfl_up_sync(FULL, incl1, d);
        if (lane >= (uint32_t)d) incl1 += o;
      }
      if (lane == 31) S.wsum[warp] = incl1;
      __syncthreads();
      uint32_t wpre1 = 0, all1 = 0;
#pragma unroll
      for (int w = 0; w < PW; ++w) { const uint32_t x = S.wsum[w]; if ((uint32_t)w < warp) wpre1 += x; all1 += x; }
      const uint32_t s1 = all0 + wpre1 + incl1 - v1;
#pragma unroll
      for (int k = 0; k < 2; ++k) {
        const uint32_t t = tid + k * PT;
        if (t < T) {
          const uint32_t b = S.tlist[t];
          uint32_t run = k ? s1 : s0;
          S.tstart[t] = run;
#pragma unroll
          for (int w = 0; w < PW; ++w) { const uint32_t c = cnt[w * NB + b]; cnt[w * NB + b] = (uint16_t)run; run += c; }
        }
      }
      if (tid == 0) { S.total = all0 + all1; S.tstart[T] = all0 + all1; }
    }
    __syncthreads();
    // ---- one segment entry per touched bucket: {chunk, bucket, start | len << 16} ----
    if (tid == 0) S.seg_base = atomicAdd(&p.st->n_segs, (unsigned long long)T);
    __syncthreads();
    for (uint32_t t = tid; t < T; t += PT) {
      const unsigned long long slot = S.seg_base + t;
      const uint32_t st = S.tstart[t], len = S.tstart[t + 1] - st;
      if (slot < p.seg_cap) p.seg_out[slot] = make_uint4((uint32_t)chunk, S.tlist[t], st | (len << 16), 0);
    }
    // ---- pass B: scatter into shared memory -------------------------------------------
#pragma unroll
    for (int r = 0; r < ROUNDS; ++r) {
      const uint32_t info = dec[r].info, c = info & 3u;
      const uint32_t pos = (uint32_t)(wrec0 + r * 32 + lane);
      if (c >= 1) sorted[row[(info >> 2) & 1023u] + (rk[r] & 0xFFFFu)] = make_uint2(dec[r].k0, pos);
      if (c == 2) sorted[row[(info >> 12) & 1023u] + (rk[r] >> 16)] = make_uint2(dec[r].k1, pos);
    }
    __syncthreads();
    // ---- write the chunk's events; reset the touched counters -----------------------------
    const uint32_t total = S.total;
    uint2* out = p.part_ev + chunk * kChunkCap;
    for (uint32_t j = tid; j < total; j += PT) out[j] = sorted[j];
    for (uint32_t t = tid; t < T * PW; t += PT) cnt[(t % PW) * NB + S.tlist[t / PW]] = 0;
    __syncthreads();
  }

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

cudaError_t launch_partition(const PartParams& p, cudaStream_t s) {
  if (p.n_chunks == 0) return cudaSuccess;
  const size_t smem = ((PW * p.n_buckets * 2 + 15) & ~15u) + (size_t)kChunkCap * sizeof(uint2);
  cudaError_t e = cudaFuncSetAttribute(k_partition, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  const uint32_t grid = (uint32_t)std::min<uint64_t>(p.n_chunks, (uint64_t)sms);
  k_partition<<<grid, PT, smem, s>>>(p);
  return cudaGetLastError();
}

}  // namespace arb
