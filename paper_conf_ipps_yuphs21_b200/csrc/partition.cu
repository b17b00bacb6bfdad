// partition.cu — A1 (ingest/decode) + A3a (stable partition by address bucket).
//
// k_partition  persistent CTAs (one per SM), one 4096-record chunk at a time.
//              The chunk's 16-B records are staged in shared memory by
//              cp.async (the next chunk is fetched while the current one is
//              ranked and written).  Each warp owns 256 consecutive records, in
//              two groups of 128: lane L decodes records L, L+32, L+64, L+96 of
//              the group (access vs control; byte range -> its 1 or 2 8-byte
//              words; word -> address bucket via the bin map), and the
//              group is ranked stably into the warp's per-bucket counters with a
//              single check when all its events hit one bucket (the common case
//              for real access streams).  Events are then written straight to
//              the chunk's slot of the output, grouped by bucket in trace order,
//              and one {chunk, bucket, start, len} entry per touched bucket is
//              appended for the replay.
#include "kcommon.cuh"
#include <algorithm>

namespace arb {

constexpr int PT = kPartThreads;            // 512 threads
constexpr int PW = kPartWarps;              // 16 warps
constexpr int GROUPS = kChunkRecords / PT / 4;  // 2 groups of 128 records per warp
constexpr int RPT = kChunkRecords / PT;     // 8 records per thread

struct PartSmem {
  uint32_t touched[kMaxBuckets / 32];       // bitmap of buckets hit by the chunk
  uint16_t tlist[kMaxBuckets];              // touched buckets, ascending
  uint32_t tstart[kMaxBuckets + 1];         // their first event in the chunk
  uint32_t wsum[PW];
  uint32_t n_touched, total;
  unsigned long long seg_base;
};

__device__ __forceinline__ void cp_async16(void* smem_dst, const void* gsrc) {
  const uint32_t d = (uint32_t)__cvta_generic_to_shared(smem_dst);
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(d), "l"(gsrc) : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
__device__ __forceinline__ void cp_async_wait_all() { asm volatile("cp.async.wait_all;" ::: "memory"); }

// Decoded record: info = cnt | b0 << 2 | b1 << 12 (cnt = tracked words 0..2),
// keys k0/k1 = op << 30 | word offset inside the bucket.
struct Dec { uint32_t info, k0, k1; };

__device__ __forceinline__ uint32_t bucket_key(const PartParams& p, uint64_t rel, uint32_t op, uint32_t& b) {
  const uint32_t m = __ldg(p.bin_map + (uint32_t)(rel >> p.coarse_bits));
  b = m & 1023u;
  return (op << 30) | (((m >> 10) << p.coarse_bits) | ((uint32_t)rel & ((1u << p.coarse_bits) - 1u)));
}

// flags: bit0 control record, bit1 malformed
__device__ __forceinline__ Dec decode(uint4 q, const PartParams& p, uint32_t& ign, uint32_t& flags) {
  Dec d{0, 0, 0};
  const uint32_t op = (q.y >> 16) & 0xFFu;
  if (op >= 4) {
    const bool ctl = op <= 14 && op >= 8 && op != 11;
    flags = ctl ? 1u : 2u;
    return d;
  }
  const uint32_t len = q.z;
  const uint64_t addr = ((uint64_t)(q.y & 0xFFFFu) << 32) | q.x;
  if ((q.w & 0xFFFFu) | (len - 1u > 7u) | (addr + len > (1ull << 48))) { flags = 2u; return d; }
  const uint64_t rel = (addr >> 3) - p.base_word;                 // wraps when below the range
  uint32_t cnt = 0, b0 = 0, b1 = 0;
  if (rel < p.n_words) { d.k0 = bucket_key(p, rel, op, b0); b1 = b0; cnt = 1; } else { ++ign; }
  if ((q.x & 7u) + len > 8u) {                                     // unaligned: a second word (Z4)
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

__device__ __forceinline__ void mark(uint32_t* touched, uint32_t b) { atomicOr(&touched[b >> 5], 1u << (b & 31)); }

// Generic stable rank of one 32-record round (record order, word0 before word1).
__device__ __forceinline__ void rank_round(uint32_t info, uint16_t* row, uint32_t* touched, uint32_t lane,
                                           uint32_t& r0, uint32_t& r1) {
  const uint32_t cnt = info & 3u, b0 = (info >> 2) & 1023u, b1 = (info >> 12) & 1023u;
  r0 = r1 = 0;
  const uint32_t lt = lanemask_lt();
  if (__any_sync(FULL, cnt == 2 && b0 != b1)) {
    // a record crossing a bucket boundary: serial over lanes
    for (uint32_t L = 0; L < 32; ++L) {
      if (lane == L) {
        if (cnt >= 1) { r0 = row[b0]; row[b0] = (uint16_t)(r0 + 1); mark(touched, b0); }
        if (cnt == 2) { r1 = row[b1]; row[b1] = (uint16_t)(r1 + 1); mark(touched, b1); }
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
    mark(touched, b0);
  }
  __syncwarp();
  r0 = base + __popc(grp & lt) + __popc(grp & lt & two);
  r1 = r0 + 1;
}

__global__ void __launch_bounds__(PT, 1) k_partition(PartParams p) {
  extern __shared__ __align__(16) uint8_t smem[];
  const uint32_t NB = p.n_buckets;
  uint4* stage = reinterpret_cast<uint4*>(smem);                            // [kChunkRecords]
  uint16_t* cnt = reinterpret_cast<uint16_t*>(smem + kChunkRecords * sizeof(uint4));   // [PW][NB]
  __shared__ PartSmem S;

  const uint32_t tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const uint32_t lt = lanemask_lt();
  for (uint32_t i = tid; i < PW * NB; i += PT) cnt[i] = 0;
  if (tid < kMaxBuckets / 32) S.touched[tid] = 0;
  uint16_t* row = cnt + warp * NB;
  uint32_t n_acc = 0, n_ign = 0;

  auto fetch = [&](uint64_t c) {
    if (c >= p.n_chunks) return;
    const uint64_t r0 = c * kChunkRecords;
#pragma unroll
    for (int k = 0; k < RPT; ++k) {
      const uint32_t j = tid + k * PT;
      if (r0 + j < p.n) cp_async16(stage + j, p.ev + r0 + j);
    }
    cp_async_commit();
  };

  uint64_t chunk = blockIdx.x;
  fetch(chunk);
  for (; chunk < p.n_chunks; chunk += gridDim.x) {
    const uint64_t rec0 = chunk * kChunkRecords;
    cp_async_wait_all();
    __syncthreads();
    // ---- pass A: decode + rank, 2 groups of 4 x 32 records per warp ---------------
    Dec dec[RPT];
    uint32_t rk[RPT];
#pragma unroll
    for (int g = 0; g < GROUPS; ++g) {
      uint32_t any_flag = 0;
#pragma unroll
      for (int k = 0; k < 4; ++k) {
        const uint32_t j = warp * 256 + g * 128 + k * 32 + lane;      // record inside the chunk
        uint32_t flags = 0;
        dec[g * 4 + k] = Dec{0, 0, 0};
        if (rec0 + j < p.n) dec[g * 4 + k] = decode(stage[j], p, n_ign, flags);
        any_flag |= flags << (2 * k);
        n_acc += dec[g * 4 + k].info & 3u;
      }
      if (__any_sync(FULL, any_flag != 0)) {
        // control / malformed records in the group (rare)
#pragma unroll
        for (int k = 0; k < 4; ++k) {
          const uint32_t j = warp * 256 + g * 128 + k * 32 + lane;
          const uint32_t f = (any_flag >> (2 * k)) & 3u;
          if (f & 2u) atomicMin(&p.st->err_pos, (unsigned long long)(rec0 + j));
          const uint32_t cm = __ballot_sync(FULL, f & 1u);
          if (cm) {
            unsigned long long base = 0;
            if (lane == 0) base = atomicAdd(&p.st->n_ctl, (unsigned long long)__popc(cm));
            base = __shfl_sync(FULL, base, 0);
            if (f & 1u) {
              const uint64_t slot = base + __popc(cm & lt);
              if (slot < p.ctl_cap) {
                const uint4 q = stage[j];
                CtlRec c;
                c.pos = rec0 + j;
                c.w0 = (uint64_t)q.x | ((uint64_t)q.y << 32);
                c.w1 = (uint64_t)q.z | ((uint64_t)q.w << 32);
                p.ctl[slot] = c;
              }
            }
          }
        }
      }
      // rank: one check for the whole group when all its events share a bucket
      uint32_t vm[4], tw[4], any = 0;
#pragma unroll
      for (int k = 0; k < 4; ++k) {
        const uint32_t c = dec[g * 4 + k].info & 3u;
        vm[k] = __ballot_sync(FULL, c != 0);
        tw[k] = __ballot_sync(FULL, c == 2);
        any |= vm[k];
      }
      if (!any) {
#pragma unroll
        for (int k = 0; k < 4; ++k) rk[g * 4 + k] = 0;
        continue;
      }
      uint32_t kl = 0;
      while (!vm[kl]) ++kl;
      const uint32_t lead = __ffs(vm[kl]) - 1;
      uint32_t bsrc = 0;
#pragma unroll
      for (int k = 0; k < 4; ++k) if ((uint32_t)k == kl) bsrc = (dec[g * 4 + k].info >> 2) & 1023u;
      const uint32_t bref = __shfl_sync(FULL, bsrc, lead);
      bool same = true;
#pragma unroll
      for (int k = 0; k < 4; ++k) {
        const uint32_t info = dec[g * 4 + k].info;
        same &= (info & 3u) == 0 || (((info >> 2) & 1023u) == bref && ((info >> 12) & 1023u) == bref);
      }
      if (__all_sync(FULL, same)) {
        const uint32_t base = row[bref];
        uint32_t run = base;
#pragma unroll
        for (int k = 0; k < 4; ++k) {
          const uint32_t r0 = run + __popc(vm[k] & lt) + __popc(tw[k] & lt);
          rk[g * 4 + k] = r0 | ((r0 + 1) << 16);
          run += __popc(vm[k]) + __popc(tw[k]);
        }
        __syncwarp();
        if (lane == 0) { row[bref] = (uint16_t)run; mark(S.touched, bref); }
        __syncwarp();
      } else {
#pragma unroll
        for (int k = 0; k < 4; ++k) {
          uint32_t r0, r1;
          rank_round(dec[g * 4 + k].info, row, S.touched, lane, r0, r1);
          rk[g * 4 + k] = r0 | (r1 << 16);
        }
      }
    }
    __syncthreads();                 // stage consumed; counters complete
    fetch(chunk + gridDim.x);        // next chunk streams in during the rest
    // ---- touched buckets, totals, per-warp offsets ------------------------------------
    if (warp == 0) {
      uint32_t base = 0;
      const uint32_t nw = (NB + 31) / 32;
      for (uint32_t w0 = 0; w0 < nw; w0 += 32) {
        const uint32_t wi = w0 + lane;
        const uint32_t bits = wi < nw ? S.touched[wi] : 0;
        if (wi < nw) S.touched[wi] = 0;
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
    if (T <= 32) {
      // the common case: one warp does the bookkeeping
      if (warp == 0) {
        uint32_t tot = 0, b = 0;
        if (lane < T) {
          b = S.tlist[lane];
#pragma unroll
          for (int w = 0; w < PW; ++w) tot += cnt[w * NB + b];
        }
        uint32_t incl = tot;
#pragma unroll
        for (int d = 1; d < 32; d <<= 1) {
          const uint32_t o = __shfl_up_sync(FULL, incl, d);
          if (lane >= (uint32_t)d) incl += o;
        }
        if (lane < T) {
          uint32_t run = incl - tot;
          S.tstart[lane] = run;
#pragma unroll
          for (int w = 0; w < PW; ++w) { const uint32_t c = cnt[w * NB + b]; cnt[w * NB + b] = (uint16_t)run; run += c; }
        }
        if (lane == 31) { S.tstart[T] = incl; S.total = incl; }
        unsigned long long sb = 0;
        if (lane == 0) sb = atomicAdd(&p.st->n_segs, (unsigned long long)T);
        sb = __shfl_sync(FULL, sb, 0);
        __syncwarp();
        if (lane < T && sb + lane < p.seg_cap)
          p.seg_out[sb + lane] = make_uint4((uint32_t)chunk, b, (incl - tot) | (tot << 16), 0);
      }
    } else {
      // many buckets (scattered chunk): all threads
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
      uint32_t all0 = 0, s0 = 0, s1 = 0, all1 = 0;
      {
        uint32_t v = mytot[0], incl = v;
#pragma unroll
        for (int d = 1; d < 32; d <<= 1) {
          const uint32_t o = __shfl_up_sync(FULL, incl, d);
          if (lane >= (uint32_t)d) incl += o;
        }
        if (lane == 31) S.wsum[warp] = incl;
        __syncthreads();
        uint32_t wpre = 0;
#pragma unroll
        for (int w = 0; w < PW; ++w) { const uint32_t x = S.wsum[w]; if ((uint32_t)w < warp) wpre += x; all0 += x; }
        s0 = wpre + incl - v;
        __syncthreads();
        uint32_t v1 = mytot[1], incl1 = v1;
#pragma unroll
        for (int d = 1; d < 32; d <<= 1) {
          const uint32_t o = __shfl_up_sync(FULL, incl1, d);
          if (lane >= (uint32_t)d) incl1 += o;
        }
        if (lane == 31) S.wsum[warp] = incl1;
        __syncthreads();
        uint32_t wpre1 = 0;
#pragma unroll
        for (int w = 0; w < PW; ++w) { const uint32_t x = S.wsum[w]; if ((uint32_t)w < warp) wpre1 += x; all1 += x; }
        s1 = all0 + wpre1 + incl1 - v1;
      }
      if (tid == 0) S.seg_base = atomicAdd(&p.st->n_segs, (unsigned long long)T);
      __syncthreads();
#pragma unroll
      for (int k = 0; k < 2; ++k) {
        const uint32_t t = tid + k * PT;
        if (t < T) {
          const uint32_t b = S.tlist[t];
          uint32_t run = k ? s1 : s0;
          const uint32_t st = run;
          S.tstart[t] = run;
#pragma unroll
          for (int w = 0; w < PW; ++w) { const uint32_t c = cnt[w * NB + b]; cnt[w * NB + b] = (uint16_t)run; run += c; }
          if (S.seg_base + t < p.seg_cap)
            p.seg_out[S.seg_base + t] = make_uint4((uint32_t)chunk, b, st | ((run - st) << 16), 0);
        }
      }
      if (tid == 0) { S.total = all0 + all1; S.tstart[T] = all0 + all1; }
    }
    __syncthreads();
    // ---- pass B: write the events straight to the chunk's output slot ---------------
    uint2* out = p.part_ev + chunk * kChunkCap;
#pragma unroll
    for (int r = 0; r < RPT; ++r) {
      const uint32_t info = dec[r].info, c = info & 3u;
      const uint32_t j = warp * 256 + (r >> 2) * 128 + (r & 3) * 32 + lane;
      const uint32_t pos = (uint32_t)(rec0 + j);
      if (c >= 1) out[row[(info >> 2) & 1023u] + (rk[r] & 0xFFFFu)] = make_uint2(dec[r].k0, pos);
      if (c == 2) out[row[(info >> 12) & 1023u] + (rk[r] >> 16)] = make_uint2(dec[r].k1, pos);
    }
    __syncthreads();
    for (uint32_t t = tid; t < T * PW; t += PT) cnt[(t % PW) * NB + S.tlist[t / PW]] = 0;
    // the next iteration's wait + barrier orders this reset before the next ranking
  }
  cp_async_wait_all();

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
  const size_t smem = (size_t)kChunkRecords * sizeof(uint4) + (size_t)PW * p.n_buckets * 2;
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
