// partition.cu — A1 (ingest/decode) + A3a (stable partition by address bucket).
//
// k_sample     sampled histogram of access addresses over coarse bins; the host
//              cuts contiguous, event-balanced address buckets from it.
// k_partition  one CTA per chunk of 4096 records: 128-bit loads of the 16-B
//              records, split access vs control records, map each access's
//              byte range to its 8-byte words (1 or 2 words), and
//              stable-partition the word-events by bucket into the chunk's slot
//              of the output (chunk-major) plus one row of the offset table.
//              Each record is decoded and ranked once; ranks stay in registers.
#include "kcommon.cuh"

namespace arb {

// Sampled histogram of access addresses over coarse bins (bucket balancing).
__global__ void k_sample(SampleParams p, uint64_t n_samples) {
  for (uint64_t k = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; k < n_samples;
       k += (uint64_t)gridDim.x * blockDim.x) {
    uint4 r = ld_stream(p.ev + k * p.stride);
    uint64_t w0 = (uint64_t)r.x | ((uint64_t)r.y << 32);
    if (((w0 >> 48) & 0xFFu) >= 4) continue;
    uint64_t x = (w0 & kMask48) >> 3;
    uint64_t rel = x - p.base_word;
    if (x >= p.base_word && rel < p.n_words) atomicAdd(&p.hist[rel >> p.coarse_bits], 1u);
  }
}

cudaError_t launch_sample(const SampleParams& p, uint64_t n_samples, cudaStream_t s) {
  if (!n_samples) return cudaSuccess;
  uint64_t g = (n_samples + 255) / 256;
  k_sample<<<(unsigned)(g > 148 * 16 ? 148 * 16 : g), 256, 0, s>>>(p, n_samples);
  return cudaGetLastError();
}

// ---- bucket cutting on the device (single CTA) ------------------------------
// Buckets start at bin 0, at every bin whose exclusive sample prefix crosses a
// multiple of `target` (quantile cuts: a heavy bin gets a bucket of its own),
// and at every multiple of 2^30 words (span cap).  Writes bin_map (see
// arb_internal.h), bucket_start [nb + 1], bucket weights [nb] and nb.
constexpr int kCutThreads = 1024;

__device__ uint32_t cta_excl_scan(uint32_t v, uint32_t* ws, uint32_t* total) {
  const uint32_t lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  uint32_t incl = v;
#pragma unroll
  for (int d = 1; d < 32; d <<= 1) {
    const uint32_t o = __shfl_up_sync(FULL, incl, d);
    if (lane >= (uint32_t)d) incl += o;
  }
  __syncthreads();
  if (lane == 31) ws[warp] = incl;
  __syncthreads();
  if (warp == 0) {
    const uint32_t x = ws[lane];
    uint32_t xi = x;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
      const uint32_t o = __shfl_up_sync(FULL, xi, d);
      if (lane >= (uint32_t)d) xi += o;
    }
    ws[lane] = xi - x;
    if (lane == 31) ws[32] = xi;
  }
  __syncthreads();
  *total = ws[32];
  return ws[warp] + incl - v;
}

__global__ void __launch_bounds__(kCutThreads) k_cut(uint32_t* hist_map, uint32_t n_bins, uint32_t coarse_bits,
                                                      uint64_t n_words, uint32_t max_buckets,
                                                      uint64_t* bucket_start, uint32_t* weight,
                                                      uint32_t* first_bin, uint32_t* nb_out) {
  __shared__ uint32_t ws[33];
  const uint32_t per = (n_bins + kCutThreads - 1) / kCutThreads;
  const uint32_t i0 = min(n_bins, threadIdx.x * per), i1 = min(n_bins, i0 + per);
  uint32_t s = 0;
  for (uint32_t i = i0; i < i1; ++i) s += hist_map[i];
  uint32_t total;
  const uint32_t pre = cta_excl_scan(s, ws, &total);
  const uint32_t levels = max(1u, max_buckets - 124);            // <= levels quantile cuts (+ span cuts <= 1024)
  const uint32_t target = max(1u, (total + levels - 1) / levels);
  const uint64_t span64 = (1ull << 30) >> coarse_bits;
  const uint32_t span_bins = span64 == 0 ? 1u : (span64 > 0xFFFFFFFFull ? 0xFFFFFFFFu : (uint32_t)span64);
  // a bucket starts at bin i when the quantile level of its exclusive prefix
  // differs from the previous bin's, or at a span boundary
  const uint32_t lev0 = (i0 == 0 || i0 >= n_bins) ? 0xFFFFFFFFu : (pre - hist_map[i0 - 1]) / target;
  uint32_t nflag = 0;
  {
    uint32_t p = pre, prev = lev0;
    for (uint32_t i = i0; i < i1; ++i) {
      const uint32_t lev = p / target;
      nflag += (i == 0 || i % span_bins == 0 || lev != prev);
      prev = lev;
      p += hist_map[i];
    }
  }
  uint32_t nb;
  uint32_t b = cta_excl_scan(nflag, ws, &nb);
  {
    uint32_t p = pre, prev = lev0;
    for (uint32_t i = i0; i < i1; ++i) {
      const uint32_t lev = p / target;
      if (i == 0 || i % span_bins == 0 || lev != prev) { first_bin[b] = i; weight[b] = p; ++b; }
      prev = lev;
      p += hist_map[i];
    }
  }
  __syncthreads();
  for (uint32_t k = threadIdx.x; k < nb; k += kCutThreads) bucket_start[k] = (uint64_t)first_bin[k] << coarse_bits;
  __syncthreads();
  uint32_t wk[4];   // weights = differences of the prefixes at the starts (nb <= 4096)
#pragma unroll
  for (int j = 0; j < 4; ++j) {
    const uint32_t k = threadIdx.x + j * kCutThreads;
    wk[j] = k < nb ? (k + 1 < nb ? weight[k + 1] : total) - weight[k] : 0;
  }
  __syncthreads();
#pragma unroll
  for (int j = 0; j < 4; ++j) {
    const uint32_t k = threadIdx.x + j * kCutThreads;
    if (k < nb) weight[k] = wk[j];
  }
  {
    // bin map: walk this thread's bins again; b = number of bucket starts before i0
    uint32_t p = pre, prev = lev0;
    int cur = (int)(b - nflag) - 1;                         // bucket open at i0 - 1 (-1: none)
    uint32_t first = (cur >= 0 && i0 < i1) ? first_bin[cur] : 0;
    for (uint32_t i = i0; i < i1; ++i) {
      const uint32_t lev = p / target;
      if (i == 0 || i % span_bins == 0 || lev != prev) { ++cur; first = i; }
      prev = lev;
      p += hist_map[i];
      hist_map[i] = cur | ((i - first) << 10);
    }
  }
  if (threadIdx.x == 0) { bucket_start[nb] = n_words; *nb_out = nb; }
}

cudaError_t launch_cut(uint32_t* hist_map, uint32_t n_bins, uint32_t coarse_bits, uint64_t n_words,
                       uint32_t max_buckets, uint64_t* bucket_start, uint32_t* weight, uint32_t* first_bin,
                       uint32_t* nb_out, cudaStream_t s) {
  k_cut<<<1, kCutThreads, 0, s>>>(hist_map, n_bins, coarse_bits, n_words, max_buckets, bucket_start, weight,
                                  first_bin, nb_out);
  return cudaGetLastError();
}

// Decoded access record, packed: info = cnt | b0 << 2 | b1 << 12, keys k0/k1 =
// op << 30 | word offset inside the bucket.  cnt = tracked words (0..2).
struct Dec { uint32_t info, k0, k1; };

__device__ __forceinline__ Dec decode(uint4 r, bool valid, const PartParams& p, uint32_t& ign, bool& ctl,
                                      bool& bad) {
  Dec d{0, 0, 0};
  ctl = false; bad = false;
  if (!valid) return d;
  const uint64_t w0 = (uint64_t)r.x | ((uint64_t)r.y << 32);
  const uint32_t op = (r.y >> 16) & 0xFFu;
  if (op < 4) {
    const uint64_t addr = w0 & kMask48;
    const uint32_t len = r.z;
    if (r.w & 0xFFFFu || len < 1 || len > 8 || addr + len > (1ull << 48)) { bad = true; return d; }
    const uint64_t x0 = addr >> 3;
    const uint32_t nw = (uint32_t)(((addr + len - 1) >> 3) - x0) + 1;   // 1 or 2 words (Z4)
    const uint32_t cmask = (1u << p.coarse_bits) - 1u;
    uint32_t cnt = 0, b0 = 0, b1 = 0;
    for (uint32_t k = 0; k < nw; ++k) {
      const uint64_t rel = x0 + k - p.base_word;
      if (x0 + k >= p.base_word && rel < p.n_words) {
        const uint32_t m = __ldg(p.bin_map + (rel >> p.coarse_bits));
        const uint32_t key = (op << 30) | (((m >> 10) << p.coarse_bits) | ((uint32_t)rel & cmask));
        if (cnt == 0) { b0 = m & 1023u; b1 = b0; d.k0 = key; } else { b1 = m & 1023u; d.k1 = key; }
        ++cnt;
      } else {
        ++ign;
      }
    }
    d.info = cnt | (b0 << 2) | (b1 << 12);
  } else if (op == OP_MAP_ENTER || op == OP_MAP_EXIT || op == OP_UPDATE ||
             op == OP_TASK_BEGIN || op == OP_TASK_END || op == OP_SYNC) {
    ctl = true;
  } else {
    bad = true;
  }
  return d;
}

// Stable rank of this round's events inside the warp's per-bucket counters
// `row` (record order, word0 before word1).  r0/r1: rank of word 0/1 inside
// its bucket's run of this warp.
__device__ __forceinline__ void rank_round(uint32_t info, uint16_t* row, uint32_t lane, uint32_t& r0,
                                           uint32_t& r1) {
  const uint32_t cnt = info & 3u, b0 = (info >> 2) & 1023u, b1 = (info >> 12) & 1023u;
  r0 = r1 = 0;
  const bool straddle = cnt == 2 && b0 != b1;
  const uint32_t vmask = __ballot_sync(FULL, cnt != 0);
  if (!vmask) return;
  if (__any_sync(FULL, straddle)) {
    // rare: a record crossing a bucket boundary somewhere in the warp; serial
    for (uint32_t L = 0; L < 32; ++L) {
      if (lane == L) {
        if (cnt >= 1) { r0 = row[b0]; row[b0] = (uint16_t)(r0 + 1); }
        if (cnt == 2) { r1 = row[b1]; row[b1] = (uint16_t)(r1 + 1); }
      }
      __syncwarp();
    }
    return;
  }
  const uint32_t two = __ballot_sync(FULL, cnt == 2);
  const uint32_t lt = lanemask_lt();
  const uint32_t lead = __ffs(vmask) - 1;
  const uint32_t bref = __shfl_sync(FULL, b0, lead);
  uint32_t grp;
  if (__all_sync(FULL, cnt == 0 || b0 == bref)) grp = vmask;      // whole warp in one bucket
  else grp = __match_any_sync(FULL, cnt ? b0 : 0xFFFFFFFFu);
  const uint32_t before = __popc(grp & lt) + __popc(grp & lt & two);
  const uint32_t total = __popc(grp) + __popc(grp & two);
  uint32_t base = 0;
  if (cnt) base = row[b0];
  __syncwarp();
  if (cnt && lane == 31u - __clz(grp)) row[b0] = (uint16_t)(base + total);
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
  constexpr int kRounds = kChunkRecords / kPartThreads;  // 8 rounds of 32 records per warp
  const uint64_t wrec0 = chunk * kChunkRecords + (uint64_t)warp * (kChunkRecords / kPartWarps);

  for (uint32_t i = tid; i < kPartWarps * NB; i += kPartThreads) hist[i] = 0;
  __syncthreads();

  uint16_t* row = hist + warp * NB;
  Dec dec[kRounds];
  uint32_t rk[kRounds];
  uint32_t n_acc = 0, n_ign = 0;
  {
    uint4 rec[kRounds];
#pragma unroll
    for (int r = 0; r < kRounds; ++r) {
      const uint64_t i = wrec0 + (uint64_t)r * 32 + lane;
      rec[r] = i < p.n ? ld_stream(p.ev + i) : make_uint4(0, 0, 0, 0);
    }
#pragma unroll
    for (int r = 0; r < kRounds; ++r) {
      const uint64_t i = wrec0 + (uint64_t)r * 32 + lane;
      bool ctl, bad;
      dec[r] = decode(rec[r], i < p.n, p, n_ign, ctl, bad);
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
      rank_round(dec[r].info, row, lane, r0, r1);
      rk[r] = r0 | (r1 << 16);
    }
  }
  __syncthreads();

  // ---- offsets: per bucket over warps, then over buckets ------------------
  // thread t owns buckets 2t and 2t+1
  uint32_t bt[2] = {0, 0};
#pragma unroll
  for (int k = 0; k < 2; ++k) {
    const uint32_t b = 2 * tid + k;
    if (b < NB) {
      uint32_t s = 0;
      for (int w = 0; w < kPartWarps; ++w) {
        const uint32_t c = hist[w * NB + b];
        hist[w * NB + b] = (uint16_t)s;
        s += c;
      }
      bt[k] = s;
    }
  }
  const uint32_t mine = bt[0] + bt[1];
  uint32_t incl = mine;
#pragma unroll
  for (int d = 1; d < 32; d <<= 1) {
    const uint32_t o = __shfl_up_sync(FULL, incl, d);
    if (lane >= (uint32_t)d) incl += o;
  }
  if (lane == 31) s_wsum[warp] = incl;
  __syncthreads();
  if (warp == 0) {
    const uint32_t v = lane < kPartWarps ? s_wsum[lane] : 0;
    uint32_t vi = v;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
      const uint32_t o = __shfl_up_sync(FULL, vi, d);
      if (lane >= (uint32_t)d) vi += o;
    }
    if (lane < kPartWarps) s_wsum[lane] = vi - v;
    if (lane == kPartWarps - 1) s_total = vi;
  }
  __syncthreads();
  const uint32_t excl = s_wsum[warp] + incl - mine;
  const uint32_t bb[2] = {excl, excl + bt[0]};
#pragma unroll
  for (int k = 0; k < 2; ++k) {
    const uint32_t b = 2 * tid + k;
    if (b < NB) {
      for (int w = 0; w < kPartWarps; ++w) hist[w * NB + b] = (uint16_t)(hist[w * NB + b] + bb[k]);
      p.part_off[(uint64_t)b * p.n_chunks + chunk] = (uint16_t)bb[k];
    }
  }
  if (tid == 0) p.part_off[(uint64_t)NB * p.n_chunks + chunk] = (uint16_t)s_total;
  __syncthreads();

  // ---- scatter into shared memory, then one coalesced write -----------------
#pragma unroll
  for (int r = 0; r < kRounds; ++r) {
    const uint32_t info = dec[r].info, cnt = info & 3u;
    const uint32_t pos = (uint32_t)(wrec0 + (uint64_t)r * 32 + lane);
    if (cnt >= 1) sorted[hist[warp * NB + ((info >> 2) & 1023u)] + (rk[r] & 0xFFFFu)] = make_uint2(dec[r].k0, pos);
    if (cnt == 2) sorted[hist[warp * NB + ((info >> 12) & 1023u)] + (rk[r] >> 16)] = make_uint2(dec[r].k1, pos);
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

cudaError_t launch_partition(const PartParams& p, cudaStream_t s) {
  if (p.n_chunks == 0) return cudaSuccess;
  const size_t smem = ((kPartWarps * p.n_buckets * 2 + 15) & ~15u) + (size_t)kChunkCap * sizeof(uint2);
  cudaError_t e = cudaFuncSetAttribute(k_partition, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  k_partition<<<p.n_chunks, kPartThreads, smem, s>>>(p);
  return cudaGetLastError();
}

}  // namespace arb
