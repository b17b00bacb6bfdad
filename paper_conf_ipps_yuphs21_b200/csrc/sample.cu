// sample.cu — address sampling and device-side bucket cutting (bucket balancing).
//
// k_sample   sampled histogram of access addresses over coarse bins.
// k_cut_*    contiguous, event-balanced address buckets: a bucket starts at
//            bin 0, at every bin whose exclusive sample prefix enters a new
//            quantile level or is at least 4 levels heavy (a heavy bin gets a
//            bucket of its own) and at every
//            2^30-word span boundary.  The histogram is rewritten in place as
//            the bin map (bucket | offset-in-bins << kBucketBits, see arb_internal.h).
//            Tiles of 1024 bins are handled by separate CTAs; two one-CTA
//            scans carry the prefixes between tiles.
#include "kcommon.cuh"

namespace arb {

__global__ void k_sample(SampleParams p, uint64_t n_samples) {
  for (uint64_t k = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; k < n_samples;
       k += (uint64_t)gridDim.x * blockDim.x) {
    // jittered sampling: record k * stride + (hash(k) mod stride) — a fixed stride
    // aliases with periodic loop bodies (e.g. one of a stencil's 8 accesses)
    uint64_t z = k * 0x9E3779B97F4A7C15ull;
    z = (z ^ (z >> 29)) * 0xBF58476D1CE4E5B9ull;
    z ^= z >> 32;
    const uint64_t idx = k * p.stride + (p.stride > 1 ? z % p.stride : 0);
    if (idx >= p.n) continue;
    const uint4 r = ld_stream(p.ev + idx);
    const uint64_t w0 = (uint64_t)r.x | ((uint64_t)r.y << 32);
    if (((w0 >> 48) & 0xFFu) >= 4) continue;
    const uint64_t x = (w0 & kMask48) >> 3;
    const uint64_t rel = x - p.base_word;
    if (x >= p.base_word && rel < p.n_words) atomicAdd(&p.hist[rel >> p.coarse_bits], 1u);
  }
}

cudaError_t launch_sample(const SampleParams& p, uint64_t n_samples, cudaStream_t s) {
  if (!n_samples) return cudaSuccess;
  const uint64_t g = (n_samples + 255) / 256;
  k_sample<<<(unsigned)(g > 148 * 16 ? 148 * 16 : g), 256, 0, s>>>(p, n_samples);
  return cudaGetLastError();
}

constexpr int kT = 1024;   // bins per tile = threads per CTA

// exclusive block scan of one value per thread (1024 threads)
__device__ __forceinline__ uint32_t scan1024(uint32_t v, uint32_t* ws, uint32_t* total) {
  const uint32_t lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  uint32_t incl = v;
#pragma unroll
  for (int d = 1; d < 32; d <<= 1) {
    const uint32_t o = __shfl_up_sync(FULL, incl, d);
    if (lane >= (uint32_t)d) incl += o;
  }
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
  const uint32_t r = ws[warp] + incl - v;
  __syncthreads();
  return r;
}

struct CutArgs {
  uint32_t* hist_map; uint32_t n_bins; uint32_t coarse_bits; uint64_t n_words; uint32_t max_buckets;
  uint64_t* bucket_start; uint32_t* weight; uint32_t* first_bin; uint32_t* nb_out;
  uint32_t* tile_a; uint32_t* tile_b;          // per-tile scratch (sums / flag counts, then prefixes)
  uint32_t* misc;                              // [0] total, [1] target, [2] span bins
  uint32_t* bucket_of;                         // per bin bucket index
};

__global__ void __launch_bounds__(kT) k_cut_sum(CutArgs a) {
  __shared__ uint32_t ws[33];
  const uint32_t i = blockIdx.x * kT + threadIdx.x;
  uint32_t tot;
  scan1024(i < a.n_bins ? a.hist_map[i] : 0, ws, &tot);
  if (threadIdx.x == 0) a.tile_a[blockIdx.x] = tot;
}

// one CTA: exclusive scan of n per-tile values in place; optional totals
__global__ void __launch_bounds__(kT) k_cut_scan(uint32_t* v, uint32_t n, uint32_t* total_out, CutArgs a,
                                                 int first) {
  __shared__ uint32_t ws[33];
  uint32_t carry = 0;
  for (uint32_t base = 0; base < n; base += kT) {
    const uint32_t i = base + threadIdx.x;
    uint32_t tot;
    const uint32_t ex = scan1024(i < n ? v[i] : 0, ws, &tot);
    if (i < n) v[i] = carry + ex;
    carry += tot;
  }
  if (threadIdx.x == 0) {
    *total_out = carry;
    if (first) {   // quantile target and span cap
      // leave room for the span cuts (n_words / 2^30 + 1 of them, <= 257)
      const uint32_t spans = (uint32_t)(a.n_words >> kMaxBucketSpanBits) + 1;
      // heavy-bin buckets (<= levels / 4 of them) need ids as well
      const uint32_t levels = max(1u, (a.max_buckets - spans - 1) * 4 / 5);
      a.misc[1] = max(1u, (carry + levels - 1) / levels);
      const uint64_t span64 = (1ull << kMaxBucketSpanBits) >> a.coarse_bits;
      a.misc[2] = span64 == 0 ? 1u : (span64 > 0xFFFFFFFFull ? 0xFFFFFFFFu : (uint32_t)span64);
    }
  }
}

// flags of the bins of one tile (needs the tile's exclusive sample prefix)
__device__ __forceinline__ bool cut_flag(const CutArgs& a, uint32_t i, uint32_t p, uint32_t h, uint32_t h_prev_known,
                                         uint32_t* levs) {
  const uint32_t target = a.misc[1], span = a.misc[2];
  const uint32_t lev = p / target;
  levs[threadIdx.x] = lev;
  __syncthreads();
  uint32_t prev;
  if (threadIdx.x > 0) prev = levs[threadIdx.x - 1];
  else prev = i == 0 ? 0xFFFFFFFFu : (p - h_prev_known) / target;   // level of the previous tile's last bin
  __syncthreads();
  // a very heavy bin (>= 4 levels: a hot word's bin) also starts a bucket of its
  // own, so the hot bucket spans one bin (the next bin is at a new level)
  return i < a.n_bins && (i == 0 || i % span == 0 || lev != prev || h >= 4 * target);
}

__global__ void __launch_bounds__(kT) k_cut_flags(CutArgs a) {
  __shared__ uint32_t ws[33];
  __shared__ uint32_t levs[kT];
  const uint32_t i = blockIdx.x * kT + threadIdx.x;
  const uint32_t h = i < a.n_bins ? a.hist_map[i] : 0;
  uint32_t tot;
  const uint32_t p = a.tile_a[blockIdx.x] + scan1024(h, ws, &tot);
  const uint32_t hprev = (i > 0 && threadIdx.x == 0) ? a.hist_map[i - 1] : 0;
  const bool f = cut_flag(a, i, p, h, hprev, levs);
  uint32_t nf;
  scan1024(f ? 1u : 0u, ws, &nf);
  if (threadIdx.x == 0) a.tile_b[blockIdx.x] = nf;
}

__global__ void __launch_bounds__(kT) k_cut_write(CutArgs a) {
  __shared__ uint32_t ws[33];
  __shared__ uint32_t levs[kT];
  const uint32_t i = blockIdx.x * kT + threadIdx.x;
  const uint32_t h = i < a.n_bins ? a.hist_map[i] : 0;
  uint32_t tot;
  const uint32_t p = a.tile_a[blockIdx.x] + scan1024(h, ws, &tot);
  const uint32_t hprev = (i > 0 && threadIdx.x == 0) ? a.hist_map[i - 1] : 0;
  const bool f = cut_flag(a, i, p, h, hprev, levs);
  uint32_t nf;
  const uint32_t b = a.tile_b[blockIdx.x] + scan1024(f ? 1u : 0u, ws, &nf);
  if (f) { a.first_bin[b] = i; a.weight[b] = p; }
  if (i < a.n_bins) a.bucket_of[i] = f ? b : b - 1;
}

__global__ void k_cut_map(CutArgs a) {
  const uint32_t nb = *a.nb_out;
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < a.n_bins; i += gridDim.x * blockDim.x) {
    const uint32_t b = a.bucket_of[i];
    a.hist_map[i] = b | ((i - a.first_bin[b]) << kBucketBits);
  }
  for (uint32_t b = blockIdx.x * blockDim.x + threadIdx.x; b <= nb; b += gridDim.x * blockDim.x) {
    if (b < nb) a.bucket_start[b] = (uint64_t)a.first_bin[b] << a.coarse_bits;
    else a.bucket_start[nb] = a.n_words;
  }
}

__global__ void k_cut_weights(CutArgs a) {   // one CTA: prefix differences
  const uint32_t nb = *a.nb_out, total = a.misc[0];
  uint32_t w[4];
#pragma unroll
  for (int j = 0; j < 4; ++j) {
    const uint32_t b = threadIdx.x + j * blockDim.x;
    w[j] = b < nb ? (b + 1 < nb ? a.weight[b + 1] : total) - a.weight[b] : 0;
  }
  __syncthreads();
#pragma unroll
  for (int j = 0; j < 4; ++j) {
    const uint32_t b = threadIdx.x + j * blockDim.x;
    if (b < nb) a.weight[b] = w[j];
  }
}

cudaError_t launch_cut(uint32_t* hist_map, uint32_t n_bins, uint32_t coarse_bits, uint64_t n_words,
                       uint32_t max_buckets, uint64_t* bucket_start, uint32_t* weight, uint32_t* first_bin,
                       uint32_t* nb_out, uint32_t* scratch, cudaStream_t s, int* launches) {
  const uint32_t nt = (n_bins + kT - 1) / kT;
  CutArgs a{hist_map, n_bins, coarse_bits, n_words, max_buckets, bucket_start, weight, first_bin, nb_out,
            scratch, scratch + nt, scratch + 2 * nt, scratch + 2 * nt + 4};
  k_cut_sum<<<nt, kT, 0, s>>>(a);
  k_cut_scan<<<1, kT, 0, s>>>(a.tile_a, nt, a.misc, a, 1);
  k_cut_flags<<<nt, kT, 0, s>>>(a);
  k_cut_scan<<<1, kT, 0, s>>>(a.tile_b, nt, nb_out, a, 0);
  k_cut_write<<<nt, kT, 0, s>>>(a);
  k_cut_map<<<148, 1024, 0, s>>>(a);
  k_cut_weights<<<1, kT, 0, s>>>(a);
  *launches += 7;
  return cudaGetLastError();
}

}  // namespace arb
