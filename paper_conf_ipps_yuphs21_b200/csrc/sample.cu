// sample.cu — address sampling and device-side bucket cutting (bucket balancing).
//
// k_sample  sampled histogram of access addresses over coarse bins.
// k_cut     single CTA: contiguous, event-balanced address buckets (quantile
//           cuts of the sampled histogram + span cuts), bin map in place.
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

}  // namespace arb
