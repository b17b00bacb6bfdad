// arbgen.cu — C API of the synthetic trace generator (libarbgen.so).
// Host fill (OpenMP), device fill, and order-preserving shard / sample filters.
// Test and bench infrastructure: not part of the replay path.
#include "arbgen.cuh"
#include <cuda_runtime.h>
#include <algorithm>
#include <vector>

using namespace arbgen;

extern "C" {

int arbgen_fill_host(const GenSeg* segs, uint32_t nseg, const GenEntry* ent, const uint64_t* lit,
                     uint64_t start, uint64_t count, uint64_t* out) {
#pragma omp parallel for schedule(static)
  for (long long k = 0; k < (long long)count; ++k)
    gen_record(segs, nseg, ent, lit, start + (uint64_t)k, &out[2 * k], &out[2 * k + 1]);
  return 0;
}

// keep control records and accesses touching a word of the sorted set `words`
// (or the range [word_lo, word_hi) if words == NULL); writes kept records and
// their global indices; returns the count.
uint64_t arbgen_filter_host(const GenSeg* segs, uint32_t nseg, const GenEntry* ent, const uint64_t* lit,
                            uint64_t start, uint64_t count, const uint64_t* words, uint64_t nwords,
                            uint64_t word_lo, uint64_t word_hi, uint64_t* out, uint64_t* gidx,
                            uint64_t cap) {
  const int nt = 64;
  std::vector<std::vector<uint64_t>> part(nt);
  uint64_t per = (count + nt - 1) / nt;
#pragma omp parallel for schedule(dynamic)
  for (int t = 0; t < nt; ++t) {
    uint64_t a = start + t * per, b = std::min(start + count, a + per);
    auto& v = part[t];
    for (uint64_t i = a; i < b; ++i) {
      uint64_t w0, w1;
      gen_record(segs, nseg, ent, lit, i, &w0, &w1);
      uint32_t op = (uint32_t)(w0 >> 48) & 0xFF;
      bool keep = op >= 4;
      if (!keep) {
        uint64_t addr = w0 & ((1ull << 48) - 1), len = w1 & ((1ull << 48) - 1);
        uint64_t x0 = addr >> 3, x1 = (addr + (len ? len : 1) - 1) >> 3;
        for (uint64_t x = x0; x <= x1 && !keep; ++x) {
          if (words) keep = std::binary_search(words, words + nwords, x);
          else keep = x >= word_lo && x < word_hi;
        }
      }
      if (keep) { v.push_back(w0); v.push_back(w1); v.push_back(i); }
    }
  }
  uint64_t n = 0;
  for (auto& v : part)
    for (size_t k = 0; k < v.size(); k += 3) {
      if (n < cap) { out[2 * n] = v[k]; out[2 * n + 1] = v[k + 1]; gidx[n] = v[k + 2]; }
      ++n;
    }
  return n;
}

}  // extern "C"

__global__ void k_gen(const GenSeg* segs, uint32_t nseg, const GenEntry* ent, const uint64_t* lit,
                      uint64_t start, uint64_t count, uint4* out) {
  for (uint64_t k = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; k < count;
       k += (uint64_t)gridDim.x * blockDim.x) {
    uint64_t w0, w1;
    gen_record(segs, nseg, ent, lit, start + k, &w0, &w1);
    out[k] = make_uint4((uint32_t)w0, (uint32_t)(w0 >> 32), (uint32_t)w1, (uint32_t)(w1 >> 32));
  }
}

constexpr int kFT = 256, kFI = 16, kFTile = kFT * kFI;

__device__ __forceinline__ bool keep_rec(uint4 r, uint64_t lo, uint64_t hi) {
  uint64_t w0 = (uint64_t)r.x | ((uint64_t)r.y << 32), w1 = (uint64_t)r.z | ((uint64_t)r.w << 32);
  uint32_t op = (uint32_t)(w0 >> 48) & 0xFF;
  if (op >= 4) return true;
  uint64_t addr = w0 & ((1ull << 48) - 1), len = w1 & ((1ull << 48) - 1);
  uint64_t x0 = addr >> 3, x1 = (addr + (len ? len : 1) - 1) >> 3;
  return x1 >= lo && x0 < hi;
}

__global__ void k_filter_count(const uint4* in, uint64_t n, uint64_t lo, uint64_t hi, uint32_t* blk) {
  __shared__ uint32_t red[kFT / 32];
  uint32_t c = 0;
  uint64_t base = blockIdx.x * (uint64_t)kFTile;
  for (int j = 0; j < kFI; ++j) {
    uint64_t i = base + (uint64_t)threadIdx.x * kFI + j;
    if (i < n) c += keep_rec(in[i], lo, hi);
  }
  for (int d = 16; d; d >>= 1) c += __shfl_xor_sync(0xFFFFFFFFu, c, d);
  if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = c;
  __syncthreads();
  if (threadIdx.x == 0) {
    uint32_t t = 0;
    for (int w = 0; w < kFT / 32; ++w) t += red[w];
    blk[blockIdx.x] = t;
  }
}

__global__ void k_scan64(const uint32_t* a, uint64_t* out, uint64_t n) {  // single CTA exclusive scan
  __shared__ uint64_t ws[32];
  __shared__ uint64_t carry;
  if (threadIdx.x == 0) carry = 0;
  __syncthreads();
  const uint32_t lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  for (uint64_t base = 0; base < n; base += 1024) {
    uint64_t i = base + threadIdx.x;
    uint64_t v = i < n ? a[i] : 0, incl = v;
    for (int d = 1; d < 32; d <<= 1) {
      uint64_t o = __shfl_up_sync(0xFFFFFFFFu, incl, d);
      if (lane >= (uint32_t)d) incl += o;
    }
    if (lane == 31) ws[warp] = incl;
    __syncthreads();
    if (warp == 0) {
      uint64_t x = ws[lane], xi = x;
      for (int d = 1; d < 32; d <<= 1) {
        uint64_t o = __shfl_up_sync(0xFFFFFFFFu, xi, d);
        if (lane >= (uint32_t)d) xi += o;
      }
      ws[lane] = xi - x;
    }
    __syncthreads();
    uint64_t c = carry;
    if (i <= n) out[i] = c + ws[warp] + incl - v;
    __syncthreads();
    if (threadIdx.x == 1023) carry = c + ws[warp] + incl;
    __syncthreads();
  }
  if (threadIdx.x == 0 && n % 1024 == 0) out[n] = carry;
}

__global__ void k_filter_write(const uint4* in, uint64_t n, uint64_t lo, uint64_t hi, const uint64_t* off,
                               uint64_t first_index, uint4* out, uint64_t* gidx) {
  __shared__ uint32_t ws[kFT / 32];
  const uint32_t lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  uint64_t base = blockIdx.x * (uint64_t)kFTile;
  bool kp[kFI];
  uint32_t c = 0;
  for (int j = 0; j < kFI; ++j) {
    uint64_t i = base + (uint64_t)threadIdx.x * kFI + j;
    kp[j] = i < n && keep_rec(in[i], lo, hi);
    c += kp[j];
  }
  uint32_t incl = c;
  for (int d = 1; d < 32; d <<= 1) {
    uint32_t o = __shfl_up_sync(0xFFFFFFFFu, incl, d);
    if (lane >= (uint32_t)d) incl += o;
  }
  if (lane == 31) ws[warp] = incl;
  __syncthreads();
  uint32_t wpre = 0;
  for (uint32_t w = 0; w < warp; ++w) wpre += ws[w];
  uint64_t o = off[blockIdx.x] + wpre + incl - c;
  for (int j = 0; j < kFI; ++j) {
    if (!kp[j]) continue;
    uint64_t i = base + (uint64_t)threadIdx.x * kFI + j;
    out[o] = in[i];
    if (gidx) gidx[o] = first_index + i;
    ++o;
  }
}

extern "C" {

int arbgen_fill_device(const GenSeg* segs, uint32_t nseg, const GenEntry* ent, const uint64_t* lit,
                       uint64_t start, uint64_t count, void* out, void* stream) {
  if (!count) return 0;
  uint64_t g = (count + 255) / 256;
  k_gen<<<(unsigned)std::min<uint64_t>(g, 148 * 32), 256, 0, (cudaStream_t)stream>>>(
      segs, nseg, ent, lit, start, count, (uint4*)out);
  return (int)cudaGetLastError();
}

// order-preserving compaction of the records touching words [lo, hi) plus every
// control record; scratch must hold ceil(n/4096)*12+16 bytes.  *n_out (host) is set.
int arbgen_filter_device(const void* in, uint64_t n, uint64_t lo, uint64_t hi, uint64_t first_index,
                         void* out, uint64_t* gidx, void* scratch, uint64_t* n_out, void* stream) {
  cudaStream_t s = (cudaStream_t)stream;
  uint64_t nb = (n + kFTile - 1) / kFTile;
  if (!nb) { *n_out = 0; return 0; }
  uint32_t* blk = (uint32_t*)scratch;
  uint64_t* off = (uint64_t*)((char*)scratch + ((nb * 4 + 15) & ~15ull));
  k_filter_count<<<(unsigned)nb, kFT, 0, s>>>((const uint4*)in, n, lo, hi, blk);
  k_scan64<<<1, 1024, 0, s>>>(blk, off, nb);
  k_filter_write<<<(unsigned)nb, kFT, 0, s>>>((const uint4*)in, n, lo, hi, off, first_index, (uint4*)out, gidx);
  uint64_t tot = 0;
  cudaMemcpyAsync(&tot, off + nb, 8, cudaMemcpyDeviceToHost, s);
  cudaError_t e = cudaStreamSynchronize(s);
  *n_out = tot;
  return (int)e;
}

}  // extern "C"
