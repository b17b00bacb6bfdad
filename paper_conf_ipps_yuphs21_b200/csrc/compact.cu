// compact.cu — canonical report order (word, record, kind) + unique:
// LSD radix sort of the report candidates, then stream compaction.
#include "kcommon.cuh"

namespace arb {

constexpr int kRsThreads = 512, kRsItems = 8, kRsTile = kRsThreads * kRsItems;

struct RsPass { int field; int shift; int bits; uint32_t div = 1; };   // digit of field / div
constexpr int kRsMaxBits = 11;                    // digits of up to 11 bits (2048 bins)
constexpr int kRsBins = 1 << kRsMaxBits;
// digit fields (64-bit): uint4 report candidates {x, y = word, z = record, w = kind}:
// 0: kind, 1: record, 5: record << 3 | kind, 6: word, 7: kind << 30 | record (records < 2^30);
// uint2 {0: x, 1: y} (w = report kind, 1..4: 3 bits)
constexpr int kKindBits = 3;
__device__ __forceinline__ uint64_t rs_field(uint4 c, int f) {
  return f == 0 ? c.w : f == 1 ? c.z : f == 5 ? ((uint64_t)c.z << kKindBits) | c.w
       : f == 6 ? ((uint64_t)c.y << 32) | c.x : ((uint64_t)c.w << 30) | c.z;
}
// uint2 {0: x, 1: y, 2: segment entry chunk (x bits 0-20 | y bit 31 << 21)}
__device__ __forceinline__ uint64_t rs_field(uint2 c, int f) {
  return f == 0 ? c.x : f == 1 ? c.y : (c.x & ((1u << kSegChunkBits) - 1u)) | ((c.y >> 31) << kSegChunkBits);
}
template <class E>
__device__ __forceinline__ uint32_t rs_digit(E c, RsPass ps) {
  uint64_t v = rs_field(c, ps.field);
  if (ps.div > 1) v /= ps.div;
  return (uint32_t)(v >> ps.shift) & ((1u << ps.bits) - 1u);
}

// A block owns `sub` consecutive tiles of kRsTile elements (fewer, larger blocks
// for large arrays: the digit-count matrix and its scan shrink by `sub`).
template <class E>
__global__ void __launch_bounds__(kRsThreads) k_rs_hist(const E* in, uint64_t n, RsPass ps, uint32_t* cnt,
                                                        uint32_t nblk, uint32_t sub) {
  __shared__ uint32_t h[kRsBins];
  const int nd = 1 << ps.bits;
  for (int i = threadIdx.x; i < nd; i += kRsThreads) h[i] = 0;
  __syncthreads();
  const uint64_t base = (uint64_t)blockIdx.x * kRsTile * sub;
  for (uint32_t j = 0; j < kRsItems * sub; ++j) {
    uint64_t i = base + (uint64_t)j * kRsThreads + threadIdx.x;
    if (i < n) atomicAdd(&h[rs_digit(in[i], ps)], 1u);
  }
  __syncthreads();
  for (int d = threadIdx.x; d < nd; d += kRsThreads) cnt[(uint64_t)d * nblk + blockIdx.x] = h[d];
}

// ---- exclusive scan of u32 values in place ------------------------------------------
// A tile is 16K values: 1024 threads owning 16 consecutive values each.
constexpr int kScanV = 16;
constexpr uint64_t kScanTile = 1024 * kScanV;

// scans a[base, base + kScanTile) ∩ [0, n) starting from `carry`; returns the
// running total after the tile (valid in every thread)
__device__ uint32_t scan_tile(uint32_t* a, uint64_t base, uint64_t n, uint32_t carry, uint32_t* ws) {
  const uint32_t lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const uint64_t i0 = base + (uint64_t)threadIdx.x * kScanV;
  uint32_t v[kScanV], s = 0;
#pragma unroll
  for (int j = 0; j < kScanV; ++j) { v[j] = i0 + j < n ? a[i0 + j] : 0; s += v[j]; }
  uint32_t incl = s;
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
    if (lane == 31) ws[32] = xi;
  }
  __syncthreads();
  uint32_t run = carry + ws[warp] + incl - s;
#pragma unroll
  for (int j = 0; j < kScanV; ++j) {
    if (i0 + j < n) a[i0 + j] = run;
    run += v[j];
  }
  const uint32_t total = carry + ws[32];
  __syncthreads();
  return total;
}

// single CTA, tile after tile
__global__ void __launch_bounds__(1024) k_scan_inplace(uint32_t* a, uint64_t n) {
  __shared__ uint32_t ws[33];
  uint32_t carry = 0;
  for (uint64_t base = 0; base < n; base += kScanTile) carry = scan_tile(a, base, n, carry, ws);
}
// one CTA per tile: local scan, tile totals to tot[]
__global__ void __launch_bounds__(1024) k_scan_tiles(uint32_t* a, uint64_t n, uint32_t* tot) {
  __shared__ uint32_t ws[33];
  const uint32_t t = scan_tile(a, blockIdx.x * kScanTile, n, 0, ws);
  if (threadIdx.x == 0) tot[blockIdx.x] = t;
}
__global__ void __launch_bounds__(1024) k_scan_add(uint32_t* a, uint64_t n, const uint32_t* off) {
  const uint32_t o = off[blockIdx.x];
  if (!o) return;
  const uint64_t i0 = blockIdx.x * kScanTile + (uint64_t)threadIdx.x * kScanV;
#pragma unroll
  for (int j = 0; j < kScanV; ++j)
    if (i0 + j < n) a[i0 + j] += o;
}
// scratch: n / kScanTile + 1 values
static void scan_u32(uint32_t* a, uint64_t n, uint32_t* scratch, cudaStream_t s, int* launches) {
  const uint64_t nt = (n + kScanTile - 1) / kScanTile;
  if (nt <= 1) {
    k_scan_inplace<<<1, 1024, 0, s>>>(a, n);
    *launches += 1;
    return;
  }
  k_scan_tiles<<<(unsigned)nt, 1024, 0, s>>>(a, n, scratch);
  k_scan_inplace<<<1, 1024, 0, s>>>(scratch, nt);
  k_scan_add<<<(unsigned)nt, 1024, 0, s>>>(a, n, scratch);
  *launches += 3;
}

// dynamic shared memory: hist[kRsThreads / 32][2^bits] u16 + dbase[2^bits] u32
template <class E>
__global__ void __launch_bounds__(kRsThreads) k_rs_scatter(const E* in, E* out, uint64_t n, RsPass ps,
                                                           const uint32_t* cnt, uint32_t nblk, uint32_t sub) {
  extern __shared__ __align__(16) uint8_t rs_smem[];
  const int nd = 1 << ps.bits;
  uint16_t* hist = reinterpret_cast<uint16_t*>(rs_smem);                     // [warp][nd]
  uint32_t* dbase = reinterpret_cast<uint32_t*>(rs_smem + (kRsThreads / 32) * nd * 2);
  const uint32_t tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  uint32_t* h32 = reinterpret_cast<uint32_t*>(hist);
  for (int d = tid; d < nd; d += kRsThreads) dbase[d] = cnt[(uint64_t)d * nblk + blockIdx.x];
  uint16_t* row = hist + warp * nd;
  const uint32_t lt = lanemask_lt();
  constexpr int kDig = kRsBins / kRsThreads;       // digits per thread in the offset pass
  // the block's tiles in order; within a tile a stable rank per warp (kRsItems
  // rounds of 32), then per-digit offsets across the warps
  for (uint32_t t = 0; t < sub; ++t) {
  const uint64_t base = ((uint64_t)blockIdx.x * sub + t) * kRsTile;
  if (base >= n) break;
  for (uint32_t i = tid; i < (uint32_t)((kRsThreads / 32) * nd / 2); i += kRsThreads) h32[i] = 0;
  __syncthreads();
  E c[kRsItems]; uint32_t rk[kRsItems], dg[kRsItems];
  for (int r = 0; r < kRsItems; ++r) {
    uint64_t i = base + warp * (32 * kRsItems) + r * 32 + lane;
    bool valid = i < n;
    if (valid) c[r] = in[i];
    uint32_t d = valid ? rs_digit(c[r], ps) : 0xFFFFu;
    uint32_t grp = __match_any_sync(FULL, d);
    uint32_t b = valid ? row[d] : 0;
    __syncwarp();
    if (valid && lane == 31u - __clz(grp)) row[d] = (uint16_t)(b + __popc(grp));
    __syncwarp();
    dg[r] = d; rk[r] = b + __popc(grp & lt);
  }
  __syncthreads();
  uint32_t tot[kDig];
#pragma unroll
  for (int k = 0; k < kDig; ++k) {
    const int d = tid + k * kRsThreads;
    uint32_t s = 0;
    if (d < nd)
      for (int w = 0; w < kRsThreads / 32; ++w) { uint32_t x = hist[w * nd + d]; hist[w * nd + d] = (uint16_t)s; s += x; }
    tot[k] = s;
  }
  __syncthreads();
  for (int r = 0; r < kRsItems; ++r) {
    uint64_t i = base + warp * (32 * kRsItems) + r * 32 + lane;
    if (i < n) out[dbase[dg[r]] + row[dg[r]] + rk[r]] = c[r];
  }
  __syncthreads();
#pragma unroll
  for (int k = 0; k < kDig; ++k)
    if (tid + k * kRsThreads < nd) dbase[tid + k * kRsThreads] += tot[k];
  }
}

// keep flags: unique (all fields differ from the predecessor), or dedup-first
// (word, kind differ from the predecessor) for the (word, kind, pos) order.
__device__ __forceinline__ bool keep_elem(const uint4* a, uint64_t i, int mode) {
  if (mode == 2) return a[i].w != 0;           // cross-flush dedup: kind 0 marks a dropped element
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
  uint32_t kc[8] = {0, 0, 0, 0, 0, 0, 0, 0};
  for (int j = 0; j < kRsItems; ++j) {
    uint64_t i = base + (uint64_t)threadIdx.x * kRsItems + j;
    if (!kp[j]) continue;
    uint4 x = a[i];
    if (final_out) {
      uint64_t word = ((uint64_t)x.x | ((uint64_t)x.y << 32)) + base_word;
      uint64_t w0 = (word & kMask48) | ((uint64_t)x.w << 48);
      uint64_t w1 = gidx ? gidx[x.z] : index_base + x.z;
      out[o] = make_uint4((uint32_t)w0, (uint32_t)(w0 >> 32), (uint32_t)w1, (uint32_t)(w1 >> 32));
      kc[x.w & 7u]++;                      // per-kind counts in n_out[1..4]
    } else {
      out[o] = x;
    }
    ++o;
  }
  if (final_out) {
#pragma unroll
    for (int k = 1; k < 5; ++k) {
      uint32_t v = kc[k];
      for (int d = 16; d; d >>= 1) v += __shfl_xor_sync(FULL, v, d);
      if (lane == 0 && v) atomicAdd(&n_out[k], (unsigned long long)v);
    }
  }
  if (blockIdx.x == nblk - 1 && threadIdx.x == kRsThreads - 1) *n_out = o;
}

// ARB_F_DEDUP_FIRST across flushes (Z3 over the whole trace, N2): the (word, kind)
// pairs reported so far live in a persistent open-addressing set of keys
// (word << 3 | kind) + 1 (0 = empty slot).  Each candidate that is the first of its
// (word, kind) in this flush is inserted; if the key was already there an earlier
// flush reported the pair, and the candidate is dropped (kind := 0).
__global__ void k_dedup_set(uint4* a, uint64_t n, unsigned long long* set, uint64_t mask,
                            unsigned long long* inserted) {
  uint32_t ins = 0;
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x) {
    uint4 x = a[i];
    const unsigned long long key = ((((unsigned long long)x.y << 32) | x.x) << 3 | (x.w & 7u)) + 1ull;
    uint64_t h = (key * 0x9E3779B97F4A7C15ull) >> 20;
    for (;;) {
      h &= mask;
      const unsigned long long old = atomicCAS(&set[h], 0ull, key);
      if (old == 0ull) { ++ins; break; }
      if (old == key) { a[i].w = 0; break; }
      ++h;
    }
  }
  for (int d = 16; d; d >>= 1) ins += __shfl_xor_sync(FULL, ins, d);
  if ((threadIdx.x & 31) == 0 && ins) atomicAdd(inserted, (unsigned long long)ins);
}
// rehash the set into a larger table
__global__ void k_dedup_rehash(const unsigned long long* old, uint64_t n_old, unsigned long long* set, uint64_t mask) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n_old; i += (uint64_t)gridDim.x * blockDim.x) {
    const unsigned long long key = old[i];
    if (!key) continue;
    uint64_t h = (key * 0x9E3779B97F4A7C15ull) >> 20;
    for (;;) {
      h &= mask;
      if (atomicCAS(&set[h], 0ull, key) == 0ull) break;
      ++h;
    }
  }
}
cudaError_t launch_dedup_rehash(const unsigned long long* old, uint64_t n_old, unsigned long long* set, uint64_t mask,
                                cudaStream_t s) {
  if (n_old) k_dedup_rehash<<<(unsigned)std::min<uint64_t>((n_old + 255) / 256, 4096), 256, 0, s>>>(old, n_old, set, mask);
  return cudaGetLastError();
}

// dedup-first (Z3): the kept candidates are sorted by (word, kind, pos) and hold at
// most one element per (word, kind), so a word's group has <= 8 elements; the
// canonical order (word, pos, kind) is a rank inside the group.  Writes the
// arb_report records (as k_keep_write with final_out) and the per-kind counts.
__global__ void k_dedup_canonical(const uint4* a, uint64_t n, uint4* out, uint64_t base_word, const uint64_t* gidx,
                                  uint64_t index_base, unsigned long long* n_out) {
  uint32_t kc[5] = {0, 0, 0, 0, 0};
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x) {
    const uint4 x = a[i];
    uint64_t g0 = i, g1 = i + 1;
    while (g0 > 0 && i - g0 < 8 && a[g0 - 1].x == x.x && a[g0 - 1].y == x.y) --g0;
    while (g1 < n && g1 - i < 8 && a[g1].x == x.x && a[g1].y == x.y) ++g1;
    uint32_t rank = 0;
    for (uint64_t j = g0; j < g1; ++j) {
      const uint4 y = a[j];
      rank += (y.z < x.z) || (y.z == x.z && y.w < x.w);
    }
    const uint64_t word = ((uint64_t)x.x | ((uint64_t)x.y << 32)) + base_word;
    const uint64_t w0 = (word & kMask48) | ((uint64_t)x.w << 48);
    const uint64_t w1 = gidx ? gidx[x.z] : index_base + x.z;
    out[g0 + rank] = make_uint4((uint32_t)w0, (uint32_t)(w0 >> 32), (uint32_t)w1, (uint32_t)(w1 >> 32));
    const uint32_t kd = x.w & 7u;
    kc[kd < 5 ? kd : 0]++;
  }
  const uint32_t lane = threadIdx.x & 31;
#pragma unroll
  for (int k = 1; k < 5; ++k) {
    uint32_t v = kc[k];
    for (int d = 16; d; d >>= 1) v += __shfl_xor_sync(FULL, v, d);
    if (lane == 0 && v) atomicAdd(&n_out[k], (unsigned long long)v);
  }
  if (blockIdx.x == 0 && threadIdx.x == 0) n_out[0] = n;
}

template <class E>
static cudaError_t radix_sort(E*& a, E*& b, uint64_t n, const RsPass* passes, int np, uint32_t* cnt,
                              cudaStream_t s, int* launches) {
  // tiles per block: the largest power of two <= 8 that still gives >= 4 blocks per SM
  // (the scatter walks its tiles one after the other)
  uint32_t sub = 1;
  while (sub < 8 && n / ((uint64_t)kRsTile * sub * 2) >= 4 * 148) sub *= 2;
  const uint32_t nblk = (uint32_t)((n + (uint64_t)kRsTile * sub - 1) / ((uint64_t)kRsTile * sub));
  const size_t smem_max = (kRsThreads / 32) * kRsBins * 2 + kRsBins * 4;
  cudaError_t e = cudaFuncSetAttribute(k_rs_scatter<E>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem_max);
  if (e != cudaSuccess) return e;
  for (int k = 0; k < np; ++k) {
    const uint64_t nd = 1ull << passes[k].bits;
    k_rs_hist<E><<<nblk, kRsThreads, 0, s>>>(a, n, passes[k], cnt, nblk, sub);
    scan_u32(cnt, (uint64_t)nblk * nd, cnt + (uint64_t)nblk * nd, s, launches);
    k_rs_scatter<E><<<nblk, kRsThreads, (kRsThreads / 32) * nd * 2 + nd * 4, s>>>(a, b, n, passes[k], cnt, nblk, sub);
    *launches += 2;
    E* t = a; a = b; b = t;
  }
  return cudaGetLastError();
}

// LSD passes over `bits` bits of a field, in near-equal digits of <= 11 bits
static int add_field_passes(RsPass* ps, int np, int field, int bits) {
  if (bits <= 0) return np;
  const int k = (bits + kRsMaxBits - 1) / kRsMaxBits;
  int sh = 0;
  for (int j = 0; j < k; ++j) {
    const int w = (bits - sh + (k - j) - 1) / (k - j);
    ps[np++] = RsPass{field, sh, w};
    sh += w;
  }
  return np;
}

// Segment entries as written by k_partition (8 B): x = bucket << 21 | chunk bits
// 0-20, y = start | len << 16 | chunk bit 21 << 31 (start < 512 with kRunFlag for a
// run; len <= 512 for stored events, < 2^15 for a run continued over chunks).
__device__ __forceinline__ uint32_t seg_bucket(uint2 e) { return e.x >> kSegChunkBits; }
__device__ __forceinline__ uint32_t seg_len(uint2 e) { return (e.y >> 16) & 0x7FFFu; }
__device__ __forceinline__ uint32_t seg_chunk(uint2 e) {
  return (e.x & ((1u << kSegChunkBits) - 1u)) | ((e.y >> 31) << kSegChunkBits);
}

// first entry of every bucket in the sorted entries
__global__ void k_seg_first(const uint2* segs, uint64_t n, uint32_t n_buckets, uint32_t* first) {
  for (uint32_t b = blockIdx.x * blockDim.x + threadIdx.x; b <= n_buckets; b += gridDim.x * blockDim.x) {
    uint64_t a = 0, z = n;                 // first entry with bucket >= b
    while (a < z) { const uint64_t mid = (a + z) >> 1; if (seg_bucket(segs[mid]) < b) a = mid + 1; else z = mid; }
    first[b] = (uint32_t)a;
  }
}

// event count of each tile of sorted entries (blocked: thread t owns 8 entries)
__global__ void __launch_bounds__(kRsThreads) k_seg_tile_sum(const uint2* segs, uint64_t n, uint32_t* blk) {
  __shared__ uint32_t red[kRsThreads / 32];
  const uint64_t base = (uint64_t)blockIdx.x * kRsTile + (uint64_t)threadIdx.x * kRsItems;
  uint32_t c = 0;
#pragma unroll
  for (int j = 0; j < kRsItems; ++j)
    if (base + j < n) c += seg_len(segs[base + j]);
  for (int d = 16; d; d >>= 1) c += __shfl_xor_sync(FULL, c, d);
  if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = c;
  __syncthreads();
  if (threadIdx.x == 0) {
    uint32_t t = 0;
    for (int w = 0; w < kRsThreads / 32; ++w) t += red[w];
    blk[blockIdx.x] = t;
  }
}
// replay form {chunk, bucket, start | len << 16, exclusive event prefix over the array}
__global__ void __launch_bounds__(kRsThreads) k_seg_cum(const uint2* segs, uint64_t n, const uint32_t* blk,
                                                        uint4* out) {
  __shared__ uint32_t ws[kRsThreads / 32];
  const uint32_t lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const uint64_t base = (uint64_t)blockIdx.x * kRsTile + (uint64_t)threadIdx.x * kRsItems;
  uint2 e[kRsItems];
  uint32_t c = 0;
#pragma unroll
  for (int j = 0; j < kRsItems; ++j) {
    e[j] = base + j < n ? segs[base + j] : make_uint2(0, 0);
    c += seg_len(e[j]);
  }
  uint32_t incl = c;
  for (int d = 1; d < 32; d <<= 1) {
    const uint32_t o = __shfl_up_sync(FULL, incl, d);
    if (lane >= (uint32_t)d) incl += o;
  }
  if (lane == 31) ws[warp] = incl;
  __syncthreads();
  uint32_t run = blk[blockIdx.x] + incl - c;
  for (uint32_t w = 0; w < warp; ++w) run += ws[w];
#pragma unroll
  for (int j = 0; j < kRsItems; ++j) {
    if (base + j < n)
      out[base + j] = make_uint4(seg_chunk(e[j]), seg_bucket(e[j]), e[j].y & 0x7FFFFFFFu, run);
    run += seg_len(e[j]);
  }
}

cudaError_t launch_sort_segments(uint2* a, uint2* b, uint64_t n, uint64_t n_chunks, uint32_t n_buckets,
                                 uint32_t* cnt, uint32_t* first, uint4* out, cudaStream_t s, int* launches) {
  RsPass ps[8];
  int np = 0;
  {
    // the partition block of the chunk (chunk / kChunkBlock); within a block the input is in chunk order
    const uint64_t nblocks = (n_chunks + kChunkBlock - 1) / kChunkBlock;
    int bb = 1;
    while ((1ull << bb) < nblocks) ++bb;
    const int k = (bb + kRsMaxBits - 1) / kRsMaxBits;
    for (int j = 0, sh = 0; j < k; ++j) {
      const int w = (bb - sh + (k - j) - 1) / (k - j);
      ps[np++] = RsPass{2, sh, w, kChunkBlock};
      sh += w;
    }
  }
  {
    int nbb = 1;
    while ((1u << nbb) < n_buckets) ++nbb;                      // bucket bits actually used
    for (int sh = kSegChunkBits, k = 0; k < 1; ++k) ps[np++] = RsPass{0, sh, nbb};
  }
  cudaError_t e = cudaSuccess;
  if (n) e = radix_sort(a, b, n, ps, np, cnt, s, launches);
  if (e != cudaSuccess) return e;
  if (n) {
    const uint32_t nblk = (uint32_t)((n + kRsTile - 1) / kRsTile);
    k_seg_tile_sum<<<nblk, kRsThreads, 0, s>>>(a, n, cnt);
    scan_u32(cnt, nblk, cnt + nblk, s, launches);
    k_seg_cum<<<nblk, kRsThreads, 0, s>>>(a, n, cnt, out);
    *launches += 2;
  }
  k_seg_first<<<(n_buckets + 256) / 256, 256, 0, s>>>(a, n, n_buckets, first);
  *launches += 1;
  return cudaGetLastError();
}

cudaError_t launch_compact(const CompactParams& p, cudaStream_t s, int* launches) {
  cudaMemsetAsync(p.n_out, 0, 8 * sizeof(unsigned long long), s);
  if (p.n_cand == 0) return cudaGetLastError();
  uint4* a = p.cand;
  uint4* b = p.tmp;
  uint64_t n = p.n_cand;
  RsPass ps[24];
  int np = 0;
  cudaError_t e;
  if (p.dedup_first) {
    // (word, kind, pos): keep the first of each (word, kind)
    np = add_field_passes(ps, np, 7, 30 + kKindBits);            // record, then kind (one field)
    np = add_field_passes(ps, np, 6, p.word_bits);
    if ((e = radix_sort<uint4>(a, b, n, ps, np, p.blk, s, launches)) != cudaSuccess) return e;
    uint32_t nblk = (uint32_t)((n + kRsTile - 1) / kRsTile);
    k_keep_count<<<nblk, kRsThreads, 0, s>>>(a, n, 1, p.blk);
    scan_u32(p.blk, nblk, p.blk + nblk, s, launches);
    k_keep_write<<<nblk, kRsThreads, 0, s>>>(a, n, 1, p.blk, b, 0, 0, nullptr, 0, p.n_out, nblk);
    *launches += 2;
    // the number kept is needed on the host side to continue; read it back
    unsigned long long kept = 0;
    cudaMemcpyAsync(&kept, p.n_out, sizeof(kept), cudaMemcpyDeviceToHost, s);
    cudaStreamSynchronize(s);
    n = kept;
    uint4* t = a; a = b; b = t;
    np = 0;
    if (p.dset && n) {               // drop the (word, kind) pairs earlier flushes reported
      k_dedup_set<<<(unsigned)std::min<uint64_t>((n + 255) / 256, 4096), 256, 0, s>>>(a, n, p.dset, p.dset_mask,
                                                                                   p.dset_count);
      nblk = (uint32_t)((n + kRsTile - 1) / kRsTile);
      k_keep_count<<<nblk, kRsThreads, 0, s>>>(a, n, 2, p.blk);
      scan_u32(p.blk, nblk, p.blk + nblk, s, launches);
      k_keep_write<<<nblk, kRsThreads, 0, s>>>(a, n, 2, p.blk, b, 0, 0, nullptr, 0, p.n_out, nblk);
      *launches += 3;
      cudaMemcpyAsync(&kept, p.n_out, sizeof(kept), cudaMemcpyDeviceToHost, s);
      cudaStreamSynchronize(s);
      n = kept;
      t = a; a = b; b = t;
    }
    if (n == 0) return cudaGetLastError();     // every pair was reported by an earlier flush
    // canonical order inside each word's group of <= 8 (one per kind): no second sort
    k_dedup_canonical<<<(unsigned)std::min<uint64_t>((n + 255) / 256, 148 * 8), 256, 0, s>>>(
        a, n, p.out, p.base_word, p.gidx, p.index_base, p.n_out);
    *launches += 1;
    return cudaGetLastError();
  }
  np = add_field_passes(ps, np, 5, p.pos_bits + kKindBits);   // record, then kind (one field)
  np = add_field_passes(ps, np, 6, p.word_bits);
  if ((e = radix_sort<uint4>(a, b, n, ps, np, p.blk, s, launches)) != cudaSuccess) return e;
  uint32_t nblk = (uint32_t)((n + kRsTile - 1) / kRsTile);
  if (n == 0) {
    cudaMemsetAsync(p.n_out, 0, 8 * sizeof(unsigned long long), s);
    return cudaGetLastError();
  }
  k_keep_count<<<nblk, kRsThreads, 0, s>>>(a, n, 0, p.blk);
  scan_u32(p.blk, nblk, p.blk + nblk, s, launches);
  k_keep_write<<<nblk, kRsThreads, 0, s>>>(a, n, 0, p.blk, p.out, 1, p.base_word, p.gidx, p.index_base,
                                           p.n_out, nblk);
  *launches += 2;
  return cudaGetLastError();
}

}  // namespace arb
