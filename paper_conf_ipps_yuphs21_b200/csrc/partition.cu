// partition.cu — A1 (ingest/decode) + A3 (stable partition by address bucket)
// in one sweep over the batch, with a decoupled look-back across CTA tiles.
//
// k_partition  persistent CTAs (one per SM, 16 warps).  A CTA tile is 16 chunks of
//              256 records (4096 records), one chunk per warp; CTAs take tiles in
//              order from a ticket counter (one tile ahead, so the next tile's
//              records stream in during this one) — tickets let the CTAs drift
//              apart, so a tile's predecessors have mostly published inclusive
//              prefixes by the time it looks back (a lockstep grid would make every
//              tile of a wave walk back to the previous wave).  Per tile:
//   1. every warp decodes its chunk (staged in its shared memory by one TMA bulk
//      copy, cp.async.bulk, completing on an mbarrier; the warp's chunk of the
//      next tile is fetched as soon as this one is decoded): access vs control
//      record, byte range -> its 1 or 2 8-byte words, word -> address
//      bucket via the bin map; events are ranked stably per bucket inside the
//      warp (a single check when the whole chunk is one bucket — the common case
//      of real access streams — else match.any per 32 records);
//   2. the union of the buckets the tile touches is collected, and for each the
//      exclusive prefix over the warps (warp order = trace order) and the tile's
//      count;
//   3. decoupled look-back: the tile publishes its per-bucket counts (aggregate)
//      in a status ring, sums the predecessors' entries back to the first
//      inclusive prefix, and publishes its own inclusive prefix — every bucket,
//      so a successor never walks past one tile;
//   4. every warp writes its events to region[b] + tile prefix + warp offset +
//      rank: each bucket's events end up contiguous and in trace order (A3),
//      with no per-chunk segment list and no sort.
// Regions are sized from the sampled histogram with a margin (launch_regions);
// if a bucket overflows its region the host re-runs the partition with the
// exact counts the look-back produced (DevStats::overflow, bucket_total).
#include "kcommon.cuh"
#include <algorithm>
#include <cmath>

namespace arb {

constexpr int PT = kPartThreads;            // 512 threads
constexpr int PW = kPartWarps;              // 16 warps
constexpr int WREC = kChunkRecords;         // 256 records per chunk
constexpr int RPL = WREC / 32;              // 8 records per lane (two groups of 4 x 32)
constexpr int NBK = kMaxBuckets;            // bucket rows are always kMaxBuckets wide
constexpr int BPT = NBK / PT;               // buckets per thread in the look-back (4)
static_assert(BPT == 4, "look-back vector width");

// shared memory: CTA part {reg_start u64, reg_cap u32, tbase u32, ttag u32}[NBK],
// ulist u16[NBK], nU u32[2] (+pad); per warp: stage[WREC] uint4, tlist[2 * WREC]
// u16, row[NBK] u16, bar u64 (+pad)
constexpr size_t kCtaSmem = (size_t)NBK * (8 + 4 + 4 + 4 + 2) + 16;
constexpr size_t kWarpSmem = sizeof(uint4) * WREC + 2 * (2 * WREC) + 2 * NBK + 16;

// Decoded record: info = cnt | b0 << 2 | b1 << kB1Shift (cnt = tracked words 0..2),
// keys k0/k1 = op << 30 | word offset inside the bucket.
struct Dec { uint32_t info, k0, k1; };
constexpr int kB1Shift = 2 + kBucketBits;

// First word of a record, branch-free (predicated) so the four records of a
// round interleave.  flags: bit0 control record, bit1 malformed.  valid =
// record exists; two = an unaligned access that also touches the next word
// (Z4, rare: handled by decode1).  b1 = b0 until decode1 says otherwise.
template <bool MD>
__device__ __forceinline__ Dec decode0(uint4 q, bool valid, const PartParams& p, uint32_t& ign, uint32_t& flags,
                                       bool& two) {
  const uint32_t op = (q.y >> 16) & 0xFFu;
  const uint32_t len = q.z, hi = q.y & 0xFFFFu;
  // malformed access: len outside 1..8 or the byte range leaving the 48-bit space
  const bool bad_acc = (q.w & 0xFFFFu) != 0 || len - 1u > 7u || (hi == 0xFFFFu && q.x > 0u - len);
  const bool ctl = op < 16 && ((0xFF00u >> op) & 1u);            // ops 8-15 (11: ARB_BASE, Z25)
  const bool acc = op < 4;
  flags = valid ? (acc ? (bad_acc ? 2u : 0u) : (ctl ? 1u : 2u)) : 0u;
  bool ok = valid && acc && !bad_acc;
  uint32_t dev = 0;
  if (MD) {                                  // several accelerators (Z24): the device of RT / WT is the arg
    dev = (op & 2u) ? q.y >> 24 : 0u;
    if (acc && dev >= p.n_dev) { flags = valid ? 2u : 0u; ok = false; }
  }
  const uint64_t rel = ((((uint64_t)hi) << 29) | (q.x >> 3)) - p.base_word;   // wraps below the range
  const bool in0 = ok && rel < p.n_words;
  two = ok && (q.x & 7u) + len > 8u;
  ign += (uint32_t)(ok && !in0);
  const uint32_t cb = p.coarse_bits;
  uint32_t m0 = 0;
  if (in0) m0 = __ldg(p.bin_map + (uint32_t)(rel >> cb));
  const uint32_t b0 = m0 & kBucketMask;                          // 0 when untracked
  Dec d;
  d.k0 = (op << 30) | ((m0 >> kBucketBits) << cb) | ((uint32_t)rel & ((1u << cb) - 1u));
  d.k1 = 0;
  d.info = (uint32_t)in0 | (b0 << 2) | (b0 << kB1Shift);
  if (MD) d.info |= (dev & 3u) << 24;
  return d;
}
// Second word of an unaligned access (the record is re-read from the stage).
template <bool MD>
__device__ __forceinline__ void decode1(Dec& d, uint4 q, const PartParams& p, uint32_t& ign) {
  const uint32_t op = (q.y >> 16) & 0xFFu;
  const uint64_t r1 = ((((uint64_t)(q.y & 0xFFFFu)) << 29) | (q.x >> 3)) - p.base_word + 1;
  if (r1 >= p.n_words) { ++ign; return; }
  const uint32_t cb = p.coarse_bits;
  const uint32_t m = __ldg(p.bin_map + (uint32_t)(r1 >> cb));
  const uint32_t b = m & kBucketMask;
  const uint32_t k = (op << 30) | ((m >> kBucketBits) << cb) | ((uint32_t)r1 & ((1u << cb) - 1u));
  const uint32_t dv = MD ? d.info & (3u << 24) : 0u;   // the device bits (Z24)
  if ((d.info & 3u) == 0) { d.k0 = k; d.info = 1u | (b << 2) | (b << kB1Shift) | dv; }
  else { d.k1 = k; d.info = 2u | (d.info & (kBucketMask << 2)) | (b << kB1Shift) | dv; }
}

// append the buckets of lanes with `is_new` to the warp's touched list
__device__ __forceinline__ void touch(uint16_t* tlist, uint32_t& nT, bool is_new, uint32_t b, uint32_t lt) {
  const uint32_t m = __ballot_sync(FULL, is_new);
  if (is_new) tlist[nT + __popc(m & lt)] = (uint16_t)b;
  nT += __popc(m);
}

// Generic stable rank of one 32-record round (record order, word0 before word1).
__device__ __forceinline__ void rank_round(uint32_t info, uint16_t* row, uint16_t* tlist, uint32_t& nT,
                                           uint32_t lane, uint32_t lt, uint32_t& r0, uint32_t& r1) {
  const uint32_t cnt = info & 3u, b0 = (info >> 2) & kBucketMask, b1 = (info >> kB1Shift) & kBucketMask;
  r0 = r1 = 0;
  if (__any_sync(FULL, cnt == 2 && b0 != b1)) {
    // a record crossing a bucket boundary: serial over lanes
    bool n0 = false, n1 = false;
    for (uint32_t L = 0; L < 32; ++L) {
      if (lane == L) {
        if (cnt >= 1) { r0 = row[b0]; row[b0] = (uint16_t)(r0 + 1); n0 = r0 == 0; }
        if (cnt == 2) { r1 = row[b1]; row[b1] = (uint16_t)(r1 + 1); n1 = r1 == 0; }
      }
      __syncwarp();
    }
    touch(tlist, nT, n0, b0, lt);
    touch(tlist, nT, n1, b1, lt);
    return;
  }
  const uint32_t two = __ballot_sync(FULL, cnt == 2);
  const uint32_t grp = __match_any_sync(FULL, cnt ? b0 : 0xFFFFFFFFu);
  const uint32_t base = cnt ? row[b0] : 0;
  __syncwarp();
  const bool leader = cnt && lane == 31u - __clz(grp);
  if (leader) row[b0] = (uint16_t)(base + __popc(grp) + __popc(grp & two));
  __syncwarp();
  touch(tlist, nT, leader && base == 0, b0, lt);
  r0 = base + __popc(grp & lt) + __popc(grp & lt & two);
  r1 = r0 + 1;
}


// The fast chunk test.  Every record must be an access (op < 4) of 1..8 bytes
// inside one 8-byte word (such an access cannot leave the 48-bit space),
// and all words must lie in one address bucket.  Buckets are contiguous word
// ranges, so the test needs only the chunk's lowest and highest word: each word
// is taken relative to record 0's word w0 (32-bit signed, |d| < 2^30 as a bucket
// spans <= 2^30 words), the warp reduces min and max, and two bin-map lookups
// decide.  A word's offset in the bucket is then off(lowest) + d - dmin.  On
// success the chunk's events are returned in the general form (dec, rk).
template <bool MD>
__device__ __forceinline__ bool fast_chunk(const uint4* st, const PartParams& p, Dec* dec, uint32_t* rk,
                                           uint32_t& bref_out, uint32_t lane) {
  const uint4 q0 = st[0];
  const uint64_t w0 = ((uint64_t)((q0.y & 0xFFFFu) >> 3) << 32) | __funnelshift_r(q0.x, q0.y, 3);
  uint32_t d[RPL], opk[RPL], bad = 0, devs = 0;
  int32_t dmin = 0, dmax = 0;
#pragma unroll
  for (int k = 0; k < RPL; ++k) {
    const uint4 q = st[k * 32 + lane];
    bad |= (q.y & 0x00FC0000u) | (q.w & 0xFFFFu) | ((q.z - 1u) & ~7u) | (((q.x & 7u) + q.z - 1u) & ~7u);
    if (MD && (q.y & (1u << 17))) {                // RT / WT on device arg (Z24)
      const uint32_t dv = q.y >> 24;
      bad |= dv >= p.n_dev;
      devs |= (dv & 3u) << (2 * k);
    }
    const uint64_t word = ((uint64_t)((q.y & 0xFFFFu) >> 3) << 32) | __funnelshift_r(q.x, q.y, 3);
    const uint64_t diff = word - w0;
    bad |= (uint32_t)((diff + (1ull << 30)) >> 31);      // d outside [-2^30, 2^30)
    d[k] = (uint32_t)diff;
    dmin = min(dmin, (int32_t)d[k]);
    dmax = max(dmax, (int32_t)d[k]);
    opk[k] = ((q.y >> 16) & 3u) << 30;
  }
  if (!__all_sync(FULL, bad == 0)) return false;
  dmin = __reduce_min_sync(FULL, dmin);
  dmax = __reduce_max_sync(FULL, dmax);
  const uint64_t rlo = w0 - p.base_word + (uint64_t)(int64_t)dmin;   // wraps below the range
  const uint64_t rhi = w0 - p.base_word + (uint64_t)(int64_t)dmax;
  if (rlo >= p.n_words || rhi >= p.n_words) return false;
  const uint32_t cb = p.coarse_bits;
  const uint32_t mlo = __ldg(p.bin_map + (uint32_t)(rlo >> cb)), mhi = __ldg(p.bin_map + (uint32_t)(rhi >> cb));
  const uint32_t bref = mlo & kBucketMask;
  if (bref != (mhi & kBucketMask)) return false;
  const uint32_t c = (((mlo >> kBucketBits) << cb) | ((uint32_t)rlo & ((1u << cb) - 1u))) - (uint32_t)dmin;
  const uint32_t info = 1u | (bref << 2) | (bref << kB1Shift);
#pragma unroll
  for (int k = 0; k < RPL; ++k) {
    dec[k].k0 = opk[k] | (d[k] + c);
    dec[k].k1 = 0;
    dec[k].info = info | (MD ? ((devs >> (2 * k)) & 3u) << 24 : 0u);
    const uint32_t r = (uint32_t)(k >> 2) * 128 + (uint32_t)(k & 3) * 32 + lane;   // record index in the chunk
    rk[k] = r | ((r + 1) << 16);
  }
  bref_out = bref;
  return true;
}

// status ring entries (kRingTiles slots x NBK buckets)
constexpr unsigned long long kFlagAgg = 1ull << 38, kFlagIncl = 2ull << 38;
constexpr unsigned long long kCountMask = (1ull << 38) - 1;
__device__ __forceinline__ unsigned long long st_tag(uint32_t tile) { return (unsigned long long)(tile + 1) << 40; }

// MD: several accelerators (Z24) — the device of RT / WT goes to bits 30-31 of the
// event position; a separate instance so that the single-device kernel is unchanged
template <bool MD>
__global__ void __launch_bounds__(PT, 1) k_partition(PartParams p) {
  extern __shared__ __align__(16) uint8_t smem[];
  const uint32_t lane = threadIdx.x & 31, warp = threadIdx.x >> 5, tid = threadIdx.x;
  const uint32_t lt = lanemask_lt();
  uint64_t* sreg = reinterpret_cast<uint64_t*>(smem);              // [NBK] region start
  uint32_t* scap = reinterpret_cast<uint32_t*>(sreg + NBK);         // [NBK] region capacity
  uint32_t* tbase = scap + NBK;                                     // [NBK] tile count, then tile prefix
  uint32_t* ttag = tbase + NBK;                                     // [NBK] local tile tag of the last touch
  uint16_t* ulist = reinterpret_cast<uint16_t*>(ttag + NBK);        // [NBK] buckets the tile touches
  uint32_t* nU = reinterpret_cast<uint32_t*>(ulist + NBK);          // [2]
  uint8_t* wbase = smem + kCtaSmem + warp * kWarpSmem;
  uint4* stage = reinterpret_cast<uint4*>(wbase);                   // [WREC]
  uint16_t* tlist = reinterpret_cast<uint16_t*>(stage + WREC);       // [2 * WREC]
  uint16_t* row = tlist + 2 * WREC;                                  // [NBK]
  uint64_t* bar = reinterpret_cast<uint64_t*>(row + NBK);
  for (uint32_t i = tid; i < NBK; i += PT) {
    sreg[i] = p.reg_start[i]; scap[i] = p.reg_cap[i]; ttag[i] = 0;
  }
  if (tid < 2) nU[tid] = 0;
  __shared__ uint32_t s_tick[2];
  if (tid == 0) {
    s_tick[0] = (uint32_t)atomicAdd(&p.st->tile_ticket, 1ull);
    s_tick[1] = (uint32_t)atomicAdd(&p.st->tile_ticket, 1ull);
  }
  for (uint32_t i = lane; i < NBK; i += 32) row[i] = 0;
  if (lane == 0) mbar_init(bar, 1);
  fence_mbar_init();
  __syncthreads();
  uint32_t n_acc = 0, n_ign = 0, phase = 0;

  // the warp's chunk arrives in its stage by one TMA bulk copy (lane 0) completing on bar
  auto fetch = [&](uint64_t c) {
    if (c < p.n_chunks && lane == 0) {
      const uint64_t r0 = c * WREC;
      const uint32_t nv = p.n - r0 < (uint64_t)WREC ? (uint32_t)(p.n - r0) : (uint32_t)WREC;
      mbar_arrive_tx(bar, nv * 16u);
      bulk_g2s(stage, p.ev + r0, nv * 16u, bar);
    }
  };
  uint32_t tile = s_tick[0], nxt = s_tick[1];
  fetch((uint64_t)tile * PW + warp);
  uint32_t tag = 0, par = 0;
  while (tile < p.n_tiles) {
    tag = tag + 1 == 0 ? 1 : tag + 1;
    const uint64_t chunk = (uint64_t)tile * PW + warp;
    const uint64_t rec0 = chunk * WREC;
    const uint32_t nvalid = chunk < p.n_chunks ? (p.n - rec0 < (uint64_t)WREC ? (uint32_t)(p.n - rec0) : (uint32_t)WREC) : 0u;
    Dec dec[RPL];
    uint32_t rk[RPL];
    uint32_t nT = 0;
    bool any2 = false;                 // some record of the chunk has two words
    // ---- 1. decode + rank (warp-local) ------------------------------------------------
    if (nvalid) {
      mbar_wait(bar, phase);
      phase ^= 1u;
    }
    uint32_t bfast = 0;
    if (nvalid == WREC && fast_chunk<MD>(stage, p, dec, rk, bfast, lane)) {
      n_acc += RPL;
      if (lane == 0) { row[bfast] = (uint16_t)WREC; tlist[0] = (uint16_t)bfast; }
      nT = 1;
    } else if (nvalid) {
      uint32_t e_lane = 0;
#pragma unroll
      for (int g = 0; g < 2; ++g) {
        uint32_t any_flag = 0, twos = 0;
#pragma unroll
        for (int k = 0; k < 4; ++k) {
          const uint32_t j = g * 128 + k * 32 + lane;
          uint32_t flags;
          bool two;
          dec[g * 4 + k] = decode0<MD>(stage[j], j < nvalid, p, n_ign, flags, two);
          any_flag |= flags << (2 * k);
          twos |= (uint32_t)two << k;
        }
        if (__any_sync(FULL, twos != 0)) {
          any2 = true;
#pragma unroll
          for (int k = 0; k < 4; ++k)
            if ((twos >> k) & 1u) decode1<MD>(dec[g * 4 + k], stage[g * 128 + k * 32 + lane], p, n_ign);
        }
#pragma unroll
        for (int k = 0; k < 4; ++k) e_lane += dec[g * 4 + k].info & 3u;
        if (__any_sync(FULL, any_flag != 0)) {
          // control / malformed records in the group (rare)
#pragma unroll
          for (int k = 0; k < 4; ++k) {
            const uint32_t j = g * 128 + k * 32 + lane;
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
        // bucket of the group's first event: round kl = first with a valid lane
        const uint32_t kl = vm[0] ? 0u : vm[1] ? 1u : vm[2] ? 2u : 3u;
        const uint32_t vml = vm[0] ? vm[0] : vm[1] ? vm[1] : vm[2] ? vm[2] : vm[3];
        const uint32_t lead = __ffs(vml) - 1;
        uint32_t bsrc = 0;
#pragma unroll
        for (int k = 0; k < 4; ++k) if ((uint32_t)k == kl) bsrc = (dec[g * 4 + k].info >> 2) & kBucketMask;
        const uint32_t bref = __shfl_sync(FULL, bsrc, lead);
        const uint32_t iref = bref << 2 | bref << kB1Shift;
        bool same = true;
#pragma unroll
        for (int k = 0; k < 4; ++k) {
          const uint32_t info = dec[g * 4 + k].info;
          same &= (info & 3u) == 0 || (info & (MD ? 0xFFFFFCu : ~3u)) == iref;
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
          if (lane == 0) {
            row[bref] = (uint16_t)run;
            if (base == 0) tlist[nT] = (uint16_t)bref;
          }
          nT += base == 0;
          __syncwarp();
        } else {
#pragma unroll
          for (int k = 0; k < 4; ++k) {
            uint32_t r0, r1;
            rank_round(dec[g * 4 + k].info, row, tlist, nT, lane, lt, r0, r1);
            rk[g * 4 + k] = r0 | (r1 << 16);
          }
        }
      }
      n_acc += e_lane;
    } else {
#pragma unroll
      for (int k = 0; k < RPL; ++k) { dec[k].info = 0; rk[k] = 0; }
    }
    __syncwarp();                      // stage reads done
    fetch((uint64_t)nxt * PW + warp);  // this warp's chunk of the CTA's next tile streams in meanwhile
    // ---- 2. the buckets the tile touches ------------------------------------------------
    for (uint32_t t = lane; t < nT; t += 32) {
      const uint32_t b = tlist[t];
      if (atomicExch(&ttag[b], tag) != tag) ulist[atomicAdd(&nU[par], 1u)] = (uint16_t)b;
    }
    __syncthreads();
    // ---- per touched bucket: exclusive prefix over the warps, tile count ----------------
    const uint32_t nu = nU[par];
    for (uint32_t i = tid; i < nu; i += PT) {
      const uint32_t b = ulist[i];
      uint32_t run = 0;
#pragma unroll
      for (uint32_t w = 0; w < PW; ++w) {
        uint16_t* r = reinterpret_cast<uint16_t*>(smem + kCtaSmem + w * kWarpSmem + sizeof(uint4) * WREC + 4 * WREC) + b;
        const uint32_t c = *r;
        if (c) *r = (uint16_t)run;     // rows of warps that did not touch b stay 0
        run += c;
      }
      tbase[b] = run;
    }
    if (tid == 0) {
      nU[par ^ 1u] = 0;
      s_tick[par] = (uint32_t)atomicAdd(&p.st->tile_ticket, 1ull);   // the tile after next
    }
    __syncthreads();
    // ---- 3. decoupled look-back over the tiles (buckets 4 tid .. 4 tid + 3) -------------
    {
      const uint32_t b0 = tid * BPT;
      uint32_t own[BPT];
      unsigned long long incl[BPT];
#pragma unroll
      for (int j = 0; j < BPT; ++j) own[j] = ttag[b0 + j] == tag ? tbase[b0 + j] : 0u;
      unsigned long long* mine = p.ring + (size_t)(tile % kRingTiles) * NBK + b0;
      const unsigned long long tg = st_tag(tile);
      if (tile == 0) {
#pragma unroll
        for (int j = 0; j < BPT; ++j) incl[j] = own[j];
      } else {
        __stcg(reinterpret_cast<ulonglong2*>(mine), make_ulonglong2(tg | kFlagAgg | own[0], tg | kFlagAgg | own[1]));
        __stcg(reinterpret_cast<ulonglong2*>(mine) + 1, make_ulonglong2(tg | kFlagAgg | own[2], tg | kFlagAgg | own[3]));
        unsigned long long pre[BPT] = {0, 0, 0, 0};
        uint32_t open = (1u << BPT) - 1;
        uint32_t q = tile - 1;
        for (;;) {
          const ulonglong2* src = reinterpret_cast<const ulonglong2*>(p.ring + (size_t)(q % kRingTiles) * NBK + b0);
          const ulonglong2 v0 = __ldcg(src), v1 = __ldcg(src + 1);
          const unsigned long long v[BPT] = {v0.x, v0.y, v1.x, v1.y};
          const unsigned long long want = st_tag(q);
          bool ready = true;
#pragma unroll
          for (int j = 0; j < BPT; ++j)
            if ((open >> j) & 1u) ready &= (v[j] & ~((1ull << 40) - 1)) == want && (v[j] & (3ull << 38)) != 0;
          if (!ready) { __nanosleep(20); continue; }     // the predecessor has not published yet
#pragma unroll
          for (int j = 0; j < BPT; ++j)
            if ((open >> j) & 1u) {
              pre[j] += v[j] & kCountMask;
              if (v[j] & kFlagIncl) open &= ~(1u << j);
            }
          if (!open || q == 0) break;
          --q;
        }
#pragma unroll
        for (int j = 0; j < BPT; ++j) { incl[j] = pre[j] + own[j]; tbase[b0 + j] = (uint32_t)pre[j]; }
      }
      __stcg(reinterpret_cast<ulonglong2*>(mine), make_ulonglong2(tg | kFlagIncl | incl[0], tg | kFlagIncl | incl[1]));
      __stcg(reinterpret_cast<ulonglong2*>(mine) + 1, make_ulonglong2(tg | kFlagIncl | incl[2], tg | kFlagIncl | incl[3]));
      if (tile == 0) {
#pragma unroll
        for (int j = 0; j < BPT; ++j) tbase[b0 + j] = 0u;
      }
#pragma unroll
      for (int j = 0; j < BPT; ++j)
        if (incl[j] > scap[b0 + j]) p.st->overflow = 1ull;   // re-run with exact counts
      if (tile + 1 == p.n_tiles) {
#pragma unroll
        for (int j = 0; j < BPT; ++j) p.bucket_total[b0 + j] = incl[j];
      }
    }
    __syncthreads();
    // ---- 4. write the events: region + tile prefix + warp offset + rank -----------------
    const uint32_t pos0 = (uint32_t)rec0 + lane;
#pragma unroll
    for (int r = 0; r < RPL; ++r) {
      const uint32_t info = dec[r].info;
      if (info & 3u) {
        const uint32_t b = (info >> 2) & kBucketMask;
        const uint32_t idx = tbase[b] + row[b] + (rk[r] & 0xFFFFu);
        const uint32_t pos = (pos0 + (r >> 2) * 128 + (r & 3) * 32) | (MD ? (info >> 24) << 30 : 0u);   // | device
        if (idx < scap[b]) p.part_ev[sreg[b] + idx] = make_uint2(dec[r].k0, pos);
      }
    }
    if (any2) {
#pragma unroll
      for (int r = 0; r < RPL; ++r) {
        const uint32_t info = dec[r].info;
        if ((info & 3u) == 2u) {
          const uint32_t b = (info >> kB1Shift) & kBucketMask;
          const uint32_t idx = tbase[b] + row[b] + (rk[r] >> 16);
          const uint32_t pos = (pos0 + (r >> 2) * 128 + (r & 3) * 32) | (MD ? (info >> 24) << 30 : 0u);
          if (idx < scap[b]) p.part_ev[sreg[b] + idx] = make_uint2(dec[r].k1, pos);
        }
      }
    }
    __syncwarp();
    for (uint32_t t = lane; t < nT; t += 32) row[tlist[t]] = 0;
    __syncwarp();
    tile = nxt;
    nxt = s_tick[par];                 // written before the look-back barrier
    par ^= 1u;
  }

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
  const size_t smem = kCtaSmem + PW * kWarpSmem;
  auto kern = p.n_dev > 1 ? k_partition<true> : k_partition<false>;
  cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  const uint32_t grid = std::min<uint32_t>(p.n_tiles, (uint32_t)sms);   // every CTA resident (look-back)
  kern<<<grid, PT, smem, s>>>(p);
  return cudaGetLastError();
}

// Bucket regions from the sampled weights (one CTA of 1024 threads, 2 buckets each).
__global__ void __launch_bounds__(1024) k_regions(const uint32_t* weight, const uint32_t* nb_dev, uint32_t n_fixed,
                                                  double stride, uint64_t capacity, uint64_t* reg_start,
                                                  uint32_t* reg_cap) {
  __shared__ unsigned long long ws[32];
  __shared__ double scale;
  const uint32_t nb = nb_dev ? *nb_dev : n_fixed;
  const uint32_t t = threadIdx.x, lane = t & 31, w = t >> 5;
  unsigned long long c[2];
#pragma unroll
  for (int j = 0; j < 2; ++j) {
    const uint32_t b = 2 * t + j;
    c[j] = 0;
    if (b < nb) {
      // the sample count is ~Poisson: cover weight + 6 sqrt(weight) + 8 samples' worth of
      // events with 10 % to spare (an overflow only costs a re-run with exact counts)
      const double wt = (double)weight[b];
      const double est = (wt + 6.0 * sqrt(wt) + 8.0) * stride * 1.10 + 64.0;
      c[j] = ((unsigned long long)est + 1ull) & ~1ull;
    }
  }
  unsigned long long v = c[0] + c[1], incl = v;
#pragma unroll
  for (int d = 1; d < 32; d <<= 1) {
    const unsigned long long o = __shfl_up_sync(FULL, incl, d);
    if (lane >= (uint32_t)d) incl += o;
  }
  if (lane == 31) ws[w] = incl;
  __syncthreads();
  if (w == 0) {
    const unsigned long long x = ws[lane];
    unsigned long long xi = x;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
      const unsigned long long o = __shfl_up_sync(FULL, xi, d);
      if (lane >= (uint32_t)d) xi += o;
    }
    ws[lane] = xi - x;
    if (lane == 31) scale = xi > capacity ? (double)capacity / (double)xi : 1.0;
  }
  __syncthreads();
  if (scale < 1.0) {            // too little room: shrink every region (overflow -> exact re-run)
#pragma unroll
    for (int j = 0; j < 2; ++j) c[j] = (unsigned long long)((double)c[j] * scale) & ~1ull;
    v = c[0] + c[1];
    incl = v;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
      const unsigned long long o = __shfl_up_sync(FULL, incl, d);
      if (lane >= (uint32_t)d) incl += o;
    }
    __syncthreads();
    if (lane == 31) ws[w] = incl;
    __syncthreads();
    if (w == 0) {
      const unsigned long long x = ws[lane];
      unsigned long long xi = x;
#pragma unroll
      for (int d = 1; d < 32; d <<= 1) {
        const unsigned long long o = __shfl_up_sync(FULL, xi, d);
        if (lane >= (uint32_t)d) xi += o;
      }
      ws[lane] = xi - x;
    }
    __syncthreads();
  }
  const unsigned long long start = ws[w] + incl - v;
#pragma unroll
  for (int j = 0; j < 2; ++j) {
    const uint32_t b = 2 * t + j;
    reg_start[b] = start + (j ? c[0] : 0);
    reg_cap[b] = (uint32_t)(c[j] < 0xFFFFFFFEull ? c[j] : 0xFFFFFFFEull);
  }
}

cudaError_t launch_regions(const uint32_t* weight, const uint32_t* nb, uint32_t n_fixed, double stride,
                           uint64_t capacity, uint64_t* reg_start, uint32_t* reg_cap, cudaStream_t s) {
  static_assert(2 * 1024 == kMaxBuckets, "k_regions: 2 buckets per thread");
  k_regions<<<1, 1024, 0, s>>>(weight, nb, n_fixed, stride, capacity, reg_start, reg_cap);
  return cudaGetLastError();
}

}  // namespace arb
