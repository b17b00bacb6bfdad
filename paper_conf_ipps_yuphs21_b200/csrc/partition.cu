// partition.cu — A1 (ingest/decode) + A3a (stable partition by address bucket).
//
// k_partition  persistent CTAs (one per SM, 16 warps).  Every warp works on its
//              own 256-record chunks with no block-level synchronisation: the
//              chunk's 16-B records are staged in the warp's shared memory by
//              one TMA bulk copy completing on an mbarrier (double-buffered: the
//              next chunk streams in while the current one is processed).  Lane L decodes records L, L+32, ...
//              (access vs control; byte range -> its 1 or 2 8-byte words, P:267;
//              word -> address bucket via the bin map) in two groups of 128, and
//              each group is ranked stably into the warp's per-bucket counters —
//              a single check when all its events hit one bucket, the common
//              case for real access streams.  First touches of a bucket append
//              it to the warp's touched list; a warp scan over that list turns
//              the counts into offsets.  Events are written straight to the
//              chunk's 512-event slot of the output, grouped by bucket in trace
//              order, and one {bucket:chunk, start | len << 16} entry per touched
//              bucket is appended (batched per warp) for the replay.
#include "kcommon.cuh"
#include <algorithm>

namespace arb {

constexpr int PT = kPartThreads;            // 512 threads
constexpr int PW = kPartWarps;              // 16 warps
constexpr int WREC = kChunkRecords;         // 256 records per chunk
constexpr int RPL = WREC / 32;              // 8 records per lane (two groups of 4 x 32)
constexpr int kSegBuf = 64;                 // segment entries buffered per warp
constexpr int NST = kPartStages;            // chunks staged per warp (prefetch distance NST - 1)

// per-warp shared memory: stage[NST][WREC] uint4, segbuf[kSegBuf] uint2,
// tlist[2 * WREC] u16, row[NB] u16 (padded to 16 B), bar[NST] u64 (padded to 16 B)
__host__ __device__ constexpr size_t warp_smem_bytes(uint32_t nb) {
  return sizeof(uint4) * NST * WREC + sizeof(uint2) * kSegBuf + 2 * (2 * WREC) + (((size_t)nb * 2 + 15) & ~(size_t)15) +
         ((8 * NST + 15) & ~15);
}

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
                                       bool& two, uint32_t& cvn) {
  const uint32_t op = (q.y >> 16) & 0xFFu;
  const uint32_t len = q.z, hi = q.y & 0xFFFFu;
  // malformed access: len outside 1..8 or the byte range leaving the 48-bit space
  const bool cv = (op & 2u) && (q.y & kCvAddrBit);                // Z26: a CV address (translated first)
  const bool bad_acc = (q.w & 0xFFFFu) != 0 || len - 1u > 7u || (hi == 0xFFFFu && q.x > 0u - len) ||
                       (!(op & 2u) && (q.y & kCvAddrBit));         // host accesses use OV addresses
  const bool ctl = op <= 16 && ((0x1FF00u >> op) & 1u);          // ops 8-16 (11 ARB_BASE, 16 ARB_CV_BASE)
  const bool acc = op < 4;
  flags = valid ? (acc ? (bad_acc ? 2u : 0u) : (ctl ? 1u : 2u)) : 0u;
  bool ok = valid && acc && !bad_acc && !cv;
  if (valid && acc && cv && !bad_acc) ++cvn;
  uint32_t dev = 0;
  if (MD) {                                  // several accelerators (Z24): the device of RT / WT is the arg
    dev = (op & 2u) ? (q.y >> 24) & 0x7Fu : 0u;
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

// The run that ended the warp's previous chunk (warp-uniform): its segment entry is
// still in the warp's buffer (segbuf[idx]), so a run of the next chunk (the warp's
// chunks are consecutive) that continues it — same op, the next word, same bucket —
// extends that entry instead of opening a new one.
struct OpenRun { uint32_t idx, op, bkt, len; uint64_t next_word; };
constexpr uint32_t kNoOpen = 0xFFFFFFFFu;
constexpr uint32_t kMaxRunLen = 0x7FFFu;      // events of a run entry (15-bit length field)

// The fast chunk test and its output.  Every record must be an access (op < 4)
// of 1..8 bytes inside one 8-byte word (such an access cannot leave the
// 48-bit space) in record 0's 2^32-byte block or a neighbouring one (so word
// differences are 32-bit).  A chunk of few runs (below) is written in run form; otherwise all
// words must lie in one address bucket or in two adjacent ones (a stable two-way
// split by the bucket boundary).  Buckets are contiguous word ranges, so the test
// needs only the chunk's lowest and highest word: each word is taken relative to
// record 0's word w0 (32-bit signed, |d| < 2^30), the warp reduces min and max,
// and two bin-map lookups decide.  A word's offset in the bucket is then
// off(lowest) + d - dmin.  Returns false (nothing written) when the test fails.
template <bool MD>
__device__ __forceinline__ bool fast_chunk(const uint4* st, const PartParams& p, uint32_t chunk, uint2* out,
                                           uint2* segbuf, uint32_t& nbuf, uint32_t lane, uint16_t* scratch,
                                           OpenRun& orun, uint32_t& n_merge) {
  const uint4 q0 = st[0];
  const uint64_t w0 = ((uint64_t)((q0.y & 0xFFFFu) >> 3) << 32) | __funnelshift_r(q0.x, q0.y, 3);
  const uint32_t x0w = __funnelshift_r(q0.x, q0.y, 3);        // record 0's word, low 32 bits
  const uint32_t h0 = (q0.y & 0xFFFFu) - 1u;                   // record 0's address bits 32-47, minus 1
  uint32_t d[RPL], opk[RPL], bad = 0, devs = 0;
  int32_t dmin = 0, dmax = 0;
#pragma unroll
  for (int k = 0; k < RPL; ++k) {
    const uint4 q = st[k * 32 + lane];
    // an access (op < 4, OV address) of 1..8 bytes inside one word, whose address
    // bits 32-47 are record 0's, or one more or less: its word is then record 0's
    // word + d with |d| < 2^30, d = the difference of the words' low 32 bits
    bad |= (q.y & (0x00FC0000u | kCvAddrBit)) | (q.w & 0xFFFFu) | ((q.y & 0xFFFFu) - h0 > 2u) |
           (((q.z - 1u) | ((q.x & 7u) + q.z - 1u)) & ~7u);
    if (MD && (q.y & (1u << 17))) {                // RT / WT on device arg (Z24)
      const uint32_t dv = q.y >> 24;
      bad |= dv >= p.n_dev;
      devs |= (dv & 3u) << (2 * k);
    }
    d[k] = __funnelshift_r(q.x, q.y, 3) - x0w;
    dmin = min(dmin, (int32_t)d[k]);
    dmax = max(dmax, (int32_t)d[k]);
    opk[k] = ((q.y >> 16) & 3u) << 30;
  }
  const OpenRun prev = orun;
  orun.idx = kNoOpen;                        // reset unless the chunk ends in a run
  if (!__all_sync(FULL, bad == 0)) return false;
  dmin = __reduce_min_sync(FULL, dmin);
  dmax = __reduce_max_sync(FULL, dmax);
  const uint64_t rlo = w0 - p.base_word + (uint64_t)(int64_t)dmin;   // wraps below the range
  const uint64_t rhi = w0 - p.base_word + (uint64_t)(int64_t)dmax;
  if (rlo >= p.n_words || rhi >= p.n_words) return false;
  const uint32_t cb = p.coarse_bits;
  const uint32_t rec0 = chunk * (uint32_t)WREC;
  const uint32_t chi = (chunk >> kSegChunkBits) << 31;
  if (!MD && !p.no_runs && (uint32_t)(dmax - dmin) < (1u << 28)) {
    // ---- run form: a run = consecutive records with the same op on
    // consecutive words (event j of the run: word + j, position + j).  Record i's
    // key (d_i - i) << 3 | op << 1 is constant along a run (exact: |d| spans < 2^28);
    // a run starts where the key changes.  A chunk of <= kMaxChunkRuns runs, each
    // inside one bucket (any buckets) or split at the boundary of two adjacent ones,
    // writes one 8-B descriptor (the piece's first event, at the slot of its first
    // record) and one segment entry (start flagged kRunFlag) per piece instead of 8 B
    // per record.
    uint32_t sm[RPL], nR = 0, rprev = 0;
#pragma unroll
    for (int k = 0; k < RPL; ++k) {
      const uint32_t key = ((d[k] - (uint32_t)(k * 32) - lane) << 3) | (opk[k] >> 29);
      const uint32_t r = __shfl_sync(FULL, key, (lane + 31) & 31);    // lane L: key of lane L - 1
      const uint32_t prev = lane ? r : rprev;                          // lane 0: lane 31 of round k - 1
      rprev = __shfl_sync(FULL, r, 0);
      sm[k] = __ballot_sync(FULL, (k == 0 && lane == 0) || key != prev);
      nR += __popc(sm[k]);
    }
    if (nR <= (uint32_t)kMaxChunkRuns) {
      uint32_t* kb = reinterpret_cast<uint32_t*>(scratch);             // [0, 16): record index, [16, 32): key
      const uint32_t lt = lanemask_lt();
      uint32_t before = 0;
#pragma unroll
      for (int k = 0; k < RPL; ++k) {
        if (sm[k]) {
          if ((sm[k] >> lane) & 1u) {
            const uint32_t rk = before + __popc(sm[k] & lt);
            kb[rk] = k * 32 + lane;
            kb[kMaxChunkRuns + rk] = ((d[k] - (uint32_t)(k * 32) - lane) << 2) | (opk[k] >> 30);
          }
          before += __popc(sm[k]);
        }
      }
      __syncwarp();
      // lane r: run r, inside one bucket or split at the boundary of two adjacent ones
      bool ok = true, split = false;
      uint32_t i = 0, len = 0, len1 = 0, bkt = 0, off = 0, opr = 0;
      uint64_t first = 0;
      if (lane < nR) {
        i = kb[lane];
        len = (lane + 1 < nR ? kb[lane + 1] : (uint32_t)WREC) - i;
        const uint32_t kv = kb[kMaxChunkRuns + lane];
        opr = kv & 3u;
        first = w0 - p.base_word + (uint64_t)(int64_t)((int32_t)kv >> 2) + i;   // d_i = v + i
        const uint64_t last = first + len - 1;
        const uint32_t m1 = __ldg(p.bin_map + (uint32_t)(first >> cb)), m2 = __ldg(p.bin_map + (uint32_t)(last >> cb));
        bkt = m1 & kBucketMask;
        const uint32_t b2 = m2 & kBucketMask;
        split = b2 == bkt + 1;
        ok = b2 == bkt || split;
        len1 = len;
        if (split) len1 = (uint32_t)((((last >> cb) - (uint64_t)(m2 >> kBucketBits)) << cb) - first);
        off = ((m1 >> kBucketBits) << cb) | ((uint32_t)first & ((1u << cb) - 1u));
      }
      __syncwarp();
      if (__all_sync(FULL, ok)) {
        const uint32_t sp = __ballot_sync(FULL, split);
        // run 0 continues the previous chunk's open run?
        const uint32_t mg = __shfl_sync(FULL, (uint32_t)(lane == 0 && prev.idx != kNoOpen && opr == prev.op &&
                                                         first == prev.next_word && bkt == prev.bkt &&
                                                         prev.len + len1 <= kMaxRunLen), 0);
        const uint32_t e = nbuf + lane + __popc(sp & lanemask_lt()) - mg;   // entry of this run's first piece
        if (lane < nR) {
          const uint32_t ck = chunk & ((1u << kSegChunkBits) - 1u);
          if (lane == 0 && mg) {
            segbuf[prev.idx].y += len1 << 16;
          } else {
            out[i] = make_uint2((opr << 30) | off, rec0 + i);
            segbuf[e] = make_uint2((bkt << kSegChunkBits) | ck, i | kRunFlag | (len1 << 16) | chi);
          }
          if (split) {                     // the rest starts at the first word of bucket bkt + 1
            out[i + len1] = make_uint2(opr << 30, rec0 + i + len1);
            segbuf[e + 1] = make_uint2(((bkt + 1) << kSegChunkBits) | ck, (i + len1) | kRunFlag | ((len - len1) << 16) | chi);
          }
        }
        // the chunk's last piece stays open for the next chunk
        const uint32_t L = nR - 1;
        const uint32_t oi = (L == 0 && mg && !split) ? prev.idx : e + (split ? 1u : 0u);
        const uint32_t ol = (L == 0 && mg && !split) ? prev.len + len1 : (split ? len - len1 : len1);
        orun.idx = __shfl_sync(FULL, oi, L);
        orun.len = __shfl_sync(FULL, ol, L);
        orun.op = __shfl_sync(FULL, opr, L);
        orun.bkt = __shfl_sync(FULL, split ? bkt + 1 : bkt, L);
        orun.next_word = __shfl_sync(FULL, first + len, L);
        nbuf += nR + __popc(sp) - mg;
        n_merge += mg;
        return true;
      }
    }
  }
  const uint32_t mlo = __ldg(p.bin_map + (uint32_t)(rlo >> cb)), mhi = __ldg(p.bin_map + (uint32_t)(rhi >> cb));
  const uint32_t bref = mlo & kBucketMask, bhi = mhi & kBucketMask;
  if (bhi != bref && bhi != bref + 1) return false;
  const uint32_t c = (((mlo >> kBucketBits) << cb) | ((uint32_t)rlo & ((1u << cb) - 1u))) - (uint32_t)dmin;
  const uint32_t ck = (bref << kSegChunkBits) | (chunk & ((1u << kSegChunkBits) - 1u));
  // Two adjacent buckets (a run crossing a bucket boundary, or two runs on either
  // side of it).  Bucket bhi starts at the first coarse bin of bhi, boundary =
  // (bin(rhi) - bin offset of rhi in bhi) << cb (relative word); a record is in bhi
  // iff d >= tb; its offset in bhi is d + cB.
  int32_t tb = 0x7FFFFFFF;
  uint32_t cB = 0;
  if (bhi != bref) {
    const uint64_t boundary = ((rhi >> cb) - (uint64_t)(mhi >> kBucketBits)) << cb;
    const uint64_t r0w = w0 - p.base_word;
    tb = (int32_t)(uint32_t)(boundary - r0w);
    cB = (uint32_t)(r0w - boundary);
  }
  if (bhi == bref) {
#pragma unroll
    for (int k = 0; k < RPL; ++k)
      out[k * 32 + lane] = make_uint2(opk[k] | (d[k] + c),
                                      (rec0 + k * 32 + lane) | (MD ? ((devs >> (2 * k)) & 3u) << 30 : 0u));
    if (lane == 0) segbuf[nbuf] = make_uint2(ck, (uint32_t)WREC << 16 | chi);
    ++nbuf;
    return true;
  }
  // Two adjacent buckets: stable two-way split, the bref events first, then the
  // bhi events, each in record order.
  uint32_t bm[RPL], nB = 0;
#pragma unroll
  for (int k = 0; k < RPL; ++k) {
    bm[k] = __ballot_sync(FULL, (int32_t)d[k] >= tb);
    nB += __popc(bm[k]);
  }
  const uint32_t nA = WREC - nB, lt = lanemask_lt();
  uint32_t runA = 0, runB = nA;
#pragma unroll
  for (int k = 0; k < RPL; ++k) {
    const bool isB = (bm[k] >> lane) & 1u;
    const uint32_t o = isB ? runB + __popc(bm[k] & lt) : runA + __popc(~bm[k] & lt);
    out[o] = make_uint2(opk[k] | (d[k] + (isB ? cB : c)),
                        (rec0 + k * 32 + lane) | (MD ? ((devs >> (2 * k)) & 3u) << 30 : 0u));
    runB += __popc(bm[k]);
    runA += 32 - __popc(bm[k]);
  }
  if (lane == 0) {
    segbuf[nbuf] = make_uint2(ck, nA << 16 | chi);
    segbuf[nbuf + 1] = make_uint2(ck + (1u << kSegChunkBits), nA | (nB << 16) | chi);
  }
  nbuf += 2;
  return true;
}

// MD: several accelerators (Z24) — the device of RT / WT goes to bits 30-31 of the
// event position; a separate instance so that the single-device kernel is unchanged
template <bool MD>
__global__ void __launch_bounds__(PT, 1) k_partition(PartParams p) {
  extern __shared__ __align__(16) uint8_t smem[];
  const uint32_t NB = p.n_buckets;
  const uint32_t lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const uint32_t lt = lanemask_lt();
  uint8_t* wbase = smem + warp * warp_smem_bytes(NB);
  uint4* stage = reinterpret_cast<uint4*>(wbase);                   // [2][WREC]
  uint2* segbuf = reinterpret_cast<uint2*>(stage + NST * WREC);     // [kSegBuf]
  uint16_t* tlist = reinterpret_cast<uint16_t*>(segbuf + kSegBuf);   // [2 * WREC]
  uint16_t* row = tlist + 2 * WREC;                                  // [NB]
  uint64_t* bar = reinterpret_cast<uint64_t*>(row + ((NB + 7) & ~7u));   // [NST]
  for (uint32_t i = lane; i < NB; i += 32) row[i] = 0;
  if (lane < NST) mbar_init(bar + lane, 1);
  fence_mbar_init();
  __syncwarp();
  uint32_t n_acc = 0, n_ign = 0, n_cv = 0, nbuf = 0, phase = 0;   // phase: parity bit of each stage's barrier
  uint32_t n_fast = 0, n_runc = 0, n_merge = 0;                    // chunks: fast path / ending in an open run

  // the chunk's records arrive in stage k by one TMA bulk copy (lane 0) that
  // completes on bar[k]
  // The warp's chunks: blocks of kChunkBlock (64) consecutive chunks taken from a ticket
  // counter — consecutive chunks let runs continue from one chunk into the next
  // (OpenRun), tickets balance the warps (general chunks cost ~10x a run chunk and
  // cluster in parts of a trace).  The segment sort keys entries by block (chunk /
  // kChunkBlock): a block's entries are in chunk order in the output.
  auto take = [&]() -> uint64_t {
    unsigned long long t = 0;
    if (lane == 0) t = atomicAdd(&p.st->part_ticket, 1ull);
    return (uint64_t)__shfl_sync(FULL, t, 0) * kChunkBlock;
  };
  auto fetch = [&](uint64_t c, uint32_t k) {
    if (c < p.n_chunks && lane == 0) {
      const uint64_t r0 = c * WREC;
      const uint32_t nv = p.n - r0 < (uint64_t)WREC ? (uint32_t)(p.n - r0) : (uint32_t)WREC;
      mbar_arrive_tx(bar + k, nv * 16u);
      bulk_g2s(stage + k * WREC, p.ev + r0, nv * 16u, bar + k);
    }
  };
  auto flush_segs = [&]() {
    __syncwarp();
    unsigned long long sb = 0;
    if (lane == 0 && nbuf) sb = atomicAdd(&p.st->n_segs, (unsigned long long)nbuf);
    sb = __shfl_sync(FULL, sb, 0);
    for (uint32_t i = lane; i < nbuf; i += 32)
      if (sb + i < p.seg_cap) p.seg_out[sb + i] = segbuf[i];
    __syncwarp();
    nbuf = 0;
  };
  OpenRun orun;
  orun.idx = kNoOpen; orun.op = orun.bkt = orun.len = 0; orun.next_word = 0;

  static_assert(NST == 2, "prefetch distance 1 (the next chunk may start another block)");
  uint32_t cur = 0;
  uint64_t chunk = take();
  uint64_t blk_end = chunk + kChunkBlock < p.n_chunks ? chunk + kChunkBlock : p.n_chunks;
  uint64_t next_blk = take();
  fetch(chunk, 0);
  auto advance = [&]() -> uint64_t {           // the warp's next chunk
    if (chunk + 1 < blk_end) return chunk + 1;
    const uint64_t c = next_blk;
    blk_end = c + kChunkBlock < p.n_chunks ? c + kChunkBlock : p.n_chunks;
    next_blk = take();
    orun.idx = kNoOpen;                        // not consecutive: no run continues into it
    return c;
  };
  for (; chunk < p.n_chunks; chunk = advance()) {
    fetch(chunk + 1 < blk_end ? chunk + 1 : next_blk, cur ^ 1u);
    mbar_wait(bar + cur, (phase >> cur) & 1u);
    phase ^= 1u << cur;
    const uint4* st = stage + cur * WREC;
    const uint64_t rec0 = chunk * WREC;
    const uint32_t nvalid = p.n - rec0 < (uint64_t)WREC ? (uint32_t)(p.n - rec0) : (uint32_t)WREC;
    // ---- fast chunk: 256 single-word tracked accesses of one bucket or two adjacent
    // ones (the common case of real access streams: runs over one array).  One bucket:
    // event j is record j, one coalesced store per record, one segment entry; two:
    // a stable two-way split and two entries.  Anything else takes the general path.
    if (nbuf + 2 * kMaxChunkRuns > kSegBuf) {
      if (orun.idx != kNoOpen) {         // keep the open run's entry (the last one) in the buffer
        const uint2 keep = segbuf[nbuf - 1];
        --nbuf;
        flush_segs();
        if (lane == 0) segbuf[0] = keep;
        __syncwarp();
        nbuf = 1; orun.idx = 0;
      } else {
        flush_segs();
      }
    }
    if (nvalid < WREC) orun.idx = kNoOpen;
    if (nvalid == WREC && fast_chunk<MD>(st, p, (uint32_t)chunk, p.part_ev + chunk * kChunkCap,
                                     segbuf, nbuf, lane, tlist, orun, n_merge)) {
      n_fast += 1u;
      n_runc += orun.idx != kNoOpen;
      n_acc += RPL;
      cur = cur + 1 == NST ? 0 : cur + 1;
      __syncwarp();                    // stage[cur] reads done before the next fetch overwrites it
      continue;
    }
    uint32_t nT = 0, e_lane = 0;
    // ---- pass A: decode + rank, 2 groups of 4 x 32 records ----------------------------
    Dec dec[RPL];
    uint32_t rk[RPL];
    bool any2 = false;                 // some record of the chunk has two words
#pragma unroll
    for (int g = 0; g < 2; ++g) {
      uint32_t any_flag = 0, twos = 0;
#pragma unroll
      for (int k = 0; k < 4; ++k) {
        const uint32_t j = g * 128 + k * 32 + lane;
        uint32_t flags;
        bool two;
        dec[g * 4 + k] = decode0<MD>(st[j], j < nvalid, p, n_ign, flags, two, n_cv);
        any_flag |= flags << (2 * k);
        twos |= (uint32_t)two << k;
      }
      if (__any_sync(FULL, twos != 0)) {
        any2 = true;
#pragma unroll
        for (int k = 0; k < 4; ++k)
          if ((twos >> k) & 1u) decode1<MD>(dec[g * 4 + k], st[g * 128 + k * 32 + lane], p, n_ign);
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
                const uint4 q = st[j];
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
    __syncwarp();
    // ---- counts -> offsets over the touched list; segment entries ------------------------
    uint2* out = p.part_ev + chunk * kChunkCap;
    uint32_t carry = 0;
    for (uint32_t t0 = 0; t0 < nT; t0 += 32) {
      const uint32_t t = t0 + lane;
      uint32_t b = 0, tot = 0;
      if (t < nT) { b = tlist[t]; tot = row[b]; }
      const uint32_t len = tot;
      uint32_t incl = len;
#pragma unroll
      for (int d = 1; d < 32; d <<= 1) {
        const uint32_t o = __shfl_up_sync(FULL, incl, d);
        if (lane >= (uint32_t)d) incl += o;
      }
      const uint32_t start = carry + incl - len;
      carry += __shfl_sync(FULL, incl, 31);
      const uint32_t n_new = min(32u, nT - t0);
      if (nbuf + n_new > kSegBuf) flush_segs();
      if (t < nT) {
        row[b] = (uint16_t)start;
        segbuf[nbuf + lane] = make_uint2((b << kSegChunkBits) | ((uint32_t)chunk & ((1u << kSegChunkBits) - 1u)),
                                         start | (len << 16) | (((uint32_t)chunk >> kSegChunkBits) << 31));
      }
      nbuf += n_new;
    }
    __syncwarp();
    // ---- pass B: write the events straight to the chunk's output slot ----------------------
    const uint32_t pos0 = (uint32_t)rec0 + lane;
#pragma unroll
    for (int r = 0; r < RPL; ++r) {
      const uint32_t info = dec[r].info;
      const uint32_t pos = (pos0 + (r >> 2) * 128 + (r & 3) * 32) | (MD ? (info >> 24) << 30 : 0u);   // | device
      if (info & 3u) out[row[(info >> 2) & kBucketMask] + (rk[r] & 0xFFFFu)] = make_uint2(dec[r].k0, pos);
    }
    if (any2) {
#pragma unroll
      for (int r = 0; r < RPL; ++r) {
        const uint32_t info = dec[r].info;
        const uint32_t pos = (pos0 + (r >> 2) * 128 + (r & 3) * 32) | (MD ? (info >> 24) << 30 : 0u);
        if ((info & 3u) == 2u) out[row[(info >> kB1Shift) & kBucketMask] + (rk[r] >> 16)] = make_uint2(dec[r].k1, pos);
      }
    }
    __syncwarp();
    for (uint32_t t = lane; t < nT; t += 32) row[tlist[t]] = 0;
    n_acc += e_lane;
    cur = cur + 1 == NST ? 0 : cur + 1;
    __syncwarp();                      // stage[cur] reads and row resets done before reuse
  }
  flush_segs();

#pragma unroll
  for (int d = 16; d; d >>= 1) {
    n_acc += __shfl_xor_sync(FULL, n_acc, d);
    n_ign += __shfl_xor_sync(FULL, n_ign, d);
    n_cv += __shfl_xor_sync(FULL, n_cv, d);
  }
  if (lane == 0) {
    if (n_acc) atomicAdd(&p.st->access_words, (unsigned long long)n_acc);
    if (n_ign) atomicAdd(&p.st->ignored_words, (unsigned long long)n_ign);
    if (n_cv) atomicAdd(&p.st->n_cv_acc, (unsigned long long)n_cv);
    if (n_fast) atomicAdd(&p.st->chunks_fast, (unsigned long long)n_fast);
    if (n_runc) atomicAdd(&p.st->chunks_run, (unsigned long long)n_runc);
    if (n_merge) atomicAdd(&p.st->run_merges, (unsigned long long)n_merge);
  }
}

cudaError_t launch_partition(const PartParams& p, cudaStream_t s) {
  if (p.n_chunks == 0) return cudaSuccess;
  const size_t smem = PW * warp_smem_bytes(p.n_buckets);
  auto kern = p.n_dev > 1 ? k_partition<true> : k_partition<false>;
  cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  kern<<<p.grid, PT, smem, s>>>(p);
  return cudaGetLastError();
}

}  // namespace arb
