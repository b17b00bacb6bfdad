// mir.cu — MIR join kernels (Theorem 1; reading Z10 of DESIGN.md).
#include "kcommon.cuh"

namespace arb {

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

// N2: the access summaries of instances carried in from earlier flushes enter
// the hash like their records would, and (iii) window range ops covering them race.
__global__ void k_mir_carry_insert(MirParams p) {
  for (uint64_t g = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; g < p.n_carry;
       g += (uint64_t)gridDim.x * blockDim.x) {
    const uint4 e = p.carry[g];
    const uint32_t qd = p.cmap[e.z];
    if (qd == 0xFFFFFFFFu) continue;            // joined before this flush's first record
    const uint64_t w = (uint64_t)e.x | ((uint64_t)e.y << 32);
    unsigned long long key = ((unsigned long long)w << 20) | (qd + 1);
    uint64_t h = hslot(key, p.hmask);
    for (;;) {
      unsigned long long old = atomicCAS(&p.hkeys[h], 0ull, key);
      if (old == 0ull || old == key) break;
      h = (h + 1) & p.hmask;
    }
    if (e.w) atomicOr(&p.hvals[h], 1u);
    for (uint32_t j = p.win_start[qd]; j < p.win_start[qd + 1]; ++j) {
      RangeRef rr = p.win_ops[j];
      if (w >= rr.lo && w < rr.hi) emit_mir(p, w, rr.pos);
    }
  }
}

// N2: summaries of the instances carried out of this flush
__global__ void k_mir_carry_extract(const unsigned long long* hkeys, const uint32_t* hvals, uint64_t hcap,
                                    const uint32_t* co_of, uint4* out, unsigned long long* n_out) {
  for (uint64_t h = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; h < hcap;
       h += (uint64_t)gridDim.x * blockDim.x) {
    const unsigned long long key = hkeys[h];
    if (!key) continue;
    const uint32_t co = co_of[(uint32_t)(key & 0xFFFFFu) - 1];
    if (co == 0xFFFFFFFFu) continue;
    const uint64_t w = key >> 20;
    const unsigned long long slot = atomicAdd(n_out, 1ull);
    out[slot] = make_uint4((uint32_t)w, (uint32_t)(w >> 32), co, hvals[h] & 1u);
  }
}

cudaError_t launch_carry_extract(const unsigned long long* hkeys, const uint32_t* hvals, uint64_t hcap,
                                 const uint32_t* co_of, uint4* out, unsigned long long* n_out, cudaStream_t s) {
  const uint64_t g = (hcap + 255) / 256;
  k_mir_carry_extract<<<(unsigned)(g > 148 * 64 ? 148 * 64 : (g ? g : 1)), 256, 0, s>>>(hkeys, hvals, hcap, co_of,
                                                                                        out, n_out);
  return cudaGetLastError();
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
  if (p.n_carry) { k_mir_carry_insert<<<grid(p.n_carry), 256, 0, s>>>(p); ++*launches; }
  if (n_qry_pos) { k_mir_query<<<grid(n_qry_pos), 256, 0, s>>>(p, n_qry_pos); ++*launches; }
  if (n_rr_words) { k_mir_ranges<<<grid(n_rr_words), 256, 0, s>>>(p, n_rr_words); ++*launches; }
  return cudaGetLastError();
}

// ---- N1 (Z25): accesses through a tagged pointer outside its base's entry ----
__global__ void k_bo_tags(const uint4* ev, uint64_t n, uint64_t base_word, uint64_t n_words,
                          const uint32_t* tag_first, const TagSeg* segs, uint4* cand, uint64_t cand_cap,
                          unsigned long long* count) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x) {
    const uint4 q = ld_stream(ev + i);
    const uint32_t op = (q.y >> 16) & 0xFFu, tag = q.w >> 16;
    if ((op != OP_RT && op != OP_WT) || tag == 0) continue;
    uint32_t a = __ldg(tag_first + tag), z = __ldg(tag_first + tag + 1);
    if (a == z || segs[a].pos > (uint32_t)i) continue;        // no base defined yet
    while (z - a > 1) {                                        // last segment starting at or before i
      const uint32_t mid = (a + z) >> 1;
      if (segs[mid].pos <= (uint32_t)i) a = mid; else z = mid;
    }
    const uint64_t lo = segs[a].lo, hi = segs[a].hi;
    const uint64_t addr = (uint64_t)q.x | ((uint64_t)(q.y & 0xFFFFu) << 32), len = q.z;
    const uint64_t w0 = addr >> 3, w1 = (addr + len - 1) >> 3;
    for (uint64_t x = w0; x <= w1; ++x) {
      if (x < base_word || x - base_word >= n_words || (x >= lo && x < hi)) continue;
      const unsigned long long slot = atomicAdd(count, 1ull);
      if (slot < cand_cap) {
        const uint64_t r = x - base_word;
        cand[slot] = make_uint4((uint32_t)r, (uint32_t)(r >> 32), (uint32_t)i, 4u);   // ARB_BO
      }
    }
  }
}

cudaError_t launch_bo_tags(const uint4* ev, uint64_t n, uint64_t base_word, uint64_t n_words,
                           const uint32_t* tag_first, const TagSeg* segs, uint4* cand, uint64_t cand_cap,
                           unsigned long long* count, cudaStream_t s) {
  if (!n) return cudaSuccess;
  const uint64_t g = (n + 255) / 256;
  k_bo_tags<<<(unsigned)std::min<uint64_t>(g, 148 * 16), 256, 0, s>>>(ev, n, base_word, n_words, tag_first, segs,
                                                                     cand, cand_cap, count);
  return cudaGetLastError();
}

// ---- N1 (Z26): CV -> OV translation of device-addressed target accesses ----------
__global__ void k_cv_translate(const uint4* in, uint4* out, uint64_t n, const uint32_t* epoch_pos,
                               const uint32_t* epoch_first, uint32_t n_epochs, const CvPlace* place) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x) {
    uint4 q = ld_stream(in + i);
    const uint32_t op = (q.y >> 16) & 0xFFu;
    if ((op == OP_RT || op == OP_WT) && (q.y & kCvAddrBit)) {
      uint32_t a = 0, z = n_epochs;                       // the epoch holding position i
      while (z - a > 1) {
        const uint32_t mid = (a + z) >> 1;
        if (epoch_pos[mid] <= (uint32_t)i) a = mid; else z = mid;
      }
      uint32_t lo = epoch_first[a], hi = epoch_first[a + 1];
      const uint64_t y = (uint64_t)q.x | ((uint64_t)(q.y & 0xFFFFu) << 32);
      while (hi - lo > 1) {                                // the last placement starting at or before y
        const uint32_t mid = (lo + hi) >> 1;
        if (place[mid].cv_lo <= y) lo = mid; else hi = mid;
      }
      if (lo < epoch_first[a + 1] && place[lo].cv_lo <= y && y < place[lo].cv_hi) {
        const uint64_t x = place[lo].ov_lo + (y - place[lo].cv_lo);
        q.x = (uint32_t)x;
        q.y = (q.y & 0x7FFF0000u) | (uint32_t)((x >> 32) & 0xFFFFu);   // OV address, CV flag cleared
      }
    }
    out[i] = q;
  }
}

cudaError_t launch_cv_translate(const uint4* in, uint4* out, uint64_t n, const uint32_t* epoch_pos,
                                const uint32_t* epoch_first, uint32_t n_epochs, const CvPlace* place,
                                cudaStream_t s) {
  if (!n) return cudaSuccess;
  k_cv_translate<<<(unsigned)std::min<uint64_t>((n + 255) / 256, 148 * 16), 256, 0, s>>>(in, out, n, epoch_pos,
                                                                                        epoch_first, n_epochs, place);
  return cudaGetLastError();
}

}  // namespace arb
