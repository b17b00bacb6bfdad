// arbgen.cuh — counter-based synthetic trace generator (host and device).
//
// Part of the input-generator module (gen/), shared by tests, bench and both
// sides of the parity check.  It writes trace records from a
// small table of segments; record i is a pure function of (table, i), keyed
// by splitmix64, so host and device produce identical bytes.  It contains none
// of the method's arithmetic.
#pragma once
#include <stdint.h>

#if defined(__CUDACC__)
#define AG_HD __host__ __device__ __forceinline__
#else
#define AG_HD inline
#endif

namespace arbgen {

enum SegType : uint32_t { SEG_LIT = 0, SEG_LOOP = 1, SEG_RUNS = 2 };
enum Mode : uint32_t { M_LINEAR = 0, M_2D = 1, M_RANDOM = 2, M_SKEW = 3 };

// one entry of a loop body: record b of iteration t
struct GenEntry {
  uint32_t op, size, mode, pad;
  uint64_t base;     // byte address
  uint64_t stride;   // bytes per step (LINEAR, 2D column, RANDOM/SKEW element)
  uint64_t range;    // 2D: row pitch in bytes; RANDOM/SKEW: number of elements
};

struct GenSeg {
  uint64_t start;    // first global record index
  uint64_t count;    // number of records
  uint32_t type;     // SegType
  uint32_t body_len; // LOOP: entries per iteration
  uint32_t body_off; // LOOP: first entry; LIT: first literal record
  uint32_t width;    // LOOP 2D: columns per row
  uint64_t t0;       // LOOP: first iteration
  uint64_t seed;
  // RUNS: p0 = first word of the section, p1 = span of run starts (words),
  //       p2 = run length L, p3 = kind (0 device WT,RT,RT; 1 host WH,RH,RH)
  //       p4 = paired device-run seed, p5 = overlap runs (MIR injection),
  //       p6 = stale-run rate (1 in p6 host runs reads a device run; 0 = never)
  uint64_t p0, p1, p2, p3, p4, p5, p6, p7;
};

AG_HD uint64_t splitmix64(uint64_t x) {
  x += 0x9E3779B97F4A7C15ull;
  uint64_t z = x;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}
AG_HD uint64_t rng(uint64_t seed, uint64_t ctr) { return splitmix64(seed * 0x632BE59BD9B4E019ull + ctr); }

AG_HD void encode(uint32_t op, uint64_t addr, uint64_t len, uint64_t* w0, uint64_t* w1) {
  *w0 = (addr & ((1ull << 48) - 1)) | ((uint64_t)op << 48);
  *w1 = len;
}

// record `j` (local index) of a LOOP segment
AG_HD void gen_loop(const GenSeg& s, const GenEntry* ent, uint64_t j, uint64_t* w0, uint64_t* w1) {
  uint64_t t = s.t0 + j / s.body_len;
  uint32_t b = (uint32_t)(j % s.body_len);
  const GenEntry& e = ent[s.body_off + b];
  uint64_t addr;
  switch (e.mode) {
    case M_2D: addr = e.base + (t / s.width) * e.range + (t % s.width) * e.stride; break;
    case M_RANDOM: addr = e.base + (rng(s.seed + b, t) % e.range) * e.stride; break;
    case M_SKEW: {
      uint64_t h1 = rng(s.seed + b, t), h2 = rng(s.seed + b + 977, t);
      addr = e.base + (h1 % (1 + h2 % e.range)) * e.stride;
      break;
    }
    default: addr = e.base + t * e.stride; break;
  }
  encode(e.op, addr, e.size, w0, w1);
}

// record `j` of a RUNS segment (config 5 group bodies)
AG_HD void gen_runs(const GenSeg& s, uint64_t j, uint64_t* w0, uint64_t* w1) {
  const uint64_t L = s.p2;
  uint64_t run = j / (3 * L);
  uint32_t phase = (uint32_t)((j / L) % 3);
  uint64_t k = j % L;
  uint64_t start = s.p0 + rng(s.seed, run) % s.p1;
  uint32_t op;
  if (s.p3 == 0) {
    op = phase == 0 ? 3u : 2u;                           // WT, RT, RT
  } else {
    op = phase == 0 ? 1u : 0u;                           // WH, RH, RH
    bool overlap = run < s.p5;                           // host run over a device run: race if not joined
    bool stale = s.p6 && (rng(s.seed ^ 0x5A5Aull, run) % s.p6) == 0;
    if (overlap || stale) start = s.p0 + rng(s.p4, run) % s.p1;
    if (stale) op = 0u;                                  // RH only: reads the device-written words
  }
  encode(op, (start + k) * 8, 8, w0, w1);
}

AG_HD uint32_t find_seg(const GenSeg* segs, uint32_t n, uint64_t i) {
  uint32_t a = 0, z = n;             // last seg with start <= i
  while (z - a > 1) { uint32_t m = (a + z) >> 1; if (segs[m].start <= i) a = m; else z = m; }
  return a;
}

AG_HD void gen_record(const GenSeg* segs, uint32_t nseg, const GenEntry* ent, const uint64_t* lit,
                      uint64_t i, uint64_t* w0, uint64_t* w1) {
  const GenSeg& s = segs[find_seg(segs, nseg, i)];
  uint64_t j = i - s.start;
  switch (s.type) {
    case SEG_LIT: *w0 = lit[2 * (s.body_off + j)]; *w1 = lit[2 * (s.body_off + j) + 1]; break;
    case SEG_RUNS: gen_runs(s, j, w0, w1); break;
    default: gen_loop(s, ent, j, w0, w1); break;
  }
}

}  // namespace arbgen
