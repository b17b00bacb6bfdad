// api.cpp — the C ABI of libarbalest (include/arbalest.h).
#include "arbalest.h"
#include "arb_internal.h"
#include "control.h"

#include <dlfcn.h>
#include <algorithm>
#include <chrono>
#include <cmath>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <new>
#include <string>
#include <vector>

using namespace arb;

namespace {

// ---- NCCL through dlopen (only needed when world > 1) ---------------------
// ncclUniqueId is a 128-byte struct passed by value
struct NcclId { char internal[128]; };
typedef int (*nccl_init_fn)(void** comm, int nranks, NcclId id, int rank);
typedef int (*nccl_allgather_fn)(const void* send, void* recv, size_t count, int dtype, void* comm, cudaStream_t s);
typedef int (*nccl_destroy_fn)(void* comm);
typedef int (*nccl_count_fn)(const void* comm, int* count);
constexpr int kNcclInt64 = 4;   // ncclInt64

template <class T>
struct DevBuf {
  T* p = nullptr;
  size_t cap = 0;
  cudaError_t ensure(size_t n) {
    if (n <= cap) return cudaSuccess;
    size_t c = std::max(n, (size_t)(cap * 3 / 2));
    if (p) cudaFree(p);
    p = nullptr; cap = 0;
    cudaError_t e = cudaMalloc(&p, c * sizeof(T) + 16);
    if (e == cudaSuccess) cap = c;
    return e;
  }
  // grow keeping the first `keep` elements (staging buffers filled across submits)
  cudaError_t ensure_keep(size_t n, size_t keep) {
    if (n <= cap) return cudaSuccess;
    size_t c = std::max(n, (size_t)(cap * 3 / 2));
    T* q = nullptr;
    cudaError_t e = cudaMalloc(&q, c * sizeof(T) + 16);
    if (e != cudaSuccess) return e;
    keep = std::min(keep, cap);
    if (p && keep) e = cudaMemcpy(q, p, keep * sizeof(T), cudaMemcpyDeviceToDevice);
    if (p) cudaFree(p);
    p = q; cap = c;
    return e;
  }
  void release() { if (p) cudaFree(p); p = nullptr; cap = 0; }
};

template <class T>
cudaError_t upload(DevBuf<T>& b, const std::vector<T>& v, cudaStream_t s) {
  cudaError_t e = b.ensure(std::max<size_t>(v.size(), 1));
  if (e != cudaSuccess || v.empty()) return e;
  return cudaMemcpyAsync(b.p, v.data(), v.size() * sizeof(T), cudaMemcpyHostToDevice, s);
}

// gidx: device global indices (on_device), or host ones read on the report path only
struct Submit { const void* ev; uint64_t n; const uint64_t* gidx; int on_device; };

// pinned host buffer (async copies, no staging through pageable memory)
template <class T>
struct HostBuf {
  T* p = nullptr;
  size_t cap = 0;
  cudaError_t ensure(size_t n) {
    if (n <= cap) return cudaSuccess;
    size_t c = std::max(n, (size_t)(cap * 3 / 2));
    if (p) cudaFreeHost(p);
    p = nullptr; cap = 0;
    cudaError_t e = cudaMallocHost(&p, c * sizeof(T));
    if (e == cudaSuccess) cap = c;
    return e;
  }
  void release() { if (p) cudaFreeHost(p); p = nullptr; cap = 0; }
};

// upload through a pinned staging buffer; the staging buffer is reused only
// after the flush's final stream synchronisation
template <class T>
cudaError_t upload_pinned(DevBuf<T>& b, HostBuf<T>& h, const std::vector<T>& v, cudaStream_t s) {
  cudaError_t e = b.ensure(std::max<size_t>(v.size(), 1));
  if (e != cudaSuccess || v.empty()) return e;
  if ((e = h.ensure(v.size())) != cudaSuccess) return e;
  std::memcpy(h.p, v.data(), v.size() * sizeof(T));
  return cudaMemcpyAsync(b.p, h.p, v.size() * sizeof(T), cudaMemcpyHostToDevice, s);
}

// Several host vectors in one pinned staging buffer and one H2D copy into one device
// buffer (16-B aligned parts); `at` gives a part's device address.
struct PackUpload {
  struct Part { const void* src; size_t bytes, off; };
  std::vector<Part> parts;
  size_t total = 0;
  template <class T>
  size_t add(const std::vector<T>& v) {
    const size_t o = total, b = v.size() * sizeof(T);
    parts.push_back({v.data(), b, o});
    total += (std::max<size_t>(b, 1) + 15) & ~(size_t)15;
    return o;
  }
  cudaError_t run(DevBuf<uint8_t>& d, HostBuf<uint8_t>& h, cudaStream_t s) {
    cudaError_t e = d.ensure(std::max<size_t>(total, 16));
    if (e == cudaSuccess) e = h.ensure(std::max<size_t>(total, 16));
    if (e != cudaSuccess) return e;
    for (const Part& q : parts)
      if (q.bytes) std::memcpy(h.p + q.off, q.src, q.bytes);
    return total ? cudaMemcpyAsync(d.p, h.p, total, cudaMemcpyHostToDevice, s) : cudaSuccess;
  }
  template <class P>
  static P at(const DevBuf<uint8_t>& d, size_t off) { return reinterpret_cast<P>(d.p + off); }
};

}  // namespace

struct arb_ctx_s {
  arb_config cfg{};
  uint64_t base_word = 0, n_words = 0;
  uint32_t bucket_bits = 0, n_buckets = 0, coarse_bits = 0, n_bins = 0;
  std::vector<uint32_t> bin_map, hist;
  std::vector<uint64_t> bucket_start;
  std::vector<uint4> items;                   // replay work items (see build_items)
  std::vector<uint4> slice_items;             // K5 phase-3 items (second replay launch)
  std::vector<uint4> hot;                     // K5 hot buckets {bucket, slices, span, 0}
  std::vector<uint64_t> hot_off;              // per bucket scratch offset (hot buckets)
  uint64_t hot_entries = 0;
  DevBuf<uint4> d_slice_items, d_hot;
  HostBuf<uint4> h_slice_items, h_hot;
  DevBuf<uint64_t> d_hot_off;
  HostBuf<uint64_t> h_hot_off;
  DevBuf<uint32_t> hot_F;
  DevBuf<uint8_t> hot_P;
  DevBuf<uint4> d_items;
  HostBuf<uint4> h_items;
  DevBuf<uint32_t> d_bin_map, d_hist, d_cut, d_cutscr;
  DevBuf<uint64_t> d_bucket_start;
  int n_sms = 148;
  uint8_t* shadow = nullptr;
  std::vector<Submit> subs;
  uint64_t pending = 0;
  bool any_gidx = false, any_nogidx = false;
  bool host_gidx = false, dev_gidx = false;   // where this batch's global indices live
  DevBuf<uint4> staging;
  DevBuf<uint64_t> gidx_staging;
  DevBuf<uint2> part_ev;
  DevBuf<uint2> seg_a, seg_b;                 // partition entries, sort ping-pong
  DevBuf<uint4> segs;                         // replay form
  DevBuf<uint32_t> seg_first;
  uint64_t seg_cap = 0;
  HostBuf<uint32_t> h_weight;
  TagBases tags;                              // N1 (Z25): pointer tag bases (committed per flush)
  DevBuf<uint4> cv_buf;                       // N1 (Z26): the batch with CV addresses translated
  DevBuf<uint32_t> d_cv_epoch_pos, d_cv_epoch_first;
  DevBuf<CvPlace> d_cv_place;
  DevBuf<uint32_t> d_tag_first;
  DevBuf<TagSeg> d_tag_segs;
  DevBuf<CtlRec> ctl;
  DevBuf<uint4> cand, cand_tmp, reports;
  DevBuf<uint32_t> blk;
  DevBuf<uint32_t> ops_start;
  DevBuf<BucketOp> ops;
  DevBuf<DevStats> dstats;
  DevBuf<unsigned long long> dcount;
  // MIR: the join plan's arrays, packed (one pinned staging buffer, one copy)
  DevBuf<uint8_t> m_pack;
  HostBuf<uint8_t> h_m_pack;
  DevBuf<unsigned long long> hkeys;
  DevBuf<uint32_t> hvals;
  // N2: nowait instances unjoined at the end of the last flush (committed with the map table)
  std::vector<CarriedInst> carried;
  LastEnded last_ended;                       // Z22 across flushes (committed with `carried`)
  // ARB_F_DEDUP_FIRST across flushes: (word, kind) keys reported so far (open addressing)
  DevBuf<unsigned long long> dset, dset_cnt;
  uint64_t dset_slots = 0, dset_n = 0;
  DevBuf<uint4> carry_ent, carry_next;        // their access summaries {word lo, word hi, carried idx, flag}
  uint64_t n_carry = 0;
  DevBuf<uint32_t> m_co_of;
  uint64_t ctl_cap = 1 << 16;
  uint64_t cand_cap = 1 << 24;
  MapTable map;
  uint64_t next_index = 0;
  uint64_t n_reports = 0;      // exact count of the last flush
  uint64_t n_stored = 0;       // reports held in `reports` (or h_reports)
  bool reports_on_host = false;             // host global indices: translated reports in h_reports
  HostBuf<uint4> h_reports;
  bool flushed = false;
  std::string err;
  arb_stats stats{};
  cudaEvent_t ev[10] = {};
  cudaStream_t aux = nullptr;                 // control-record copies beside the main stream
  HostBuf<DevStats> h_stats;
  HostBuf<uint32_t> h_nb, h_ops_start;
  HostBuf<uint64_t> h_bstart;
  HostBuf<CtlRec> h_ctl;
  HostBuf<BucketOp> h_ops;
  // NCCL
  void* nccl_lib = nullptr;
  void* comm = nullptr;
  nccl_allgather_fn nccl_allgather = nullptr;
  nccl_destroy_fn nccl_destroy = nullptr;
  DevBuf<int64_t> counts;                     // [world] x {status, report count} + own pair
  int comm_ranks = 0;
};

// every ARB_F_* bit arb_init accepts (the two ARB_F_DEVICES bits included)
constexpr uint32_t kKnownFlags = ARB_F_DEDUP_FIRST | ARB_F_TIMING | ARB_F_SMALL_PARTS | ARB_F_BO | ARB_F_UNIFIED |
                                 (3u << ARB_F_DEVICES_SHIFT);

static int fail(arb_ctx c, int rc, const std::string& msg) {
  if (c) c->err = msg;
  return rc;
}
static int cuda_fail(arb_ctx c, cudaError_t e, const char* where) {
  return fail(c, ARB_ECUDA, std::string(where) + ": " + cudaGetErrorString(e));
}
#define CK(call, where)                                    \
  do {                                                     \
    cudaError_t _e = (call);                               \
    if (_e != cudaSuccess) return cuda_fail(ctx, _e, where); \
  } while (0)

// ncclAllGather of one {a, b} pair per rank (stream-ordered, then synchronised);
// all = world pairs in rank order.  ARB_ECUDA if NCCL or CUDA fails.
static int nccl_exchange(arb_ctx ctx, cudaStream_t s, int64_t a, int64_t b, std::vector<int64_t>& all) {
  const int w = ctx->cfg.world;
  int64_t mine[2] = {a, b};
  all.assign(2 * (size_t)w, 0);
  int64_t* own = ctx->counts.p + 2 * w;
  if (cudaMemcpyAsync(own, mine, sizeof(mine), cudaMemcpyHostToDevice, s) != cudaSuccess)
    return fail(ctx, ARB_ECUDA, "count exchange: copy");
  if (ctx->nccl_allgather(own, ctx->counts.p, 2, kNcclInt64, ctx->comm, s) != 0)
    return fail(ctx, ARB_ECUDA, "ncclAllGather failed");
  if (cudaMemcpyAsync(all.data(), ctx->counts.p, 16 * (size_t)w, cudaMemcpyDeviceToHost, s) != cudaSuccess ||
      cudaStreamSynchronize(s) != cudaSuccess)
    return fail(ctx, ARB_ECUDA, "count exchange: read-back");
  return ARB_OK;
}

extern "C" int arb_init(const arb_config* cfg, arb_ctx* out) {
  if (!out) return ARB_EINVAL;
  *out = nullptr;
  if (!cfg || (cfg->addr_base & 7) || (cfg->addr_bytes & 7) || cfg->addr_bytes == 0 ||
      cfg->addr_base + cfg->addr_bytes > (1ull << 48) || cfg->world < 1 || cfg->rank < 0 ||
      cfg->rank >= cfg->world || (cfg->world > 1 && !cfg->nccl_unique_id) || (cfg->flags & ~kKnownFlags) ||
      ((cfg->flags & ARB_F_BO) && (cfg->flags & ARB_F_UNIFIED)) || ((cfg->flags >> ARB_F_DEVICES_SHIFT) & 3u) > 2u ||
      (((cfg->flags >> ARB_F_DEVICES_SHIFT) & 3u) && (cfg->flags & (ARB_F_BO | ARB_F_UNIFIED))))
    return ARB_EINVAL;
  arb_ctx ctx = new (std::nothrow) arb_ctx_s();
  if (!ctx) return ARB_ENOMEM;
  ctx->cfg = *cfg;
  ctx->base_word = cfg->addr_base >> 3;
  ctx->n_words = cfg->addr_bytes >> 3;
  // Address buckets.  bucket_bits != 0: fixed buckets of 2^bits words (<= 2048
  // of them).  0: buckets balanced per flush on a sampled address histogram over
  // <= 2^18 coarse bins (<= 2048 buckets of <= 2^30 words).
  if (ctx->n_words > (1ull << 38)) { delete ctx; return ARB_EINVAL; }
  uint32_t bits = cfg->bucket_bits;
  if (bits) {
    uint64_t nb = (ctx->n_words + (1ull << bits) - 1) >> bits;
    if (bits > kMaxBucketSpanBits || nb > (uint64_t)kMaxBuckets) { delete ctx; return ARB_EINVAL; }
    ctx->coarse_bits = bits;
    ctx->bin_map.resize(nb);
    ctx->bucket_start.clear();
    for (uint64_t b = 0; b < nb; ++b) { ctx->bin_map[b] = (uint32_t)b; ctx->bucket_start.push_back(b << bits); }
    ctx->bucket_start.push_back(ctx->n_words);
  } else {
    uint32_t cb = 0;
    while (((ctx->n_words + (1ull << cb) - 1) >> cb) > (uint64_t)kMaxCoarseBins) ++cb;
    ctx->coarse_bits = cb;
  }
  ctx->bucket_bits = bits;
  ctx->n_bins = (uint32_t)((ctx->n_words + (1ull << ctx->coarse_bits) - 1) >> ctx->coarse_bits);
  if (cfg->report_capacity) ctx->cand_cap = cfg->report_capacity;
  cudaError_t e = cudaSetDevice(cfg->device);
  if (e != cudaSuccess) { delete ctx; return ARB_ECUDA; }
  cudaDeviceGetAttribute(&ctx->n_sms, cudaDevAttrMultiProcessorCount, cfg->device);
  e = cudaMalloc(&ctx->shadow, ctx->n_words + 16);
  if (e != cudaSuccess) { delete ctx; return ARB_ENOMEM; }
  e = cudaMemset(ctx->shadow, 0, ctx->n_words);                 // all invalid
  if (e == cudaSuccess) e = ctx->dstats.ensure(1);
  if (e == cudaSuccess) e = ctx->dcount.ensure(8);
  if (e == cudaSuccess) e = ctx->ctl.ensure(ctx->ctl_cap);
  for (int i = 0; i < 10 && e == cudaSuccess; ++i) e = cudaEventCreate(&ctx->ev[i]);
  if (e == cudaSuccess) e = cudaStreamCreateWithFlags(&ctx->aux, cudaStreamNonBlocking);
  if (e == cudaSuccess) e = ctx->h_stats.ensure(1);
  if (e == cudaSuccess) e = ctx->h_nb.ensure(1);
  if (e == cudaSuccess) e = ctx->h_bstart.ensure(kMaxBuckets + 1);
  if (e == cudaSuccess) e = ctx->h_weight.ensure(kMaxBuckets);
  if (e == cudaSuccess) e = cudaDeviceSynchronize();
  if (e != cudaSuccess) { arb_destroy(ctx); return ARB_ENOMEM; }
  if (cfg->nccl_unique_id) {
    // world > 1: the address-sharded job's communicator; world == 1 with an id: a
    // 1-rank communicator, so that the exchange path runs on a single GPU too
    ctx->nccl_lib = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
    if (!ctx->nccl_lib) { arb_destroy(ctx); return ARB_ECUDA; }
    auto init = (nccl_init_fn)dlsym(ctx->nccl_lib, "ncclCommInitRank");
    auto count = (nccl_count_fn)dlsym(ctx->nccl_lib, "ncclCommCount");
    ctx->nccl_allgather = (nccl_allgather_fn)dlsym(ctx->nccl_lib, "ncclAllGather");
    ctx->nccl_destroy = (nccl_destroy_fn)dlsym(ctx->nccl_lib, "ncclCommDestroy");
    if (!init || !count || !ctx->nccl_allgather || !ctx->nccl_destroy) { arb_destroy(ctx); return ARB_ECUDA; }
    NcclId id;
    std::memcpy(id.internal, cfg->nccl_unique_id, sizeof(id.internal));
    if (init(&ctx->comm, cfg->world, id, cfg->rank) != 0 || ctx->counts.ensure(2 * cfg->world + 2) != cudaSuccess ||
        count(ctx->comm, &ctx->comm_ranks) != 0 || ctx->comm_ranks != cfg->world) {
      arb_destroy(ctx);
      return ARB_ECUDA;
    }
    ctx->stats.nccl_ranks = (uint64_t)ctx->comm_ranks;
  }
  *out = ctx;
  return ARB_OK;
}

extern "C" int arb_destroy(arb_ctx ctx) {
  if (!ctx) return ARB_OK;
  if (ctx->comm && ctx->nccl_destroy) ctx->nccl_destroy(ctx->comm);
  if (ctx->shadow) cudaFree(ctx->shadow);
  ctx->staging.release(); ctx->gidx_staging.release(); ctx->part_ev.release(); ctx->seg_a.release(); ctx->seg_b.release(); ctx->segs.release(); ctx->seg_first.release();
  ctx->h_weight.release();
  ctx->d_tag_first.release(); ctx->d_tag_segs.release(); ctx->cv_buf.release(); ctx->d_cv_epoch_pos.release();
  ctx->d_cv_epoch_first.release(); ctx->d_cv_place.release();
  ctx->ctl.release(); ctx->cand.release(); ctx->cand_tmp.release(); ctx->reports.release(); ctx->blk.release();
  ctx->ops_start.release(); ctx->ops.release(); ctx->dstats.release(); ctx->dcount.release();
  ctx->m_pack.release(); ctx->h_m_pack.release(); ctx->hkeys.release(); ctx->hvals.release(); ctx->counts.release();
  ctx->carry_ent.release(); ctx->carry_next.release(); ctx->dset.release(); ctx->dset_cnt.release(); ctx->m_co_of.release();
  ctx->d_bin_map.release(); ctx->d_items.release(); ctx->h_items.release();
  ctx->d_slice_items.release(); ctx->h_slice_items.release(); ctx->d_hot.release(); ctx->h_hot.release();
  ctx->d_hot_off.release(); ctx->h_hot_off.release(); ctx->hot_F.release(); ctx->hot_P.release(); ctx->d_hist.release(); ctx->d_bucket_start.release(); ctx->d_cut.release();
  for (auto& e : ctx->ev) if (e) cudaEventDestroy(e);
  if (ctx->aux) cudaStreamDestroy(ctx->aux);
  ctx->h_stats.release(); ctx->h_nb.release(); ctx->h_ops_start.release(); ctx->h_bstart.release();
  ctx->h_ctl.release(); ctx->h_ops.release(); ctx->h_reports.release();
  if (ctx->nccl_lib) dlclose(ctx->nccl_lib);
  delete ctx;
  return ARB_OK;
}

extern "C" const char* arb_last_error(arb_ctx ctx) {
  if (!ctx) return "null context";
  return ctx->err.c_str();
}

extern "C" int arb_submit_events(arb_ctx ctx, const arb_event* ev, uint64_t n, const uint64_t* global_index,
                                 int ev_on_device, void* stream) {
  if (!ctx) return ARB_EINVAL;
  if (n == 0) return ARB_OK;
  if (!ev) return fail(ctx, ARB_EINVAL, "null event pointer");
  if (ctx->pending + n > kMaxBatchRecords) return fail(ctx, ARB_EINVAL, "batch exceeds 2^30 records");
  if (((ctx->cfg.flags >> ARB_F_DEVICES_SHIFT) & 3u) && ctx->pending + n > (kMaxBatchRecords >> 1))
    return fail(ctx, ARB_EINVAL, "several accelerators: a batch holds at most 2^29 records");
  if ((global_index != nullptr && ctx->any_nogidx) || (global_index == nullptr && ctx->any_gidx))
    return fail(ctx, ARB_EINVAL, "global_index must be given for every submit of a batch or for none");
  cudaSetDevice(ctx->cfg.device);
  cudaStream_t s = (cudaStream_t)stream;
  if (!ev_on_device) {
    // host records are copied now (stream-ordered) into the staging buffer
    uint64_t off = ctx->pending;
    // keep earlier device submits: move them into staging first
    cudaError_t e = cudaStreamSynchronize(s);
    if (e == cudaSuccess) e = ctx->staging.ensure_keep(off + n, off);
    if (e != cudaSuccess) return fail(ctx, ARB_ENOMEM, "staging buffer");
    e = cudaMemcpyAsync(ctx->staging.p + off, ev, n * sizeof(arb_event), cudaMemcpyHostToDevice, s);
    if (e != cudaSuccess) return cuda_fail(ctx, e, "copy host records");
    const uint64_t* host_gi = nullptr;
    if (global_index && ctx->dev_gidx) {
      // the batch's other indices are on the device: copy these next to them
      if ((e = ctx->gidx_staging.ensure_keep(off + n, off)) != cudaSuccess) return fail(ctx, ARB_ENOMEM, "gidx staging");
      e = cudaMemcpyAsync(ctx->gidx_staging.p + off, global_index, n * 8, cudaMemcpyHostToDevice, s);
      if (e != cudaSuccess) return cuda_fail(ctx, e, "copy host global_index");
    } else if (global_index) {
      host_gi = global_index;      // read on the report path only (no H2D copy, §8(b))
      ctx->host_gidx = true;
    }
    e = cudaStreamSynchronize(s);  // the caller may free the host records on return
    if (e != cudaSuccess) return cuda_fail(ctx, e, "submit sync");
    ctx->subs.push_back(Submit{nullptr, n, host_gi, 0});
  } else {
    if (global_index && ctx->host_gidx)
      return fail(ctx, ARB_EINVAL, "global_index of one batch: host arrays (host submits) or device arrays, not both");
    if (global_index) ctx->dev_gidx = true;
    ctx->subs.push_back(Submit{ev, n, global_index, 1});
  }
  if (global_index) ctx->any_gidx = true; else ctx->any_nogidx = true;
  ctx->pending += n;
  return ARB_OK;
}

static void reset_batch(arb_ctx ctx) {
  ctx->subs.clear();
  ctx->pending = 0;
  ctx->any_gidx = ctx->any_nogidx = false;
  ctx->host_gidx = ctx->dev_gidx = false;
}

// Replay work items, heaviest first.  A bucket whose range ops cover many words
// compared with its events is split into parts (contiguous word ranges, 16-word
// aligned): each part replays all of the bucket's events but acts only on its own
// words, so the range-op streaming of one huge bucket spreads over many CTAs.
// Cost model (per CTA): ~600 range-op words stream in the time of one event.
//
// Hot buckets (K5): a bucket of <= kHotSpan words whose estimated events exceed
// 1.25x the per-CTA share of the flush (and 2^17) would be the replay's critical
// path; it is cut into time slices of ~2^17 events: phase 1 (kItemSummary, in the
// first replay launch) composes each slice's per-word transition functions,
// k_carry (phase 2) carries the states across the slices and writes the final
// shadow, and phase 3 (kItemSlice, second launch) replays each slice against its
// carried-in states to classify its reads.
static void build_items(arb_ctx ctx, const FlushPlan& plan, const std::vector<double>& bucket_events) {
  constexpr double kWordsPerEvent = 600.0;
  constexpr uint32_t kMaxParts = 64, kMaxSlices = 64;
  constexpr double kSliceEvents = double(1u << 17);
  const bool small = ctx->cfg.flags & ARB_F_SMALL_PARTS;
  const double kPartWords = small ? 1024.0 : double(1u << 24);
  const uint32_t nb = ctx->n_buckets;
  std::vector<uint32_t> parts(nb, 1);
  std::vector<double> rws(nb, 0.0);
  bool any_split = false;
  for (uint32_t b = 0; b < nb; ++b) {
    double rw = 0;
    for (uint32_t k = plan.ops_start[b]; k < plan.ops_start[b + 1]; ++k) rw += double(plan.ops[k].hi - plan.ops[k].lo);
    rws[b] = rw;
    const double ev = b < bucket_events.size() ? bucket_events[b] : 0.0;
    const uint64_t span = ctx->bucket_start[b + 1] - ctx->bucket_start[b];
    if (rw > 2 * kPartWords && span >= 32) {
      const double by_range = rw / kPartWords, by_events = small ? by_range : rw / (ev * kWordsPerEvent + 1.0);
      uint32_t np = (uint32_t)std::max(1.0, std::min<double>(std::min(by_range, by_events), kMaxParts));
      np = (uint32_t)std::min<uint64_t>(np, span / 16);
      parts[b] = np;
      any_split |= np > 1;
    }
  }
  // hot buckets
  ctx->hot.clear(); ctx->slice_items.clear(); ctx->hot_entries = 0;
  double ev_tot = 0;
  for (double e : bucket_events) ev_tot += e;
  const double share = ev_tot / double(std::max(1, ctx->n_sms * kReplayCtasPerSm));
  const bool force_hot = ctx->cfg.flags & ARB_F_SMALL_PARTS;     // test knob: slice every small busy bucket
  std::vector<uint32_t> slices(nb, 0);
  constexpr uint64_t kMaxHotEntries = 1ull << 29;      // K5 scratch: 5 B per entry
  uint64_t hot_total = 0;
  for (uint32_t b = 0; b < nb && b < bucket_events.size(); ++b) {
    const uint64_t span = ctx->bucket_start[b + 1] - ctx->bucket_start[b];
    const double ev = bucket_events[b];
    if (parts[b] != 1 || span > kHotSpan) continue;
    const bool hot = force_hot ? ev >= 64.0 : (ev > 1.25 * share && ev > kSliceEvents);
    if (!hot) continue;
    const double want = force_hot ? 3.0 : std::ceil(ev / kSliceEvents);
    uint32_t ns = (uint32_t)std::max(2.0, std::min<double>(want, kMaxSlices));
    const uint64_t span16 = (span + 15) & ~15ull;
    ns = (uint32_t)std::min<uint64_t>(ns, kMaxHotEntries / 8 / span16);        // scratch per bucket
    if (ns < 2 || hot_total + ns * span16 > kMaxHotEntries) continue;           // scratch per flush
    hot_total += ns * span16;
    slices[b] = ns;
  }
  bool any_hot = false;
  ctx->hot_off.assign(nb, 0);
  for (uint32_t b = 0; b < nb; ++b) {
    if (!slices[b]) continue;
    any_hot = true;
    const uint32_t span = (uint32_t)(ctx->bucket_start[b + 1] - ctx->bucket_start[b]);
    ctx->hot_off[b] = ctx->hot_entries;
    ctx->hot_entries += (uint64_t)slices[b] * ((span + 15) & ~15u);
    ctx->hot.push_back(make_uint4(b, slices[b], span, 0u));
    for (uint32_t k = 0; k < slices[b]; ++k) ctx->slice_items.push_back(make_uint4(b, k, slices[b], kItemSlice));
  }
  ctx->items.clear();
  if (!any_split && !any_hot) {
    // every bucket whole: order by sampled events, heaviest first (ties: bucket id)
    std::vector<uint64_t> key(nb);
    for (uint32_t b = 0; b < nb; ++b) {
      const double ev = b < bucket_events.size() ? bucket_events[b] : 0.0;
      const uint64_t w = (uint64_t)std::min(ev, 4.0e9);
      key[b] = ((0xFFFFFFFFull - w) << 32) | b;
    }
    std::sort(key.begin(), key.end());
    for (uint64_t k : key) {
      const uint32_t b = (uint32_t)k;
      ctx->items.push_back(make_uint4(b, 0, (uint32_t)(ctx->bucket_start[b + 1] - ctx->bucket_start[b]), 0u));
    }
    return;
  }
  struct It { double cost; uint4 v; };
  std::vector<It> its;
  its.reserve(nb);
  for (uint32_t b = 0; b < nb; ++b) {
    const double ev = b < bucket_events.size() ? bucket_events[b] : 0.0;
    const uint64_t span = ctx->bucket_start[b + 1] - ctx->bucket_start[b];
    if (slices[b]) {                   // phase-1 items of a hot bucket
      for (uint32_t k = 0; k < slices[b]; ++k)
        its.push_back(It{ev / slices[b] * kWordsPerEvent, make_uint4(b, k, slices[b], kItemSummary)});
      continue;
    }
    const uint32_t np = parts[b];
    const uint64_t step = ((span + np - 1) / np + 15) & ~15ull;
    for (uint32_t q = 0; q < np; ++q) {
      const uint64_t lo = std::min<uint64_t>(span, q * step), hi = std::min<uint64_t>(span, lo + step);
      if (lo >= hi && np > 1) continue;
      const double cost = ev * kWordsPerEvent + (np == 1 ? 0.0 : rws[b] * double(hi - lo) / double(span));
      its.push_back(It{cost, make_uint4(b, (uint32_t)lo, (uint32_t)hi, np > 1 ? kItemPart : kItemWhole)});
    }
  }
  std::stable_sort(its.begin(), its.end(), [](const It& x, const It& y) { return x.cost > y.cost; });
  ctx->items.resize(its.size());
  for (size_t i = 0; i < its.size(); ++i) ctx->items[i] = its[i].v;
}

extern "C" int arb_flush(arb_ctx ctx, void* stream, uint64_t* n_reports_local, uint64_t* report_offset_global) {
  if (!ctx) return ARB_EINVAL;
  cudaSetDevice(ctx->cfg.device);
  cudaStream_t s = (cudaStream_t)stream;
  const bool timing = ctx->cfg.flags & ARB_F_TIMING;
  int launches = 0;
  const uint64_t n = ctx->pending;
  arb_stats& S = ctx->stats;
  S.exchanges = 0;
  S.records = n; S.access_words = S.range_words = S.control_records = S.range_ops = S.tasks = 0;
  S.reports = 0; std::memset(S.reports_by_kind, 0, sizeof(S.reports_by_kind)); S.ignored_words = 0;
  S.ms_partition = S.ms_control = S.ms_replay = S.ms_mir = S.ms_reports = S.ms_total = 0;
  S.ms_segsort = S.ms_host_control = 0;
  S.steps_run = S.segments = S.chunks = S.chunks_fast = S.chunks_run = S.run_merges = 0;
  S.buckets = ctx->n_buckets; S.bucket_bits = ctx->bucket_bits; S.max_bucket_events = 0;

  // Phase A (validation): decode + partition and control resolution.  Nothing
  // committed changes here, so an error discards the batch and leaves the context
  // usable.  With a communicator every rank then exchanges its phase-A status, and
  // a batch any rank rejects is discarded by all of them (ARB_EPEER on the others):
  // the ranks stay in lockstep and nobody waits in a collective a peer skipped.
  const uint4* ev = nullptr;
  const uint64_t* gidx = nullptr;
  const uint64_t index_base = ctx->next_index;
  const bool balanced = ctx->bucket_bits == 0;
  DevStats& hst = *ctx->h_stats.p;
  std::vector<double> bucket_events;      // estimated events per bucket (sampled)
  MapTable map;
  FlushPlan plan;
  std::chrono::steady_clock::time_point t_host0, t_host1;
  int rc = [&]() -> int {
  // ---- resolve the batch into one device array ---------------------------
  if (n) {
    bool single_dev = ctx->subs.size() == 1 && ctx->subs[0].on_device;
    if (single_dev) {
      ev = reinterpret_cast<const uint4*>(ctx->subs[0].ev);
      gidx = ctx->subs[0].gidx;
    } else {
      // gather device submits into staging (host submits are already there)
      uint64_t off = 0;
      CK(cudaStreamSynchronize(s), "staging sync");
      CK(ctx->staging.ensure_keep(n, n), "staging");
      if (ctx->any_gidx && !ctx->host_gidx) CK(ctx->gidx_staging.ensure_keep(n, n), "gidx staging");
      for (const Submit& sb : ctx->subs) {
        if (sb.on_device) {
          CK(cudaMemcpyAsync(ctx->staging.p + off, sb.ev, sb.n * 16, cudaMemcpyDeviceToDevice, s), "gather");
          if (sb.gidx && !ctx->host_gidx)
            CK(cudaMemcpyAsync(ctx->gidx_staging.p + off, sb.gidx, sb.n * 8, cudaMemcpyDeviceToDevice, s), "gather gidx");
        }
        off += sb.n;
      }
      ev = ctx->staging.p;
      gidx = ctx->any_gidx && !ctx->host_gidx ? ctx->gidx_staging.p : nullptr;
    }
  }
  if (timing) cudaEventRecord(ctx->ev[0], s);
  // N1 (Z26): a batch with CV-addressed target accesses runs this part twice: the
  // first pass finds them (left untracked) and resolves the CV placements, the
  // second partitions a copy with those accesses translated to OV addresses
  for (bool translated = false;;) {
    // ---- bucket balancing on a sampled address histogram (all on the device) ----
    if (balanced) {
      CK(ctx->d_hist.ensure(ctx->n_bins), "alloc hist");
      CK(cudaMemsetAsync(ctx->d_hist.p, 0, ctx->n_bins * sizeof(uint32_t), s), "hist clear");
      SampleParams sp{};
      sp.ev = ev; sp.n = n; sp.stride = std::max<uint64_t>(1, n / kSampleCap);
      sp.base_word = ctx->base_word; sp.n_words = ctx->n_words; sp.coarse_bits = ctx->coarse_bits;
      sp.hist = ctx->d_hist.p;
      const uint64_t n_samples = n ? (n + sp.stride - 1) / sp.stride : 0;
      CK(launch_sample(sp, n_samples, s), "k_sample");
      launches += n_samples ? 1 : 0;
      // cut balanced buckets; the histogram becomes the bin map in place
      if (ctx->d_bucket_start.cap == 0) {       // the read-back below copies every slot
        CK(ctx->d_bucket_start.ensure(kMaxBuckets + 1), "alloc buckets");
        CK(cudaMemsetAsync(ctx->d_bucket_start.p, 0, (kMaxBuckets + 1) * 8, s), "clear buckets");
      }
      if (ctx->d_cut.cap == 0) {
        CK(ctx->d_cut.ensure(2 * kMaxBuckets + 2), "alloc cut scratch");
        CK(cudaMemsetAsync(ctx->d_cut.p, 0, (2 * kMaxBuckets + 2) * 4, s), "clear cut scratch");
      }
      CK(ctx->d_cutscr.ensure(2 * ((ctx->n_bins + 1023) / 1024) + 4 + ctx->n_bins), "alloc cut scratch");
      CK(launch_cut(ctx->d_hist.p, ctx->n_bins, ctx->coarse_bits, ctx->n_words, kMaxBuckets, ctx->d_bucket_start.p,
                    ctx->d_cut.p, ctx->d_cut.p + kMaxBuckets, ctx->d_cut.p + 2 * kMaxBuckets, ctx->d_cutscr.p,
                    s, &launches), "k_cut");
      // the bucket count and starts come back with the partition's counters (one sync)
      CK(cudaMemcpyAsync(ctx->h_nb.p, ctx->d_cut.p + 2 * kMaxBuckets, 4, cudaMemcpyDeviceToHost, s), "nb d2h");
      CK(cudaMemcpyAsync(ctx->h_bstart.p, ctx->d_bucket_start.p, (kMaxBuckets + 1) * 8, cudaMemcpyDeviceToHost, s),
         "buckets d2h");
      CK(cudaMemcpyAsync(ctx->h_weight.p, ctx->d_cut.p, kMaxBuckets * 4, cudaMemcpyDeviceToHost, s), "weights d2h");
    } else if (ctx->d_bin_map.cap == 0) {
      CK(upload(ctx->d_bin_map, ctx->bin_map, s), "upload bin map");
      CK(upload(ctx->d_bucket_start, ctx->bucket_start, s), "upload bucket starts");
    }
    if (!balanced) ctx->n_buckets = (uint32_t)ctx->bucket_start.size() - 1;   // fixed buckets
    if (timing) cudaEventRecord(ctx->ev[7], s);
    // ---- A1/A3a: decode + partition ------------------------------------------
    const uint32_t n_chunks = (uint32_t)((n + kChunkRecords - 1) / kChunkRecords);
    CK(ctx->part_ev.ensure((size_t)std::max<uint32_t>(n_chunks, 1) * kChunkCap), "alloc part_ev");
    if (ctx->seg_cap < (uint64_t)n_chunks * 2 + 4096) ctx->seg_cap = (uint64_t)n_chunks * 2 + 4096;
    CK(ctx->seg_a.ensure(std::max<uint64_t>(ctx->seg_cap, 1)), "alloc segments");
    PartParams pp{};
    for (int attempt = 0; attempt < 2; ++attempt) {
      CK(cudaMemsetAsync(ctx->dstats.p, 0, sizeof(DevStats), s), "stats init");
      CK(cudaMemsetAsync(&ctx->dstats.p->err_pos, 0xFF, sizeof(unsigned long long), s), "stats init");
      pp.ev = ev; pp.n = n; pp.base_word = ctx->base_word; pp.n_words = ctx->n_words;
      pp.coarse_bits = ctx->coarse_bits; pp.bin_map = balanced ? ctx->d_hist.p : ctx->d_bin_map.p;
      pp.bucket_bits = ctx->bucket_bits; pp.n_buckets = balanced ? (uint32_t)kMaxBuckets : ctx->n_buckets;
      pp.n_chunks = n_chunks;
      pp.n_dev = 1u + ((ctx->cfg.flags >> ARB_F_DEVICES_SHIFT) & 3u);
      pp.part_ev = ctx->part_ev.p; pp.seg_out = ctx->seg_a.p; pp.seg_cap = ctx->seg_cap;
      pp.no_runs = getenv("ARB_NO_RUNS") != nullptr;
      pp.grid = (uint32_t)std::max<uint64_t>(1, std::min<uint64_t>((n_chunks + kPartWarps - 1) / kPartWarps,
                                                                   (uint64_t)ctx->n_sms));
      pp.ctl = ctx->ctl.p; pp.ctl_cap = ctx->ctl_cap;
      pp.st = ctx->dstats.p;
      CK(launch_partition(pp, s), "k_partition");
      launches += n_chunks ? 1 : 0;
      CK(cudaMemcpyAsync(&hst, ctx->dstats.p, sizeof(hst), cudaMemcpyDeviceToHost, s), "stats d2h");
      CK(cudaStreamSynchronize(s), "partition sync");
      if (hst.n_ctl <= ctx->ctl_cap && hst.n_segs <= ctx->seg_cap) break;
      if (hst.n_ctl > ctx->ctl_cap) ctx->ctl_cap = hst.n_ctl + hst.n_ctl / 2;
      if (hst.n_segs > ctx->seg_cap) ctx->seg_cap = hst.n_segs + hst.n_segs / 4;
      CK(ctx->ctl.ensure(ctx->ctl_cap), "grow ctl");
      CK(ctx->seg_a.ensure(ctx->seg_cap), "grow segments");
    }
    if (timing) cudaEventRecord(ctx->ev[1], s);
    if (hst.err_pos != ~0ull)
      return fail(ctx, ARB_ETRACE, "malformed record at batch position " + std::to_string(hst.err_pos));
    if (balanced) {
      const uint32_t nb = *ctx->h_nb.p;
      ctx->bucket_start.assign(ctx->h_bstart.p, ctx->h_bstart.p + nb + 1);
      const double stride = (double)std::max<uint64_t>(1, n / kSampleCap);
      bucket_events.resize(nb);
      for (uint32_t b = 0; b < nb; ++b) bucket_events[b] = ctx->h_weight.p[b] * stride;
    }
    ctx->n_buckets = (uint32_t)ctx->bucket_start.size() - 1;
    S.buckets = ctx->n_buckets;
    S.access_words = hst.access_words;
    S.control_records = hst.n_ctl;

    // ---- A3b: segment entries sorted by (bucket, chunk) — on the GPU while the
    // host resolves the control records ------------------------------------------------
    {
      const uint64_t ns = hst.n_segs;
      CK(ctx->seg_b.ensure(std::max<uint64_t>(ns, 1)), "alloc segments");
      CK(ctx->segs.ensure(std::max<uint64_t>(ns, 1)), "alloc segments");
      CK(ctx->seg_first.ensure(ctx->n_buckets + 1), "alloc seg_first");
      CK(ctx->blk.ensure((ns + 4095) / 4096 * 2049 + 4096), "alloc blk");   // 2048-bin digit counters + scan scratch
      CK(launch_sort_segments(ctx->seg_a.p, ctx->seg_b.p, ns, n_chunks, ctx->n_buckets, ctx->blk.p, ctx->seg_first.p,
                              ctx->segs.p, s, &launches), "sort segments");
      if (timing) cudaEventRecord(ctx->ev[8], s);
    }
    t_host0 = std::chrono::steady_clock::now();

    // ---- A2: control resolution on the host -------------------------------------
    std::vector<CtlRec> ctl(hst.n_ctl);
    if (hst.n_ctl) {
      CK(ctx->h_ctl.ensure(hst.n_ctl), "pinned ctl");
      CK(cudaMemcpyAsync(ctx->h_ctl.p, ctx->ctl.p, hst.n_ctl * sizeof(CtlRec), cudaMemcpyDeviceToHost, ctx->aux),
         "ctl d2h");
      CK(cudaStreamSynchronize(ctx->aux), "ctl sync");
      std::memcpy(ctl.data(), ctx->h_ctl.p, hst.n_ctl * sizeof(CtlRec));
      std::sort(ctl.begin(), ctl.end(), [](const CtlRec& a, const CtlRec& b) { return a.pos < b.pos; });
    }
    t_host1 = std::chrono::steady_clock::now();
    map = ctx->map;
    resolve_control(ctl, n, ctx->base_word, ctx->n_words, ctx->bucket_start, map, plan,
                    (ctx->cfg.flags & ARB_F_BO) != 0, &ctx->carried, (ctx->cfg.flags & ARB_F_UNIFIED) != 0,
                    1u + ((ctx->cfg.flags >> ARB_F_DEVICES_SHIFT) & 3u), &ctx->last_ended, &ctx->tags,
                  hst.n_cv_acc != 0);
    if (plan.rc != 0)
      return fail(ctx, plan.rc, plan.err + " (batch position " + std::to_string(plan.err_pos) + ")");
  if (hst.n_cv_acc && !translated) {
    if ((ctx->cfg.flags >> ARB_F_DEVICES_SHIFT) & 3u)
      return fail(ctx, ARB_ETRACE, "CV-addressed accesses (Z26) with several accelerators are oracle-only");
    CK(upload(ctx->d_cv_epoch_pos, plan.cv_epoch_pos, s), "cv epochs");
    CK(upload(ctx->d_cv_epoch_first, plan.cv_epoch_first, s), "cv epochs");
    CK(upload(ctx->d_cv_place, plan.cv_place, s), "cv placements");
    CK(ctx->cv_buf.ensure(n), "cv copy");
    CK(launch_cv_translate(ev, ctx->cv_buf.p, n, ctx->d_cv_epoch_pos.p, ctx->d_cv_epoch_first.p,
                           (uint32_t)plan.cv_epoch_pos.size(), ctx->d_cv_place.p, s), "k_cv_translate");
    launches += 1;
    ev = ctx->cv_buf.p;
    translated = true;
    continue;
  }
  break;
  }
  return ARB_OK;
  }();
  {   // every rank learns whether every rank's batch is valid
    int64_t peer = 0;
    if (ctx->comm) {
      std::vector<int64_t> all;
      if (nccl_exchange(ctx, s, rc, 0, all) != ARB_OK) { reset_batch(ctx); return ARB_ECUDA; }
      for (int r = 0; r < (int)all.size() / 2; ++r)
        if (r != ctx->cfg.rank && all[2 * r] < 0) peer = all[2 * r];
      S.exchanges += 1;
    }
    if (rc == ARB_OK && peer < 0) rc = fail(ctx, ARB_EPEER, "another rank rejected its part of the batch (" +
                                                                   std::to_string(peer) + "); batch discarded");
  }
  if (rc != ARB_OK) {
    cudaStreamSynchronize(s);
    reset_batch(ctx);
    return rc;
  }
  S.range_words = plan.range_words;
  S.range_ops = plan.range_ops.size();
  S.tasks = plan.tasks;
  S.ignored_words = hst.ignored_words + plan.ignored_words;
  // Phase B: replay (commits the shadow), MIR join, report compaction.  A failure
  // here is ARB_ENOMEM / ARB_ECUDA: the context must be destroyed (on every rank);
  // the count exchange still runs so that no peer waits for this rank.
  uint64_t n_vsm = 0, kept_vsm = 0, n_carry_next = 0;
  int rcb = [&]() -> int {
  const auto t_host2 = std::chrono::steady_clock::now();
  build_items(ctx, plan, bucket_events);
  if (getenv("ARB_HOST_PROFILE")) {
    const auto t3 = std::chrono::steady_clock::now();
    auto ms = [](auto a, auto b) { return std::chrono::duration<double, std::milli>(b - a).count(); };
    fprintf(stderr, "arb host: ctl d2h+sort %.3f ms (%llu ctl), resolve %.3f ms (%zu range ops, %zu bucket ops), "
            "items %.3f ms\n", ms(t_host0, t_host1), (unsigned long long)hst.n_ctl, ms(t_host1, t_host2),
            plan.range_ops.size(), plan.ops.size(), ms(t_host2, t3));
  }
  S.work_items = ctx->items.size() + ctx->slice_items.size();
  S.hot_buckets = ctx->hot.size();
  S.ms_host_control = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t_host0).count();
  CK(upload_pinned(ctx->d_items, ctx->h_items, ctx->items, s), "upload work items");
  if (!ctx->hot.empty()) {
    CK(upload_pinned(ctx->d_slice_items, ctx->h_slice_items, ctx->slice_items, s), "upload slice items");
    CK(upload_pinned(ctx->d_hot, ctx->h_hot, ctx->hot, s), "upload hot buckets");
    CK(upload_pinned(ctx->d_hot_off, ctx->h_hot_off, ctx->hot_off, s), "upload hot offsets");
    CK(ctx->hot_F.ensure(ctx->hot_entries), "alloc hot F");
    CK(ctx->hot_P.ensure(ctx->hot_entries), "alloc hot P");
  }
  CK(upload_pinned(ctx->ops_start, ctx->h_ops_start, plan.ops_start, s), "upload ops_start");
  CK(upload_pinned(ctx->ops, ctx->h_ops, plan.ops, s), "upload ops");
  CK(ctx->cand.ensure(ctx->cand_cap), "alloc candidates");
  if (timing) cudaEventRecord(ctx->ev[2], s);

  // ---- A3b/A4/A5: replay ---------------------------------------------------------
  ReplayParams rp{};
  rp.part_ev = ctx->part_ev.p; rp.segs = ctx->segs.p; rp.seg_first = ctx->seg_first.p;
  rp.n_buckets = ctx->n_buckets; rp.bucket_bits = ctx->bucket_bits; rp.n_words = ctx->n_words;
  rp.bucket_start = ctx->d_bucket_start.p;
  rp.items = ctx->d_items.p; rp.n_items = (uint32_t)ctx->items.size();
  rp.shadow = ctx->shadow; rp.bo = (ctx->cfg.flags & ARB_F_BO) ? 1u : 0u;
  rp.um = (ctx->cfg.flags & ARB_F_UNIFIED) ? 1u : 0u;
  rp.md = ((ctx->cfg.flags >> ARB_F_DEVICES_SHIFT) & 3u) ? 1u : 0u; rp.ops_start = ctx->ops_start.p; rp.ops = ctx->ops.p;
  rp.cand = ctx->cand.p; rp.cand_cap = ctx->cand_cap; rp.st = ctx->dstats.p;
  rp.no_run_steps = getenv("ARB_NO_RUN_STEPS") != nullptr;
  rp.no_run_prep = getenv("ARB_NO_RUN_PREP") != nullptr;
  rp.run_step_max = getenv("ARB_RUN_STEP_MAX") ? (uint32_t)std::max(256, atoi(getenv("ARB_RUN_STEP_MAX"))) : 16384u;
  rp.hot_off = ctx->d_hot_off.p; rp.hot_F = ctx->hot_F.p; rp.hot_P = ctx->hot_P.p;
  int n_ctas = std::max(1, std::min<int>((int)ctx->items.size(), ctx->n_sms * kReplayCtasPerSm));
  CK(launch_replay(rp, std::max(n_ctas, 1), s), "k_replay");
  if (!ctx->hot.empty()) {
    // K5 phases 2 and 3 (see build_items)
    uint32_t max_span = 0;
    for (const uint4& h : ctx->hot) max_span = std::max(max_span, h.z);
    CK(launch_carry(ctx->d_hot.p, (uint32_t)ctx->hot.size(), max_span, ctx->d_bucket_start.p, ctx->d_hot_off.p,
                    ctx->hot_F.p, ctx->hot_P.p, ctx->shadow, (ctx->cfg.flags & ARB_F_BO) ? 1 : 0,
                    ((ctx->cfg.flags >> ARB_F_DEVICES_SHIFT) & 3u) ? 1 : 0, s), "k_carry");
    CK(cudaMemsetAsync(&ctx->dstats.p->work, 0, sizeof(unsigned long long), s), "work reset");
    ReplayParams r3 = rp;
    r3.items = ctx->d_slice_items.p; r3.n_items = (uint32_t)ctx->slice_items.size();
    const int n3 = std::max(1, std::min<int>((int)ctx->slice_items.size(), ctx->n_sms * kReplayCtasPerSm));
    CK(launch_replay(r3, n3, s), "k_replay slices");
    launches += 2;
  }
  launches += 1;
  if (timing) cudaEventRecord(ctx->ev[3], s);
  CK(cudaMemcpyAsync(&hst, ctx->dstats.p, sizeof(hst), cudaMemcpyDeviceToHost, s), "stats d2h");
  CK(cudaStreamSynchronize(s), "replay sync");
  n_vsm = hst.n_cand;                                // exact: VSM candidates are unique
  kept_vsm = std::min(n_vsm, ctx->cand_cap);
  S.max_bucket_events = hst.max_bucket_events;
  S.steps_fast = hst.steps_fast;
  S.steps_sort = hst.steps_sort;
  S.steps_run = hst.steps_run;
  S.segments = hst.n_segs;
  S.chunks = (n + kChunkRecords - 1) / kChunkRecords; S.chunks_fast = hst.chunks_fast; S.chunks_run = hst.chunks_run;
  S.run_merges = hst.run_merges;

  // ---- A6: MIR join ---------------------------------------------------------------
  uint64_t n_mir = 0;
  const bool carry_in = ctx->n_carry && !plan.carry_in_dense.empty();
  if (!plan.mir.empty() || carry_in || !plan.carry_out.empty()) {
    MirPlanH& M = plan.mir;
    uint64_t hcap = 1;
    while (hcap < 2 * (2 * M.n_ins_pos + (carry_in ? ctx->n_carry : 0) + 1)) hcap <<= 1;
    CK(ctx->hkeys.ensure(hcap), "alloc hash");
    CK(ctx->hvals.ensure(hcap), "alloc hash");
    PackUpload pk;
    const size_t o_cmap = pk.add(plan.carry_in_dense);
    const size_t o_ins_lo = pk.add(M.ins_lo), o_ins_cum = pk.add(M.ins_cum), o_ins_inst = pk.add(M.ins_inst);
    const size_t o_qry_lo = pk.add(M.qry_lo), o_qry_cum = pk.add(M.qry_cum), o_qos = pk.add(M.qry_open_start);
    const size_t o_open = pk.add(M.open_list), o_own_start = pk.add(M.own_start), o_win_start = pk.add(M.win_start);
    const size_t o_own = pk.add(M.own_ops), o_win = pk.add(M.win_ops), o_rr = pk.add(M.rr), o_rr_cum = pk.add(M.rr_cum);
    CK(pk.run(ctx->m_pack, ctx->h_m_pack, s), "upload mir plan");
    const DevBuf<uint8_t>& D = ctx->m_pack;
    for (int attempt = 0; attempt < 2; ++attempt) {
      CK(cudaMemsetAsync(ctx->hkeys.p, 0, hcap * sizeof(unsigned long long), s), "hash clear");
      CK(cudaMemsetAsync(ctx->hvals.p, 0, hcap * sizeof(uint32_t), s), "hash clear");
      CK(cudaMemsetAsync(&ctx->dstats.p->n_mir_cand, 0, sizeof(unsigned long long), s), "mir count");
      MirParams mp{};
      mp.ev = ev; mp.base_word = ctx->base_word; mp.n_words = ctx->n_words;
      mp.ins_lo = PackUpload::at<decltype(mp.ins_lo)>(D, o_ins_lo);
      mp.ins_cum = PackUpload::at<decltype(mp.ins_cum)>(D, o_ins_cum);
      mp.ins_inst = PackUpload::at<decltype(mp.ins_inst)>(D, o_ins_inst);
      mp.n_ins = (uint32_t)M.ins_lo.size();
      mp.qry_lo = PackUpload::at<decltype(mp.qry_lo)>(D, o_qry_lo);
      mp.qry_cum = PackUpload::at<decltype(mp.qry_cum)>(D, o_qry_cum);
      mp.qry_open_start = PackUpload::at<decltype(mp.qry_open_start)>(D, o_qos);
      mp.n_qry = (uint32_t)M.qry_lo.size();
      mp.open_list = PackUpload::at<decltype(mp.open_list)>(D, o_open);
      mp.own_start = PackUpload::at<decltype(mp.own_start)>(D, o_own_start);
      mp.own_ops = PackUpload::at<decltype(mp.own_ops)>(D, o_own);
      mp.win_start = PackUpload::at<decltype(mp.win_start)>(D, o_win_start);
      mp.win_ops = PackUpload::at<decltype(mp.win_ops)>(D, o_win);
      mp.hkeys = ctx->hkeys.p; mp.hvals = ctx->hvals.p; mp.hmask = hcap - 1;
      mp.rr = PackUpload::at<decltype(mp.rr)>(D, o_rr);
      mp.rr_cum = PackUpload::at<decltype(mp.rr_cum)>(D, o_rr_cum);
      mp.n_rr = (uint32_t)M.rr.size();
      mp.carry = ctx->carry_ent.p; mp.n_carry = carry_in ? ctx->n_carry : 0;
      mp.cmap = carry_in ? PackUpload::at<decltype(mp.cmap)>(D, o_cmap) : nullptr;
      mp.cand = ctx->cand.p + kept_vsm; mp.cand_cap = ctx->cand.cap - kept_vsm; mp.st = ctx->dstats.p;
      CK(launch_mir(mp, M.n_ins_pos, M.n_qry_pos, M.n_rr_words, s, &launches), "k_mir");
      unsigned long long c = 0;
      CK(cudaMemcpyAsync(&c, &ctx->dstats.p->n_mir_cand, sizeof(c), cudaMemcpyDeviceToHost, s), "mir d2h");
      CK(cudaStreamSynchronize(s), "mir sync");
      n_mir = c;
      if (kept_vsm + n_mir <= ctx->cand.cap) break;
      // MIR kernels only read: grow and run them again
      DevBuf<uint4> bigger;
      CK(bigger.ensure(kept_vsm + n_mir), "grow candidates");
      if (kept_vsm) CK(cudaMemcpyAsync(bigger.p, ctx->cand.p, kept_vsm * 16, cudaMemcpyDeviceToDevice, s), "copy cand");
      CK(cudaStreamSynchronize(s), "copy sync");
      ctx->cand.release();
      ctx->cand = bigger;
    }
    if (!plan.carry_out.empty()) {
      // N2: the access summaries of the instances still unjoined go to the next flush
      CK(upload(ctx->m_co_of, plan.dense_carry_out, s), "carry map");
      CK(ctx->carry_next.ensure(hcap), "alloc carry");
      CK(cudaMemsetAsync(&ctx->dstats.p->n_carry_out, 0, sizeof(unsigned long long), s), "carry count");
      CK(launch_carry_extract(ctx->hkeys.p, ctx->hvals.p, hcap, ctx->m_co_of.p, ctx->carry_next.p,
                              &ctx->dstats.p->n_carry_out, s), "carry extract");
      launches += 1;
      unsigned long long c = 0;
      CK(cudaMemcpyAsync(&c, &ctx->dstats.p->n_carry_out, sizeof(c), cudaMemcpyDeviceToHost, s), "carry d2h");
      CK(cudaStreamSynchronize(s), "carry sync");
      n_carry_next = c;
    }
  }
  // ---- N1 (Z25): accesses through a tagged pointer outside its base's entry ------------
  if (!plan.tag_first.empty() && n) {
    CK(upload(ctx->d_tag_first, plan.tag_first, s), "tag table");
    CK(upload(ctx->d_tag_segs, plan.tag_segs, s), "tag segments");
    for (int attempt = 0; attempt < 2; ++attempt) {
      const uint64_t used = kept_vsm + n_mir;
      CK(cudaMemsetAsync(&ctx->dstats.p->n_bo_cand, 0, sizeof(unsigned long long), s), "bo count");
      CK(launch_bo_tags(ev, n, ctx->base_word, ctx->n_words, ctx->d_tag_first.p, ctx->d_tag_segs.p,
                        ctx->cand.p + used, ctx->cand.cap - used, &ctx->dstats.p->n_bo_cand, s), "k_bo_tags");
      launches += 1;
      unsigned long long c = 0;
      CK(cudaMemcpyAsync(&c, &ctx->dstats.p->n_bo_cand, sizeof(c), cudaMemcpyDeviceToHost, s), "bo d2h");
      CK(cudaStreamSynchronize(s), "bo sync");
      if (used + c <= ctx->cand.cap) { n_mir += c; break; }
      DevBuf<uint4> bigger;                    // read-only kernel: grow and run it again
      CK(bigger.ensure(used + c), "grow candidates");
      if (used) CK(cudaMemcpyAsync(bigger.p, ctx->cand.p, used * 16, cudaMemcpyDeviceToDevice, s), "copy cand");
      CK(cudaStreamSynchronize(s), "copy sync");
      ctx->cand.release();
      ctx->cand = bigger;
    }
  }
  if (timing) cudaEventRecord(ctx->ev[4], s);

  // ---- canonical order + unique ---------------------------------------------------
  const uint64_t n_cand = kept_vsm + n_mir;
  CK(ctx->cand_tmp.ensure(std::max<uint64_t>(n_cand, 1)), "alloc cand tmp");
  CK(ctx->reports.ensure(std::max<uint64_t>(n_cand, 1)), "alloc reports");
  uint64_t nblk = (n_cand + 4095) / 4096;
  CK(ctx->blk.ensure(nblk * 2049 + 4096), "alloc blk");
  CompactParams cp{};
  cp.cand = ctx->cand.p; cp.n_cand = n_cand; cp.tmp = ctx->cand_tmp.p; cp.blk = ctx->blk.p;
  cp.blk_cap = ctx->blk.cap; cp.base_word = ctx->base_word;
  int wb = 1; while (wb < 64 && (ctx->n_words - 1) >> wb) ++wb;
  int pb = 1; while (pb < 32 && (n ? (n - 1) >> pb : 0)) ++pb;
  cp.word_bits = wb; cp.pos_bits = pb;
  cp.dedup_first = (ctx->cfg.flags & ARB_F_DEDUP_FIRST) ? 1 : 0;
  // host global indices: positions now, translated on the host below
  cp.gidx = ctx->host_gidx ? nullptr : gidx; cp.index_base = ctx->host_gidx ? 0 : index_base;
  cp.out = ctx->reports.p; cp.n_out = ctx->dcount.p;
  if (cp.dedup_first) {
    // the persistent (word, kind) set of earlier flushes: keep its load <= 1/2
    const uint64_t need = 2 * (ctx->dset_n + n_cand);
    if (ctx->dset_slots < need) {
      uint64_t slots = 1ull << 16;
      while (slots < need) slots <<= 1;
      DevBuf<unsigned long long> nb;
      CK(nb.ensure(slots), "alloc dedup set");
      CK(cudaMemsetAsync(nb.p, 0, slots * 8, s), "clear dedup set");
      if (ctx->dset_slots) CK(launch_dedup_rehash(ctx->dset.p, ctx->dset_slots, nb.p, slots - 1, s), "rehash");
      CK(cudaStreamSynchronize(s), "rehash sync");
      ctx->dset.release();
      ctx->dset = nb;
      ctx->dset_slots = slots;
    }
    CK(ctx->dset_cnt.ensure(1), "alloc dedup count");
    CK(cudaMemsetAsync(ctx->dset_cnt.p, 0, 8, s), "dedup count");
    cp.dset = ctx->dset.p; cp.dset_mask = ctx->dset_slots - 1; cp.dset_count = ctx->dset_cnt.p;
  }
  CK(launch_compact(cp, s, &launches), "compact");
  unsigned long long dset_new = 0;
  if (cp.dedup_first) CK(cudaMemcpyAsync(&dset_new, ctx->dset_cnt.p, 8, cudaMemcpyDeviceToHost, s), "dedup count d2h");
  unsigned long long cnt4[8] = {0, 0, 0, 0, 0, 0, 0, 0};   // [0] total, [k] kind k
  CK(cudaMemcpyAsync(cnt4, ctx->dcount.p, sizeof(cnt4), cudaMemcpyDeviceToHost, s), "count d2h");
  if (timing) cudaEventRecord(ctx->ev[5], s);
  CK(cudaStreamSynchronize(s), "compact sync");
  const uint64_t n_out = cnt4[0];
  ctx->n_stored = n_out;
  ctx->reports_on_host = ctx->host_gidx;
  if (ctx->host_gidx && n_out) {
    // the report path reads the host global indices: position -> global_index[position]
    CK(ctx->h_reports.ensure(n_out), "pinned reports");
    CK(cudaMemcpyAsync(ctx->h_reports.p, ctx->reports.p, n_out * 16, cudaMemcpyDeviceToHost, s), "reports d2h");
    CK(cudaStreamSynchronize(s), "reports sync");
    std::vector<uint64_t> off(ctx->subs.size() + 1, 0);
    for (size_t k = 0; k < ctx->subs.size(); ++k) off[k + 1] = off[k] + ctx->subs[k].n;
    for (uint64_t i = 0; i < n_out; ++i) {
      uint4& r = ctx->h_reports.p[i];
      const uint64_t pos = (uint64_t)r.z | ((uint64_t)r.w << 32);
      const size_t k = (size_t)(std::upper_bound(off.begin(), off.end(), pos) - off.begin()) - 1;
      const uint64_t g = ctx->subs[k].gidx ? ctx->subs[k].gidx[pos - off[k]] : ctx->next_index + pos;
      r.z = (uint32_t)g; r.w = (uint32_t)(g >> 32);
    }
  }
  for (int k = 1; k < 4; ++k) S.reports_by_kind[k] = cnt4[k];
  S.reports_bo = cnt4[ARB_BO];
  ctx->dset_n += dset_new;
  // dropped VSM candidates are unique and distinct from every retained one (raw
  // mode; with ARB_F_DEDUP_FIRST an upper bound, see arbalest.h)
  ctx->n_reports = n_out + (n_vsm - kept_vsm);
  return ARB_OK;
  }();

  // ---- A7: multi-GPU count exchange --------------------------------
  // One ncclAllGather of {status, report count} per rank; the exclusive prefix of
  // the counts in rank order is this rank's offset in the global report list.
  uint64_t offset = 0;
  if (ctx->comm) {
    std::vector<int64_t> all;
    const int e = nccl_exchange(ctx, s, rcb, rcb < 0 ? 0 : (int64_t)ctx->n_reports, all);
    if (e != ARB_OK) { reset_batch(ctx); return ARB_ECUDA; }
    S.exchanges += 1;
    launches += 1;
    int64_t peer = 0;
    for (int r = 0; r < (int)all.size() / 2; ++r) {
      if (r < ctx->cfg.rank) offset += (uint64_t)all[2 * r + 1];
      if (r != ctx->cfg.rank && all[2 * r] < 0) peer = all[2 * r];
    }
    if (rcb == ARB_OK && peer < 0)
      rcb = fail(ctx, ARB_EPEER, "another rank failed while replaying its part of the batch; destroy the context");
  }
  if (rcb != ARB_OK) {
    reset_batch(ctx);
    return rcb;
  }
  rc = n_vsm > kept_vsm ? ARB_TRUNCATED : ARB_OK;
  if (rc == ARB_TRUNCATED) ctx->err = "report candidates exceeded report_capacity";
  if (timing) {
    cudaEventRecord(ctx->ev[6], s);
    cudaEventSynchronize(ctx->ev[6]);
    float ms;
    cudaEventElapsedTime(&ms, ctx->ev[0], ctx->ev[1]); S.ms_partition = ms;
    cudaEventElapsedTime(&ms, ctx->ev[0], ctx->ev[7]); S.ms_sample = ms;
    cudaEventElapsedTime(&ms, ctx->ev[1], ctx->ev[2]); S.ms_control = ms;
    cudaEventElapsedTime(&ms, ctx->ev[1], ctx->ev[8]); S.ms_segsort = ms;
    cudaEventElapsedTime(&ms, ctx->ev[2], ctx->ev[3]); S.ms_replay = ms;
    cudaEventElapsedTime(&ms, ctx->ev[3], ctx->ev[4]); S.ms_mir = ms;
    cudaEventElapsedTime(&ms, ctx->ev[4], ctx->ev[5]); S.ms_reports = ms;
    cudaEventElapsedTime(&ms, ctx->ev[0], ctx->ev[6]); S.ms_total = ms;
  }
  ctx->map.swap(map);
  ctx->carried.swap(plan.carry_out);          // N2: committed with the map table
  ctx->last_ended.swap(plan.last_ended_out);
  ctx->tags.swap(plan.tags_out);
  std::swap(ctx->carry_ent, ctx->carry_next);
  ctx->n_carry = n_carry_next;
  ctx->next_index += n;
  ctx->flushed = true;
  S.reports = ctx->n_reports;
  S.kernel_launches = launches;
  S.total_records += n;
  S.total_word_events += S.access_words + S.range_words;
  S.total_reports += ctx->n_reports;
  S.flushes += 1;
  reset_batch(ctx);
  if (n_reports_local) *n_reports_local = ctx->n_reports;
  if (report_offset_global) *report_offset_global = offset;
  return rc;
}

extern "C" int arb_get_reports(arb_ctx ctx, arb_report* out, uint64_t cap, uint64_t* n_written, int out_on_device) {
  if (!ctx) return ARB_EINVAL;
  if (!ctx->flushed) return fail(ctx, ARB_ESTATE, "no flush yet");
  uint64_t k = std::min(cap, ctx->n_stored);
  if (k) {
    if (!out) return fail(ctx, ARB_EINVAL, "null output");
    cudaError_t e;
    if (ctx->reports_on_host) {
      if (out_on_device) e = cudaMemcpy(out, ctx->h_reports.p, k * sizeof(arb_report), cudaMemcpyHostToDevice);
      else { std::memcpy(out, ctx->h_reports.p, k * sizeof(arb_report)); e = cudaSuccess; }
    } else {
      e = cudaMemcpy(out, ctx->reports.p, k * sizeof(arb_report),
                     out_on_device ? cudaMemcpyDeviceToDevice : cudaMemcpyDeviceToHost);
    }
    if (e != cudaSuccess) return cuda_fail(ctx, e, "get_reports");
  }
  if (n_written) *n_written = k;
  return cap < ctx->n_reports ? ARB_TRUNCATED : ARB_OK;
}

extern "C" int arb_get_shadow(arb_ctx ctx, uint64_t word_lo, uint64_t n, uint8_t* out, int out_on_device) {
  if (!ctx) return ARB_EINVAL;
  if (word_lo < ctx->base_word || word_lo + n > ctx->base_word + ctx->n_words || (n && !out))
    return fail(ctx, ARB_EINVAL, "shadow range outside the tracked range");
  if (!n) return ARB_OK;
  cudaError_t e = cudaMemcpy(out, ctx->shadow + (word_lo - ctx->base_word), n,
                             out_on_device ? cudaMemcpyDeviceToDevice : cudaMemcpyDeviceToHost);
  if (e != cudaSuccess) return cuda_fail(ctx, e, "get_shadow");
  return ARB_OK;
}

extern "C" int arb_get_stats(arb_ctx ctx, arb_stats* out) {
  if (!ctx || !out) return ARB_EINVAL;
  *out = ctx->stats;
  return ARB_OK;
}
