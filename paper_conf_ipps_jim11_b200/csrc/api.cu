// api.cpp — the libbmr C ABI (include/bmr.h) and the host job runtime: state machine, buffer
// sizing, overflow detection + replay, sort-pass planning, output assembly and fetch.
// Every computational step runs in the CUDA kernels of map.cu / sort.cu / reduce.cu; this file
// only orchestrates launches on the job stream.  There is no CPU fallback: without a CUDA
// device every call that needs one fails with MR_ERR_CUDA.
#include <cuda_runtime.h>

#include <algorithm>
#include <atomic>
#include <cstdio>
#include <cstring>
#include <new>
#include <string>
#include <vector>

#include "bmr.h"
#include "comm.h"
#include "kernels.h"

using namespace bmr;

std::atomic<unsigned long long> bmr::g_kernel_launches{0};

namespace {

enum State { kCreated = 0, kMapped = 1, kGrouped = 2, kReduced = 3, kPartitioned = 4 };

template <typename T>
struct DBuf {
  T* p = nullptr;
  uint64_t n = 0;
  // grow-only with 1/16 headroom: sizes that drift by a few elements between runs (e.g. the
  // number of flush filler pairs) must not trigger a multi-GB cudaFree/cudaMalloc per step
  cudaError_t ensure(uint64_t need) {
    if (need <= n && p) return cudaSuccess;
    release();
    const uint64_t cnt = std::max<uint64_t>(need + need / 16, 1);
    cudaError_t e = cudaMalloc(reinterpret_cast<void**>(&p), cnt * sizeof(T));
    if (e != cudaSuccess) { p = nullptr; n = 0; cudaGetLastError(); return e; }
    n = cnt;
    return cudaSuccess;
  }
  void release() { if (p) cudaFree(p); p = nullptr; n = 0; }
};

template <typename T>
struct HBuf {  // pinned host
  T* p = nullptr;
  uint64_t n = 0;
  cudaError_t ensure(uint64_t need) {
    if (need <= n && p) return cudaSuccess;
    release();
    const uint64_t cnt = std::max<uint64_t>(need, 1);
    cudaError_t e = cudaMallocHost(reinterpret_cast<void**>(&p), cnt * sizeof(T));
    if (e != cudaSuccess) { p = nullptr; n = 0; cudaGetLastError(); return e; }
    n = cnt;
    return cudaSuccess;
  }
  void release() { if (p) cudaFreeHost(p); p = nullptr; n = 0; }
};

// MR_FLAG_PROFILE: CUDA events around each phase on the job stream; elapsed times are
// collected at the next synchronisation point.
struct Prof {
  struct Span { cudaEvent_t a, b; double* acc; };
  std::vector<cudaEvent_t> pool;
  std::vector<Span> open;
  size_t used = 0;
  bool on = false;
  cudaEvent_t get() {
    if (used == pool.size()) {
      cudaEvent_t e;
      cudaEventCreate(&e);
      pool.push_back(e);
    }
    return pool[used++];
  }
  void begin(cudaStream_t s, Span& sp) { sp.a = get(); cudaEventRecord(sp.a, s); }
  void end(cudaStream_t s, Span& sp, double* acc) {
    sp.b = get();
    cudaEventRecord(sp.b, s);
    sp.acc = acc;
    open.push_back(sp);
  }
  void collect() {  // call after the stream was synchronised
    for (auto& sp : open) {
      float ms = 0;
      if (cudaEventElapsedTime(&ms, sp.a, sp.b) == cudaSuccess) *sp.acc += ms;
    }
    cudaGetLastError();
    open.clear();
    used = 0;
  }
  void release() { for (auto e : pool) cudaEventDestroy(e); pool.clear(); open.clear(); used = 0; }
};

struct Batch {
  const uint8_t* rec;
  const uint64_t* off;
  uint64_t n, nbytes, gbase;   // text: nbytes / gbase live in the batch's device descriptor
  uint32_t di;                 // descriptor index (text)
};

// Sort workspace shared by mr_group and mr_sort_u64.
struct SortWork {
  DBuf<uint64_t> ka, kb, status;
  DBuf<uint32_t> ia, ib, hist, bases;
  DBuf<uint32_t> ka32, kb32;      // u32 keys-only ping-pong (WC exact stream)
  HBuf<uint32_t> hist_h, bases_h;
  uint32_t epoch = 1;
  uint64_t passes = 0;
  void release() {
    ka.release(); kb.release(); status.release(); ia.release(); ib.release(); hist.release(); bases.release();
    hist_h.release(); bases_h.release(); ka32.release(); kb32.release();
  }
};

__global__ void k_iota_u32(uint32_t* p, uint64_t n) {
  const uint64_t i = blockIdx.x * static_cast<uint64_t>(blockDim.x) + threadIdx.x;
  if (i < n) p[i] = static_cast<uint32_t>(i);
}

int sm_count(int dev) {
  int v = 148;
  if (cudaDeviceGetAttribute(&v, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess) { cudaGetLastError(); v = 148; }
  return v;
}

// Radix sort of m keys on their low key_width bits: writes *out_keys / *out_perm pointing into
// the workspace (or to `keys` + an identity permutation when every digit is constant).
// out_perm == nullptr: keys only (no permutation payload).  8-bit digits; constant digits are
// skipped.
cudaError_t run_sort(SortWork& W, const uint64_t* keys, uint64_t m, const uint64_t** out_keys,
                     const uint32_t** out_perm, DevState* st, int nsm, cudaStream_t s, Prof* prof = nullptr,
                     double* hist_ms = nullptr, double* pass_ms = nullptr, int key_width = 64) {
  cudaError_t e;
  const bool pay = out_perm != nullptr;
  const int bits = 8, bins = 1 << bits;
  const int ndig = std::min(8, (key_width + bits - 1) / bits);
  if ((e = W.ka.ensure(m + 1)) || (e = W.kb.ensure(m + 1))) return e;   // +1: seg_start sentinel
  if (pay && ((e = W.ia.ensure(m)) || (e = W.ib.ensure(m)))) return e;
  const uint64_t tile = pay ? sort_tile() : sort_tile_keys();
  const uint64_t tiles = (m + tile - 1) / tile;
  const uint64_t need_status = tiles * bins;
  if (W.status.n < need_status || !W.status.p) {
    if ((e = W.status.ensure(need_status))) return e;
    if ((e = cudaMemsetAsync(W.status.p, 0, W.status.n * sizeof(uint64_t), s))) return e;
  }
  if ((e = W.hist.ensure(8 * kBinStride)) || (e = W.bases.ensure(8 * kBinStride))) return e;
  if ((e = W.hist_h.ensure(8 * kBinStride)) || (e = W.bases_h.ensure(8 * kBinStride))) return e;
  {
    Prof::Span sp{};
    if (prof && prof->on) prof->begin(s, sp);
    if ((e = launch_hist(keys, m, W.hist.p, ndig, bits, nsm, s))) return e;
    if (prof && prof->on) prof->end(s, sp, hist_ms);
  }
  if ((e = cudaMemcpyAsync(W.hist_h.p, W.hist.p, 8 * kBinStride * sizeof(uint32_t), cudaMemcpyDeviceToHost, s)))
    return e;
  if ((e = cudaStreamSynchronize(s))) return e;
  int digits[8];
  int nd = 0;
  for (int d = 0; d < ndig; ++d) {
    uint32_t run = 0;
    int nonzero = 0;
    for (int b = 0; b < bins; ++b) {
      const uint32_t c = W.hist_h.p[d * kBinStride + b];
      W.bases_h.p[d * kBinStride + b] = run;
      run += c;
      nonzero += c ? 1 : 0;
    }
    if (nonzero > 1) digits[nd++] = d;  // constant digits are skipped
  }
  W.passes = nd;
  if (nd == 0) {
    *out_keys = keys;
    if (!pay) return cudaSuccess;
    k_iota_u32<<<static_cast<unsigned>((m + 255) / 256 + 1), 256, 0, s>>>(W.ia.p, m);
    count_launch();
    *out_perm = W.ia.p;
    return cudaGetLastError();
  }
  if ((e = cudaMemcpyAsync(W.bases.p, W.bases_h.p, 8 * kBinStride * sizeof(uint32_t), cudaMemcpyHostToDevice, s)))
    return e;
  const uint64_t* kin = keys;
  const uint32_t* iin = nullptr;
  Prof::Span sp2{};
  if (prof && prof->on) prof->begin(s, sp2);
  for (int p = 0; p < nd; ++p) {
    uint64_t* kout = (p & 1) ? W.kb.p : W.ka.p;
    uint32_t* iout = pay ? ((p & 1) ? W.ib.p : W.ia.p) : nullptr;
    const int rk = pay ? kRankMatch : choose_rank_kind32(W.hist_h.p + digits[p] * kBinStride, m, p == 0);
    if ((e = launch_onesweep(kin, iin, kout, iout, m, digits[p], bits, W.bases.p, W.status.p, W.epoch++,
                             &st->tile_counter[0], s, rk)))
      return e;
    kin = kout;
    iin = iout;
  }
  if (prof && prof->on) prof->end(s, sp2, pass_ms);
  *out_keys = kin;
  if (pay) *out_perm = iin;
  return cudaSuccess;
}


// Keys-only radix sort of m u32 keys on their low key_width bits (the WC exact stream):
// *out_keys points into the workspace (or at `keys` when every digit is constant).
cudaError_t run_sort32(SortWork& W, const uint32_t* keys, uint64_t m, const uint32_t** out_keys, DevState* st,
                       int nsm, cudaStream_t s, Prof* prof, double* hist_ms, double* pass_ms, int key_width) {
  cudaError_t e;
  const int bits = 8, bins = 1 << bits;
  const int ndig = std::min(4, (key_width + bits - 1) / bits);
  if ((e = W.ka32.ensure(m + 1)) || (e = W.kb32.ensure(m + 1))) return e;
  const uint64_t tiles = (m + sort_tile_keys32() - 1) / sort_tile_keys32();
  const uint64_t need_status = tiles * bins;
  if (W.status.n < need_status || !W.status.p) {
    if ((e = W.status.ensure(need_status))) return e;
    if ((e = cudaMemsetAsync(W.status.p, 0, W.status.n * sizeof(uint64_t), s))) return e;
  }
  if ((e = W.hist.ensure(8 * kBinStride)) || (e = W.bases.ensure(8 * kBinStride))) return e;
  if ((e = W.hist_h.ensure(8 * kBinStride)) || (e = W.bases_h.ensure(8 * kBinStride))) return e;
  {
    Prof::Span sp{};
    if (prof && prof->on) prof->begin(s, sp);
    if ((e = launch_hist32(keys, m, W.hist.p, ndig, bits, nsm, s))) return e;
    if (prof && prof->on) prof->end(s, sp, hist_ms);
  }
  if ((e = cudaMemcpyAsync(W.hist_h.p, W.hist.p, 8 * kBinStride * sizeof(uint32_t), cudaMemcpyDeviceToHost, s)))
    return e;
  if ((e = cudaStreamSynchronize(s))) return e;
  int digits[4];
  int nd = 0;
  for (int d = 0; d < ndig; ++d) {
    uint32_t run = 0;
    int nonzero = 0;
    for (int b = 0; b < bins; ++b) {
      const uint32_t c = W.hist_h.p[d * kBinStride + b];
      W.bases_h.p[d * kBinStride + b] = run;
      run += c;
      nonzero += c ? 1 : 0;
    }
    if (nonzero > 1) digits[nd++] = d;  // constant digits are skipped
  }
  W.passes = nd;
  *out_keys = keys;
  if (nd == 0) return cudaSuccess;
  if ((e = cudaMemcpyAsync(W.bases.p, W.bases_h.p, 8 * kBinStride * sizeof(uint32_t), cudaMemcpyHostToDevice, s)))
    return e;
  const uint32_t* kin = keys;
  Prof::Span sp2{};
  if (prof && prof->on) prof->begin(s, sp2);
  for (int p = 0; p < nd; ++p) {
    uint32_t* kout = (p & 1) ? W.kb32.p : W.ka32.p;
    const int rk = choose_rank_kind32(W.hist_h.p + digits[p] * kBinStride, m, p == 0);
    if ((e = launch_onesweep32(kin, kout, m, digits[p], bits, W.bases.p, W.status.p, W.epoch++,
                               &st->tile_counter[0], s, rk)))
      return e;
    kin = kout;
  }
  if (prof && prof->on) prof->end(s, sp2, pass_ms);
  *out_keys = kin;
  return cudaSuccess;
}

}  // namespace

struct mr_job {
  mr_config cfg{};
  mr_sm_params sm{};
  uint32_t k = 0;
  std::vector<float> cent_h;
  int state = kCreated;
  cudaStream_t stream = nullptr;
  bool own_stream = false;
  int nsm = 148;
  std::string err;
  DevState* st = nullptr;
  HBuf<DevState> st_h;
  HBuf<uint64_t> tmp_h;
  DBuf<float> cent;
  DBuf<uint64_t> h, kref, tb;
  DBuf<uint32_t> hx;              // WC exact stream keys (u32)
  // WC in-SMEM combiner (f-1): partial entries (key | count << 32), their sort / segments / merge
  DBuf<uint64_t> hp, seg_startp, psum, pxcounts;
  DBuf<uint32_t> midx, xkeys;
  uint64_t cap_p = 0, mp = 0, nseg_p = 0, n_extra = 0;
  const uint64_t* skeysp = nullptr;
  DBuf<uint8_t> v;
  uint64_t cap = 0;
  std::vector<Batch> batches;
  uint64_t next_base = 0;        // fixed-stride batches: running global byte base
  // text batches: device descriptors (nbytes, ntiles, gbase, tile-cap overflow) written by
  // k_tile_bounds, 4 u64 per batch since the last reset; tile-bounds capacity in tiles
  DBuf<uint64_t> bdesc;
  HBuf<uint64_t> bdesc_h;
  uint32_t ndesc = 0;
  uint64_t tb_cap = 0;
  std::vector<void*> owned;       // reserved
  std::vector<DBuf<uint8_t>> host_rec;   // device copies made by mr_map_host (reused after reset)
  std::vector<DBuf<uint64_t>> host_off;
  size_t host_batches = 0;
  cudaStream_t cstream = nullptr;        // copy stream of mr_map_host_lines
  std::vector<cudaEvent_t> line_ev;
  Prof prof;
  unsigned long long launches0 = 0;
  SortWork sw, swb, swc, swp;
  const uint64_t* skeys = nullptr;
  const uint32_t* skeysx = nullptr;   // WC exact stream, sorted (u32)
  const uint32_t* perm = nullptr;
  uint64_t m = 0, nseg = 0, key_bytes = 0;
  // WC hashed stream (the exact stream uses h / skeys / seg_start): pairs, sorted, segments
  DBuf<uint64_t> hb, krefb, seg_startb;
  uint64_t* sega = nullptr;       // exact-stream segment starts (seg_startx)
  DBuf<uint64_t> seg_startx;
  uint64_t cap_b = 0, mb = 0, nseg_a = 0, nseg_b = 0;
  // WC mid stream (6..8-byte words, exact 48-bit keys, keys only)
  DBuf<uint64_t> hc;
  uint64_t cap_c = 0, mc = 0, nseg_c = 0;
  const uint64_t* skeysc = nullptr;
  uint64_t* segc = nullptr;
  const uint64_t* skeysb = nullptr;
  const uint32_t* permb = nullptr;
  uint32_t key_bits_b = 48;
  DBuf<uint64_t> scan_status;     // look-back words of the single-pass scans (epoch-tagged)
  uint32_t scan_epoch = 1;
  DBuf<uint32_t> seg_counts;
  DBuf<uint64_t> tile_base, seg_start, key_off, val_off, counts, worklist, gathered;
  DBuf<uint8_t> keys_out, vals_out, vsorted;
  DBuf<double> sums;
  DBuf<unsigned long long> cnts;
  // fetched result
  HBuf<uint8_t> keys_h, vals_h;
  HBuf<uint64_t> key_off_h, val_off_h;
  // multi-GPU exchange (§8(e))
  XSource xs;
  uint32_t key_bits = 64;         // current sort-key width (WC maps with 48; re-hash -> 64)
  // WC Map output = exact stream + hashed stream (values 1, not stored); ingested WC pairs are
  // one general stream (key, kref, u64 partial count) like II
  bool split() const { return cfg.workload == MR_WORDCOUNT && !ingested; }
  bool wc_comb() const { return split() && !(cfg.flags & MR_FLAG_NO_MAP_COMBINE); }
  // second combiner level: exact words that miss the SMEM table go to an L2-resident count table
  // (the raw multi-GPU exchange, MR_FLAG_NO_COMBINE, keeps the literal pair streams)
  bool wc_table() const {
    return tables_on && wc_comb() && map_wc_table_ok(cfg.flags) && !(cfg.flags & MR_FLAG_NO_COMBINE);
  }
  // per run, from the first batch's size: the tables (tables_on; BMR_TABLE_MIN_BYTES, default 0)
  // and among them the direct-address exact-key table (xtab_on; BMR_XTAB_MIN_BYTES, default
  // 64 MiB): extracting it streams 4 GiB (~0.6 ms), so a small input (C1: 1 MiB) counts its
  // exact words in the mid table instead ("small-table mode": the Map's exact-word combiner
  // misses probe the open-addressing table; no sort, no 4 GiB scan)
  bool tables_on = true;
  bool xtab_on = true;
  DBuf<uint32_t> xtab;            // 2^30 u32 counts by exact key (zero between runs)
  // mid words (6..8 symbols): open-addressing table of 48-bit exact keys + counts (2^mbits slots)
  DBuf<uint64_t> mtab_keys;
  DBuf<uint32_t> mtab_cnt;
  uint32_t mbits = 18;
  bool xtab_dirty = false;        // a Map fed the tables since their last extraction
  bool mid_from_table = false;    // this group's mid keys / counts come from the mid table
  DBuf<uint64_t> mkeys_out, mcounts;
  // long words (9..16 symbols): open-addressing table of their 16 zero-padded key bytes + counts
  DBuf<uint64_t> ltab_keys;
  DBuf<uint32_t> ltab_cnt;
  uint32_t lbits = 19;   // (table mode: also the words of 6..8 symbols, BMR_WC_UNITAB)
  DBuf<uint64_t> lkeys_out, lkref_out, lcounts;
  uint64_t nseg_l = 0;            // long-table keys of this group (the output's last list)
  // KM: the Map accumulates the cluster sums itself (k <= 64; not for ingested partials)
  bool km_comb() const {
    return cfg.workload == MR_KMEANS && k <= 64 && !km_partial && !(cfg.flags & MR_FLAG_NO_MAP_COMBINE);
  }
  bool km_combined = false;       // KM: sums / cnts were produced by the Map combiner
  bool ingested = false;          // pairs come from mr_ingest (WC values are u64 partial counts)
  bool km_partial = false;        // KM: sums/cnts hold ingested partials; finalise owned clusters
  int vb_cur = 0;                 // value bytes of the current pairs
  DBuf<unsigned long long> xcounts, xcursors, xheapbase;
  HBuf<unsigned long long> xcounts_h;
  DBuf<uint64_t> src_e, src_h;
  DBuf<XWindow> xwin;             // f-3: receive windows of the fused Map flush (InvertedIndex)
  // the exchange inside mr_group (nranks > 1 with cfg.nccl_comm): send / receive buffers (the
  // received heap holds the key bytes the ingested pairs reference until mr_reduce completes)
  DBuf<uint8_t> xsend_e, xsend_h, xrecv_e, xrecv_h;
  DBuf<uint64_t> xrecv_counts;
  bool in_exchange = false;       // mr_group called by the exchange's own combiner step
  bool exchanged = false;         // this run's pairs already went through an exchange (mr_ingest)
  // WC batch combine (MR_FLAG_BATCH_COMBINE, SURVEY §8(e) strong scaling; "batched
  // processing at another level"): every batch is grouped + reduced when the next one is mapped
  // (or at mr_group) and its (key, count) partials appended to an arena of 16-B entries + key
  // bytes; mr_group then ingests the arena and groups the partials (counts summed exactly)
  DBuf<uint8_t> acc_e, acc_h;
  uint64_t acc_ne = 0, acc_nh = 0;
  uint32_t nfolds = 0;
  bool in_fold = false;
  mr_stats fold_stats{};          // per-group counters of the folded batches (added at the end)
  uint32_t xranks = 0;
  DBuf<uint32_t> km_list;
  uint32_t km_nlist = 0;
  uint64_t out_keys_bytes = 0, out_vals_bytes = 0, out_n = 0;
  mr_stats stats{};
};

namespace {

mr_status fail(mr_job* j, mr_status s, const std::string& msg) {
  if (j) j->err = msg;
  return s;
}
mr_status cuda_fail(mr_job* j, cudaError_t e, const char* where) {
  std::string m = std::string(where) + ": " + cudaGetErrorString(e);
  cudaGetLastError();
  return fail(j, e == cudaErrorMemoryAllocation ? MR_ERR_OOM : MR_ERR_CUDA, m);
}
#define CK(expr, where)                                  \
  do {                                                   \
    cudaError_t e_ = (expr);                             \
    if (e_ != cudaSuccess) return cuda_fail(job, e_, where); \
  } while (0)

uint64_t initial_cap(const mr_job* job, uint64_t nbytes, uint64_t n) {
  if (job->cfg.max_pairs_hint) return job->cfg.max_pairs_hint;
  switch (job->cfg.workload) {
    case MR_WORDCOUNT: return nbytes / 4 + 4096;
    case MR_STRINGMATCH: return nbytes / 256 + 4096;
    case MR_KMEANS: return n + 4096;
    default: return nbytes / 32 + 4096;
  }
}

// cap_b / cap_c: WC hashed / mid stream capacities (0 for the other workloads)
cudaError_t ensure_pairs(mr_job* job, uint64_t cap, uint64_t cap_b, uint64_t cap_c) {
  cudaError_t e;
  if (job->split()) {
    if ((e = job->hx.ensure(cap))) return e;
  } else if ((e = job->h.ensure(cap))) {
    return e;
  }
  if (has_kref(job->cfg.workload) && (e = job->kref.ensure(cap))) return e;
  const int vb = vbytes_of(job->cfg.workload);
  if (vb && (e = job->v.ensure(cap * vb))) return e;
  job->cap = cap;
  if (cap_b) {
    if ((e = job->hb.ensure(cap_b)) || (e = job->krefb.ensure(cap_b))) return e;
  }
  job->cap_b = cap_b;
  if (cap_c && (e = job->hc.ensure(cap_c))) return e;
  job->cap_c = cap_c;
  return cudaSuccess;
}
void release_pairs(mr_job* job) {
  job->hp.release(); job->cap_p = 0;
  job->h.release(); job->hx.release(); job->kref.release(); job->v.release(); job->hb.release(); job->krefb.release();
  job->hc.release();
  job->cap = job->cap_b = job->cap_c = 0;
}

cudaError_t launch_batch(mr_job* job, const Batch& b) {
  MapArgs a;
  a.workload = job->cfg.workload;
  a.flags = job->cfg.flags;
  a.records = b.rec;
  a.offsets = b.off;
  a.n = b.n;
  a.nbytes = b.nbytes;
  a.stride = job->cfg.record_stride;
  a.gbase = b.gbase;
  std::memcpy(a.pattern, job->sm.pattern, 16);
  a.centroids = job->cent.p;
  a.k = job->k;
  a.out.h = job->h.p;
  a.out.hx = job->hx.p;
  a.out.hp = job->wc_comb() ? job->hp.p : nullptr;
  a.out.xtab = job->wc_table() && job->xtab_on ? job->xtab.p : nullptr;
  a.out.mkeys = job->wc_table() ? job->mtab_keys.p : nullptr;
  a.out.mcnt = job->wc_table() ? job->mtab_cnt.p : nullptr;
  a.out.mbits = job->mbits;
  a.out.lkeys = job->wc_table() ? job->ltab_keys.p : nullptr;
  a.out.lcnt = job->wc_table() ? job->ltab_cnt.p : nullptr;
  a.out.lbits = job->lbits;
  if (a.out.xtab || a.out.mkeys) job->xtab_dirty = true;
  a.out.km_sums = job->km_comb() ? job->sums.p : nullptr;
  a.out.km_cnts = job->km_comb() ? job->cnts.p : nullptr;
  a.out.cap_p = job->cap_p;
  a.out.kref = job->kref.p;
  a.out.v = job->v.p;
  a.out.cap = job->cap;
  a.out.hb = job->hb.p;
  a.out.krefb = job->krefb.p;
  a.out.cap_b = job->cap_b;
  a.out.hc = job->hc.p;
  a.out.cap_c = job->cap_c;
  a.st = job->st;
  a.hash_seed = 0x5EEDB200ULL;
  a.key_bits = job->key_bits;
  a.xwin = job->xranks ? job->xwin.p : nullptr;
  a.xranks = job->xranks;
  if (a.workload != kKM) {   // text: dimensions on the device
    cudaError_t e = job->tb.ensure(2 * job->tb_cap + 2);
    if (e) return e;
    a.desc = job->bdesc.p + 4ULL * b.di;
    a.prev_desc = b.di ? job->bdesc.p + 4ULL * (b.di - 1) : nullptr;
    a.input_base = job->cfg.input_base;
    a.tb_cap = job->tb_cap;
  } else {
    job->stats.map_tiles += map_tiles(a);
  }
  a.tile_bounds = job->tb.p;
  return launch_map(a, job->nsm, job->stream);
}

cudaError_t read_state(mr_job* job) {
  cudaError_t e = cudaMemcpyAsync(job->st_h.p, job->st, sizeof(DevState), cudaMemcpyDeviceToHost, job->stream);
  if (e) return e;
  return cudaStreamSynchronize(job->stream);
}

// Look-back workspace for a scan of n elements (k_scan: 2048 per tile, 3 words per tile).
cudaError_t scan_ws(mr_job* job, uint64_t n, uint64_t** status, uint32_t* epoch) {
  const uint64_t need = 3 * ((n + 2047) / 2048) + 3;
  if (job->scan_status.n < need || !job->scan_status.p) {
    cudaError_t e = job->scan_status.ensure(need);
    if (e == cudaSuccess) e = cudaMemsetAsync(job->scan_status.p, 0, job->scan_status.n * 8, job->stream);
    if (e != cudaSuccess) return e;
  }
  *status = job->scan_status.p;
  *epoch = job->scan_epoch++;
  return cudaSuccess;
}

// Segment heads of one sorted stream -> seg_start[0..nseg] (seg_start[nseg] = m).
mr_status do_segments(mr_job* job, const uint64_t* skeys, const uint32_t* perm, const uint64_t* kref, uint64_t m,
                      uint32_t key_bits, DBuf<uint64_t>& seg_start, uint64_t& nseg) {
  const uint64_t tiles = (m + 4095) / 4096;
  CK(job->seg_counts.ensure(tiles + 1), "alloc seg counts");
  CK(job->tile_base.ensure(tiles + 1), "alloc tile base");
  CK(cudaMemsetAsync(&job->st->collisions, 0, sizeof(unsigned int), job->stream), "memset");
  CK(launch_seg_count(skeys, perm, kref, m, job->seg_counts.p, job->st, key_bits, ~0ULL, job->stream), "seg_count");
  uint64_t* ss;
  uint32_t ep;
  CK(scan_ws(job, tiles, &ss, &ep), "alloc scan workspace");
  CK(launch_scan_u32to64(job->seg_counts.p, job->tile_base.p, tiles, &job->st->seg_total, ss, ep,
                         &job->st->tile_counter[1], job->stream),
     "scan tiles");
  CK(read_state(job), "sync segments");
  nseg = m ? job->st_h.p->seg_total : 0;
  CK(seg_start.ensure(nseg + 1), "alloc seg_start");
  CK(launch_seg_write(skeys, m, job->tile_base.p, seg_start.p, ~0ULL, job->stream), "seg_write");
  return MR_OK;
}

// Keys-only stream: heads counted, scanned and written into a caller-provided seg_start (m + 1).
mr_status do_segments_into(mr_job* job, const uint64_t* skeys, uint64_t m, uint64_t* seg_start, uint64_t& nseg,
                           uint64_t kmask = ~0ULL) {
  const uint64_t tiles = (m + 4095) / 4096;
  CK(job->seg_counts.ensure(tiles + 1), "alloc seg counts");
  CK(job->tile_base.ensure(tiles + 1), "alloc tile base");
  CK(launch_seg_count(skeys, nullptr, nullptr, m, job->seg_counts.p, job->st, 48, kmask, job->stream), "seg_count");
  uint64_t* ss;
  uint32_t ep;
  CK(scan_ws(job, tiles, &ss, &ep), "alloc scan workspace");
  CK(launch_scan_u32to64(job->seg_counts.p, job->tile_base.p, tiles, &job->st->seg_total, ss, ep,
                         &job->st->tile_counter[1], job->stream),
     "scan tiles");
  CK(launch_seg_write(skeys, m, job->tile_base.p, seg_start, kmask, job->stream), "seg_write");
  CK(read_state(job), "sync segments");
  nseg = m ? job->st_h.p->seg_total : 0;
  return MR_OK;
}

// Keys-only u32 stream (WC exact): heads counted and scanned; seg_start sized from the count.
mr_status do_segments32(mr_job* job, const uint32_t* skeys, uint64_t m, DBuf<uint64_t>& seg_start, uint64_t& nseg) {
  const uint64_t tiles = (m + 4095) / 4096;
  CK(job->seg_counts.ensure(tiles + 1), "alloc seg counts");
  CK(job->tile_base.ensure(tiles + 1), "alloc tile base");
  CK(launch_seg_count32(skeys, m, job->seg_counts.p, job->stream), "seg_count");
  uint64_t* ss;
  uint32_t ep;
  CK(scan_ws(job, tiles, &ss, &ep), "alloc scan workspace");
  CK(launch_scan_u32to64(job->seg_counts.p, job->tile_base.p, tiles, &job->st->seg_total, ss, ep,
                         &job->st->tile_counter[1], job->stream),
     "scan tiles");
  CK(read_state(job), "sync segments");
  nseg = m ? job->st_h.p->seg_total : 0;
  CK(seg_start.ensure(nseg + 1), "alloc seg_start");
  CK(launch_seg_write32(skeys, m, job->tile_base.p, seg_start.p, job->stream), "seg_write");
  return MR_OK;
}

// D7: settle the Map of every batch.  The cursors counted demand past capacity: grow the pair
// buffers and replay every batch.  Leaves the final DevState in st_h.
cudaError_t clear_tables(mr_job* job);

mr_status settle_map(mr_job* job) {
  CK(read_state(job), "map (async)");
  DevState* hs = job->st_h.p;
  if (hs->err & kErrNullRecords) return fail(job, MR_ERR_INVALID, "records is NULL for a non-empty batch");
  if (hs->err & kErrKeyTooLong) return fail(job, MR_ERR_OVERFLOW, "an emitted key exceeds 65535 bytes");
  if (job->ingested) return MR_OK;   // ingested pairs: exact count, written into buffers sized for it
  // text batches: the dimensions the device derived (stats; tile-bounds capacity)
  uint64_t max_tiles = 0;
  if (job->cfg.record_stride == 0 && job->ndesc) {
    CK(job->bdesc_h.ensure(4ULL * job->ndesc), "alloc host descriptors");
    CK(cudaMemcpyAsync(job->bdesc_h.p, job->bdesc.p, 32ULL * job->ndesc, cudaMemcpyDeviceToHost, job->stream),
       "D2H descriptors");
    CK(cudaStreamSynchronize(job->stream), "sync descriptors");
    uint64_t bytes = 0, tiles = 0;
    for (uint32_t i = 0; i < job->ndesc; ++i) {
      bytes += job->bdesc_h.p[4 * i];
      tiles += job->bdesc_h.p[4 * i + 1];
      max_tiles = std::max(max_tiles, job->bdesc_h.p[4 * i + 1]);
    }
    job->stats.input_bytes = bytes;
    job->stats.map_tiles = tiles;
  }
  const bool tile_over = (hs->err & kErrTileCap) != 0;
  const bool mid_over = (hs->err & kErrMidTable) != 0;
  const bool long_over = (hs->err & kErrLongTable) != 0;
  if (long_over) {   // long-word table too full: 4x larger, then the replay below
    job->lbits += 2;
    job->ltab_keys.release();
    job->ltab_cnt.release();
    CK(job->ltab_keys.ensure(2ULL << job->lbits), "grow long table");
    CK(job->ltab_cnt.ensure((1ULL << job->lbits) * kMidStripes), "grow long table");
  }
  if (mid_over) {   // mid table too full: a table 4x larger (grow-only), then the replay below
    job->mbits += 2;
    job->mtab_keys.release();
    job->mtab_cnt.release();
    CK(job->mtab_keys.ensure(1ULL << job->mbits), "grow mid table");
    CK(job->mtab_cnt.ensure((1ULL << job->mbits) * kMidStripes), "grow mid table");
  }
  // Grow from the demand counted past capacity and replay every batch.  The demand of a run is
  // not exactly that of the next: flush / spill padding and the warp-private chunks depend on
  // which warps and CTAs took which windows and tiles (dynamic scheduling), so a replay that
  // still overflows grows again from its own demand (up to kMaxReplays rounds).
  constexpr int kMaxReplays = 4;
  for (int round = 0;; ++round) {
    const uint64_t m = hs->pair_cursor, mb = job->split() ? hs->pair_cursor_b : 0;
    const uint64_t mc = job->split() ? hs->pair_cursor_c : 0;
    const uint64_t mp = job->wc_comb() ? hs->pair_cursor_p : 0;
    const bool t_over = (hs->err & kErrTileCap) != 0, m_over = (hs->err & kErrMidTable) != 0;
    const bool l_over = (hs->err & kErrLongTable) != 0;
    if (!(t_over || m_over || l_over || m > job->cap || mb > job->cap_b || mc > job->cap_c || mp > job->cap_p))
      return MR_OK;
    if (round == kMaxReplays) return fail(job, MR_ERR_OOM, "replay still overflows");
    if (round > 0) {   // tables overflowing again after a replay: grow them again
      if (l_over) {
        job->lbits += 2;
        job->ltab_keys.release();
        job->ltab_cnt.release();
        CK(job->ltab_keys.ensure(2ULL << job->lbits), "grow long table");
        CK(job->ltab_cnt.ensure((1ULL << job->lbits) * kMidStripes), "grow long table");
      }
      if (m_over) {
        job->mbits += 2;
        job->mtab_keys.release();
        job->mtab_cnt.release();
        CK(job->mtab_keys.ensure(1ULL << job->mbits), "grow mid table");
        CK(job->mtab_cnt.ensure((1ULL << job->mbits) * kMidStripes), "grow mid table");
      }
      if (t_over) {   // (the descriptors of the replay)
        CK(job->bdesc_h.ensure(4ULL * job->ndesc), "alloc host descriptors");
        CK(cudaMemcpyAsync(job->bdesc_h.p, job->bdesc.p, 32ULL * job->ndesc, cudaMemcpyDeviceToHost, job->stream),
           "D2H descriptors");
        CK(cudaStreamSynchronize(job->stream), "sync descriptors");
        for (uint32_t i = 0; i < job->ndesc; ++i) max_tiles = std::max(max_tiles, job->bdesc_h.p[4 * i + 1]);
      }
    }
    if (t_over) job->tb_cap = max_tiles + 1024;   // (tb itself is grown by launch_batch)
    const uint64_t ncap_p = job->wc_comb() ? std::max(job->cap_p, mp + mp / 8 + 4096) : 0;
    const uint64_t ncap = std::max(job->cap, m + m / 8 + 4096);
    // the mid / hashed streams are appended in warp-private chunks (map.cu kLChunk = 256 entries):
    // a run may leave up to a chunk unused per map warp
    const uint64_t chunk_slack = static_cast<uint64_t>(job->nsm) * 24u * 256u;
    const uint64_t ncap_b = job->split() ? std::max(job->cap_b, mb + mb / 8 + 4096 + chunk_slack) : 0;
    const uint64_t ncap_c = job->split() ? std::max(job->cap_c, mc + mc / 8 + 4096 + chunk_slack) : 0;
    if (ncap > job->cap || ncap_b > job->cap_b || ncap_c > job->cap_c) {
      release_pairs(job);
      CK(ensure_pairs(job, ncap, ncap_b, ncap_c), "grow intermediate");
    }
    if (ncap_p > job->cap_p) {
      CK(job->hp.ensure(ncap_p), "grow partials");
      job->cap_p = ncap_p;
    }
    job->stats.capacity_pairs = job->cap + job->cap_b + job->cap_c;
    CK(cudaMemsetAsync(job->st, 0, sizeof(DevState), job->stream), "reset cursor");
    if (job->xtab_dirty || m_over || l_over) CK(clear_tables(job), "clear the tables");
    if (job->km_comb()) {
      CK(cudaMemsetAsync(job->sums.p, 0, 64ULL * job->k, job->stream), "reset sums");
      CK(cudaMemsetAsync(job->cnts.p, 0, 8ULL * job->k, job->stream), "reset counts");
    }
    for (const Batch& b : job->batches) CK(launch_batch(job, b), "replay");
    job->stats.replays += job->batches.size();
    CK(read_state(job), "replay (async)");
  }
  return MR_OK;
}

}  // namespace

extern "C" mr_status mr_partition_count(mr_job* job, uint64_t* counts, uint64_t* entry_bytes);
extern "C" mr_status mr_partition_write(mr_job* job, void* entries, void* heap);
extern "C" mr_status mr_ingest(mr_job* job, const void* entries, const void* heap, const uint64_t* recv_counts);
namespace {
mr_status ingest_impl(mr_job* job, const void* entries, const void* heap, const uint64_t* recv_counts, uint32_t R);
mr_status fold(mr_job* job);
mr_status fold_finish(mr_job* job);
mr_status tables_extract(mr_job* job);
cudaError_t clear_tables(mr_job* job);
}

namespace {

// The one exchange of the multi-GPU group-by (SURVEY §8(b) mr_group with R > 1, §8(e); PAPER.md
// L51-52: the shuffle between Map and Reduce is the framework's): partition by destination rank
// (WC / KM: after the local combiner), ncclAlltoAll of the R x (entries, heap bytes) count
// matrix, then ONE NCCL group of send / recv pairs for the entry and key-byte slices, all on the
// job stream, then mr_ingest of what arrived.  Synchronises twice (the counts size the receive
// buffers; the ingest needs the received counts on the host).
mr_status exchange(mr_job* job) {
  const NcclApi* a = nccl_api();
  if (!a->ok) return fail(job, MR_ERR_NCCL, "NCCL unavailable: " + a->err);
  const int R = job->cfg.nranks;
  void* comm = job->cfg.nccl_comm;
  cudaStream_t s = job->stream;
  std::vector<uint64_t> cnt(2 * R), rc(2 * R);
  uint64_t eb = 0;
  job->in_exchange = true;
  mr_status st = mr_partition_count(job, cnt.data(), &eb);   // (its local group + reduce time their own phases)
  job->in_exchange = false;
  if (st != MR_OK) return st;
  Prof::Span sp{};
  if (job->prof.on) job->prof.begin(s, sp);
  std::vector<uint64_t> se(R + 1, 0), sh(R + 1, 0), re(R + 1, 0), rh(R + 1, 0);
  for (int r = 0; r < R; ++r) {
    se[r + 1] = se[r] + cnt[2 * r] * eb;
    sh[r + 1] = sh[r] + cnt[2 * r + 1];
  }
  CK(job->xsend_e.ensure(se[R] + 16), "alloc send entries");
  CK(job->xsend_h.ensure(sh[R] + 16), "alloc send heap");
  st = mr_partition_write(job, job->xsend_e.p, job->xsend_h.p);
  if (st != MR_OK) return st;
  CK(job->xrecv_counts.ensure(2 * R), "alloc receive counts");
  int nr = 0;
  CK(nccl_alltoall_u64x2(a, reinterpret_cast<const uint64_t*>(job->xcounts.p), job->xrecv_counts.p, R, comm, s, &nr),
     "count exchange");
  if (nr) return fail(job, MR_ERR_NCCL, "ncclAlltoAll (counts): " + nccl_error(a, nr));
  CK(cudaMemcpyAsync(rc.data(), job->xrecv_counts.p, 2 * R * 8, cudaMemcpyDeviceToHost, s), "D2H receive counts");
  CK(cudaStreamSynchronize(s), "sync count exchange");
  for (int r = 0; r < R; ++r) {
    re[r + 1] = re[r] + rc[2 * r] * eb;
    rh[r + 1] = rh[r] + rc[2 * r + 1];
  }
  CK(job->xrecv_e.ensure(re[R] + 16), "alloc receive entries");
  CK(job->xrecv_h.ensure(rh[R] + 16), "alloc receive heap");
  nr = nccl_alltoallv2(a, job->xsend_e.p, se.data(), job->xrecv_e.p, re.data(), job->xsend_h.p, sh.data(),
                       job->xrecv_h.p, rh.data(), R, comm, s);
  if (nr) return fail(job, MR_ERR_NCCL, "NCCL send/recv: " + nccl_error(a, nr));
  job->stats.xchg_send_bytes += se[R] + sh[R];
  job->stats.xchg_recv_bytes += re[R] + rh[R];
  if (job->prof.on) job->prof.end(s, sp, &job->stats.xchg_ms);
  job->exchanged = true;
  return ingest_impl(job, job->xrecv_e.p, job->xrecv_h.p, rc.data(), static_cast<uint32_t>(R));
}

// grow a device array to >= need elements, keeping its first `used` elements
template <typename T>
cudaError_t grow_keep(DBuf<T>& b, uint64_t used, uint64_t need, cudaStream_t s) {
  if (need <= b.n && b.p) return cudaSuccess;
  DBuf<T> nb;
  cudaError_t e = nb.ensure(std::max<uint64_t>(need, 2 * b.n));
  if (e != cudaSuccess) return e;
  if (used && (e = cudaMemcpyAsync(nb.p, b.p, used * sizeof(T), cudaMemcpyDeviceToDevice, s)) != cudaSuccess) return e;
  if ((e = cudaStreamSynchronize(s)) != cudaSuccess) return e;
  b.release();
  b = nb;
  nb.p = nullptr;
  nb.n = 0;
  return cudaSuccess;
}

// WC batch combine: group + reduce the batches mapped since the last fold (the local combiner,
// exact integer sums) and append their (key, count) partials to the arena; the job is then ready
// to map the next batch.  Synchronises.
mr_status fold(mr_job* job) {
  cudaStream_t s = job->stream;
  job->in_fold = true;
  mr_status st = mr_group(job);
  if (st == MR_OK) st = mr_reduce(job);
  job->in_fold = false;
  if (st != MR_OK) return st;
  mr_stats& f = job->fold_stats;
  f.pairs += job->stats.pairs;
  f.pairs_hashed += job->stats.pairs_hashed;
  f.pairs_mid += job->stats.pairs_mid;
  f.pairs_partial += job->stats.pairs_partial;
  f.words_combined += job->stats.words_combined;
  f.flushes += job->stats.flushes;
  XSource xs;
  xs.nranks = 1;
  xs.mode = kXSegs;
  xs.n = job->nseg;
  xs.keys = job->keys_out.p;
  xs.key_off = job->key_off.p;
  xs.counts = job->counts.p;
  CK(job->xcounts.ensure(2), "alloc counts");
  CK(job->xcursors.ensure(2), "alloc cursors");
  CK(job->xheapbase.ensure(1), "alloc heap base");
  CK(job->xcounts_h.ensure(4), "alloc host counts");
  CK(launch_x_count(xs, job->xcounts.p, job->nsm, s), "fold count");
  CK(cudaMemcpyAsync(job->xcounts_h.p, job->xcounts.p, 16, cudaMemcpyDeviceToHost, s), "D2H fold counts");
  CK(cudaStreamSynchronize(s), "sync fold counts");
  const uint64_t ne = job->xcounts_h.p[0], nh = job->xcounts_h.p[1];
  CK(grow_keep(job->acc_e, job->acc_ne * sizeof(XEntry), (job->acc_ne + ne) * sizeof(XEntry) + 64, s), "grow arena");
  CK(grow_keep(job->acc_h, job->acc_nh, job->acc_nh + nh + 64, s), "grow arena");
  unsigned long long* cur = job->xcounts_h.p + 2;   // entries / heap cursors at the arena's ends
  cur[0] = job->acc_ne;
  cur[1] = job->acc_nh;
  CK(cudaMemcpyAsync(job->xcursors.p, cur, 16, cudaMemcpyHostToDevice, s), "H2D cursors");
  CK(cudaMemsetAsync(job->xheapbase.p, 0, 8, s), "heap base");   // entry key offsets = arena offsets
  xs.heap_base = job->xheapbase.p;
  CK(launch_x_scatter(xs, job->xcursors.p, job->acc_e.p, job->acc_h.p, s), "fold scatter");
  CK(cudaStreamSynchronize(s), "sync fold");
  job->acc_ne += ne;
  job->acc_nh += nh;
  ++job->nfolds;
  // a fresh Map state for the next batch (buffers kept; the folded batches may be released)
  job->batches.clear();
  CK(cudaMemsetAsync(job->st, 0, sizeof(DevState), s), "reset state");
  job->state = kCreated;
  return MR_OK;
}

// mr_group of a folded job: fold the pending batches, then ingest every batch's partials (one
// source) as the pairs to group (u64 counts, keys by reference into the arena)
mr_status fold_finish(mr_job* job) {
  if (!job->batches.empty()) {
    mr_status st = fold(job);
    if (st != MR_OK) return st;
  }
  const uint64_t rc[2] = {job->acc_ne, job->acc_nh};
  mr_status st = ingest_impl(job, job->acc_e.p, job->acc_h.p, rc, 1);
  job->nfolds = 0;   // (the arena stays referenced until mr_reduce; reset clears it)
  return st;
}

// both WC tables back to empty (after a replay's first Map or a reset without mr_group)
cudaError_t clear_tables(mr_job* job) {
  cudaError_t e = cudaSuccess;
  if (job->xtab.p) e = cudaMemsetAsync(job->xtab.p, 0, job->xtab.n * 4, job->stream);
  if (e == cudaSuccess && job->mtab_keys.p) e = cudaMemsetAsync(job->mtab_keys.p, 0xFF, job->mtab_keys.n * 8, job->stream);
  if (e == cudaSuccess && job->mtab_cnt.p) e = cudaMemsetAsync(job->mtab_cnt.p, 0, job->mtab_cnt.n * 4, job->stream);
  if (e == cudaSuccess && job->ltab_keys.p) e = cudaMemsetAsync(job->ltab_keys.p, 0, job->ltab_keys.n * 8, job->stream);
  if (e == cudaSuccess && job->ltab_cnt.p) e = cudaMemsetAsync(job->ltab_cnt.p, 0, job->ltab_cnt.n * 4, job->stream);
  return e;
}

// WC tables -> the group's exact keys (xkeys / pxcounts, the "partial-only" list: every key once)
// and mid keys (mkeys_out / mcounts, with identity segments): no sort, no merge.  Grows the
// output lists when they overflow (the entries past capacity stay in the table for a second
// pass).  Synchronises.
mr_status tables_extract(mr_job* job) {
  cudaStream_t s = job->stream;
  unsigned long long* cur = &job->st->n_extra;   // scratch cursors: n_extra, words_comb
  unsigned long long* wsum = &job->st->words_comb;
  CK(cudaMemsetAsync(cur, 0, 2 * sizeof(unsigned long long), s), "memset cursor");
  if (job->xkeys.n < 4096) { CK(job->xkeys.ensure(1 << 20), "alloc keys"); CK(job->pxcounts.ensure(1 << 20), "alloc counts"); }
  uint64_t cap = std::min(job->xkeys.n, job->pxcounts.n);
  uint64_t t = 0;
  if (job->xtab_on) {   // (small-table mode: the exact words are in the mid table)
  CK(launch_xtab_extract_list(job->xtab.p, job->xtab.n, job->xkeys.p, job->pxcounts.p, cap, cur, wsum, job->nsm, s),
     "table extract");
  CK(read_state(job), "sync table extract");
  t = job->st_h.p->n_extra;
  }
  if (t > cap) {
    CK(grow_keep(job->xkeys, cap, t + t / 8 + 4096, s), "grow keys");
    CK(grow_keep(job->pxcounts, cap, t + t / 8 + 4096, s), "grow counts");
    job->tmp_h.p[4] = cap;
    CK(cudaMemcpyAsync(cur, job->tmp_h.p + 4, 8, cudaMemcpyHostToDevice, s), "set cursor");
    const uint64_t cap2 = std::min(job->xkeys.n, job->pxcounts.n);
    CK(launch_xtab_extract_list(job->xtab.p, job->xtab.n, job->xkeys.p, job->pxcounts.p, cap2, cur, wsum, job->nsm, s),
       "table extract");
    CK(read_state(job), "sync table extract");
    t = job->st_h.p->n_extra;
    if (t > cap2) return fail(job, MR_ERR_OOM, "table extraction still overflows");
  }
  job->n_extra = t;
  // mid table
  CK(cudaMemsetAsync(cur, 0, sizeof(unsigned long long), s), "memset cursor");
  if (job->mkeys_out.n < 4096) { CK(job->mkeys_out.ensure(1 << 18), "alloc mid keys"); CK(job->mcounts.ensure(1 << 18), "alloc mid counts"); }
  cap = std::min(job->mkeys_out.n, job->mcounts.n);
  CK(launch_mtab_extract(job->mtab_keys.p, job->mtab_cnt.p, job->mtab_keys.n, job->mbits, job->mkeys_out.p, job->mcounts.p, cap, cur,
                         wsum, job->nsm, s),
     "mid table extract");
  CK(read_state(job), "sync mid table extract");
  t = job->st_h.p->n_extra;
  if (t > cap) {
    CK(grow_keep(job->mkeys_out, cap, t + t / 8 + 4096, s), "grow mid keys");
    CK(grow_keep(job->mcounts, cap, t + t / 8 + 4096, s), "grow mid counts");
    job->tmp_h.p[4] = cap;
    CK(cudaMemcpyAsync(cur, job->tmp_h.p + 4, 8, cudaMemcpyHostToDevice, s), "set cursor");
    const uint64_t cap2 = std::min(job->mkeys_out.n, job->mcounts.n);
    CK(launch_mtab_extract(job->mtab_keys.p, job->mtab_cnt.p, job->mtab_keys.n, job->mbits, job->mkeys_out.p, job->mcounts.p, cap2,
                           cur, wsum, job->nsm, s),
       "mid table extract");
    CK(read_state(job), "sync mid table extract");
    t = job->st_h.p->n_extra;
    if (t > cap2) return fail(job, MR_ERR_OOM, "mid table extraction still overflows");
  }
  job->nseg_c = t;
  // long-word table
  CK(cudaMemsetAsync(cur, 0, sizeof(unsigned long long), s), "memset cursor");
  {   // (the table holds at most one key per slot: output lists of the slot count never overflow)
    const uint64_t slots = job->ltab_keys.n / 2;
    CK(job->lkeys_out.ensure(2 * slots), "alloc long keys");
    CK(job->lkref_out.ensure(slots), "alloc long keys");
    CK(job->lcounts.ensure(slots), "alloc long counts");
  }
  uint64_t lcap = std::min({job->lkeys_out.n / 2, job->lkref_out.n, job->lcounts.n});
  CK(launch_ltab_extract(job->ltab_keys.p, job->ltab_cnt.p, job->ltab_keys.n / 2, job->lbits, job->lkeys_out.p, job->lkref_out.p,
                         job->lcounts.p, lcap, cur, wsum, job->nsm, s),
     "long table extract");
  CK(read_state(job), "sync long table extract");
  uint64_t tl = job->st_h.p->n_extra;
  if (tl > lcap) {   // (the references point into lkeys_out: grow it first, then re-extract everything)
    return fail(job, MR_ERR_OOM, "long table extraction overflow");
  }
  job->nseg_l = tl;
  job->stats.words_combined = job->st_h.p->words_comb;   // exact + mid + long words counted by the tables
  CK(job->seg_startx.ensure(t + 2), "alloc mid segments");
  CK(launch_iota_scaled(t, 1, job->seg_startx.p, s), "mid segments");   // one segment per mid key
  job->segc = job->seg_startx.p;
  job->skeysc = job->mkeys_out.p;
  job->mid_from_table = true;
  CK(cudaMemsetAsync(cur, 0, 2 * sizeof(unsigned long long), s), "memset cursor");
  job->xtab_dirty = false;
  return MR_OK;
}


}  // namespace

extern "C" {

const char* mr_status_string(mr_status s) {
  switch (s) {
    case MR_OK: return "MR_OK";
    case MR_ERR_INVALID: return "MR_ERR_INVALID";
    case MR_ERR_STATE: return "MR_ERR_STATE";
    case MR_ERR_OOM: return "MR_ERR_OOM";
    case MR_ERR_OVERFLOW: return "MR_ERR_OVERFLOW";
    case MR_ERR_CUDA: return "MR_ERR_CUDA";
    case MR_ERR_NCCL: return "MR_ERR_NCCL";
    case MR_ERR_UNSUPPORTED: return "MR_ERR_UNSUPPORTED";
  }
  return "MR_ERR_UNKNOWN";
}

const char* mr_last_error(const mr_job* job) { return job ? job->err.c_str() : "null job"; }

mr_status mr_job_create(const mr_config* cfg, mr_job** out) {
  if (!cfg || !out) return MR_ERR_INVALID;
  *out = nullptr;
  if (cfg->abi_version != MR_ABI_VERSION) return MR_ERR_INVALID;
  if (cfg->workload < MR_WORDCOUNT || cfg->workload > MR_INVINDEX) return MR_ERR_INVALID;
  if (cfg->nranks < 1 || cfg->nranks > kMaxRanks || cfg->rank < 0 || cfg->rank >= cfg->nranks) return MR_ERR_INVALID;
  if (cfg->workload == MR_KMEANS) {
    const mr_km_params* p = static_cast<const mr_km_params*>(cfg->params);
    if (!p || !p->centroids || p->dim != 8 || p->k < 1 || p->k > 1024 || cfg->record_stride != 32)
      return MR_ERR_INVALID;
  } else if (cfg->record_stride != 0) {
    return MR_ERR_INVALID;
  }
  if (cfg->workload == MR_STRINGMATCH && !cfg->params) return MR_ERR_INVALID;
  mr_job* job = new (std::nothrow) mr_job();
  if (!job) return MR_ERR_OOM;
  job->cfg = *cfg;
  job->cfg.params = nullptr;
  if (cfg->workload == MR_STRINGMATCH) job->sm = *static_cast<const mr_sm_params*>(cfg->params);
  cudaError_t e = cudaSetDevice(cfg->device);
  if (e == cudaSuccess && cfg->workload == MR_KMEANS) {
    const mr_km_params* p = static_cast<const mr_km_params*>(cfg->params);
    job->k = p->k;
    job->cent_h.assign(p->centroids, p->centroids + static_cast<size_t>(p->k) * 8);
  }
  // cfg->stream == NULL is CUDA's default stream (what torch's default stream handle is), so a
  // job always orders with the caller's stream; MR_FLAG_OWN_STREAM asks for a private stream.
  if (e == cudaSuccess) {
    if (cfg->flags & MR_FLAG_OWN_STREAM) {
      e = cudaStreamCreateWithFlags(&job->stream, cudaStreamNonBlocking);
      job->own_stream = (e == cudaSuccess);
    } else {
      job->stream = static_cast<cudaStream_t>(cfg->stream);
    }
  }
  if (e == cudaSuccess) e = cudaMalloc(reinterpret_cast<void**>(&job->st), sizeof(DevState));
  if (e == cudaSuccess) e = job->st_h.ensure(1);
  if (e == cudaSuccess) e = job->tmp_h.ensure(16);
  if (e == cudaSuccess) e = cudaMemsetAsync(job->st, 0, sizeof(DevState), job->stream);
  if (e == cudaSuccess && job->k) {
    e = job->cent.ensure(job->k * 8);
    if (e == cudaSuccess)
      e = cudaMemcpyAsync(job->cent.p, job->cent_h.data(), job->k * 32, cudaMemcpyHostToDevice, job->stream);
    if (e == cudaSuccess) e = cudaStreamSynchronize(job->stream);
  }
  if (e != cudaSuccess) {
    cudaGetLastError();
    mr_job_destroy(job);
    return e == cudaErrorMemoryAllocation ? MR_ERR_OOM : MR_ERR_CUDA;
  }
  job->nsm = sm_count(cfg->device);
  job->prof.on = (cfg->flags & MR_FLAG_PROFILE) != 0;
  job->key_bits = (cfg->workload == MR_WORDCOUNT || cfg->workload == MR_INVINDEX) ? 48u : 64u;
  job->launches0 = g_kernel_launches.load();
  *out = job;
  return MR_OK;
}

mr_status mr_job_reset(mr_job* job) {
  if (!job) return MR_ERR_INVALID;
  CK(cudaSetDevice(job->cfg.device), "set device");
  CK(cudaStreamSynchronize(job->stream), "sync");
  for (void* p : job->owned) cudaFree(p);
  job->owned.clear();
  job->host_batches = 0;
  job->ingested = false;
  job->exchanged = false;
  job->nfolds = 0;
  job->acc_ne = job->acc_nh = 0;
  job->fold_stats = mr_stats{};
  job->km_partial = false;
  job->km_combined = false;
  job->key_bits = (job->cfg.workload == MR_WORDCOUNT || job->cfg.workload == MR_INVINDEX) ? 48u : 64u;
  job->key_bits_b = 48;
  job->mb = job->nseg_a = job->nseg_b = job->mc = job->nseg_c = 0;
  job->mp = job->nseg_p = job->n_extra = 0;
  job->skeysp = nullptr;
  job->skeysc = nullptr;
  job->segc = nullptr;
  job->skeysb = nullptr;
  job->permb = nullptr;
  job->prof.collect();
  job->batches.clear();
  job->next_base = 0;
  job->ndesc = 0;
  job->m = job->nseg = job->key_bytes = 0;
  job->skeys = nullptr;
  job->perm = nullptr;
  const uint64_t cap = job->stats.capacity_pairs;
  job->stats = mr_stats{};
  job->stats.capacity_pairs = cap;
  job->launches0 = g_kernel_launches.load();
  CK(cudaMemsetAsync(job->st, 0, sizeof(DevState), job->stream), "reset state");
  if (job->xtab_dirty) {   // a Map fed the tables but no mr_group extracted them
    CK(clear_tables(job), "clear the tables");
    job->xtab_dirty = false;
  }
  job->mid_from_table = false;
  job->state = kCreated;
  return MR_OK;
}

// known_nbytes: the batch length when the caller knows it (mr_map_host_lines), else ~0 (read
// offsets[n] back from the device)
static mr_status map_common(mr_job* job, const uint8_t* records, const uint64_t* offsets, uint64_t n,
                            uint64_t known_nbytes = ~0ULL) {
  if (job->state != kCreated && job->state != kMapped) return fail(job, MR_ERR_STATE, "mr_map after mr_group");
  const bool fixed = job->cfg.record_stride > 0;
  if (fixed != (offsets == nullptr)) return fail(job, MR_ERR_INVALID, "offsets must be NULL iff record_stride > 0");
  if (fixed && (reinterpret_cast<uintptr_t>(records) & 15u))
    return fail(job, MR_ERR_INVALID, "fixed-stride records must be 16-byte aligned");
  if ((reinterpret_cast<uintptr_t>(records) >> 48) != 0) return fail(job, MR_ERR_INVALID, "records address >= 2^48");
  // Text batches are enqueued without a host round trip: the batch length offsets[n], its tile
  // count and global base are derived on the device (map.cu k_tile_bounds) and read back at the
  // next synchronising call (settle_map).  known_nbytes (mr_map_host_lines) only sizes buffers.
  uint64_t nbytes = ~0ULL;
  if (fixed) {
    nbytes = n * job->cfg.record_stride;
    if (nbytes && !records) return fail(job, MR_ERR_INVALID, "records is NULL");
  } else if (job->cfg.flags & MR_FLAG_VALIDATE) {
    std::vector<uint64_t> o(n + 1);
    CK(cudaMemcpyAsync(o.data(), offsets, (n + 1) * 8, cudaMemcpyDeviceToHost, job->stream), "read offsets");
    CK(cudaStreamSynchronize(job->stream), "sync");
    if (o[0] != 0) return fail(job, MR_ERR_INVALID, "offsets[0] != 0");
    for (uint64_t i = 0; i < n; ++i)
      if (o[i + 1] < o[i]) return fail(job, MR_ERR_INVALID, "offsets not non-decreasing");
    nbytes = o[n];
    if (nbytes && !records) return fail(job, MR_ERR_INVALID, "records is NULL");
  } else if (known_nbytes != ~0ULL) {
    nbytes = known_nbytes;
  }
  // sizing estimate for the first batch's buffers (text of unknown length: <= 32 B per record
  // assumed; overflow is caught by the demand counters and replayed at mr_group)
  const uint64_t est = nbytes != ~0ULL ? nbytes : 32 * n;
  if (job->batches.empty() && job->nfolds == 0 && !job->ingested) {
    const char* tm = getenv("BMR_TABLE_MIN_BYTES");   // (tests: 1 << 40 = the sorted streams)
    job->tables_on = est >= (tm ? strtoull(tm, nullptr, 10) : 0ULL);
    const char* xm = getenv("BMR_XTAB_MIN_BYTES");    // (tests: 0 = always the exact-key table)
    job->xtab_on = est >= (xm ? strtoull(xm, nullptr, 10) : (64ULL << 20));
    if (!job->xtab_on && !map_wc_tab()) job->tables_on = false;   // small-table mode needs wc_window_tab
  }
  if ((job->cfg.flags & MR_FLAG_BATCH_COMBINE) && job->cfg.workload == MR_WORDCOUNT && !job->ingested &&
      !job->batches.empty()) {
    mr_status fs = fold(job);   // WC batch combine: the previous batches become (key, count) partials
    if (fs != MR_OK) return fs;
  }
  if (job->cap == 0) {
    // WC: ~1 word per 6 bytes, a few % of them longer than 7 bytes (hashed stream)
    const bool wc = job->cfg.workload == MR_WORDCOUNT;
    const uint64_t hint = job->cfg.max_pairs_hint;
    const uint64_t cap_b = !wc ? 0 : hint ? hint : est / 48 + 4096;
    const uint64_t cap_c = !wc ? 0 : hint ? hint : est / 32 + 4096;
    CK(ensure_pairs(job, initial_cap(job, est, n), cap_b, cap_c), "alloc intermediate");
    if (job->wc_comb()) {   // combiner partials: <= 2^kCombBits per CTA per batch (grown + replayed if exceeded)
      job->cap_p = job->cfg.max_pairs_hint ? job->cfg.max_pairs_hint : 2ULL * 4096 * job->nsm + 4096;
      CK(job->hp.ensure(job->cap_p), "alloc partials");
    }
    job->stats.capacity_pairs = job->cap + job->cap_b + job->cap_c;
  }
  if (job->wc_table() && job->xtab_on && !job->xtab.p) {   // emptied once (extraction re-empties it)
    CK(job->xtab.ensure(1ULL << kExactBits), "alloc count table");
    CK(cudaMemsetAsync(job->xtab.p, 0, job->xtab.n * 4, job->stream), "empty the count table");
  }
  if (job->wc_table() && !job->mtab_keys.p) {   // the mid / long tables, emptied once
    CK(job->mtab_keys.ensure(1ULL << job->mbits), "alloc mid table");
    CK(job->mtab_cnt.ensure((1ULL << job->mbits) * kMidStripes), "alloc mid table");
    CK(job->ltab_keys.ensure(2ULL << job->lbits), "alloc long table");
    CK(job->ltab_cnt.ensure((1ULL << job->lbits) * kMidStripes), "alloc long table");
    CK(clear_tables(job), "empty the tables");
  }
  if (job->batches.empty() && job->km_comb()) {   // KM combiner accumulators (summed over batches)
    CK(job->sums.ensure(8ULL * job->k), "alloc sums");
    CK(job->cnts.ensure(job->k), "alloc counts");
    CK(cudaMemsetAsync(job->sums.p, 0, 64ULL * job->k, job->stream), "zero sums");
    CK(cudaMemsetAsync(job->cnts.p, 0, 8ULL * job->k, job->stream), "zero counts");
  }
  Batch b{records, offsets, n, fixed ? nbytes : 0, fixed ? job->cfg.input_base + job->next_base : 0, 0};
  if (fixed) {
    job->next_base += nbytes;
    job->stats.input_bytes += nbytes;
  } else {
    if (job->tb_cap == 0) job->tb_cap = (std::max<uint64_t>(est, 128 * n) + kMapTileBytes - 1) / kMapTileBytes + 1024;
    if (job->ndesc + 1 > job->bdesc.n / 4) {   // descriptor table (grown keeping earlier batches')
      DBuf<uint64_t> nb;
      CK(nb.ensure(4ULL * std::max<uint32_t>(256, 2 * job->ndesc)), "alloc batch descriptors");
      if (job->ndesc) {
        CK(cudaMemcpyAsync(nb.p, job->bdesc.p, 32ULL * job->ndesc, cudaMemcpyDeviceToDevice, job->stream), "copy descriptors");
        CK(cudaStreamSynchronize(job->stream), "sync descriptors");
      }
      job->bdesc.release();
      job->bdesc = nb;
    }
    b.di = job->ndesc++;
  }
  job->batches.push_back(b);
  Prof::Span sp{};
  if (job->prof.on) job->prof.begin(job->stream, sp);
  CK(launch_batch(job, b), "map kernel launch");
  if (job->prof.on) job->prof.end(job->stream, sp, &job->stats.map_ms);
  job->state = kMapped;
  return MR_OK;
}

mr_status mr_map(mr_job* job, const uint8_t* records, const uint64_t* offsets, uint64_t n) {
  if (!job) return MR_ERR_INVALID;
  CK(cudaSetDevice(job->cfg.device), "set device");
  return map_common(job, records, offsets, n);
}

mr_status mr_map_host(mr_job* job, const uint8_t* records, const uint64_t* offsets, uint64_t n) {
  if (!job) return MR_ERR_INVALID;
  CK(cudaSetDevice(job->cfg.device), "set device");
  const bool fixed = job->cfg.record_stride > 0;
  if (fixed != (offsets == nullptr)) return fail(job, MR_ERR_INVALID, "offsets must be NULL iff record_stride > 0");
  const uint64_t nbytes = fixed ? n * job->cfg.record_stride : offsets[n];
  if (nbytes && !records) return fail(job, MR_ERR_INVALID, "records is NULL");
  const size_t i = job->host_batches++;
  if (job->host_rec.size() <= i) { job->host_rec.resize(i + 1); job->host_off.resize(i + 1); }
  CK(job->host_rec[i].ensure(std::max<uint64_t>(nbytes, 16)), "alloc device records");
  if (nbytes) CK(cudaMemcpyAsync(job->host_rec[i].p, records, nbytes, cudaMemcpyHostToDevice, job->stream), "H2D records");
  const uint64_t* doff = nullptr;
  if (!fixed) {
    CK(job->host_off[i].ensure(n + 1), "alloc device offsets");
    CK(cudaMemcpyAsync(job->host_off[i].p, offsets, (n + 1) * 8, cudaMemcpyHostToDevice, job->stream), "H2D offsets");
    doff = job->host_off[i].p;
  }
  return map_common(job, job->host_rec[i].p, doff, n, fixed ? ~0ULL : nbytes);
}

// mr_map_host_lines batch size (BMR_LINE_CHUNK bytes, default 256 MiB): copies of batch b + 1
// overlap the line split and Map of batch b
static uint64_t line_chunk() {   // read per call (tests shrink it to force many batches)
  const char* e = getenv("BMR_LINE_CHUNK");
  return e ? std::max<uint64_t>(strtoull(e, nullptr, 10), 64) : (256ULL << 20);
}

mr_status mr_map_host_lines(mr_job* job, const uint8_t* text, uint64_t nbytes) {
  const uint64_t kLineChunk = line_chunk();
  if (!job) return MR_ERR_INVALID;
  if (job->cfg.record_stride > 0) return fail(job, MR_ERR_INVALID, "mr_map_host_lines: text workloads only");
  if (nbytes && !text) return fail(job, MR_ERR_INVALID, "text is NULL");
  if (job->state != kCreated && job->state != kMapped) return fail(job, MR_ERR_STATE, "mr_map after mr_group");
  if (nbytes == 0) {   // no records: nothing to copy or map
    job->state = kMapped;
    return MR_OK;
  }
  CK(cudaSetDevice(job->cfg.device), "set device");
  if (!job->cstream) {
    CK(cudaStreamCreateWithFlags(&job->cstream, cudaStreamNonBlocking), "copy stream");
  }
  // batches of ~kLineChunk bytes ending after a '\n' (host-side memrchr on the caller's text)
  std::vector<uint64_t> cut{0};
  while (cut.back() < nbytes) {
    uint64_t end = std::min(nbytes, cut.back() + kLineChunk);
    if (end < nbytes) {
      const void* nl = memrchr(text + cut.back(), '\n', end - cut.back());
      if (nl) end = static_cast<const uint8_t*>(nl) - text + 1;
      else {  // a line longer than a chunk: extend to its end
        const void* f = memchr(text + end, '\n', nbytes - end);
        end = f ? static_cast<const uint8_t*>(f) - text + 1 : nbytes;
      }
    }
    cut.push_back(end);
  }
  const size_t nb = cut.size() - 1;
  const size_t ti = job->host_batches++;
  if (job->host_rec.size() <= ti) { job->host_rec.resize(ti + 1); job->host_off.resize(ti + 1); }
  CK(job->host_rec[ti].ensure(nbytes + 64), "alloc device text");
  uint8_t* dtext = job->host_rec[ti].p;
  // copies on the copy stream, one event per batch; the job stream waits per batch
  if (job->line_ev.size() < nb) {
    const size_t old = job->line_ev.size();
    job->line_ev.resize(nb);
    for (size_t b = old; b < nb; ++b) CK(cudaEventCreateWithFlags(&job->line_ev[b], cudaEventDisableTiming), "event");
  }
  CK(cudaEventRecord(job->line_ev[0], job->stream), "event");   // copies start after earlier work
  CK(cudaStreamWaitEvent(job->cstream, job->line_ev[0], 0), "wait");
  for (size_t b = 0; b < nb; ++b) {
    CK(cudaMemcpyAsync(dtext + cut[b], text + cut[b], cut[b + 1] - cut[b], cudaMemcpyHostToDevice, job->cstream),
       "H2D text");
    CK(cudaEventRecord(job->line_ev[b], job->cstream), "event");
  }
  for (size_t b = 0; b < nb; ++b) {
    const uint64_t lo = cut[b], hi = cut[b + 1];
    CK(cudaStreamWaitEvent(job->stream, job->line_ev[b], 0), "wait text");
    const uint64_t tiles = line_tiles(lo, hi);
    CK(job->seg_counts.ensure(tiles + 1), "alloc line counts");
    CK(job->tile_base.ensure(tiles + 1), "alloc line bases");
    CK(launch_line_count(dtext, lo, hi, job->seg_counts.p, job->stream), "line count");
    uint64_t* ss;
    uint32_t ep;
    CK(scan_ws(job, tiles, &ss, &ep), "alloc scan workspace");
    CK(launch_scan_u32to64(job->seg_counts.p, job->tile_base.p, tiles, &job->st->seg_total, ss, ep,
                           &job->st->tile_counter[1], job->stream),
       "scan line counts");
    CK(read_state(job), "sync line count");
    const uint64_t nl = job->st_h.p->seg_total;
    const bool open_end = text[hi - 1] != '\n';
    const uint64_t n = nl + (open_end ? 1 : 0);
    const size_t oi = job->host_batches++;
    if (job->host_rec.size() <= oi) { job->host_rec.resize(oi + 1); job->host_off.resize(oi + 1); }
    CK(job->host_off[oi].ensure(n + 1), "alloc device offsets");
    uint64_t* off = job->host_off[oi].p;
    CK(cudaMemsetAsync(off, 0, 8, job->stream), "offsets[0]");
    CK(launch_line_write(dtext, lo, hi, job->tile_base.p, off, job->stream), "line offsets");
    if (open_end) {
      job->tmp_h.p[1] = hi - lo;
      CK(cudaMemcpyAsync(off + n, job->tmp_h.p + 1, 8, cudaMemcpyHostToDevice, job->stream), "offsets[n]");
    }
    mr_status st = map_common(job, dtext + lo, off, n, hi - lo);
    if (st != MR_OK) return st;
  }
  return MR_OK;
}

mr_status mr_group(mr_job* job) {
  if (!job) return MR_ERR_INVALID;
  if (job->state != kMapped && job->state != kCreated) return fail(job, MR_ERR_STATE, "mr_group out of order");
  CK(cudaSetDevice(job->cfg.device), "set device");
  if (job->nfolds && !job->in_fold) {   // WC batch combine: fold the last batch, ingest all partials
    mr_status fs = fold_finish(job);
    if (fs != MR_OK) return fs;
  }
  if (job->cfg.nranks > 1 && job->cfg.nccl_comm && !job->in_exchange && !job->in_fold && !job->exchanged &&
      job->cfg.workload != MR_STRINGMATCH) {
    mr_status xs = exchange(job);   // -> ingested pairs (or KM partials) of the keys this rank owns
    if (xs != MR_OK) return xs;
  }
  if (job->km_partial) {           // ingested KM partials: grouping happened at the owner (atomics)
    job->state = kGrouped;
    return MR_OK;
  }
  mr_status st = settle_map(job);
  if (st != MR_OK) return st;
  DevState* hs = job->st_h.p;
  const bool split = job->split();
  const uint64_t m_total = hs->pair_cursor;            // includes the flush filler pairs (sentinel keys)
  const uint64_t m = m_total - hs->pads;
  // WC mid / hashed streams: slots taken (incl. the sentinel-filled chunk tails) and real entries
  const uint64_t mb_total = split ? hs->pair_cursor_b : 0, mc_total = split ? hs->pair_cursor_c : 0;
  const uint64_t mb = split ? mb_total - hs->pads_b : 0;
  const uint64_t mc = split ? mc_total - hs->pads_c : 0;
  job->m = m;
  job->mb = mb;
  job->mc = mc;
  job->mp = job->wc_comb() ? hs->pair_cursor_p : 0;
  const bool tables = job->wc_table();   // exact + mid words were counted by the tables, not emitted
  job->stats.pairs_partial = job->mp;
  job->stats.pairs = m + mb + mc;
  job->stats.pairs_hashed = mb;
  job->stats.pairs_mid = mc;
  job->stats.flushes = hs->flushes;
  job->stats.map_seal_waits = hs->seal_waits;
  job->stats.map_spills = hs->spills;
  job->stats.km_points_scanned = hs->km_scanned;
  if (m_total >= (1ULL << 32) - 1 || mb >= (1ULL << 32) - 1 || mc >= (1ULL << 32) - 1)
    return fail(job, MR_ERR_UNSUPPORTED, ">= 2^32 intermediate pairs in one group");
  if (job->km_comb()) {   // KM combiner: the Map produced the cluster sums; nothing to group
    uint64_t pts = 0;
    for (const Batch& b : job->batches) pts += b.n;
    job->stats.words_combined = pts;
    job->km_combined = true;
    job->nseg = job->k;
    if (job->prof.on) job->prof.collect();
    job->state = kGrouped;
    return MR_OK;
  }
  if (job->cfg.workload == MR_STRINGMATCH && (job->cfg.flags & MR_FLAG_SM_LINES)) {
    // per-line output (L125): one record start per match -> sort + unique (the group-by path)
    CK(run_sort(job->sw, job->h.p, m, &job->skeys, nullptr, job->st, job->nsm, job->stream, &job->prof,
                &job->stats.hist_ms, &job->stats.sort_ms, 64),
       "radix sort (lines)");
    job->stats.sort_passes += job->sw.passes;
    job->perm = nullptr;
    CK(job->seg_start.ensure(m + 1), "alloc segments");
    st = do_segments_into(job, job->skeys, m, job->seg_start.p, job->nseg);
    if (st != MR_OK) return st;
    job->stats.n_keys = job->nseg;
    if (job->prof.on) job->prof.collect();
    job->state = kGrouped;
    return MR_OK;
  }
  if (job->cfg.workload == MR_STRINGMATCH) {  // Map-only
    job->nseg = m;
    if (job->prof.on) job->prof.collect();      // settle_map synchronised the stream
    job->state = kGrouped;
    return MR_OK;
  }
  job->nseg_b = job->nseg_c = 0;
  job->nseg_p = job->n_extra = 0;   // (ingested jobs have no combiner partials)
  job->skeysb = nullptr;
  job->permb = nullptr;
  job->skeysc = nullptr;
  job->segc = nullptr;
  job->mid_from_table = false;
  job->nseg_l = 0;
  if (split && tables) {
    // the two tables hold every exact and mid word: their nonzero counts are the final keys
    Prof::Span sp{};
    if (job->prof.on) job->prof.begin(job->stream, sp);
    job->nseg_a = 0;
    job->nseg_p = 0;
    job->mp = 0;
    job->skeysp = nullptr;
    job->perm = nullptr;
    st = tables_extract(job);
    if (st != MR_OK) return st;
    CK(job->seg_counts.ensure(1), "alloc");
    job->sega = job->tile_base.p;   // (no exact segments)
    if (job->prof.on) job->prof.end(job->stream, sp, &job->stats.seg_ms);
  } else if (split) {
    // exact stream: keys only (the key is the record), no byte verification needed
    CK(run_sort32(job->sw, job->hx.p, m_total, &job->skeysx, job->st, job->nsm, job->stream, &job->prof,
                  &job->stats.hist_ms, &job->stats.sort_keys_ms, kExactBits),   // exact keys < 2^30
       "radix sort (exact)");
    job->stats.sort_passes += job->sw.passes;
    job->stats.sort_passes_keys += job->sw.passes;
    job->perm = nullptr;
    Prof::Span sp{};
    if (job->prof.on) job->prof.begin(job->stream, sp);
    // heads (count, scan, write) into seg_startx.
    // (A single-pass select with a decoupled look-back over the 4096-key tiles measured slower:
    // 5.4 ms against 3.3 + 2.2 ms on C5.)
    st = do_segments32(job, job->skeysx, m, job->seg_startx, job->nseg_a);
    if (st != MR_OK) return st;
    job->sega = job->seg_startx.p;
    // combiner partials: sort (keys-only, 30-bit key, count above bit 32), segments, then merge
    // into the exact segments or the extra list of partial-only keys
    job->nseg_p = job->n_extra = 0;
    job->skeysp = nullptr;
    if (job->mp) {
      const uint64_t mp = job->mp;
      CK(run_sort(job->swp, job->hp.p, mp, &job->skeysp, nullptr, job->st, job->nsm, job->stream, nullptr,
                  nullptr, nullptr, kExactBits),
         "radix sort (partials)");
      job->stats.sort_passes += job->swp.passes;
      CK(job->seg_startp.ensure(mp + 1), "alloc partial segments");
      st = do_segments_into(job, job->skeysp, mp, job->seg_startp.p, job->nseg_p, (1ULL << kExactBits) - 1);
      if (st != MR_OK) return st;
      const uint64_t np = job->nseg_p;
      CK(job->midx.ensure(np + 1), "alloc merge");
      CK(job->psum.ensure(np + 1), "alloc merge");
      CK(job->xkeys.ensure(np + 1), "alloc merge");
      CK(job->pxcounts.ensure(np + 1), "alloc merge");
      CK(cudaMemsetAsync(&job->st->n_extra, 0, 2 * sizeof(unsigned long long), job->stream), "memset");
      CK(launch_comb_merge(job->seg_startp.p, np, job->skeysp, job->sega, job->nseg_a, job->skeysx, job->midx.p,
                           job->psum.p, job->xkeys.p, job->pxcounts.p, &job->st->n_extra, job->stream),
         "combiner merge");
      CK(read_state(job), "sync merge");
      job->n_extra = hs->n_extra;
      job->stats.words_combined = hs->words_comb;
    }
    if (job->prof.on) job->prof.end(job->stream, sp, &job->stats.seg_ms);
    // mid stream: exact 48-bit keys, keys only (no fillers: plain stores)
    CK(run_sort(job->swc, job->hc.p, mc_total, &job->skeysc, nullptr, job->st, job->nsm, job->stream, &job->prof,
                &job->stats.hist_ms, &job->stats.sort_ms, kMidBits),
       "radix sort (mid)");
    job->stats.sort_passes += job->swc.passes;
    job->stats.sort_passes_mid += job->swc.passes;
    Prof::Span spc{};
    if (job->prof.on) job->prof.begin(job->stream, spc);
    job->segc = (job->skeysc == job->swc.ka.p) ? job->swc.kb.p : job->swc.ka.p;
    st = do_segments_into(job, job->skeysc, mc, job->segc, job->nseg_c);
    if (st != MR_OK) return st;
    if (job->prof.on) job->prof.end(job->stream, spc, &job->stats.seg_ms);
  }
  // general stream (II / KM / ingested WC) or the WC hashed stream: sort with the permutation,
  // verify equal hashes byte for byte, re-hash and re-sort on a collision (slow path)
  {
    uint64_t* keys = split ? job->hb.p : job->h.p;
    const uint64_t* kref = split ? job->krefb.p : (has_kref(job->cfg.workload) || job->ingested ? job->kref.p : nullptr);
    const uint64_t n = split ? mb_total : m_total;   // (sentinel entries sort after every real key)
    const uint64_t nreal = split ? mb : m;
    uint32_t& kbits = split ? job->key_bits_b : job->key_bits;
    SortWork& W = split ? job->swb : job->sw;
    const uint64_t** sk = split ? &job->skeysb : &job->skeys;
    const uint32_t** pm = split ? &job->permb : &job->perm;
    DBuf<uint64_t>& seg = split ? job->seg_startb : job->seg_start;
    uint64_t& ns = split ? job->nseg_b : job->nseg_a;
    for (int attempt = 0;; ++attempt) {
      // sentinel keys sort after every real key: the first nreal sorted positions are the real pairs
      CK(run_sort(W, keys, n, sk, pm, job->st, job->nsm, job->stream, &job->prof, &job->stats.hist_ms,
                  &job->stats.sort_ms, static_cast<int>(kbits)),
         "radix sort");
      job->stats.sort_passes += W.passes;
      Prof::Span sp2{};
      if (job->prof.on) job->prof.begin(job->stream, sp2);
      st = do_segments(job, *sk, *pm, kref, nreal, kbits, seg, ns);
      if (st != MR_OK) return st;
      if (job->prof.on) job->prof.end(job->stream, sp2, &job->stats.seg_ms);
      const uint32_t coll = hs->collisions;
      if (coll == 0) break;
      job->stats.collisions += coll;
      if (attempt >= 3) return fail(job, MR_ERR_UNSUPPORTED, "unresolvable 64-bit hash collision");
      // slow path: recompute every hashed key with a fresh full-width hash, then sort again
      CK(launch_rehash(keys, kref, n, 0xC0111DE5ULL + attempt, job->stream), "rehash");
      kbits = 64;
    }
    if (!split) { job->nseg_a = ns; }
  }
  job->nseg = job->nseg_a + job->n_extra + job->nseg_c + job->nseg_b + (job->mid_from_table ? job->nseg_l : 0);
  job->stats.n_keys = job->nseg;
  Prof::Span sp3{};
  if (job->prof.on) job->prof.begin(job->stream, sp3);
  if (job->cfg.workload == MR_WORDCOUNT || job->cfg.workload == MR_INVINDEX) {
    CK(job->key_off.ensure(job->nseg + 1), "alloc key offsets");
    if (split) {
      const uint64_t na = job->nseg_a + job->n_extra;   // exact segments, then partial-only keys
      CK(launch_key_lengths_exact32(job->sega, job->nseg_a, job->skeysx, job->key_off.p, job->stream),
         "key lengths (exact)");
      CK(launch_key_lengths_list32(job->xkeys.p, job->n_extra, job->key_off.p + job->nseg_a, job->stream),
         "key lengths (partial-only)");
      CK(launch_key_lengths_exact(job->segc, job->nseg_c, job->skeysc, job->key_off.p + na, job->stream),
         "key lengths (mid)");
      CK(launch_key_lengths(job->seg_startb.p, job->nseg_b, job->permb, job->krefb.p,
                            job->key_off.p + na + job->nseg_c,
                            job->stream),
         "key lengths (hashed)");
      if (job->mid_from_table && job->nseg_l)   // the long-word table's keys (a reference list)
        CK(launch_key_lengths(nullptr, job->nseg_l, nullptr, job->lkref_out.p,
                              job->key_off.p + na + job->nseg_c + job->nseg_b, job->stream),
           "key lengths (long table)");
    } else {
      CK(launch_key_lengths(job->seg_start.p, job->nseg, job->perm, job->kref.p, job->key_off.p, job->stream),
         "key lengths");
    }
    uint64_t* ss;
    uint32_t ep;
    CK(scan_ws(job, job->nseg, &ss, &ep), "alloc scan workspace");
    CK(launch_scan_u64(job->key_off.p, job->key_off.p, job->nseg,
                       reinterpret_cast<unsigned long long*>(job->key_off.p + job->nseg), ss, ep,
                       &job->st->tile_counter[2], job->stream),
       "scan key lengths");
    CK(cudaMemcpyAsync(job->tmp_h.p, job->key_off.p + job->nseg, 8, cudaMemcpyDeviceToHost, job->stream), "read key bytes");
    CK(cudaStreamSynchronize(job->stream), "sync key bytes");
    job->key_bytes = job->tmp_h.p[0];
  }
  if (job->prof.on) { job->prof.end(job->stream, sp3, &job->stats.seg_ms); CK(cudaStreamSynchronize(job->stream), "sync"); job->prof.collect(); }
  if (!job->in_fold && !job->in_exchange) {   // the folded batches' own group-by counters
    const mr_stats& f = job->fold_stats;
    job->stats.pairs += f.pairs;
    job->stats.pairs_hashed += f.pairs_hashed;
    job->stats.pairs_mid += f.pairs_mid;
    job->stats.pairs_partial += f.pairs_partial;
    job->stats.words_combined += f.words_combined;
    job->stats.flushes += f.flushes;
  }
  job->state = kGrouped;
  return MR_OK;
}

mr_status mr_reduce(mr_job* job) {
  if (!job) return MR_ERR_INVALID;
  if (job->state != kGrouped) return fail(job, MR_ERR_STATE, "mr_reduce before mr_group");
  CK(cudaSetDevice(job->cfg.device), "set device");
  const uint64_t S = job->nseg, m = job->m;
  cudaStream_t s = job->stream;
  Prof::Span sp{};
  if (job->prof.on) job->prof.begin(s, sp);
  switch (job->cfg.workload) {
    case MR_WORDCOUNT: {
      CK(job->counts.ensure(S + 1), "alloc counts");
      CK(job->keys_out.ensure(job->key_bytes + 1), "alloc keys");
      if (job->split()) {
        // every Map value is 1: a key's count is its segment length (exact stream first, then
        // the hashed stream; the output order is the sorted order of each stream)
        const uint64_t na = job->nseg_a + job->n_extra;
        CK(launch_seg_lengths(job->sega, job->nseg_a, job->counts.p, s), "counts (exact)");
        CK(launch_comb_add(job->midx.p, job->psum.p, job->nseg_p, job->counts.p, s), "counts (combined)");
        if (job->n_extra)
          CK(cudaMemcpyAsync(job->counts.p + job->nseg_a, job->pxcounts.p, job->n_extra * 8, cudaMemcpyDeviceToDevice, s),
             "counts (partial-only)");
        if (job->mid_from_table)
          CK(cudaMemcpyAsync(job->counts.p + na, job->mcounts.p, job->nseg_c * 8, cudaMemcpyDeviceToDevice, s),
             "counts (mid)");
        else
          CK(launch_seg_lengths(job->segc, job->nseg_c, job->counts.p + na, s), "counts (mid)");
        CK(launch_seg_lengths(job->seg_startb.p, job->nseg_b, job->counts.p + na + job->nseg_c, s),
           "counts (hashed)");
        CK(launch_key_decode(job->segc, job->nseg_c, job->skeysc, job->key_off.p + na, job->keys_out.p, s),
           "key decode (mid)");
        CK(launch_key_decode_list32(job->xkeys.p, job->n_extra, job->key_off.p + job->nseg_a, job->keys_out.p, s),
           "key decode (partial-only)");
        CK(launch_key_decode32(job->sega, job->nseg_a, job->skeysx, job->key_off.p, job->keys_out.p, s),
           "key decode");
        CK(launch_key_copy(job->seg_startb.p, job->nseg_b, job->permb, job->krefb.p,
                           job->key_off.p + na + job->nseg_c,
                           job->keys_out.p, s),
           "key copy");
        if (job->mid_from_table && job->nseg_l) {   // the long-word table's keys and counts
          const uint64_t nl0 = na + job->nseg_c + job->nseg_b;
          CK(launch_key_copy(nullptr, job->nseg_l, nullptr, job->lkref_out.p, job->key_off.p + nl0, job->keys_out.p, s),
             "key copy (long table)");
          CK(cudaMemcpyAsync(job->counts.p + nl0, job->lcounts.p, job->nseg_l * 8, cudaMemcpyDeviceToDevice, s),
             "counts (long table)");
        }
      } else {
        CK(job->worklist.ensure(m / 1024 + 64), "alloc worklist");
        CK(launch_reduce_wc(job->seg_start.p, S, job->skeys, job->perm, job->v.p, 1, job->counts.p, job->worklist.p,
                            job->st, job->nsm, s),
           "reduce wc");
        CK(launch_key_copy(job->seg_start.p, S, job->perm, job->kref.p, job->key_off.p, job->keys_out.p, s),
           "key copy");
      }
      CK(job->val_off.ensure(S + 1), "alloc val offsets");
      CK(launch_iota_scaled(S, 8, job->val_off.p, s), "val offsets");
      job->out_n = S;
      job->out_keys_bytes = job->key_bytes;
      job->out_vals_bytes = S * 8;
      break;
    }
    case MR_INVINDEX: {
      CK(job->gathered.ensure(m + 1), "alloc values");
      CK(launch_gather_u64(job->perm, job->v.p, m, job->gathered.p, s), "gather values");
      CK(job->val_off.ensure(S + 1), "alloc val offsets");
      CK(launch_offsets_scaled(job->seg_start.p, S, 8, job->val_off.p, s), "val offsets");
      CK(job->keys_out.ensure(job->key_bytes + 1), "alloc keys");
      CK(launch_key_copy(job->seg_start.p, S, job->perm, job->kref.p, job->key_off.p, job->keys_out.p, s), "key copy");
      job->out_n = S;
      job->out_keys_bytes = job->key_bytes;
      job->out_vals_bytes = m * 8;
      break;
    }
    case MR_KMEANS: {
      const uint32_t k = job->k;
      CK(job->sums.ensure(8ULL * k), "alloc sums");
      CK(job->cnts.ensure(k), "alloc counts");
      if (!job->km_partial && !job->km_combined) {
        CK(job->worklist.ensure(m / 1024 + 64), "alloc worklist");
        CK(launch_reduce_km(job->seg_start.p, S, job->skeys, job->perm, job->v.p, job->sums.p, job->cnts.p, k,
                            job->worklist.p, job->st, job->nsm, s),
           "reduce km");
      }
      const uint32_t* list = job->km_partial ? job->km_list.p : nullptr;
      const uint32_t nout = job->km_partial ? job->km_nlist : k;
      CK(job->keys_out.ensure(4ULL * k), "alloc keys");
      CK(job->vals_out.ensure(40ULL * k), "alloc vals");
      CK(job->key_off.ensure(k + 1), "alloc key offsets");
      CK(job->val_off.ensure(k + 1), "alloc val offsets");
      CK(launch_km_finalize(job->sums.p, job->cnts.p, job->cent.p, k, list, nout, job->vals_out.p, job->val_off.p,
                            job->keys_out.p, job->key_off.p, s),
         "km finalize");
      job->out_n = nout;
      job->out_keys_bytes = 4ULL * nout;
      job->out_vals_bytes = 40ULL * nout;
      break;
    }
    case MR_STRINGMATCH: {
      const uint64_t n = S;   // matches, or (per-line output) distinct record starts
      if (job->cfg.flags & MR_FLAG_SM_LINES) {
        CK(job->keys_out.ensure(8 * n + 8), "alloc keys");
        CK(launch_seg_keys(job->seg_start.p, n, job->skeys, reinterpret_cast<uint64_t*>(job->keys_out.p), s),
           "line keys");
      }
      CK(job->key_off.ensure(n + 1), "alloc key offsets");
      CK(job->val_off.ensure(n + 1), "alloc val offsets");
      CK(launch_iota_scaled(n, 8, job->key_off.p, s), "key offsets");
      CK(cudaMemsetAsync(job->val_off.p, 0, (n + 1) * 8, s), "val offsets");
      job->out_n = n;
      job->out_keys_bytes = n * 8;
      job->out_vals_bytes = 0;
      break;
    }
  }
  if (job->prof.on) job->prof.end(s, sp, &job->stats.reduce_ms);
  job->state = kReduced;
  return MR_OK;
}

mr_status mr_fetch(mr_job* job, mr_result* out) {
  if (!job || !out) return MR_ERR_INVALID;
  if (job->state != kReduced) return fail(job, MR_ERR_STATE, "mr_fetch before mr_reduce");
  CK(cudaSetDevice(job->cfg.device), "set device");
  cudaStream_t s = job->stream;
  const uint64_t n = job->out_n;
  CK(job->keys_h.ensure(job->out_keys_bytes + 1), "alloc host keys");
  CK(job->vals_h.ensure(job->out_vals_bytes + 1), "alloc host vals");
  CK(job->key_off_h.ensure(n + 1), "alloc host key offsets");
  CK(job->val_off_h.ensure(n + 1), "alloc host val offsets");
  const uint8_t* dkeys = (job->cfg.workload == MR_STRINGMATCH && !(job->cfg.flags & MR_FLAG_SM_LINES))
                             ? reinterpret_cast<const uint8_t*>(job->h.p)
                             : job->keys_out.p;
  const uint8_t* dvals = job->cfg.workload == MR_WORDCOUNT ? reinterpret_cast<const uint8_t*>(job->counts.p)
                         : job->cfg.workload == MR_INVINDEX ? reinterpret_cast<const uint8_t*>(job->gathered.p)
                                                            : job->vals_out.p;
  if (job->out_keys_bytes) CK(cudaMemcpyAsync(job->keys_h.p, dkeys, job->out_keys_bytes, cudaMemcpyDeviceToHost, s), "D2H keys");
  if (job->out_vals_bytes) CK(cudaMemcpyAsync(job->vals_h.p, dvals, job->out_vals_bytes, cudaMemcpyDeviceToHost, s), "D2H vals");
  CK(cudaMemcpyAsync(job->key_off_h.p, job->key_off.p, (n + 1) * 8, cudaMemcpyDeviceToHost, s), "D2H key offsets");
  CK(cudaMemcpyAsync(job->val_off_h.p, job->val_off.p, (n + 1) * 8, cudaMemcpyDeviceToHost, s), "D2H val offsets");
  CK(cudaStreamSynchronize(s), "fetch");
  if (job->prof.on) job->prof.collect();
  out->n_keys = n;
  out->keys = job->keys_h.p;
  out->key_offsets = job->key_off_h.p;
  out->vals = job->vals_h.p;
  out->val_offsets = job->val_off_h.p;
  return MR_OK;
}

// ---------------------------------------------------------------- multi-GPU exchange (§8(e))
mr_status mr_partition_count(mr_job* job, uint64_t* counts, uint64_t* entry_bytes) {
  if (!job || !counts) return MR_ERR_INVALID;
  if (job->state != kMapped && job->state != kCreated) return fail(job, MR_ERR_STATE, "mr_partition_count out of order");
  CK(cudaSetDevice(job->cfg.device), "set device");
  const uint32_t R = static_cast<uint32_t>(job->cfg.nranks);
  const int w = job->cfg.workload;
  if (w == MR_STRINGMATCH) return fail(job, MR_ERR_UNSUPPORTED, "StringMatch is Map-only: no exchange");
  const bool combine = (w == MR_KMEANS) || (w == MR_WORDCOUNT && !(job->cfg.flags & MR_FLAG_NO_COMBINE));
  XSource xs;
  xs.nranks = R;
  if (combine) {
    // combiner (SURVEY §8(e) reading): local group + reduce, exchange partial aggregates
    mr_status st = mr_group(job);
    if (st != MR_OK) return st;
    st = mr_reduce(job);
    if (st != MR_OK) return st;
    if (w == MR_WORDCOUNT) {
      xs.mode = kXSegs;
      xs.n = job->nseg;
      xs.keys = job->keys_out.p;
      xs.key_off = job->key_off.p;
      xs.counts = job->counts.p;
    } else {
      xs.mode = kXKM;
      xs.n = job->k;
      xs.sums = job->sums.p;
      xs.cnts = job->cnts.p;
    }
  } else {
    // raw pairs: settle the Map (capacity check / replay) without grouping
    mr_status st = settle_map(job);
    if (st != MR_OK) return st;
    DevState* hs = job->st_h.p;
    const uint64_t m = hs->pair_cursor;
    job->m = m - hs->pads;
    job->mb = job->split() ? hs->pair_cursor_b - hs->pads_b : 0;
    job->mc = job->split() ? hs->pair_cursor_c - hs->pads_c : 0;
    job->stats.pairs = job->m + job->mb + job->mc;
    if (job->split()) {
      xs.mode = kXSplit;
      xs.hx = job->hx.p;
      xs.nx = m;
      xs.hc = job->hc.p;
      xs.nc = hs->pair_cursor_c;   // (all slots: sentinel entries are skipped)
      xs.hp = job->hp.p;
      xs.np = job->wc_comb() ? hs->pair_cursor_p : 0;   // (no tables on the raw exchange path: wc_table)
      xs.n = m + xs.np + hs->pair_cursor_c + hs->pair_cursor_b;
      xs.kref = job->krefb.p;
    } else {
      xs.mode = kXPairs;
      xs.n = m;
      xs.kref = job->kref.p;
      xs.v = job->v.p;
      xs.vbytes = vbytes_of(w);
    }
  }
  CK(job->xcounts.ensure(2 * R), "alloc counts");
  CK(job->xcursors.ensure(2 * R), "alloc cursors");
  CK(job->xheapbase.ensure(R), "alloc heap base");
  CK(job->xcounts_h.ensure(4 * R), "alloc host counts");
  CK(launch_x_count(xs, job->xcounts.p, job->nsm, job->stream), "partition count");
  CK(cudaMemcpyAsync(job->xcounts_h.p, job->xcounts.p, 2 * R * 8, cudaMemcpyDeviceToHost, job->stream), "D2H counts");
  CK(cudaStreamSynchronize(job->stream), "sync counts");
  unsigned long long* cur = job->xcounts_h.p + 2 * R;   // host staging for cursors
  unsigned long long e = 0, hb = 0;
  std::vector<unsigned long long> hbase(R);
  for (uint32_t r = 0; r < R; ++r) {
    counts[2 * r] = job->xcounts_h.p[2 * r];
    counts[2 * r + 1] = job->xcounts_h.p[2 * r + 1];
    cur[2 * r] = e;
    cur[2 * r + 1] = hb;
    hbase[r] = hb;
    e += counts[2 * r];
    hb += counts[2 * r + 1];
  }
  CK(cudaMemcpyAsync(job->xcursors.p, cur, 2 * R * 8, cudaMemcpyHostToDevice, job->stream), "H2D cursors");
  CK(cudaMemcpyAsync(job->xheapbase.p, hbase.data(), R * 8, cudaMemcpyHostToDevice, job->stream), "H2D heap base");
  CK(cudaStreamSynchronize(job->stream), "sync cursors");
  xs.heap_base = job->xheapbase.p;
  job->xs = xs;
  if (entry_bytes) *entry_bytes = (xs.mode == kXKM) ? sizeof(XEntryKM) : sizeof(XEntry);
  job->state = kPartitioned;
  return MR_OK;
}

mr_status mr_partition_write(mr_job* job, void* entries, void* heap) {
  if (!job) return MR_ERR_INVALID;
  if (job->state != kPartitioned) return fail(job, MR_ERR_STATE, "mr_partition_write before mr_partition_count");
  CK(cudaSetDevice(job->cfg.device), "set device");
  if (job->xs.n && !entries) return fail(job, MR_ERR_INVALID, "entries is NULL");
  CK(launch_x_scatter(job->xs, job->xcursors.p, static_cast<uint8_t*>(entries), static_cast<uint8_t*>(heap),
                      job->stream),
     "partition scatter");
  return MR_OK;
}

mr_status mr_ingest(mr_job* job, const void* entries, const void* heap, const uint64_t* recv_counts) {
  if (!job || !recv_counts) return MR_ERR_INVALID;
  if (job->state != kPartitioned) return fail(job, MR_ERR_STATE, "mr_ingest before mr_partition_write");
  CK(cudaSetDevice(job->cfg.device), "set device");
  job->exchanged = true;
  return ingest_impl(job, entries, heap, recv_counts, static_cast<uint32_t>(job->cfg.nranks));
}

}  // extern "C"

namespace {
// received entries of R sources (recv_counts[2r], [2r+1]) -> the job's ingested pair stream (or,
// for KM, the owner's partial sums)
mr_status ingest_impl(mr_job* job, const void* entries, const void* heap, const uint64_t* recv_counts, uint32_t R) {
  std::vector<uint64_t> se(R + 1, 0), sh(R + 1, 0);
  for (uint32_t r = 0; r < R; ++r) {
    se[r + 1] = se[r] + recv_counts[2 * r];
    sh[r + 1] = sh[r] + recv_counts[2 * r + 1];
  }
  const uint64_t n = se[R];
  if (n && !entries) return fail(job, MR_ERR_INVALID, "entries is NULL");
  cudaStream_t s = job->stream;
  job->batches.clear();
  if (job->cfg.workload == MR_KMEANS) {
    const uint32_t k = job->k;
    CK(job->sums.ensure(8ULL * k), "alloc sums");
    CK(job->cnts.ensure(k), "alloc counts");
    CK(cudaMemsetAsync(job->sums.p, 0, 64ULL * k, s), "memset sums");
    CK(cudaMemsetAsync(job->cnts.p, 0, 8ULL * k, s), "memset counts");
    CK(launch_x_ingest_km(entries, n, job->sums.p, job->cnts.p, k, s), "ingest km");
    std::vector<uint32_t> own;
    for (uint32_t j = 0; j < k; ++j)
      if (km_owner(j, static_cast<uint32_t>(job->cfg.nranks)) == static_cast<uint32_t>(job->cfg.rank)) own.push_back(j);
    CK(job->km_list.ensure(own.size() + 1), "alloc owner list");
    if (!own.empty())
      CK(cudaMemcpyAsync(job->km_list.p, own.data(), own.size() * 4, cudaMemcpyHostToDevice, s), "H2D owners");
    CK(cudaStreamSynchronize(s), "sync owners");
    job->km_nlist = static_cast<uint32_t>(own.size());
    job->km_partial = true;
    job->state = kMapped;
    return MR_OK;
  }
  // The ingested stream lives in h / kref / v (u64 values).  The Map's own buffers stay as they
  // are (a WordCount job's split streams hx / hb / hc / hp are untouched), so the job can be reset
  // and mapped again; the ingested count is exact, so settle_map skips the capacity check.
  CK(job->h.ensure(n + 1), "alloc pairs");
  CK(job->kref.ensure(n + 1), "alloc pairs");
  CK(job->v.ensure((n + 1) * 8), "alloc pairs");
  if (!job->split()) job->cap = std::min<uint64_t>(std::min(job->h.n, job->kref.n), job->v.n / 8);
  CK(job->src_e.ensure(R + 1), "alloc src");
  CK(job->src_h.ensure(R + 1), "alloc src");
  CK(cudaMemcpyAsync(job->src_e.p, se.data(), (R + 1) * 8, cudaMemcpyHostToDevice, s), "H2D src");
  CK(cudaMemcpyAsync(job->src_h.p, sh.data(), (R + 1) * 8, cudaMemcpyHostToDevice, s), "H2D src");
  CK(launch_x_ingest(entries, static_cast<const uint8_t*>(heap), n, job->src_e.p, job->src_h.p, R, job->h.p,
                     job->kref.p, reinterpret_cast<uint64_t*>(job->v.p), 0x5EEDB200ULL,
                     (job->cfg.flags & MR_FLAG_WEAK_HASH_DEBUG) ? 1u : 0u, job->key_bits, s),
     "ingest");
  CK(cudaMemsetAsync(job->st, 0, sizeof(DevState), s), "reset state");
  job->tmp_h.p[0] = n;
  CK(cudaMemcpyAsync(&job->st->pair_cursor, job->tmp_h.p, 8, cudaMemcpyHostToDevice, s), "set pair count");
  CK(cudaStreamSynchronize(s), "sync ingest");
  job->ingested = true;
  job->state = kMapped;
  return MR_OK;
}
}  // namespace

extern "C" {

mr_status mr_set_xwindows(mr_job* job, uint32_t nranks, void* const* entries, void* const* heaps,
                          uint64_t* const* cursors, uint64_t entry_cap, uint64_t heap_cap) {
  if (!job) return MR_ERR_INVALID;
  if (nranks == 0) { job->xranks = 0; return MR_OK; }
  if (job->cfg.workload != MR_INVINDEX) return fail(job, MR_ERR_INVALID, "fused windows: InvertedIndex only");
  if (nranks > static_cast<uint32_t>(kMaxRanks) || !entries || !heaps || !cursors)
    return fail(job, MR_ERR_INVALID, "bad window arrays");
  if (job->state != kCreated) return fail(job, MR_ERR_STATE, "mr_set_xwindows after mr_map");
  std::vector<XWindow> w(nranks);
  for (uint32_t r = 0; r < nranks; ++r) {
    if (!entries[r] || !heaps[r] || !cursors[r] || (reinterpret_cast<uintptr_t>(entries[r]) & 15u) ||
        (reinterpret_cast<uintptr_t>(heaps[r]) & 7u) || (reinterpret_cast<uintptr_t>(cursors[r]) & 7u))
      return fail(job, MR_ERR_INVALID, "window pointer NULL or misaligned");
    w[r] = XWindow{static_cast<uint8_t*>(entries[r]), static_cast<uint8_t*>(heaps[r]),
                   reinterpret_cast<unsigned long long*>(cursors[r]), entry_cap, heap_cap};
  }
  CK(cudaSetDevice(job->cfg.device), "set device");
  CK(job->xwin.ensure(nranks), "alloc windows");
  CK(cudaMemcpyAsync(job->xwin.p, w.data(), nranks * sizeof(XWindow), cudaMemcpyHostToDevice, job->stream),
     "H2D windows");
  CK(cudaStreamSynchronize(job->stream), "sync windows");
  job->xranks = nranks;
  return MR_OK;
}

mr_status mr_ingest_xwindow(mr_job* job, const void* entries, const void* heap, const uint64_t* cursor,
                            uint64_t entry_cap, uint64_t heap_cap) {
  if (!job || !cursor) return MR_ERR_INVALID;
  if (job->cfg.workload != MR_INVINDEX) return fail(job, MR_ERR_INVALID, "fused windows: InvertedIndex only");
  if (job->state != kMapped && job->state != kCreated)
    return fail(job, MR_ERR_STATE, "mr_ingest_xwindow after mr_group");
  CK(cudaSetDevice(job->cfg.device), "set device");
  // this rank's Map errors first (read_state synchronises the job stream): a URL clamped to
  // 65535 bytes in the Map's queue must reject the batch here too, as settle_map does
  CK(read_state(job), "map (async)");
  if (job->st_h.p->err & kErrKeyTooLong) return fail(job, MR_ERR_OVERFLOW, "an emitted key exceeds 65535 bytes");
  uint64_t* c = job->tmp_h.p + 2;
  CK(cudaMemcpyAsync(c, cursor, 2 * sizeof(uint64_t), cudaMemcpyDeviceToHost, job->stream), "D2H window cursor");
  CK(cudaStreamSynchronize(job->stream), "sync window cursor");
  if (c[0] > entry_cap || c[1] > heap_cap)
    return fail(job, MR_ERR_OOM, "receive window overflow: " + std::to_string(c[0]) + " entries / " +
                                          std::to_string(c[1]) + " heap bytes needed");
  const uint32_t R = static_cast<uint32_t>(std::max(1, job->cfg.nranks));
  std::vector<uint64_t> counts(2 * R, 0);
  counts[0] = c[0];   // one contiguous block (source order is irrelevant after the sort)
  counts[1] = c[1];
  job->state = kPartitioned;
  return mr_ingest(job, entries, heap, counts.data());
}

// ---- device memory + CUDA IPC helpers for receive windows shared between processes ----
mr_status mr_dev_alloc(int device, uint64_t bytes, void** dptr) {
  if (!dptr) return MR_ERR_INVALID;
  *dptr = nullptr;
  if (cudaSetDevice(device) != cudaSuccess) { cudaGetLastError(); return MR_ERR_CUDA; }
  if (cudaMalloc(dptr, std::max<uint64_t>(bytes, 256)) != cudaSuccess) { cudaGetLastError(); *dptr = nullptr; return MR_ERR_OOM; }
  return MR_OK;
}
mr_status mr_dev_free(void* dptr) {
  if (dptr && cudaFree(dptr) != cudaSuccess) { cudaGetLastError(); return MR_ERR_CUDA; }
  return MR_OK;
}
mr_status mr_dev_copy(void* dst, const void* src, uint64_t bytes) {   // synchronous, any direction
  if (bytes && (!dst || !src)) return MR_ERR_INVALID;
  if (bytes && cudaMemcpy(dst, src, bytes, cudaMemcpyDefault) != cudaSuccess) { cudaGetLastError(); return MR_ERR_CUDA; }
  return MR_OK;
}
mr_status mr_dev_zero(void* dptr, uint64_t bytes) {
  if (bytes && !dptr) return MR_ERR_INVALID;
  if (bytes && cudaMemset(dptr, 0, bytes) != cudaSuccess) { cudaGetLastError(); return MR_ERR_CUDA; }
  return MR_OK;
}
mr_status mr_ipc_handle(const void* dptr, void* handle) {
  if (!dptr || !handle) return MR_ERR_INVALID;
  cudaIpcMemHandle_t h;
  if (cudaIpcGetMemHandle(&h, const_cast<void*>(dptr)) != cudaSuccess) { cudaGetLastError(); return MR_ERR_CUDA; }
  static_assert(sizeof(h) == MR_IPC_HANDLE_BYTES, "IPC handle size");
  std::memcpy(handle, &h, sizeof(h));
  return MR_OK;
}
mr_status mr_ipc_open(int device, const void* handle, void** dptr) {
  if (!handle || !dptr) return MR_ERR_INVALID;
  *dptr = nullptr;
  cudaIpcMemHandle_t h;
  std::memcpy(&h, handle, sizeof(h));
  if (cudaSetDevice(device) != cudaSuccess) { cudaGetLastError(); return MR_ERR_CUDA; }
  if (cudaIpcOpenMemHandle(dptr, h, cudaIpcMemLazyEnablePeerAccess) != cudaSuccess) {
    cudaGetLastError();
    *dptr = nullptr;
    return MR_ERR_CUDA;
  }
  return MR_OK;
}
mr_status mr_ipc_close(void* dptr) {
  if (dptr && cudaIpcCloseMemHandle(dptr) != cudaSuccess) { cudaGetLastError(); return MR_ERR_CUDA; }
  return MR_OK;
}

mr_status mr_get_stats(const mr_job* job, void* stats, size_t bytes) {
  if (!job || !stats) return MR_ERR_INVALID;
  mr_stats st = job->stats;
  st.kernel_launches = g_kernel_launches.load() - job->launches0;
  st.sort_ms += st.sort_keys_ms;   // sort_ms covers both streams
  std::memcpy(stats, &st, std::min(bytes, sizeof(mr_stats)));
  return MR_OK;
}

mr_status mr_job_destroy(mr_job* job) {
  if (!job) return MR_OK;
  cudaSetDevice(job->cfg.device);
  cudaStreamSynchronize(job->stream);
  for (void* p : job->owned) cudaFree(p);
  for (auto& b : job->host_rec) b.release();
  for (auto& b : job->host_off) b.release();
  job->prof.release();
  job->xcounts.release(); job->xcursors.release(); job->xheapbase.release(); job->xcounts_h.release();
  job->src_e.release(); job->src_h.release(); job->km_list.release(); job->xwin.release();
  job->xsend_e.release(); job->xsend_h.release(); job->xrecv_e.release(); job->xrecv_h.release();
  job->xrecv_counts.release(); job->acc_e.release(); job->acc_h.release(); job->xtab.release(); job->mtab_keys.release();
  job->mtab_cnt.release(); job->mkeys_out.release(); job->mcounts.release();
  job->ltab_keys.release(); job->ltab_cnt.release(); job->lkeys_out.release(); job->lkref_out.release();
  job->lcounts.release();
  job->cent.release(); release_pairs(job); job->tb.release();
  job->swp.release(); job->seg_startp.release(); job->psum.release(); job->pxcounts.release();
  job->midx.release(); job->xkeys.release();
  job->sw.release(); job->swb.release(); job->swc.release(); job->seg_startb.release(); job->seg_startx.release();
  job->scan_status.release();
  job->seg_counts.release(); job->tile_base.release(); job->seg_start.release(); job->key_off.release();
  job->val_off.release(); job->counts.release(); job->worklist.release(); job->gathered.release();
  job->keys_out.release(); job->vals_out.release(); job->vsorted.release(); job->sums.release(); job->cnts.release();
  job->keys_h.release(); job->vals_h.release(); job->key_off_h.release(); job->val_off_h.release();
  job->st_h.release(); job->tmp_h.release();
  if (job->st) cudaFree(job->st);
  for (cudaEvent_t e : job->line_ev) cudaEventDestroy(e);
  if (job->cstream) cudaStreamDestroy(job->cstream);
  if (job->own_stream && job->stream) cudaStreamDestroy(job->stream);
  cudaGetLastError();
  delete job;
  return MR_OK;
}

mr_status mr_sort_u64(const uint64_t* keys, uint64_t* keys_out, uint32_t* perm_out, uint64_t n, void* stream) {
  if ((n && (!keys || !keys_out || !perm_out)) || n >= (1ULL << 32) - 1) return MR_ERR_INVALID;
  if (n == 0) return MR_OK;
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  SortWork W;
  DevState* st = nullptr;
  int dev = 0;
  cudaGetDevice(&dev);
  cudaError_t e = cudaMalloc(reinterpret_cast<void**>(&st), sizeof(DevState));
  if (e == cudaSuccess) e = cudaMemsetAsync(st, 0, sizeof(DevState), s);
  const uint64_t* ko = nullptr;
  const uint32_t* po = nullptr;
  if (e == cudaSuccess) e = run_sort(W, keys, n, &ko, &po, st, sm_count(dev), s);
  if (e == cudaSuccess) e = cudaMemcpyAsync(keys_out, ko, n * 8, cudaMemcpyDeviceToDevice, s);
  if (e == cudaSuccess) e = cudaMemcpyAsync(perm_out, po, n * 4, cudaMemcpyDeviceToDevice, s);
  if (e == cudaSuccess) e = cudaStreamSynchronize(s);
  W.release();
  if (st) cudaFree(st);
  if (e != cudaSuccess) { cudaGetLastError(); return e == cudaErrorMemoryAllocation ? MR_ERR_OOM : MR_ERR_CUDA; }
  return MR_OK;
}

}  // extern "C"
