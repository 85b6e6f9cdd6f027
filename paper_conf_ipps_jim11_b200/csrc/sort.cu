// sort.cu — group-by-key, part 1: a hand-written onesweep-style LSD radix
// sort of the 64-bit intermediate sort keys with a u32 permutation payload, plus the generic
// single-pass (decoupled look-back) exclusive scan used by the segment and output steps.
//
// The paper reuses Mars's shuffle unchanged and does not describe it (PAPER.md L295, L305:
// "Word Count is an example where there is a large shuffle phase").  B200 design:
//   * one histogram pass computes all eight 8-bit digit histograms (k_hist); digits whose
//     histogram has a single non-empty bin are skipped by the host (constant-digit skip);
//   * each remaining digit is one pass of k_onesweep: a 4096-key tile is ranked with
//     warp-private counters + match.any (stable: warp-striped order == element order), the tile
//     count of every digit is published and the exclusive prefix over earlier tiles is obtained
//     by decoupled look-back on per-(tile, digit) status words; keys and payload are then
//     scattered through SMEM so that global writes are contiguous runs per digit.
// Look-back status words: [epoch:30 | kind:2 | value:32]; every launch uses a fresh epoch so
// the status buffer never needs clearing.
#include <algorithm>
#include <cmath>
#include <cstdio>
#include <cstdlib>

#include "common.cuh"

namespace bmr {
namespace {

constexpr uint32_t kAgg = 1u, kPrefix = 2u;
constexpr int kWarps = kSortThreads / 32;

__device__ __forceinline__ uint64_t pack_status(uint32_t epoch, uint32_t kind, uint32_t v) {
  return (static_cast<uint64_t>(epoch) << 34) | (static_cast<uint64_t>(kind) << 32) | v;
}

// Digit histograms of the first nd digits of `bits` bits (8 or 9): one read of the keys (16-byte
// loads: two u64 or four u32 keys each), shared atomics into a per-block nd x 512 table (stride
// kBinStride).
template <typename K>
__global__ void __launch_bounds__(256) k_hist(const K* __restrict__ keys, uint64_t m, uint32_t nd, uint32_t bits,
                                            uint32_t* hist) {
  constexpr int kPer = 16 / sizeof(K);
  __shared__ uint32_t sh[8 * kBinStride];
  for (int i = threadIdx.x; i < 8 * kBinStride; i += blockDim.x) sh[i] = 0;
  __syncthreads();
  const uint32_t mask = (1u << bits) - 1u;
  const uint64_t stride = static_cast<uint64_t>(gridDim.x) * blockDim.x;
  const uint64_t mv = m / kPer;
  const uint4* k4 = reinterpret_cast<const uint4*>(keys);
  for (uint64_t i = blockIdx.x * static_cast<uint64_t>(blockDim.x) + threadIdx.x; i < mv; i += stride) {
    const uint4 raw = __ldcs(k4 + i);
    K kk[kPer];
    memcpy(kk, &raw, 16);
#pragma unroll
    for (uint32_t d = 0; d < 8; ++d) {
      if (d >= nd) break;
#pragma unroll
      for (int q = 0; q < kPer; ++q) atomicAdd(&sh[d * kBinStride + (static_cast<uint32_t>(kk[q] >> (bits * d)) & mask)], 1u);
    }
  }
  if (blockIdx.x == 0 && threadIdx.x < m % kPer) {
    const K k = keys[mv * kPer + threadIdx.x];
    for (uint32_t d = 0; d < nd; ++d) atomicAdd(&sh[d * kBinStride + (static_cast<uint32_t>(k >> (bits * d)) & mask)], 1u);
  }
  __syncthreads();
  for (int i = threadIdx.x; i < static_cast<int>(nd) * kBinStride; i += blockDim.x)
    if (sh[i]) atomicAdd(&hist[i], sh[i]);
}

template <typename K, int IPT, bool kPay, int kBins, int kSlots = 0>
struct SortSmem {
  static constexpr int kTile = kSortThreads * IPT;
  uint32_t mm[kSlots > 0 ? kSlots : 1][kWarps][kSlots > 0 ? kBins : 1];   // match masks (kOrMatch)
  K keys[kTile];
  uint32_t idx[kPay ? kTile : 1];
  uint32_t wcnt[kWarps][kBins];    // per-warp digit counters, then warp-exclusive offsets
  uint32_t hist[kBins];
  uint32_t goff[kBins];
  uint32_t wsum[kWarps];
  uint32_t tile;
};


// One LSD pass over the digit [shift, shift + 8) (256 bins, one digit per thread).
// kOrMatch: rank with shared-memory match masks (one RED.OR of the lane bit per key into a
// per-warp digit slot, 4 slots in flight) instead of match.any — faster for a first pass whose
// 32-key groups carry many distinct digits (choose_rank_kind32).
// kPay: carry the u32 permutation payload (false: keys only, idx_in / idx_out unused).
// The tile histogram is built before the ranking and published at once as the tile's early
// aggregate; kLookWindow predecessor status words are fetched per look-back step (per digit).
template <typename K, bool kFirst, bool kOrMatch, int IPT, int MINB, bool kPay, int kLookWindow = 4>
__global__ void __launch_bounds__(kSortThreads, MINB) k_onesweep(const K* __restrict__ keys_in,
                                                               const uint32_t* __restrict__ idx_in,
                                                               K* __restrict__ keys_out,
                                                               uint32_t* __restrict__ idx_out, uint64_t m,
                                                               uint32_t shift, const uint32_t* __restrict__ bases,
                                                               uint64_t* status, uint32_t epoch,
                                                               unsigned int* tile_counter) {
  constexpr int kBins = 256, kDPT = kBins / kSortThreads;
  constexpr uint32_t kMask = kBins - 1;
  constexpr int kSortIPT = IPT;
  constexpr int kSlots = kOrMatch ? 4 : 0;
  using Smem = SortSmem<K, IPT, kPay, kBins, kSlots>;
  constexpr int kSortTile = Smem::kTile;
  static_assert(kDPT >= 1 && kDPT * kSortThreads == kBins, "bins must be a multiple of the block size");
  extern __shared__ __align__(16) uint8_t raw[];
  Smem& S = *reinterpret_cast<Smem*>(raw);
  const uint32_t tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  if (tid == 0) S.tile = atomicAdd(tile_counter, 1u);
  for (uint32_t i = tid; i < kWarps * kBins; i += kSortThreads) (&S.wcnt[0][0])[i] = 0;
  for (uint32_t i = tid; i < kBins; i += kSortThreads) S.hist[i] = 0;
  if constexpr (kOrMatch)
    for (uint32_t i = tid; i < kSlots * kWarps * kBins; i += kSortThreads) (&S.mm[0][0][0])[i] = 0;
  __syncthreads();
  const uint32_t tile = S.tile;
  const uint64_t tbase = static_cast<uint64_t>(tile) * kSortTile;
  const uint64_t wbase = tbase + static_cast<uint64_t>(warp) * 32 * kSortIPT;
  K key[kSortIPT];
  uint32_t rank[kSortIPT];
#pragma unroll
  for (int j = 0; j < kSortIPT; ++j) {
    const uint64_t e = wbase + j * 32 + lane;
    key[j] = e < m ? keys_in[e] : static_cast<K>(~static_cast<K>(0));  // padding sorts last (top digit value, after every real key)
  }
  const uint32_t d0 = tid * kDPT;   // this thread's digits: d0 .. d0 + kDPT - 1
  uint32_t tcount[kDPT];
  uint64_t* my = status + static_cast<uint64_t>(tile) * kBins + d0;
  if constexpr (kOrMatch) {
    // peer masks through shared memory (read back after a warp barrier, cleared by the group's
    // leader); the leader issues the tile histogram and warp-counter atomics (applied in issue
    // order: stable ranks)
#pragma unroll
    for (int j0 = 0; j0 < kSortIPT; j0 += kSlots) {
      uint32_t pm[kSlots];
#pragma unroll
      for (int q = 0; q < kSlots; ++q) {
        if (j0 + q >= kSortIPT) break;
        const uint32_t dj = static_cast<uint32_t>(key[j0 + q] >> shift) & kMask;
        atomicOr(&S.mm[q][warp][dj], 1u << lane);
      }
      __syncwarp();
#pragma unroll
      for (int q = 0; q < kSlots; ++q) {
        if (j0 + q >= kSortIPT) break;
        pm[q] = S.mm[q][warp][static_cast<uint32_t>(key[j0 + q] >> shift) & kMask];
      }
      __syncwarp();
#pragma unroll
      for (int q = 0; q < kSlots; ++q) {
        if (j0 + q >= kSortIPT) break;
        const uint32_t dj = static_cast<uint32_t>(key[j0 + q] >> shift) & kMask;
        rank[j0 + q] = 0;
        if (lane == 31u - __clz(pm[q])) {
          S.mm[q][warp][dj] = 0;
          atomicAdd(&S.hist[dj], __popc(pm[q]));
          rank[j0 + q] = atomicAdd(&S.wcnt[warp][dj], __popc(pm[q]));
        }
      }
#pragma unroll
      for (int q = 0; q < kSlots; ++q) {
        if (j0 + q >= kSortIPT) break;
        rank[j0 + q] = __shfl_sync(0xffffffffu, rank[j0 + q], 31 - __clz(pm[q])) + __popc(pm[q] & lanemask_lt());
      }
    }
    __syncthreads();
#pragma unroll
    for (int q = 0; q < kDPT; ++q) {
      tcount[q] = S.hist[d0 + q];
      st_relaxed_gpu_u64(my + q, pack_status(epoch, tile == 0 ? kPrefix : kAgg, tcount[q]));
    }
  } else {
    // 1. tile histogram first, published immediately (early aggregate for the successors)
#pragma unroll
    for (int j = 0; j < kSortIPT; ++j) atomicAdd(&S.hist[static_cast<uint32_t>(key[j] >> shift) & kMask], 1u);
    __syncthreads();
#pragma unroll
    for (int q = 0; q < kDPT; ++q) {
      tcount[q] = S.hist[d0 + q];
      st_relaxed_gpu_u64(my + q, pack_status(epoch, tile == 0 ? kPrefix : kAgg, tcount[q]));
    }
    // 2. stable warp-level ranking (element order == (j, lane) order inside the warp): match.any
    //    groups, the group leader reads and advances the warp's digit counter
#pragma unroll
    for (int j = 0; j < kSortIPT; ++j) {
      const uint32_t dj = static_cast<uint32_t>(key[j] >> shift) & kMask;
      const uint32_t peers = __match_any_sync(0xffffffffu, dj);
      const uint32_t leader = __ffs(peers) - 1;
      uint32_t before = 0;
      if (lane == leader) {
        before = S.wcnt[warp][dj];
        S.wcnt[warp][dj] = before + __popc(peers);
      }
      __syncwarp();   // order this step's counter updates before the next step's reads
      before = __shfl_sync(0xffffffffu, before, leader);
      rank[j] = before + __popc(peers & lanemask_lt());
    }
  }
  __syncthreads();
  // (a thread reads and rewrites only the counters of its own digits: no barrier needed here)
  // 3. per digit: the tile-local digit start (block scan of the tile counts), then every warp's
  //    counter becomes its tile-local scatter base for the digit (digit start + earlier warps)
  uint32_t tsum = 0;
#pragma unroll
  for (int q = 0; q < kDPT; ++q) tsum += tcount[q];
  const uint32_t inc = warp_inclusive_add(tsum);
  if (lane == 31) S.wsum[warp] = inc;
  __syncthreads();
  uint32_t dsq[kDPT];
  {
    uint32_t wpre = 0;
#pragma unroll
    for (int w = 0; w < kWarps; ++w) wpre += (w < static_cast<int>(warp)) ? S.wsum[w] : 0u;
    uint32_t ds = wpre + inc - tsum;
#pragma unroll
    for (int q = 0; q < kDPT; ++q) {
      dsq[q] = ds;
      uint32_t run = ds;
#pragma unroll
      for (int w = 0; w < kWarps; ++w) {
        const uint32_t c = S.wcnt[w][d0 + q];
        S.wcnt[w][d0 + q] = run;
        run += c;
      }
      ds += tcount[q];
    }
  }
  __syncthreads();
  // 4. scatter into SMEM in tile-sorted order (payload loaded here, after ranking); frees the
  //    key and rank registers before the look-back
#pragma unroll
  for (int j = 0; j < kSortIPT; ++j) {
    const uint64_t e = wbase + j * 32 + lane;
    const uint32_t dj = static_cast<uint32_t>(key[j] >> shift) & kMask;
    const uint32_t lp = S.wcnt[warp][dj] + rank[j];
    S.keys[lp] = key[j];
    if constexpr (kPay) S.idx[lp] = kFirst ? static_cast<uint32_t>(e) : (e < m ? idx_in[e] : 0u);
  }
  {
    // 5. decoupled look-back, kLookWindow predecessors per round trip, all digits of the thread
    //    in flight together
    uint32_t excl[kDPT];
#pragma unroll
    for (int q = 0; q < kDPT; ++q) excl[q] = 0;
    if (tile > 0) {
      long long p[kDPT];
      bool done[kDPT];
#pragma unroll
      for (int q = 0; q < kDPT; ++q) { p[q] = static_cast<long long>(tile) - 1; done[q] = false; }
      for (;;) {
        uint64_t sv[kDPT][kLookWindow];
#pragma unroll
        for (int q = 0; q < kDPT; ++q)
#pragma unroll
          for (int i = 0; i < kLookWindow; ++i)
            sv[q][i] = (!done[q] && p[q] - i >= 0)
                           ? ld_relaxed_gpu_u64(status + static_cast<uint64_t>(p[q] - i) * kBins + d0 + q)
                           : 0;
        bool all = true;
#pragma unroll
        for (int q = 0; q < kDPT; ++q) {
          if (done[q]) continue;
          int adv = 0;
          bool fin = false;
#pragma unroll
          for (int i = 0; i < kLookWindow; ++i) {
            if (fin || adv != i) continue;             // stop at the first not-ready / prefix word
            const uint32_t ep = static_cast<uint32_t>(sv[q][i] >> 34), kind = static_cast<uint32_t>(sv[q][i] >> 32) & 3u;
            if (ep != epoch || kind == 0) continue;     // not ready yet: retry from here
            excl[q] += static_cast<uint32_t>(sv[q][i]);
            ++adv;
            if (kind == kPrefix) fin = true;
          }
          if (fin) done[q] = true;
          else { p[q] -= adv; all = false; }
        }
        if (all) break;
      }
#pragma unroll
      for (int q = 0; q < kDPT; ++q) st_relaxed_gpu_u64(my + q, pack_status(epoch, kPrefix, excl[q] + tcount[q]));
    }
    // global position of tile-sorted slot i with digit d: i + (digit base + earlier tiles - digit start)
#pragma unroll
    for (int q = 0; q < kDPT; ++q) S.goff[d0 + q] = bases[d0 + q] + excl[q] - dsq[q];
  }
  __syncthreads();
  // 6. contiguous per-digit runs to global memory
  const uint32_t nvalid = static_cast<uint32_t>(min(static_cast<uint64_t>(kSortTile), m - tbase));
  if (nvalid == static_cast<uint32_t>(kSortTile)) {
    // full tile: unrolled in groups of 8, so the SMEM reads of 8 elements are in flight together
    // (a rolled loop serialises LDS key -> LDS goff -> STG per element)
#pragma unroll
    for (int j0 = 0; j0 < kSortIPT; j0 += 8) {
      K kk[8];
      uint32_t pp[8];
#pragma unroll
      for (int j = 0; j < 8 && j0 + j < kSortIPT; ++j) kk[j] = S.keys[(j0 + j) * kSortThreads + tid];
#pragma unroll
      for (int j = 0; j < 8 && j0 + j < kSortIPT; ++j)
        pp[j] = S.goff[static_cast<uint32_t>(kk[j] >> shift) & kMask] + (j0 + j) * kSortThreads + tid;
#pragma unroll
      for (int j = 0; j < 8 && j0 + j < kSortIPT; ++j) {
        keys_out[pp[j]] = kk[j];
        if constexpr (kPay) idx_out[pp[j]] = S.idx[(j0 + j) * kSortThreads + tid];
      }
    }
    return;
  }
  for (uint32_t i = tid; i < nvalid; i += kSortThreads) {
    const K k = S.keys[i];
    const uint32_t dk = static_cast<uint32_t>(k >> shift) & kMask;
    const uint32_t pos = S.goff[dk] + i;
    keys_out[pos] = k;
    if constexpr (kPay) idx_out[pos] = S.idx[i];
  }
}

// ---- single-pass exclusive scan (u32 or u64 input -> u64 output), decoupled look-back ----
constexpr int kScanThreads = 256, kScanIPT = 8, kScanTile = kScanThreads * kScanIPT;

template <typename T>
__global__ void __launch_bounds__(kScanThreads) k_scan(const T* __restrict__ in, uint64_t* out, uint64_t n,
                                                     unsigned long long* total, uint64_t* status, uint32_t epoch,
                                                     unsigned int* tile_counter) {
  __shared__ uint64_t wsum[kScanThreads / 32];
  __shared__ uint64_t s_excl;
  __shared__ uint32_t s_tile;
  const uint32_t tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  if (tid == 0) s_tile = atomicAdd(tile_counter, 1u);
  __syncthreads();
  const uint32_t tile = s_tile;
  const uint64_t base = static_cast<uint64_t>(tile) * kScanTile + static_cast<uint64_t>(tid) * kScanIPT;
  uint64_t v[kScanIPT];
  uint64_t tsum = 0;
#pragma unroll
  for (int j = 0; j < kScanIPT; ++j) {
    v[j] = (base + j < n) ? static_cast<uint64_t>(in[base + j]) : 0ULL;
    tsum += v[j];
  }
  const uint64_t inc = warp_inclusive_add64(tsum);
  if (lane == 31) wsum[warp] = inc;
  __syncthreads();
  uint64_t wpre = 0, tile_sum = 0;
#pragma unroll
  for (int w = 0; w < kScanThreads / 32; ++w) {
    wpre += (w < static_cast<int>(warp)) ? wsum[w] : 0ULL;
    tile_sum += wsum[w];
  }
  if (tid == 0) {
    // status layout per tile: [flag, aggregate, inclusive prefix]
    uint64_t* my = status + 3ULL * tile;
    uint64_t excl = 0;
    if (tile == 0) {
      st_volatile_u64(my + 2, tile_sum);
      __threadfence();
      st_volatile_u64(my, pack_status(epoch, kPrefix, 0));
    } else {
      st_volatile_u64(my + 1, tile_sum);
      __threadfence();
      st_volatile_u64(my, pack_status(epoch, kAgg, 0));
      long long p = static_cast<long long>(tile) - 1;
      while (p >= 0) {
        const uint64_t f = ld_volatile_u64(status + 3ULL * p);
        const uint32_t ep = static_cast<uint32_t>(f >> 34), kind = static_cast<uint32_t>(f >> 32) & 3u;
        if (ep != epoch || kind == 0) continue;
        __threadfence();
        if (kind == kPrefix) { excl += ld_volatile_u64(status + 3ULL * p + 2); break; }
        excl += ld_volatile_u64(status + 3ULL * p + 1);
        --p;
      }
      st_volatile_u64(my + 2, excl + tile_sum);
      __threadfence();
      st_volatile_u64(my, pack_status(epoch, kPrefix, 0));
    }
    s_excl = excl;
    if (total && (static_cast<uint64_t>(tile) + 1) * kScanTile >= n) *total = excl + tile_sum;
  }
  __syncthreads();
  uint64_t run = s_excl + wpre + inc - tsum;
#pragma unroll
  for (int j = 0; j < kScanIPT; ++j) {
    if (base + j < n) out[base + j] = run;
    run += v[j];
  }
}

}  // namespace

template <typename K>
static cudaError_t hist_impl(const K* keys, uint64_t m, uint32_t* hist, int nd, int bits, int num_sms,
                             cudaStream_t s) {
  cudaError_t e = cudaMemsetAsync(hist, 0, 8 * kBinStride * sizeof(uint32_t), s);
  if (e != cudaSuccess || m == 0) return e;
  while (reinterpret_cast<uintptr_t>(keys) & 15u) {   // 16-B loads: peel keys off a misaligned start
    k_hist<K><<<1, 32, 0, s>>>(keys, 1, static_cast<uint32_t>(nd), static_cast<uint32_t>(bits), hist);
    count_launch();
    ++keys;
    if (--m == 0) return cudaGetLastError();
  }
  constexpr uint64_t kPer = 16 / sizeof(K);
  uint64_t blocks = std::min<uint64_t>(static_cast<uint64_t>(num_sms) * 8, (m / kPer + 255) / 256 + 1);
  k_hist<K><<<static_cast<unsigned>(blocks), 256, 0, s>>>(keys, m, static_cast<uint32_t>(nd),
                                                          static_cast<uint32_t>(bits), hist);
  count_launch();
  return cudaGetLastError();
}
cudaError_t launch_hist(const uint64_t* keys, uint64_t m, uint32_t* hist, int nd, int bits, int num_sms,
                        cudaStream_t s) {
  return hist_impl<uint64_t>(keys, m, hist, nd, bits, num_sms, s);
}
cudaError_t launch_hist32(const uint32_t* keys, uint64_t m, uint32_t* hist, int nd, int bits, int num_sms,
                          cudaStream_t s) {
  return hist_impl<uint32_t>(keys, m, hist, nd, bits, num_sms, s);
}

// Tile shapes (keys per thread x 256 threads, CTAs per SM), measured on C5 in round 1 (16 keys
// with the early tile histogram and a look-back window of 4 was the fastest u64 shape among
// 8/12/16/20/24 keys, 9-bit digits, windows 1..16, spin back-off and match-aggregated histogram
// atomics; 24 keys x 3 CTAs the fastest u32 keys-only shape among 16/20/24/32; ballot-sliced
// peer masks and larger look-back windows were slower — tools/micro/sort_bench.cu):
//   payload passes (u64 key + u32 index): 16 keys, 3 CTAs/SM
//   keys-only u64 passes: 16 keys, 3 CTAs/SM; keys-only u32 passes: 24 keys, 3 CTAs/SM
constexpr int kIptPay = 16, kIptKeys = 16, kIptKeys32 = 24;
// u32 pass ranking by digit statistics: E = expected number of distinct digits among 32 keys
// (sum over bins of 1 - (1 - p_b)^32).  match.any slows down with many distinct values per warp,
// the shared-memory OR masks with many equal ones (same-address atomics serialise); measured with
// tools/micro/sort_bench (round 1): first pass over Zipf keys (E 28.6) 3.37 vs 4.59 ms.  Only the
// first pass sees the input order: after it, equal keys are adjacent and the warps' digits are
// far less diverse than E says (later passes: match 2.4-3.4 ms, OR masks 3.8-4.6 ms), so they
// keep match.any.  Threshold 24 on E.
int choose_rank_kind32(const uint32_t* hist, uint64_t m, bool first_pass) {
  if (m == 0) return kRankMatch;
  double e = 0;
  for (int b = 0; b < 256; ++b) e += 1.0 - std::pow(1.0 - static_cast<double>(hist[b]) / static_cast<double>(m), 32);
  return (first_pass && e >= 24.0) ? kRankOrMask : kRankMatch;
}

int sort_tile() { return kSortThreads * kIptPay; }
int sort_tile_keys() { return kSortThreads * kIptKeys; }
int sort_tile_keys32() { return kSortThreads * kIptKeys32; }

template <typename K, bool kFirst, bool kOrMatch, int IPT, int MINB, bool kPay>
static void launch_os(unsigned tiles, const K* keys_in, const uint32_t* idx_in, K* keys_out, uint32_t* idx_out,
                      uint64_t m, uint32_t shift, const uint32_t* bases, uint64_t* status, uint32_t epoch,
                      unsigned int* tile_counter, cudaStream_t s) {
  const auto k = &k_onesweep<K, kFirst, kOrMatch, IPT, MINB, kPay>;
  const size_t smem = sizeof(SortSmem<K, IPT, kPay, 256, kOrMatch ? 4 : 0>);
  cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, static_cast<int>(smem));
  k<<<tiles, kSortThreads, smem, s>>>(keys_in, idx_in, keys_out, idx_out, m, shift, bases, status, epoch,
                                      tile_counter);
}

#define BMR_OS_ARGS tiles, keys_in, idx_in, keys_out, idx_out, m, shift, bases, status, epoch, tile_counter, s
template <typename K>
static cudaError_t onesweep_impl(const K* keys_in, const uint32_t* idx_in, K* keys_out, uint32_t* idx_out, uint64_t m,
                                 int digit, int bits, const uint32_t* bases_all, uint64_t* status, uint32_t epoch,
                                 unsigned int* tile_counter, cudaStream_t s, int rank_kind) {
  if (m == 0) return cudaSuccess;
  const bool keys_only = idx_out == nullptr;
  if (bits != 8) return cudaErrorInvalidValue;
  if (sizeof(K) == 4 && !keys_only) return cudaErrorInvalidValue;
  const uint64_t tile = sizeof(K) == 4 ? sort_tile_keys32() : keys_only ? sort_tile_keys() : sort_tile();
  const unsigned tiles = static_cast<unsigned>((m + tile - 1) / tile);
  cudaError_t e = cudaMemsetAsync(tile_counter, 0, sizeof(unsigned int), s);
  if (e != cudaSuccess) return e;
  const uint32_t shift = static_cast<uint32_t>(bits * digit);
  const uint32_t* bases = bases_all + kBinStride * digit;
  const bool orm = rank_kind == kRankOrMask;
  if constexpr (sizeof(K) == 4) {
    if (orm) launch_os<K, false, true, kIptKeys32, 3, false>(BMR_OS_ARGS);
    else launch_os<K, false, false, kIptKeys32, 3, false>(BMR_OS_ARGS);
  } else if (keys_only) {
    if (orm) launch_os<K, false, true, kIptKeys, 3, false>(BMR_OS_ARGS);
    else launch_os<K, false, false, kIptKeys, 3, false>(BMR_OS_ARGS);
  } else if (idx_in == nullptr) {   // first payload pass: identity permutation
    launch_os<K, true, false, kIptPay, 3, true>(BMR_OS_ARGS);
  } else {
    launch_os<K, false, false, kIptPay, 3, true>(BMR_OS_ARGS);
  }
  count_launch();
  return cudaGetLastError();
}
#undef BMR_OS_ARGS

cudaError_t launch_onesweep(const uint64_t* keys_in, const uint32_t* idx_in, uint64_t* keys_out, uint32_t* idx_out,
                            uint64_t m, int digit, int bits, const uint32_t* bases_all, uint64_t* status,
                            uint32_t epoch, unsigned int* tile_counter, cudaStream_t s, int rank_kind) {
  return onesweep_impl<uint64_t>(keys_in, idx_in, keys_out, idx_out, m, digit, bits, bases_all, status, epoch,
                                 tile_counter, s, rank_kind);
}
cudaError_t launch_onesweep32(const uint32_t* keys_in, uint32_t* keys_out, uint64_t m, int digit, int bits,
                              const uint32_t* bases_all, uint64_t* status, uint32_t epoch,
                              unsigned int* tile_counter, cudaStream_t s, int rank_kind) {
  return onesweep_impl<uint32_t>(keys_in, nullptr, keys_out, nullptr, m, digit, bits, bases_all, status, epoch,
                                 tile_counter, s, rank_kind);
}

template <typename T>
static cudaError_t scan_impl(const T* in, uint64_t* out, uint64_t n, unsigned long long* total, uint64_t* status,
                             uint32_t epoch, unsigned int* tile_counter, cudaStream_t s) {
  if (n == 0) {
    if (total) return cudaMemsetAsync(total, 0, sizeof(unsigned long long), s);
    return cudaSuccess;
  }
  cudaError_t e = cudaMemsetAsync(tile_counter, 0, sizeof(unsigned int), s);
  if (e != cudaSuccess) return e;
  const uint64_t tiles = (n + kScanTile - 1) / kScanTile;
  k_scan<T><<<static_cast<unsigned>(tiles), kScanThreads, 0, s>>>(in, out, n, total, status, epoch, tile_counter);
  count_launch();
  return cudaGetLastError();
}

cudaError_t launch_scan_u64(const uint64_t* in, uint64_t* out, uint64_t n, unsigned long long* total,
                            uint64_t* status, uint32_t epoch, unsigned int* tile_counter, cudaStream_t s) {
  return scan_impl<uint64_t>(in, out, n, total, status, epoch, tile_counter, s);
}
cudaError_t launch_scan_u32to64(const uint32_t* in, uint64_t* out, uint64_t n, unsigned long long* total,
                                uint64_t* status, uint32_t epoch, unsigned int* tile_counter, cudaStream_t s) {
  return scan_impl<uint32_t>(in, out, n, total, status, epoch, tile_counter, s);
}

}  // namespace bmr
