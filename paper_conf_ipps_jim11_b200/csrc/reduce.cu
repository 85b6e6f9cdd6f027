// reduce.cu — group-by-key, part 2 (segment boundaries) and the Reduce phase
// with output assembly (a9).
//
// Segments: after the radix sort equal sort keys are adjacent.  head[i] = (i == 0) ||
// key[i] != key[i-1].  For hashed keys (top bit set) equal hashes are verified byte-for-byte
// against the neighbouring pair (C-3 #13: distinct keys must never merge); a mismatch is
// counted in DevState::collisions and the host re-sorts with a fresh hash (slow path).
//
// Reduce (§IV-C, §IV-E): TR = one thread per key set, BR = a block per key
// set; the paper found TR better for WC's 10,000s of small key sets and BR better for KM's
// dozens of large ones.  B200 re-derivation, segment-size aware:
//   * small segments (<= kSmall pairs): one warp per segment, lanes stride the segment and the
//     warp reduces with shuffles (TR's parallelism across key sets, without per-thread serial
//     loops over Zipf-heavy sets);
//   * large segments: split into kLargeTile-pair work items appended to a work list; persistent
//     blocks reduce one item each and combine with one global atomic per item (BR).
// KM partial sums are fp32 over <= 32 values per lane, combined in fp64 (north_star: "fp32 on
// GPU"; tolerance derivation in DESIGN.md).
#include <algorithm>

#include "common.cuh"

#ifndef BMR_XTAB_BPS
#define BMR_XTAB_BPS 256   // table extraction: blocks per SM (C5: 8 -> 1.21 ms, 64 -> 0.98, 512 -> 0.94; short-lived blocks keep more loads in flight)
#endif
#ifndef BMR_XTAB_UNROLL
#define BMR_XTAB_UNROLL 1   // (2 and 4 in-flight loads per thread measured no better: 1.0 vs 1.0 / 1.34 ms)
#endif

namespace bmr {
namespace {

constexpr int kSegThreads = 256, kSegIPT = 16, kSegTile = kSegThreads * kSegIPT;
constexpr uint64_t kSmallWC = 4096, kSmallKM = 1024;
constexpr uint64_t kLargeTile = 8192;

__device__ __forceinline__ uint64_t warp_sum_u64(uint64_t v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  return v;
}

// 8 key bytes starting at p (little-endian); reads only the aligned 8-byte words that hold
// bytes [p, p + need), need <= 8, so it never touches a word outside the key's own words.

// Byte equality of two keys given as kref = (address << 16) | length.
__device__ bool key_bytes_equal(uint64_t ka, uint64_t kb) {
  const uint32_t la = static_cast<uint32_t>(ka & 0xFFFF), lb = static_cast<uint32_t>(kb & 0xFFFF);
  if (la != lb) return false;
  const uint8_t* pa = reinterpret_cast<const uint8_t*>(ka >> 16);
  const uint8_t* pb = reinterpret_cast<const uint8_t*>(kb >> 16);
  // no early exit inside the loop: equal keys (the common case) read every chunk anyway, and
  // independent iterations let the loads of several chunks be in flight together
  uint64_t diff = 0;
#pragma unroll 4
  for (uint32_t i = 0; i < la; i += 8) {
    const uint32_t need = min(8u, la - i);
    const uint64_t mask = need == 8 ? ~0ULL : ((1ULL << (8 * need)) - 1ULL);
    diff |= (load8(pa + i, need) ^ load8(pb + i, need)) & mask;
  }
  return diff == 0;
}

// Each warp owns 512 consecutive sorted positions (16 steps of 32 lanes: coalesced loads);
// a lane compares its key with the previous position's key (shuffle from the previous lane).
constexpr int kSegWarp = 32 * kSegIPT;   // positions per warp

template <bool kVerify, typename K = uint64_t>
__global__ void __launch_bounds__(kSegThreads) k_seg_count(const K* __restrict__ sk,
                                                         const uint32_t* __restrict__ perm,
                                                         const uint64_t* __restrict__ kref, uint64_t m,
                                                         uint32_t* counts, DevState* st, uint64_t hbit,
                                                         uint64_t kmask) {
  __shared__ uint32_t red[kSegThreads / 32];
  const uint32_t lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const uint64_t wbase = static_cast<uint64_t>(blockIdx.x) * kSegTile + static_cast<uint64_t>(warp) * kSegWarp;
  uint32_t heads = 0, coll = 0;
  K carry_k = (wbase > 0 && wbase - 1 < m) ? sk[wbase - 1] : 0;            // key before this step
  uint64_t carry_r = 0;                                                     // its kref (if loaded)
  bool carry_has_r = false;
#pragma unroll 4
  for (int j = 0; j < kSegIPT; ++j) {
    const uint64_t i = wbase + static_cast<uint64_t>(j) * 32 + lane;
    const bool valid = i < m;
    const K k = valid ? sk[i] : 0;
    K prev = __shfl_up_sync(0xffffffffu, k, 1);
    if (lane == 0) prev = carry_k;
    const bool head = valid && (i == 0 || ((k ^ prev) & static_cast<K>(kmask)) != 0);
    heads += head ? 1u : 0u;
    carry_k = __shfl_sync(0xffffffffu, k, 31);
    if constexpr (kVerify) {
      // byte verification of equal hashed keys (C-3 #13): adjacent pairs inside an equal-hash run
      const bool hashed_run = valid && (k & hbit) && !head;
      const bool need_r = valid && (k & hbit);
      const unsigned any = __ballot_sync(0xffffffffu, need_r);
      uint64_t r = 0;
      if (any) {
        if (need_r) r = kref[perm[i]];
        uint64_t rp = __shfl_up_sync(0xffffffffu, r, 1);
        if (lane == 0) rp = carry_has_r ? carry_r : ((hashed_run && i > 0) ? kref[perm[i - 1]] : 0);
        // keys of <= 16 bytes: every lane reads its OWN key bytes once and compares them with
        // the previous lane's by shuffles (one random read per element instead of two; C5's long
        // words; longer keys such as C4's URLs keep the two-pointer comparison)
        const uint32_t len = static_cast<uint32_t>(r & 0xFFFF);
        uint64_t b[2] = {0, 0};
        if (need_r && len <= 16) {
          const uint8_t* kp = reinterpret_cast<const uint8_t*>(r >> 16);
#pragma unroll
          for (int q = 0; q < 2; ++q) {
            const uint32_t off = 8u * q;
            if (off < len) {
              const uint32_t need = min(8u, len - off);
              b[q] = load8(kp + off, need) & (need == 8 ? ~0ULL : ((1ULL << (8 * need)) - 1ULL));
            }
          }
        }
        uint64_t pb[2];
#pragma unroll
        for (int q = 0; q < 2; ++q) pb[q] = __shfl_up_sync(0xffffffffu, b[q], 1);
        const uint32_t plen = static_cast<uint32_t>(rp & 0xFFFF);
        if (hashed_run) {
          bool eq;
          if (lane != 0 && len <= 16 && plen <= 16) eq = len == plen && b[0] == pb[0] && b[1] == pb[1];
          else eq = key_bytes_equal(r, rp);
          if (!eq) ++coll;
        }
      }
      carry_r = __shfl_sync(0xffffffffu, r, 31);
      carry_has_r = __shfl_sync(0xffffffffu, need_r ? 1u : 0u, 31) != 0;
    }
  }
  if (coll) atomicAdd(&st->collisions, coll);
  const uint32_t w = __reduce_add_sync(0xffffffffu, heads);
  if (lane == 0) red[warp] = w;
  __syncthreads();
  if (threadIdx.x == 0) {
    uint32_t t = 0;
    for (int q = 0; q < kSegThreads / 32; ++q) t += red[q];
    counts[blockIdx.x] = t;
  }
}

template <typename K = uint64_t>
__global__ void __launch_bounds__(kSegThreads) k_seg_write(const K* __restrict__ sk, uint64_t m,
                                                         const uint64_t* __restrict__ tile_base,
                                                         uint64_t* seg_start, uint64_t kmask) {
  __shared__ uint32_t wsum[kSegThreads / 32];
  const uint32_t lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const uint64_t wbase = static_cast<uint64_t>(blockIdx.x) * kSegTile + static_cast<uint64_t>(warp) * kSegWarp;
  // pass 1: heads of this warp's 512 positions (bitmask per step kept in registers)
  uint32_t hm[kSegIPT];
  uint32_t wcount = 0;
  K carry_k = (wbase > 0 && wbase - 1 < m) ? sk[wbase - 1] : 0;
#pragma unroll
  for (int j = 0; j < kSegIPT; ++j) {
    const uint64_t i = wbase + static_cast<uint64_t>(j) * 32 + lane;
    const bool valid = i < m;
    const K k = valid ? sk[i] : 0;
    K prev = __shfl_up_sync(0xffffffffu, k, 1);
    if (lane == 0) prev = carry_k;
    hm[j] = __ballot_sync(0xffffffffu, valid && (i == 0 || ((k ^ prev) & static_cast<K>(kmask)) != 0));
    wcount += __popc(hm[j]);
    carry_k = __shfl_sync(0xffffffffu, k, 31);
  }
  if (lane == 0) wsum[warp] = wcount;
  __syncthreads();
  uint32_t wpre = 0, tot = 0;
  for (int w = 0; w < kSegThreads / 32; ++w) {
    wpre += (w < static_cast<int>(warp)) ? wsum[w] : 0u;
    tot += wsum[w];
  }
  uint64_t r = tile_base[blockIdx.x] + wpre;
#pragma unroll
  for (int j = 0; j < kSegIPT; ++j) {
    const uint64_t i = wbase + static_cast<uint64_t>(j) * 32 + lane;
    if ((hm[j] >> lane) & 1u) seg_start[r + __popc(hm[j] & lanemask_lt())] = i;
    r += __popc(hm[j]);
  }
  const uint64_t tile_end = static_cast<uint64_t>(blockIdx.x + 1) * kSegTile;
  if (threadIdx.x == 0 && tile_end >= m) seg_start[tile_base[blockIdx.x] + tot] = m;  // sentinel S -> m
}

// ---------------------------------------------------------------- WordCount reduce (u64 sums)
// Segment-size-aware WC reduce.  A warp takes 32 consecutive segments: tiny ones (<= 32 pairs,
// the long tail of the Zipf vocabulary) are summed by their own lane (TR, L181); medium ones
// (<= kSmallWC) by the whole warp in turn; large ones become kLargeTile work items for the
// block-level kernel below (BR).
// Value of sorted position i: gathered through perm (u32 / u64 value arrays) or, for packed WC
// pairs, read from the top 16 bits of the sorted 64-bit word itself (no gather at all).
template <int kMode>   // 0: u32 v[perm[i]], 1: u64 v[perm[i]], 2: packed sk[i] >> 48
__device__ __forceinline__ uint64_t val_at(const uint64_t* __restrict__ sk, const uint32_t* __restrict__ perm,
                                           const void* __restrict__ v, uint64_t i) {
  if constexpr (kMode == 2) return sk[i] >> 48;
  else if constexpr (kMode == 1) return static_cast<const uint64_t*>(v)[perm[i]];
  else return static_cast<const uint32_t*>(v)[perm[i]];
}

// Segment-size-aware WC reduce.  A warp takes 32 consecutive
// segments: tiny ones (<= 32 pairs, the long tail of the Zipf vocabulary) are summed by their
// own lane (TR, L181); medium ones (<= kSmallWC) by the whole warp in turn; large ones become
// kLargeTile work items for the block-level kernel below (BR).
template <int kMode>
__global__ void k_reduce_wc_small(const uint64_t* __restrict__ seg, uint64_t nseg, const uint64_t* __restrict__ sk,
                                  const uint32_t* __restrict__ perm, const void* __restrict__ v, uint64_t* counts,
                                  uint64_t* worklist, DevState* st) {
  const uint64_t gw = (blockIdx.x * static_cast<uint64_t>(blockDim.x) + threadIdx.x) >> 5;
  const uint64_t nw = (static_cast<uint64_t>(gridDim.x) * blockDim.x) >> 5;
  const uint32_t lane = threadIdx.x & 31;
  for (uint64_t s0 = gw * 32; s0 < nseg; s0 += nw * 32) {
    const uint64_t s = s0 + lane;
    uint64_t a = 0, b = 0;
    if (s < nseg) { a = seg[s]; b = seg[s + 1]; }
    const uint64_t size = b - a;
    if (s < nseg && size <= 32) {                       // thread per key set
      uint64_t sum = 0;
      for (uint64_t i = a; i < b; ++i) sum += val_at<kMode>(sk, perm, v, i);
      counts[s] = sum;
    } else if (s < nseg && size > kSmallWC) {           // block-level work items
      counts[s] = 0;
      const uint64_t nt = (size + kLargeTile - 1) / kLargeTile;
      const uint64_t at = atomicAdd(&st->large_items, static_cast<unsigned long long>(nt));
      for (uint64_t t = 0; t < nt; ++t) worklist[at + t] = (s << 24) | t;
    }
    uint32_t med = __ballot_sync(0xffffffffu, s < nseg && size > 32 && size <= kSmallWC);
    while (med) {                                        // warp per medium key set
      const int L = __ffs(med) - 1;
      med &= med - 1;
      const uint64_t ma = __shfl_sync(0xffffffffu, a, L), mb = __shfl_sync(0xffffffffu, b, L);
      uint64_t sum = 0;
#pragma unroll 4
      for (uint64_t i = ma + lane; i < mb; i += 32) sum += val_at<kMode>(sk, perm, v, i);
      sum = warp_sum_u64(sum);
      if (lane == 0) counts[s0 + L] = sum;
    }
  }
}

template <int kMode>
__global__ void __launch_bounds__(256) k_reduce_wc_large(const uint64_t* __restrict__ seg,
                                                       const uint64_t* __restrict__ sk,
                                                       const uint32_t* __restrict__ perm, const void* __restrict__ v,
                                                       uint64_t* counts, const uint64_t* __restrict__ worklist,
                                                       DevState* st) {
  __shared__ unsigned long long item;
  __shared__ uint64_t red[8];
  const unsigned long long nitems = st->large_items;
  for (;;) {
    if (threadIdx.x == 0) item = atomicAdd(&st->large_done, 1ULL);
    __syncthreads();
    const unsigned long long it = item;
    if (it >= nitems) break;
    const uint64_t w = worklist[it], s = w >> 24, t = w & 0xFFFFFF;
    const uint64_t a = seg[s] + t * kLargeTile, b = min(seg[s + 1], a + kLargeTile);
    uint64_t sum = 0;
#pragma unroll 8
    for (uint64_t i = a + threadIdx.x; i < b; i += blockDim.x) sum += val_at<kMode>(sk, perm, v, i);
    sum = warp_sum_u64(sum);
    if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = sum;
    __syncthreads();
    if (threadIdx.x == 0) {
      uint64_t tot = 0;
      for (int i = 0; i < 8; ++i) tot += red[i];
      atomicAdd(reinterpret_cast<unsigned long long*>(&counts[s]), static_cast<unsigned long long>(tot));
    }
    __syncthreads();
  }
}

// ---------------------------------------------------------------- KMeans reduce
__device__ __forceinline__ void load_point(const uint8_t* v, uint32_t p, float (&x)[8]) {
  const float4* q = reinterpret_cast<const float4*>(v + static_cast<uint64_t>(p) * 32);
  const float4 a = q[0], b = q[1];
  x[0] = a.x; x[1] = a.y; x[2] = a.z; x[3] = a.w; x[4] = b.x; x[5] = b.y; x[6] = b.z; x[7] = b.w;
}

__global__ void k_reduce_km_small(const uint64_t* __restrict__ seg, uint64_t nseg, const uint64_t* __restrict__ sk,
                                  const uint32_t* __restrict__ perm, const uint8_t* __restrict__ v, double* sums,
                                  unsigned long long* cnts, uint32_t k, uint64_t* worklist, DevState* st) {
  const uint64_t gw = (blockIdx.x * static_cast<uint64_t>(blockDim.x) + threadIdx.x) >> 5;
  const uint64_t nw = (static_cast<uint64_t>(gridDim.x) * blockDim.x) >> 5;
  const uint32_t lane = threadIdx.x & 31;
  for (uint64_t s = gw; s < nseg; s += nw) {
    const uint64_t a = seg[s], b = seg[s + 1], size = b - a;
    const uint64_t cid = sk[a];
    if (cid >= k) continue;
    if (size <= kSmallKM) {
      float acc[8] = {0, 0, 0, 0, 0, 0, 0, 0};
      for (uint64_t i = a + lane; i < b; i += 32) {   // <= 32 fp32 adds per lane
        float x[8];
        load_point(v, perm[i], x);
#pragma unroll
        for (int t = 0; t < 8; ++t) acc[t] = __fadd_rn(acc[t], x[t]);
      }
#pragma unroll
      for (int t = 0; t < 8; ++t) {
        double d = static_cast<double>(acc[t]);
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) d += __shfl_xor_sync(0xffffffffu, d, o);
        if (lane == 0) atomicAdd(&sums[cid * 8 + t], d);
      }
      if (lane == 0) atomicAdd(&cnts[cid], static_cast<unsigned long long>(size));
    } else if (lane == 0) {
      atomicAdd(&cnts[cid], static_cast<unsigned long long>(size));
      const uint64_t nt = (size + kLargeTile - 1) / kLargeTile;
      const uint64_t at = atomicAdd(&st->large_items, static_cast<unsigned long long>(nt));
      for (uint64_t t = 0; t < nt; ++t) worklist[at + t] = (s << 24) | t;
    }
  }
}

// Large cluster segments in 8192-position work items (block reduce, BR — PAPER.md L181, L286:
// KM-BR gains from staging its input in shared memory): the block stages the item's points in
// SMEM, kKmStage at a time, with asynchronous 16-B gathers (cp.async: the whole sub-tile's random
// reads are in flight together instead of one dependent load chain per thread), then every thread
// adds its points from SMEM (<= 32 fp32 adds per thread and item, reading 5) and the
// block combines in fp64.
constexpr int kKmStage = 1024;   // points per staged sub-tile (32 KB)
__device__ __forceinline__ void cp_async16(void* sdst, const void* gsrc) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(static_cast<uint32_t>(__cvta_generic_to_shared(sdst))),
               "l"(gsrc)
               : "memory");
}
__global__ void __launch_bounds__(256) k_reduce_km_large(const uint64_t* __restrict__ seg,
                                                       const uint64_t* __restrict__ sk,
                                                       const uint32_t* __restrict__ perm,
                                                       const uint8_t* __restrict__ v, double* sums,
                                                       const uint64_t* __restrict__ worklist, DevState* st) {
  extern __shared__ __align__(16) float4 stg[];   // kKmStage x 2 float4
  __shared__ unsigned long long item;
  __shared__ double red[8][8];
  const unsigned long long nitems = st->large_items;
  const uint32_t lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  for (;;) {
    if (threadIdx.x == 0) item = atomicAdd(&st->large_done, 1ULL);
    __syncthreads();
    const unsigned long long it = item;
    if (it >= nitems) break;
    const uint64_t w = worklist[it], s = w >> 24, t = w & 0xFFFFFF;
    const uint64_t a = seg[s] + t * kLargeTile, b = min(seg[s + 1], a + kLargeTile);
    const uint64_t cid = sk[seg[s]];
    float acc[8] = {0, 0, 0, 0, 0, 0, 0, 0};           // kLargeTile / 256 = 32 fp32 adds per thread
    for (uint64_t sub = a; sub < b; sub += kKmStage) {
      const uint32_t n = static_cast<uint32_t>(min(static_cast<uint64_t>(kKmStage), b - sub));
      for (uint32_t i = threadIdx.x; i < 2 * n; i += blockDim.x) {   // two 16-B halves per point
        const uint8_t* src = v + static_cast<uint64_t>(perm[sub + (i >> 1)]) * 32 + (i & 1u) * 16;
        cp_async16(&stg[i], src);
      }
      asm volatile("cp.async.commit_group;\n\tcp.async.wait_group 0;" ::: "memory");
      __syncthreads();
      for (uint32_t i = threadIdx.x; i < n; i += blockDim.x) {
        const float4 p0 = stg[2 * i], p1 = stg[2 * i + 1];
        acc[0] = __fadd_rn(acc[0], p0.x); acc[1] = __fadd_rn(acc[1], p0.y);
        acc[2] = __fadd_rn(acc[2], p0.z); acc[3] = __fadd_rn(acc[3], p0.w);
        acc[4] = __fadd_rn(acc[4], p1.x); acc[5] = __fadd_rn(acc[5], p1.y);
        acc[6] = __fadd_rn(acc[6], p1.z); acc[7] = __fadd_rn(acc[7], p1.w);
      }
      __syncthreads();   // the next sub-tile overwrites the stage
    }
#pragma unroll
    for (int q = 0; q < 8; ++q) {
      double d = static_cast<double>(acc[q]);
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) d += __shfl_xor_sync(0xffffffffu, d, o);
      if (lane == 0) red[warp][q] = d;
    }
    __syncthreads();
    if (threadIdx.x < 8) {
      double d = 0;
      for (int ww = 0; ww < 8; ++ww) d += red[ww][threadIdx.x];
      atomicAdd(&sums[cid * 8 + threadIdx.x], d);
    }
    __syncthreads();
  }
}

__global__ void k_km_finalize(const double* sums, const unsigned long long* cnts, const float* cent, uint32_t k,
                              const uint32_t* list, uint32_t nlist, uint8_t* vals, uint64_t* val_off, uint8_t* keys,
                              uint64_t* key_off) {
  const uint32_t n = list ? nlist : k;
  const uint32_t o = blockIdx.x * blockDim.x + threadIdx.x;   // output slot
  if (o > n) return;
  if (o == n) { val_off[n] = 40ULL * n; key_off[n] = 4ULL * n; return; }
  const uint32_t j = list ? list[o] : o;
  const unsigned long long c = cnts[j];
  float* out = reinterpret_cast<float*>(vals + 40ULL * o);
  for (int t = 0; t < 8; ++t)
    out[t] = c ? static_cast<float>(__ddiv_rn(sums[j * 8 + t], static_cast<double>(c))) : cent[j * 8 + t];
  *reinterpret_cast<unsigned long long*>(vals + 40ULL * o + 32) = c;
  *reinterpret_cast<uint32_t*>(keys + 4ULL * o) = j;
  val_off[o] = 40ULL * o;
  key_off[o] = 4ULL * o;
}

// ---------------------------------------------------------------- output assembly
__global__ void k_key_lengths(const uint64_t* seg, uint64_t nseg, const uint32_t* perm, const uint64_t* kref,
                              uint64_t* lens) {
  const uint64_t s = blockIdx.x * static_cast<uint64_t>(blockDim.x) + threadIdx.x;
  if (s < nseg) lens[s] = kref[seg ? perm[seg[s]] : s] & 0xFFFF;   // (seg == nullptr: kref is the key list)
}
__global__ void k_key_copy(const uint64_t* seg, uint64_t nseg, const uint32_t* perm, const uint64_t* kref,
                           const uint64_t* key_off, uint8_t* keys) {
  // one thread per key resolves its reference (seg -> perm -> kref: three dependent random loads,
  // 32 keys of a warp in flight together), then the warp copies its 32 keys one after another
  // with the lanes on consecutive bytes (a warp per key serialised the three loads per key:
  // C4 1.7 ms per step, ncu launch list round 1)
  const uint64_t s = blockIdx.x * static_cast<uint64_t>(blockDim.x) + threadIdx.x;
  const uint32_t lane = threadIdx.x & 31;
  uint64_t kr = 0, d = 0;
  if (s < nseg) {
    kr = kref[seg ? perm[seg[s]] : s];   // (seg == nullptr: kref is the key list)
    d = key_off[s];
  }
#pragma unroll 4
  for (int q = 0; q < 32; ++q) {
    const uint64_t kq = __shfl_sync(0xffffffffu, kr, q), dq = __shfl_sync(0xffffffffu, d, q);
    const uint8_t* src = reinterpret_cast<const uint8_t*>(kq >> 16);
    const uint32_t len = static_cast<uint32_t>(kq & 0xFFFF);
    for (uint32_t i = lane; i < len; i += 32) keys[dq + i] = src[i];
  }
}
// WC exact stream: the key is the record (value 1) -> count = segment length, key bytes decoded
// from the key itself.
__global__ void k_seg_lengths(const uint64_t* seg, uint64_t nseg, uint64_t* out) {
  const uint64_t s = blockIdx.x * static_cast<uint64_t>(blockDim.x) + threadIdx.x;
  if (s < nseg) out[s] = seg[s + 1] - seg[s];
}
template <typename K>
__global__ void k_key_lengths_exact(const uint64_t* seg, uint64_t nseg, const K* sk, uint64_t* lens) {
  const uint64_t s = blockIdx.x * static_cast<uint64_t>(blockDim.x) + threadIdx.x;
  if (s >= nseg) return;
  uint32_t len;
  exact_key_bytes(sk[seg[s]], len);
  lens[s] = len;
}
template <typename K>
__global__ void k_key_decode(const uint64_t* seg, uint64_t nseg, const K* sk, const uint64_t* key_off,
                             uint8_t* keys) {
  const uint64_t s = blockIdx.x * static_cast<uint64_t>(blockDim.x) + threadIdx.x;
  if (s >= nseg) return;
  uint32_t len;
  const uint64_t b = exact_key_bytes(sk[seg[s]], len);
  uint8_t* dst = keys + key_off[s];
  for (uint32_t i = 0; i < len; ++i) dst[i] = static_cast<uint8_t>(b >> (8 * i));
}
// WC combiner partials (f-1), after their own sort + segments: the summed count of every partial
// key, then a binary search of the key among the exact stream's segment keys (ascending).  Found:
// midx = that segment (its count is augmented in mr_reduce); not found: the key is appended to
// the extra list (keys that only the combiner saw).
__global__ void k_comb_merge(const uint64_t* __restrict__ segp, uint64_t nsegp, const uint64_t* __restrict__ skp,
                             const uint64_t* __restrict__ sega, uint64_t nsega, const uint32_t* __restrict__ skx,
                             uint32_t* midx, uint64_t* psum, uint32_t* xkeys, uint64_t* xcounts,
                             unsigned long long* nextra) {   // nextra[1]: words absorbed (sum of counts)
  const uint64_t s = blockIdx.x * static_cast<uint64_t>(blockDim.x) + threadIdx.x;
  const bool live = s < nsegp;
  uint64_t sum = 0;
  uint32_t key = 0;
  bool extra = false;
  if (live) {
    const uint64_t a = segp[s], b = segp[s + 1];
    key = static_cast<uint32_t>(skp[a] & 0x3FFFFFFFULL);
    for (uint64_t i = a; i < b; ++i) sum += skp[i] >> 32;
    uint64_t lo = 0, hi = nsega;   // first exact segment with key >= `key`
    while (lo < hi) {
      const uint64_t mid = (lo + hi) >> 1;
      if (skx[sega[mid]] < key) lo = mid + 1; else hi = mid;
    }
    if (lo < nsega && skx[sega[lo]] == key) {
      midx[s] = static_cast<uint32_t>(lo);
      psum[s] = sum;
    } else {
      midx[s] = 0xFFFFFFFFu;
      extra = true;
    }
  }
  // warp-aggregated global atomics (per-thread ones serialised on these two addresses)
  const uint32_t lane = threadIdx.x & 31;
  const uint64_t wsum = warp_inclusive_add64(sum);
  const uint32_t me = __ballot_sync(0xffffffffu, extra);
  unsigned long long base = 0;
  if (lane == 31 && wsum) atomicAdd(nextra + 1, static_cast<unsigned long long>(wsum));   // (the warp's total)
  if (lane == 0 && me) base = atomicAdd(nextra, static_cast<unsigned long long>(__popc(me)));
  base = __shfl_sync(0xffffffffu, base, 0);
  if (extra) {
    const unsigned long long e = base + __popc(me & lanemask_lt());
    xkeys[e] = key;
    xcounts[e] = sum;
  }
}
__global__ void k_comb_add(const uint32_t* midx, const uint64_t* psum, uint64_t nsegp, uint64_t* counts) {
  const uint64_t s = blockIdx.x * static_cast<uint64_t>(blockDim.x) + threadIdx.x;
  if (s < nsegp && midx[s] != 0xFFFFFFFFu) counts[midx[s]] += psum[s];   // distinct keys: distinct targets
}
__global__ void k_key_lengths_list32(const uint32_t* keys, uint64_t n, uint64_t* lens) {
  const uint64_t s = blockIdx.x * static_cast<uint64_t>(blockDim.x) + threadIdx.x;
  if (s >= n) return;
  uint32_t len;
  exact_key_bytes(keys[s], len);
  lens[s] = len;
}
__global__ void k_key_decode_list32(const uint32_t* keys, uint64_t n, const uint64_t* key_off, uint8_t* out) {
  const uint64_t s = blockIdx.x * static_cast<uint64_t>(blockDim.x) + threadIdx.x;
  if (s >= n) return;
  uint32_t len;
  const uint64_t b = exact_key_bytes(keys[s], len);
  uint8_t* dst = out + key_off[s];
  for (uint32_t i = 0; i < len; ++i) dst[i] = static_cast<uint8_t>(b >> (8 * i));
}
// keys at the segment heads of a sorted keys-only stream (SM per-line output: unique record starts)
__global__ void k_seg_keys(const uint64_t* seg, uint64_t nseg, const uint64_t* sk, uint64_t* out) {
  const uint64_t s = blockIdx.x * static_cast<uint64_t>(blockDim.x) + threadIdx.x;
  if (s < nseg) out[s] = sk[seg[s]];
}
__global__ void k_gather_u64(const uint32_t* perm, const uint64_t* v, uint64_t m, uint64_t* out) {
  const uint64_t i = blockIdx.x * static_cast<uint64_t>(blockDim.x) + threadIdx.x;
  if (i < m) out[i] = v[perm[i]];
}
__global__ void k_offsets_scaled(const uint64_t* seg, uint64_t nseg, uint64_t scale, uint64_t* out) {
  const uint64_t s = blockIdx.x * static_cast<uint64_t>(blockDim.x) + threadIdx.x;
  if (s <= nseg) out[s] = seg[s] * scale;
}
__global__ void k_iota_scaled(uint64_t n, uint64_t scale, uint64_t* out) {
  const uint64_t s = blockIdx.x * static_cast<uint64_t>(blockDim.x) + threadIdx.x;
  if (s <= n) out[s] = s * scale;
}
__global__ void k_rehash(uint64_t* h, const uint64_t* kref, uint64_t m, uint64_t seed) {
  const uint64_t i = blockIdx.x * static_cast<uint64_t>(blockDim.x) + threadIdx.x;
  if (i >= m) return;
  const uint64_t kr = kref[i];
  if (kr == 0) { h[i] = sentinel_of(64); return; }   // flush filler
  h[i] = key_of_bytes(reinterpret_cast<const uint8_t*>(kr >> 16), static_cast<uint32_t>(kr & 0xFFFF), seed, false, 64);
}

inline unsigned blocks_for(uint64_t n, unsigned t) { return static_cast<unsigned>((n + t - 1) / t); }

}  // namespace

cudaError_t launch_seg_count(const uint64_t* skeys, const uint32_t* perm, const uint64_t* kref, uint64_t m,
                             uint32_t* counts, DevState* st, uint32_t key_bits, uint64_t kmask, cudaStream_t s) {
  if (m == 0) return cudaSuccess;
  if (kref)
    k_seg_count<true><<<blocks_for(m, kSegTile), kSegThreads, 0, s>>>(skeys, perm, kref, m, counts, st,
                                                                      hashed_bit(key_bits), kmask);
  else   // keys-only streams: equal keys are equal records, nothing to verify
    k_seg_count<false><<<blocks_for(m, kSegTile), kSegThreads, 0, s>>>(skeys, perm, kref, m, counts, st,
                                                                       hashed_bit(key_bits), kmask);
  count_launch();
  return cudaGetLastError();
}
cudaError_t launch_seg_write(const uint64_t* skeys, uint64_t m, const uint64_t* tile_base, uint64_t* seg_start,
                             uint64_t kmask, cudaStream_t s) {
  if (m == 0) return cudaMemsetAsync(seg_start, 0, sizeof(uint64_t), s);
  k_seg_write<<<blocks_for(m, kSegTile), kSegThreads, 0, s>>>(skeys, m, tile_base, seg_start, kmask);
  count_launch();
  return cudaGetLastError();
}
cudaError_t launch_seg_count32(const uint32_t* skeys, uint64_t m, uint32_t* counts, cudaStream_t s) {
  if (m == 0) return cudaSuccess;
  k_seg_count<false, uint32_t><<<blocks_for(m, kSegTile), kSegThreads, 0, s>>>(skeys, nullptr, nullptr, m, counts,
                                                                               nullptr, 0, ~0ULL);
  count_launch();
  return cudaGetLastError();
}
cudaError_t launch_seg_write32(const uint32_t* skeys, uint64_t m, const uint64_t* tile_base, uint64_t* seg_start,
                               cudaStream_t s) {
  if (m == 0) return cudaMemsetAsync(seg_start, 0, sizeof(uint64_t), s);
  k_seg_write<uint32_t><<<blocks_for(m, kSegTile), kSegThreads, 0, s>>>(skeys, m, tile_base, seg_start, ~0ULL);
  count_launch();
  return cudaGetLastError();
}
cudaError_t launch_key_lengths(const uint64_t* seg_start, uint64_t nseg, const uint32_t* perm, const uint64_t* kref,
                               uint64_t* lens, cudaStream_t s) {
  if (nseg == 0) return cudaSuccess;
  k_key_lengths<<<blocks_for(nseg, 256), 256, 0, s>>>(seg_start, nseg, perm, kref, lens);
  count_launch();
  return cudaGetLastError();
}
cudaError_t launch_key_copy(const uint64_t* seg_start, uint64_t nseg, const uint32_t* perm, const uint64_t* kref,
                            const uint64_t* key_off, uint8_t* keys, cudaStream_t s) {
  if (nseg == 0) return cudaSuccess;
  k_key_copy<<<blocks_for(nseg, 256), 256, 0, s>>>(seg_start, nseg, perm, kref, key_off, keys);
  count_launch();
  return cudaGetLastError();
}
cudaError_t launch_reduce_wc(const uint64_t* seg_start, uint64_t nseg, const uint64_t* skeys, const uint32_t* perm,
                             const uint8_t* v, int vmode, uint64_t* counts, uint64_t* worklist, DevState* st,
                             int num_sms, cudaStream_t s) {
  if (nseg == 0) return cudaSuccess;
  cudaError_t e = cudaMemsetAsync(&st->large_items, 0, 2 * sizeof(unsigned long long), s);
  if (e != cudaSuccess) return e;
  const unsigned g1 = static_cast<unsigned>(std::min<uint64_t>(blocks_for(nseg, 256), 148ULL * 32));
  if (vmode == 2) {
    k_reduce_wc_small<2><<<g1, 256, 0, s>>>(seg_start, nseg, skeys, perm, v, counts, worklist, st);
    k_reduce_wc_large<2><<<num_sms * 4, 256, 0, s>>>(seg_start, skeys, perm, v, counts, worklist, st);
  } else if (vmode == 1) {
    k_reduce_wc_small<1><<<g1, 256, 0, s>>>(seg_start, nseg, skeys, perm, v, counts, worklist, st);
    k_reduce_wc_large<1><<<num_sms * 4, 256, 0, s>>>(seg_start, skeys, perm, v, counts, worklist, st);
  } else {
    k_reduce_wc_small<0><<<g1, 256, 0, s>>>(seg_start, nseg, skeys, perm, v, counts, worklist, st);
    k_reduce_wc_large<0><<<num_sms * 4, 256, 0, s>>>(seg_start, skeys, perm, v, counts, worklist, st);
  }
  count_launch(2);
  return cudaGetLastError();
}
cudaError_t launch_reduce_km(const uint64_t* seg_start, uint64_t nseg, const uint64_t* skeys, const uint32_t* perm,
                             const uint8_t* v, double* sums, unsigned long long* cnts, uint32_t k,
                             uint64_t* worklist, DevState* st, int num_sms, cudaStream_t s) {
  cudaError_t e = cudaMemsetAsync(&st->large_items, 0, 2 * sizeof(unsigned long long), s);
  if (e == cudaSuccess) e = cudaMemsetAsync(sums, 0, sizeof(double) * 8 * k, s);
  if (e == cudaSuccess) e = cudaMemsetAsync(cnts, 0, sizeof(unsigned long long) * k, s);
  if (e != cudaSuccess || nseg == 0) return e;
  const unsigned g1 = static_cast<unsigned>(std::min<uint64_t>(blocks_for(nseg * 32, 256), 148ULL * 64));
  k_reduce_km_small<<<g1, 256, 0, s>>>(seg_start, nseg, skeys, perm, v, sums, cnts, k, worklist, st);
  count_launch();
  k_reduce_km_large<<<num_sms * 4, 256, kKmStage * 32, s>>>(seg_start, skeys, perm, v, sums, worklist, st);
  count_launch();
  return cudaGetLastError();
}
cudaError_t launch_km_finalize(const double* sums, const unsigned long long* cnts, const float* centroids, uint32_t k,
                               const uint32_t* list, uint32_t nlist, uint8_t* vals, uint64_t* val_off, uint8_t* keys,
                               uint64_t* key_off, cudaStream_t s) {
  const uint32_t n = list ? nlist : k;
  k_km_finalize<<<blocks_for(n + 1, 128), 128, 0, s>>>(sums, cnts, centroids, k, list, nlist, vals, val_off, keys,
                                                       key_off);
  count_launch();
  return cudaGetLastError();
}
cudaError_t launch_seg_lengths(const uint64_t* seg_start, uint64_t nseg, uint64_t* out, cudaStream_t s) {
  if (nseg == 0) return cudaSuccess;
  k_seg_lengths<<<blocks_for(nseg, 256), 256, 0, s>>>(seg_start, nseg, out);
  count_launch();
  return cudaGetLastError();
}
cudaError_t launch_key_lengths_exact(const uint64_t* seg_start, uint64_t nseg, const uint64_t* skeys, uint64_t* lens,
                                     cudaStream_t s) {
  if (nseg == 0) return cudaSuccess;
  k_key_lengths_exact<<<blocks_for(nseg, 256), 256, 0, s>>>(seg_start, nseg, skeys, lens);
  count_launch();
  return cudaGetLastError();
}
cudaError_t launch_key_decode(const uint64_t* seg_start, uint64_t nseg, const uint64_t* skeys, const uint64_t* key_off,
                              uint8_t* keys, cudaStream_t s) {
  if (nseg == 0) return cudaSuccess;
  k_key_decode<<<blocks_for(nseg, 256), 256, 0, s>>>(seg_start, nseg, skeys, key_off, keys);
  count_launch();
  return cudaGetLastError();
}
cudaError_t launch_key_lengths_exact32(const uint64_t* seg_start, uint64_t nseg, const uint32_t* skeys, uint64_t* lens,
                                       cudaStream_t s) {
  if (nseg == 0) return cudaSuccess;
  k_key_lengths_exact<<<blocks_for(nseg, 256), 256, 0, s>>>(seg_start, nseg, skeys, lens);
  count_launch();
  return cudaGetLastError();
}
cudaError_t launch_key_decode32(const uint64_t* seg_start, uint64_t nseg, const uint32_t* skeys,
                                const uint64_t* key_off, uint8_t* keys, cudaStream_t s) {
  if (nseg == 0) return cudaSuccess;
  k_key_decode<<<blocks_for(nseg, 256), 256, 0, s>>>(seg_start, nseg, skeys, key_off, keys);
  count_launch();
  return cudaGetLastError();
}
cudaError_t launch_comb_merge(const uint64_t* segp, uint64_t nsegp, const uint64_t* skp, const uint64_t* sega,
                              uint64_t nsega, const uint32_t* skx, uint32_t* midx, uint64_t* psum, uint32_t* xkeys,
                              uint64_t* xcounts, unsigned long long* nextra, cudaStream_t s) {
  if (nsegp == 0) return cudaSuccess;
  k_comb_merge<<<blocks_for(nsegp, 256), 256, 0, s>>>(segp, nsegp, skp, sega, nsega, skx, midx, psum, xkeys, xcounts,
                                                      nextra);
  count_launch();
  return cudaGetLastError();
}
cudaError_t launch_comb_add(const uint32_t* midx, const uint64_t* psum, uint64_t nsegp, uint64_t* counts,
                            cudaStream_t s) {
  if (nsegp == 0) return cudaSuccess;
  k_comb_add<<<blocks_for(nsegp, 256), 256, 0, s>>>(midx, psum, nsegp, counts);
  count_launch();
  return cudaGetLastError();
}
// WordCount two-level combiner (MapCG-style grouping by table):
// the L2-resident count table the Map fed with one RED per exact word that missed the SMEM table
// is turned into combiner partials.  One streaming read of the table (16 B per thread step, the
// nonzero entries are sparse: a warp ballot skips empty steps); a warp's nonzero entries take one
// global atomic for their output slots; written entries are zeroed, so the table is clean for the
// next Map.
template <bool kList>
__global__ void __launch_bounds__(256) k_xtab_extract(uint32_t* __restrict__ tab, uint64_t nv4, uint64_t* out,
                                                    uint32_t* okeys, uint64_t* ocounts, uint64_t cap,
                                                    unsigned long long* cursor, unsigned long long* wsum) {
  const uint32_t lane = threadIdx.x & 31;
  const uint64_t stride = static_cast<uint64_t>(gridDim.x) * blockDim.x;
  uint4* t4 = reinterpret_cast<uint4*>(tab);
  uint64_t csum = 0;
  // (kXU 16-B loads in flight per thread: one load per step left the stream at ~4.5 TB/s)
  constexpr int kXU = BMR_XTAB_UNROLL;
  for (uint64_t i0 = blockIdx.x * static_cast<uint64_t>(blockDim.x) * kXU + threadIdx.x; i0 - lane < nv4;
       i0 += stride * kXU) {
    uint4 vv[kXU];
#pragma unroll
    for (int u = 0; u < kXU; ++u) {
      const uint64_t i = i0 + static_cast<uint64_t>(u) * blockDim.x;
      vv[u] = i < nv4 ? __ldcs(t4 + i) : make_uint4(0, 0, 0, 0);
    }
    uint32_t any = 0;
#pragma unroll
    for (int u = 0; u < kXU; ++u) any |= vv[u].x | vv[u].y | vv[u].z | vv[u].w;
    if (!__any_sync(0xffffffffu, any != 0)) continue;
#pragma unroll 1
    for (int u = 0; u < kXU; ++u) {
    const uint64_t i = i0 + static_cast<uint64_t>(u) * blockDim.x;
    const uint4 v = vv[u];
    const uint32_t nz = (v.x != 0) + (v.y != 0) + (v.z != 0) + (v.w != 0);
    if (!__any_sync(0xffffffffu, nz != 0)) continue;
    const uint32_t incl = warp_inclusive_add(nz);
    const uint32_t tot = __shfl_sync(0xffffffffu, incl, 31);
    unsigned long long base = 0;
    if (lane == 31) base = atomicAdd(cursor, static_cast<unsigned long long>(tot));
    base = __shfl_sync(0xffffffffu, base, 31);
    uint64_t o = base + incl - nz;
    uint32_t c[4] = {v.x, v.y, v.z, v.w};
    bool wrote = false;
    for (int q = 0; q < 4; ++q) {
      if (!c[q]) continue;
      if (o < cap) {
        if constexpr (kList) {
          okeys[o] = static_cast<uint32_t>(4 * i + q);
          ocounts[o] = c[q];
          csum += c[q];
        } else {
          out[o] = (4 * i + q) | (static_cast<uint64_t>(c[q]) << 32);
        }
        c[q] = 0;
        wrote = true;
      }
      ++o;
    }
    if (wrote) t4[i] = make_uint4(c[0], c[1], c[2], c[3]);   // (entries past cap stay for the next call)
    }
  }
  if constexpr (kList) {
    const uint64_t w = warp_inclusive_add64(csum);
    if (lane == 31 && w) atomicAdd(wsum, static_cast<unsigned long long>(w));
  }
}

cudaError_t launch_xtab_extract(uint32_t* tab, uint64_t nent, uint64_t* out, uint64_t cap, unsigned long long* cursor,
                                int num_sms, cudaStream_t s) {
  const uint64_t nv4 = nent / 4;
  k_xtab_extract<false><<<static_cast<unsigned>(std::min<uint64_t>(8ULL * num_sms, (nv4 + 256 * BMR_XTAB_UNROLL - 1) / (256 * BMR_XTAB_UNROLL))), 256, 0, s>>>(
      tab, nv4, out, nullptr, nullptr, cap, cursor, nullptr);
  count_launch();
  return cudaGetLastError();
}
cudaError_t launch_xtab_extract_list(uint32_t* tab, uint64_t nent, uint32_t* okeys, uint64_t* ocounts, uint64_t cap,
                                     unsigned long long* cursor, unsigned long long* wsum, int num_sms, cudaStream_t s) {
  const uint64_t nv4 = nent / 4;
  k_xtab_extract<true><<<static_cast<unsigned>(std::min<uint64_t>(static_cast<uint64_t>(BMR_XTAB_BPS) * num_sms, (nv4 + 256 * BMR_XTAB_UNROLL - 1) / (256 * BMR_XTAB_UNROLL))), 256, 0, s>>>(
      tab, nv4, nullptr, okeys, ocounts, cap, cursor, wsum);
  count_launch();
  return cudaGetLastError();
}

// WC mid table -> (key, count) lists.  Each key sits in exactly one slot (the Map's inserts find an
// existing key before any empty slot), so the lists are the final mid keys; slots past `cap` stay.
__global__ void __launch_bounds__(256) k_mtab_extract(uint64_t* __restrict__ mkeys, uint32_t* __restrict__ mcnt, uint32_t bits,
                                                    uint64_t nslots, uint64_t* okeys, uint64_t* ocounts,
                                                    uint64_t cap, unsigned long long* cursor,
                                                    unsigned long long* wsum) {
  const uint32_t lane = threadIdx.x & 31;
  uint64_t csum = 0;
  const uint64_t stride = static_cast<uint64_t>(gridDim.x) * blockDim.x;
  for (uint64_t i = blockIdx.x * static_cast<uint64_t>(blockDim.x) + threadIdx.x; i - lane < nslots; i += stride) {
    const uint64_t k = i < nslots ? mkeys[i] : kMidEmpty;
    const bool full = k != kMidEmpty;
    const uint32_t m = __ballot_sync(0xffffffffu, full);
    if (!m) continue;
    unsigned long long base = 0;
    if (lane == 0) base = atomicAdd(cursor, static_cast<unsigned long long>(__popc(m)));
    base = __shfl_sync(0xffffffffu, base, 0);
    const uint64_t o = base + __popc(m & lanemask_lt());
    if (full && o < cap) {
      uint64_t c = 0;
#pragma unroll
      for (uint32_t q = 0; q < kMidStripes; ++q) c += mcnt[stripe_at(i, q, bits)];
      okeys[o] = k;
      ocounts[o] = c;
      csum += c;
      mkeys[i] = kMidEmpty;
      for (uint32_t q = 0; q < kMidStripes; ++q) mcnt[stripe_at(i, q, bits)] = 0;
    }
  }
  const uint64_t w = warp_inclusive_add64(csum);
  if (lane == 31 && w) atomicAdd(wsum, static_cast<unsigned long long>(w));
}

__global__ void __launch_bounds__(256) k_ltab_extract(uint64_t* __restrict__ lkeys, uint32_t* __restrict__ lcnt, uint32_t bits,
                                                    uint64_t nslots, uint64_t* okeys, uint64_t* okref,
                                                    uint64_t* ocounts, uint64_t cap, unsigned long long* cursor,
                                                    unsigned long long* wsum) {
  const uint32_t lane = threadIdx.x & 31;
  const uint64_t stride = static_cast<uint64_t>(gridDim.x) * blockDim.x;
  uint64_t csum = 0;
  for (uint64_t i = blockIdx.x * static_cast<uint64_t>(blockDim.x) + threadIdx.x; i - lane < nslots; i += stride) {
    const uint64_t lo = i < nslots ? lkeys[2 * i] : 0, hi = i < nslots ? lkeys[2 * i + 1] : 0;
    const bool full = lo != 0;   // (a word's first byte is never 0)
    const uint32_t m = __ballot_sync(0xffffffffu, full);
    if (!m) continue;
    unsigned long long base = 0;
    if (lane == 0) base = atomicAdd(cursor, static_cast<unsigned long long>(__popc(m)));
    base = __shfl_sync(0xffffffffu, base, 0);
    const uint64_t o = base + __popc(m & lanemask_lt());
    if (full && o < cap) {
      uint64_t c = 0;
#pragma unroll
      for (uint32_t q = 0; q < kMidStripes; ++q) c += lcnt[stripe_at(i, q, bits)];
      okeys[2 * o] = lo;
      okeys[2 * o + 1] = hi;
      // length = the number of nonzero (word) bytes of the zero-padded key
      // (hi == kShortHi: a word of <= 8 bytes, its length from lo)
      const uint32_t len = hi == kShortHi ? (64u - static_cast<uint32_t>(__clzll(static_cast<long long>(lo))) + 7u) / 8u
                           : 8u + (hi ? (64u - static_cast<uint32_t>(__clzll(static_cast<long long>(hi))) + 7u) / 8u : 0u);
      okref[o] = (reinterpret_cast<uint64_t>(okeys + 2 * o) << 16) | len;
      ocounts[o] = c;
      csum += c;
      lkeys[2 * i] = 0;
      lkeys[2 * i + 1] = 0;
      for (uint32_t q = 0; q < kMidStripes; ++q) lcnt[stripe_at(i, q, bits)] = 0;
    }
  }
  const uint64_t w = warp_inclusive_add64(csum);
  if (lane == 31 && w) atomicAdd(wsum, static_cast<unsigned long long>(w));
}

cudaError_t launch_ltab_extract(uint64_t* lkeys, uint32_t* lcnt, uint64_t nslots, uint32_t bits, uint64_t* okeys, uint64_t* okref,
                                uint64_t* ocounts, uint64_t cap, unsigned long long* cursor, unsigned long long* wsum,
                                int num_sms, cudaStream_t s) {
  k_ltab_extract<<<static_cast<unsigned>(std::min<uint64_t>(8ULL * num_sms, (nslots + 255) / 256)), 256, 0, s>>>(
      lkeys, lcnt, bits, nslots, okeys, okref, ocounts, cap, cursor, wsum);
  count_launch();
  return cudaGetLastError();
}

cudaError_t launch_mtab_extract(uint64_t* mkeys, uint32_t* mcnt, uint64_t nslots, uint32_t bits, uint64_t* okeys, uint64_t* ocounts,
                                uint64_t cap, unsigned long long* cursor, unsigned long long* wsum, int num_sms,
                                cudaStream_t s) {
  k_mtab_extract<<<static_cast<unsigned>(std::min<uint64_t>(8ULL * num_sms, (nslots + 255) / 256)), 256, 0, s>>>(
      mkeys, mcnt, bits, nslots, okeys, ocounts, cap, cursor, wsum);
  count_launch();
  return cudaGetLastError();
}

cudaError_t launch_key_lengths_list32(const uint32_t* keys, uint64_t n, uint64_t* lens, cudaStream_t s) {
  if (n == 0) return cudaSuccess;
  k_key_lengths_list32<<<blocks_for(n, 256), 256, 0, s>>>(keys, n, lens);
  count_launch();
  return cudaGetLastError();
}
cudaError_t launch_key_decode_list32(const uint32_t* keys, uint64_t n, const uint64_t* key_off, uint8_t* out,
                                     cudaStream_t s) {
  if (n == 0) return cudaSuccess;
  k_key_decode_list32<<<blocks_for(n, 256), 256, 0, s>>>(keys, n, key_off, out);
  count_launch();
  return cudaGetLastError();
}
cudaError_t launch_seg_keys(const uint64_t* seg, uint64_t nseg, const uint64_t* sk, uint64_t* out, cudaStream_t s) {
  if (nseg == 0) return cudaSuccess;
  k_seg_keys<<<blocks_for(nseg, 256), 256, 0, s>>>(seg, nseg, sk, out);
  count_launch();
  return cudaGetLastError();
}
cudaError_t launch_gather_u64(const uint32_t* perm, const uint8_t* v, uint64_t m, uint64_t* out, cudaStream_t s) {
  if (m == 0) return cudaSuccess;
  k_gather_u64<<<blocks_for(m, 256), 256, 0, s>>>(perm, reinterpret_cast<const uint64_t*>(v), m, out);
  count_launch();
  return cudaGetLastError();
}
cudaError_t launch_offsets_scaled(const uint64_t* seg_start, uint64_t nseg, uint64_t scale, uint64_t* out,
                                  cudaStream_t s) {
  k_offsets_scaled<<<blocks_for(nseg + 1, 256), 256, 0, s>>>(seg_start, nseg, scale, out);
  count_launch();
  return cudaGetLastError();
}
cudaError_t launch_iota_scaled(uint64_t n, uint64_t scale, uint64_t* out, cudaStream_t s) {
  k_iota_scaled<<<blocks_for(n + 1, 256), 256, 0, s>>>(n, scale, out);
  count_launch();
  return cudaGetLastError();
}
cudaError_t launch_rehash(uint64_t* h, const uint64_t* kref, uint64_t m, uint64_t seed, cudaStream_t s) {
  if (m == 0) return cudaSuccess;
  k_rehash<<<blocks_for(m, 256), 256, 0, s>>>(h, kref, m, seed);
  count_launch();
  return cudaGetLastError();
}

}  // namespace bmr
