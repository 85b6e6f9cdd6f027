// lines.cu — record directory of '\n'-terminated text on the device (the record model of every
// text config: a record is a line, Table II "a line", L195-270).
//
// mr_map_host_lines copies host text to the device in chunks and derives each chunk's offsets
// here while the next chunk is still in flight, so the host never touches (or sends) an offsets
// array.  Two passes over the chunk's bytes [lo, hi) of the device text buffer, both on 16-byte
// loads in the absolute (256-B aligned allocation) frame with the bytes outside [lo, hi) masked:
//   k_line_count: '\n' count per 16 KiB tile;
//   (exclusive scan of the tile counts: k_scan in sort.cu)
//   k_line_write: offsets[1 + rank] = (position of the rank-th '\n') + 1 - lo.
// offsets[0] = 0 and, for an unterminated last line, offsets[n] = hi - lo are set by the host.
#include "common.cuh"

namespace bmr {
namespace {

constexpr int kLineThreads = 256;
constexpr int kLineBytesPerThread = 64;
constexpr uint64_t kLineTile = static_cast<uint64_t>(kLineThreads) * kLineBytesPerThread;   // 16 KiB

// 64-bit mask of the '\n' bytes of the 64 bytes at absolute position p (bytes outside [lo, hi)
// are ignored).  `a` is the 16-B aligned buffer base.
__device__ __forceinline__ uint64_t nl_mask64(const uint8_t* a, uint64_t p, uint64_t lo, uint64_t hi) {
  uint64_t m = 0;
#pragma unroll
  for (int v = 0; v < 4; ++v) {
    const uint64_t q = p + 16 * v;
    if (q + 16 <= lo || q >= hi) continue;
    const uint4 w = __ldcs(reinterpret_cast<const uint4*>(a + q));
    const uint32_t ww[4] = {w.x, w.y, w.z, w.w};
#pragma unroll
    for (int i = 0; i < 4; ++i) {
      const uint32_t e = __vcmpeq4(ww[i], 0x0A0A0A0Au);                     // 0xFF per '\n' byte
      const uint32_t b4 = ((((e >> 7) & 0x01010101u) * 0x01020408u) >> 24) & 0xFu;
      m |= static_cast<uint64_t>(b4) << (16 * v + 4 * i);
    }
  }
  // clip to [lo, hi)
  if (p < lo) m &= (lo - p >= 64) ? 0ULL : (~0ULL << (lo - p));
  if (p + 64 > hi) m &= (hi <= p) ? 0ULL : (~0ULL >> (64 - (hi - p)));
  return m;
}

__global__ void __launch_bounds__(kLineThreads) k_line_count(const uint8_t* __restrict__ a, uint64_t lo, uint64_t hi,
                                                           uint32_t* counts) {
  __shared__ uint32_t ws[kLineThreads / 32];
  const uint64_t a0 = lo & ~15ULL;
  const uint64_t p = a0 + blockIdx.x * kLineTile + static_cast<uint64_t>(threadIdx.x) * kLineBytesPerThread;
  const uint32_t c = __popcll(nl_mask64(a, p, lo, hi));
  const uint32_t w = __reduce_add_sync(0xffffffffu, c);
  if ((threadIdx.x & 31) == 0) ws[threadIdx.x >> 5] = w;
  __syncthreads();
  if (threadIdx.x == 0) {
    uint32_t t = 0;
    for (int i = 0; i < kLineThreads / 32; ++i) t += ws[i];
    counts[blockIdx.x] = t;
  }
}

__global__ void __launch_bounds__(kLineThreads) k_line_write(const uint8_t* __restrict__ a, uint64_t lo, uint64_t hi,
                                                           const uint64_t* __restrict__ tile_base, uint64_t* off) {
  __shared__ uint32_t ws[kLineThreads / 32];
  const uint32_t lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const uint64_t a0 = lo & ~15ULL;
  const uint64_t p = a0 + blockIdx.x * kLineTile + static_cast<uint64_t>(threadIdx.x) * kLineBytesPerThread;
  uint64_t m = nl_mask64(a, p, lo, hi);
  const uint32_t c = __popcll(m);
  const uint32_t inc = warp_inclusive_add(c);
  if (lane == 31) ws[warp] = inc;
  __syncthreads();
  uint32_t pre = 0;
#pragma unroll
  for (int i = 0; i < kLineThreads / 32; ++i) pre += (i < static_cast<int>(warp)) ? ws[i] : 0u;
  uint64_t r = tile_base[blockIdx.x] + pre + inc - c;
  while (m) {
    const int j = __ffsll(static_cast<long long>(m)) - 1;
    m &= m - 1;
    off[1 + r++] = p + j + 1 - lo;
  }
}

inline unsigned tiles_of(uint64_t lo, uint64_t hi) {
  const uint64_t a0 = lo & ~15ULL;
  return static_cast<unsigned>((hi - a0 + kLineTile - 1) / kLineTile);
}

}  // namespace

uint64_t line_tiles(uint64_t lo, uint64_t hi) { return hi > lo ? tiles_of(lo, hi) : 0; }

cudaError_t launch_line_count(const uint8_t* base, uint64_t lo, uint64_t hi, uint32_t* counts, cudaStream_t s) {
  if (hi <= lo) return cudaSuccess;
  k_line_count<<<tiles_of(lo, hi), kLineThreads, 0, s>>>(base, lo, hi, counts);
  count_launch();
  return cudaGetLastError();
}

cudaError_t launch_line_write(const uint8_t* base, uint64_t lo, uint64_t hi, const uint64_t* tile_base, uint64_t* off,
                              cudaStream_t s) {
  if (hi <= lo) return cudaSuccess;
  k_line_write<<<tiles_of(lo, hi), kLineThreads, 0, s>>>(base, lo, hi, tile_base, off);
  count_launch();
  return cudaGetLastError();
}

}  // namespace bmr
