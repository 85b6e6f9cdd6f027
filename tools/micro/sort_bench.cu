// Microbenchmark of the u32 keys-only onesweep passes (links build/sort.o): m random keys of
// `bits` bits, Zipf-like or uniform; times the histogram and each LSD pass with CUDA events,
// every pass ranked with match.any (rank 0) or the shared-memory OR masks (rank 1).
// usage: sort_bench M_millions key_bits zipf(0/1) rank(0/1)
#include <cstdio>
#include <cstdlib>
#include <vector>
#include <atomic>
#include <cmath>
#include "../../paper_conf_ipps_jim11_b200/csrc/kernels.h"
namespace bmr { std::atomic<unsigned long long> g_kernel_launches{0}; }
using namespace bmr;
__global__ void gen(uint32_t* k, uint64_t m, uint32_t bits, int zipf) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < m; i += (uint64_t)gridDim.x * blockDim.x) {
    uint64_t z = i * 0x9E3779B97F4A7C15ull + 12345;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull; z = (z ^ (z >> 27)) * 0x94D049BB133111EBull; z ^= z >> 31;
    uint32_t v;
    if (zipf) {  // rank ~ 2^(20 u) (log-uniform, Zipf-like), then a fixed scramble of the rank into the key space
      const double u = (z >> 11) * (1.0 / 9007199254740992.0);
      const uint32_t r = (uint32_t)exp2(20.0 * u);
      v = (r * 2654435761u) ^ (r >> 7);
    } else v = (uint32_t)z;
    k[i] = v & ((1u << bits) - 1u);
  }
}
int main(int argc, char** argv) {
  const uint64_t m = (uint64_t)(argc > 1 ? atof(argv[1]) : 672) * 1000000ull;
  const int bits = argc > 2 ? atoi(argv[2]) : 30, zipf = argc > 3 ? atoi(argv[3]) : 1;
  const int rank = argc > 4 ? atoi(argv[4]) : 0;
  uint32_t *a, *b, *c, *hist, *bases; uint64_t* status; unsigned* tc;
  cudaMalloc(&a, m * 4); cudaMalloc(&b, m * 4); cudaMalloc(&c, m * 4);
  cudaMalloc(&hist, 8 * kBinStride * 4); cudaMalloc(&bases, 8 * kBinStride * 4);
  const uint64_t tiles = m / 4096 + 2;
  cudaMalloc(&status, tiles * 256 * 8); cudaMemset(status, 0, tiles * 256 * 8); cudaMalloc(&tc, 4);
  gen<<<148 * 8, 256>>>(a, m, bits, zipf);
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  std::vector<uint32_t> h(8 * kBinStride), bs(8 * kBinStride);
  uint32_t epoch = 1; float ms;
  for (int rep = 0; rep < 3; ++rep) {
    cudaEventRecord(e0);
    launch_hist32(a, m, hist, 4, 8, 148, 0);
    cudaEventRecord(e1); cudaEventSynchronize(e1); cudaEventElapsedTime(&ms, e0, e1);
    if (rep == 2) printf("hist %.3f ms\n", ms);
    cudaMemcpy(h.data(), hist, h.size() * 4, cudaMemcpyDeviceToHost);
    for (int d = 0; d < 4; ++d) { uint32_t run = 0; for (int x = 0; x < 256; ++x) { bs[d * kBinStride + x] = run; run += h[d * kBinStride + x]; } }
    if (rep == 2)
      for (int d = 0; d < 4; ++d) {
        double e = 0; for (int x = 0; x < 256; ++x) { const double p = (double)h[d * kBinStride + x] / m; e += 1 - pow(1 - p, 32); }
        printf("digit %d: expected distinct digits per 32 keys %.2f\n", d, e);
      }
    cudaMemcpy(bases, bs.data(), bs.size() * 4, cudaMemcpyHostToDevice);
    const uint32_t* kin = a; float tot = 0;
    for (int d = 0; d < 4; ++d) {
      uint32_t* kout = (d & 1) ? c : b;
      cudaEventRecord(e0);
      launch_onesweep32(kin, kout, m, d, 8, bases, status, epoch++, tc, 0, rank ? kRankOrMask : kRankMatch);
      cudaEventRecord(e1); cudaEventSynchronize(e1); cudaEventElapsedTime(&ms, e0, e1);
      tot += ms;
      if (rep == 2) printf("pass %d %.3f ms (%.1f GB/s)\n", d, ms, m * 8.0 / ms / 1e6);
      kin = kout;
    }
    if (rep == 2) {
      std::vector<uint32_t> o(m);
      cudaMemcpy(o.data(), kin, m * 4, cudaMemcpyDeviceToHost);
      uint64_t bad = 0; for (uint64_t i = 1; i < m; ++i) bad += o[i - 1] > o[i];
      printf("total %.3f ms, %s (%llu inversions), err %s\n", tot, bad ? "NOT SORTED" : "sorted", (unsigned long long)bad,
             cudaGetErrorString(cudaGetLastError()));
    }
  }
  return 0;
}
