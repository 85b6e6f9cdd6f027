// gen_device.cu — device (sm_100a) build of the seeded input generators in bmr_gen.h.
// Test/bench infrastructure only (no MapReduce arithmetic): lets bench.py and the full-size
// parity tests create multi-GiB inputs directly in HBM.  Bytes are identical to the host
// build (gen_host.c) for the same parameters (tests/test_gen_device.py).
#include <cuda_runtime.h>
#include "bmr_gen.h"

__global__ void k_pages(bmrg_text_params P, uint64_t page0, uint64_t npages, uint8_t* out,
                        uint32_t* page_lines) {
  uint64_t p = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
  if (p >= npages) return;
  uint8_t* o = out + p * (uint64_t)P.page_bytes;
  uint64_t gbase = (page0 + p) * (uint64_t)P.page_bytes;
  uint32_t nl = (P.kind == BMRG_HTML) ? bmrg_html_page(&P, page0 + p, o, gbase, nullptr)
                                      : bmrg_text_page(&P, page0 + p, o, gbase, nullptr);
  page_lines[p] = nl;
}

// one warp per page: offsets[k+1] = (page byte) + 1 for every '\n', k from line_base[p]
__global__ void k_offsets(const uint8_t* data, uint64_t npages, uint32_t pb,
                          const uint64_t* line_base, uint64_t* offsets) {
  uint64_t p = (blockIdx.x * (uint64_t)blockDim.x + threadIdx.x) >> 5;
  int lane = threadIdx.x & 31;
  if (p >= npages) return;
  const uint8_t* d = data + p * (uint64_t)pb;
  uint64_t k = line_base[p];
  if (p == 0 && lane == 0) offsets[0] = 0;
  for (uint32_t c = 0; c < pb; c += 32 * 16) {
    uint32_t i0 = c + lane * 16;
    uint32_t m = 0;
    if (i0 < pb) {
      for (int j = 0; j < 16 && i0 + j < pb; ++j) m |= (d[i0 + j] == '\n' ? 1u : 0u) << j;
    }
    uint32_t cnt = __popc(m), inc = cnt;
    for (int s = 1; s < 32; s <<= 1) {
      uint32_t v = __shfl_up_sync(0xffffffffu, inc, s);
      if (lane >= s) inc += v;
    }
    uint64_t w = k + inc - cnt;
    while (m) {
      int j = __ffs(m) - 1; m &= m - 1;
      offsets[++w] = p * (uint64_t)pb + i0 + j + 1;
    }
    k += __shfl_sync(0xffffffffu, inc, 31);
  }
}

__global__ void k_km(uint64_t seed, uint64_t i0, uint64_t n, const int32_t* centres, uint32_t k, float* out) {
  uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
  if (i >= n) return;
  float x[8];
  bmrg_km_point(seed, i0 + i, centres, k, x);
  float4* o = reinterpret_cast<float4*>(out + i * 8);
  o[0] = make_float4(x[0], x[1], x[2], x[3]);
  o[1] = make_float4(x[4], x[5], x[6], x[7]);
}

extern "C" {
// P: host struct whose table pointers are DEVICE pointers.
int bmrg_dev_pages(const bmrg_text_params* P, uint64_t page0, uint64_t npages, uint8_t* out,
                   uint32_t* page_lines, void* stream) {
  if (!P || !out || !page_lines) return 1;
  if (!npages) return 0;
  unsigned blocks = (unsigned)((npages + 63) / 64);
  k_pages<<<blocks, 64, 0, (cudaStream_t)stream>>>(*P, page0, npages, out, page_lines);
  return cudaGetLastError() == cudaSuccess ? 0 : 2;
}
int bmrg_dev_offsets(const uint8_t* data, uint64_t npages, uint32_t page_bytes,
                     const uint64_t* line_base, uint64_t* offsets, void* stream) {
  if (!npages) return 0;
  unsigned blocks = (unsigned)((npages * 32 + 255) / 256);
  k_offsets<<<blocks, 256, 0, (cudaStream_t)stream>>>(data, npages, page_bytes, line_base, offsets);
  return cudaGetLastError() == cudaSuccess ? 0 : 2;
}
int bmrg_dev_km(uint64_t seed, uint64_t i0, uint64_t n, const int32_t* centres, uint32_t k,
                float* out, void* stream) {
  if (!n) return 0;
  unsigned blocks = (unsigned)((n + 255) / 256);
  k_km<<<blocks, 256, 0, (cudaStream_t)stream>>>(seed, i0, n, centres, k, out);
  return cudaGetLastError() == cudaSuccess ? 0 : 2;
}
}
