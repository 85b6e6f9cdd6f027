// exchange.cu — multi-GPU group-by: partition intermediate records by destination
// rank and ingest the records received from one all-to-all.
//
// Map shards by byte range with no communication.  Group/Reduce need exactly one exchange:
// destination = mix64(partition hash of the key bytes) mod R, so equal keys meet on one rank.
// The partition hash is computed from the key BYTES (not from the local sort key), so it is the
// same on every rank even if a rank re-hashed after a collision.  Records travel as fixed
// entries plus a byte heap for the keys:
//   WC / II entry (16 B): (heap offset << 16 | key length, value u64)
//   KM entry (80 B):      (cluster id, count, 8 x fp64 partial sums)
// The caller (torch.distributed over NCCL) moves the per-destination slices; mr_ingest turns the
// received entries back into SoA pairs (key by reference into the received heap) or, for KM,
// accumulates the partial sums.
#include <algorithm>

#include "common.cuh"

namespace bmr {
namespace {

constexpr int kXThreads = 256;
__device__ __forceinline__ uint32_t dest_of_id(uint64_t id, uint32_t R) {
  return static_cast<uint32_t>(mix64(id ^ kPartSeed) % R);
}

// Record i of the source: key bytes (ptr, len — or inline bytes), value, destination, heap bytes.
struct Rec {
  const uint8_t* kp;
  uint64_t kin;   // key bytes of an exact WC key (kp == nullptr)
  uint32_t klen;
  uint64_t v;
  uint32_t dest;
  uint32_t heap;  // bytes in the heap (key length rounded up to 8)
  __device__ __forceinline__ uint8_t byte(uint32_t k) const {
    return kp ? kp[k] : static_cast<uint8_t>(kin >> (8 * k));
  }
};

__device__ __forceinline__ Rec get_rec(const XSource& S, uint64_t i) {
  Rec r{};
  if (S.mode == kXSplit) {   // WC Map output: exact, combiner partials, mid, then hashed stream
    r.v = 1;
    if (i < S.nx + S.np + S.nc) {
      if (i < S.nx && S.hx[i] == 0xFFFFFFFFu) { r.dest = ~0u; return r; }   // flush filler (exact stream)
      uint64_t key;
      if (i < S.nx) {
        key = S.hx[i];
      } else if (i < S.nx + S.np) {   // combiner partial: exact key, value = its count
        key = S.hp[i - S.nx] & 0x3FFFFFFFULL;
        r.v = S.hp[i - S.nx] >> 32;
      } else {
        key = S.hc[i - S.nx - S.np];
        if (key == (1ULL << kMidBits) - 1ULL) { r.dest = ~0u; return r; }   // chunk-tail sentinel
      }
      r.kin = exact_key_bytes(key, r.klen);
      r.dest = dest_of_bytes(reinterpret_cast<const uint8_t*>(&r.kin), r.klen, S.nranks);
      r.heap = (r.klen + 7u) & ~7u;
      return r;
    }
    const uint64_t kr = S.kref[i - S.nx - S.np - S.nc];
    if (kr == 0) { r.dest = ~0u; return r; }   // chunk-tail sentinel (hashed stream)
    r.kp = reinterpret_cast<const uint8_t*>(kr >> 16);
    r.klen = static_cast<uint32_t>(kr & 0xFFFF);
  } else if (S.mode == kXPairs) {
    const uint64_t kr = S.kref[i];   // 0 = flush filler (sentinel) pair: not a record
    if (kr == 0) { r.dest = ~0u; return r; }
    r.kp = reinterpret_cast<const uint8_t*>(kr >> 16);
    r.klen = static_cast<uint32_t>(kr & 0xFFFF);
    r.v = S.vbytes == 4 ? reinterpret_cast<const uint32_t*>(S.v)[i] : reinterpret_cast<const uint64_t*>(S.v)[i];
  } else {  // kXSegs: combined WC (key blob + u64 counts)
    const uint64_t a = S.key_off[i], b = S.key_off[i + 1];
    r.kp = S.keys + a;
    r.klen = static_cast<uint32_t>(b - a);
    r.v = S.counts[i];
  }
  r.dest = dest_of_bytes(r.kp, r.klen, S.nranks);
  r.heap = (r.klen + 7u) & ~7u;
  return r;
}

__global__ void __launch_bounds__(kXThreads) k_x_count(XSource S, unsigned long long* counts) {
  __shared__ unsigned long long c[2 * kMaxRanks];
  for (uint32_t d = threadIdx.x; d < 2 * kMaxRanks; d += blockDim.x) c[d] = 0;
  __syncthreads();
  const uint64_t stride = static_cast<uint64_t>(gridDim.x) * blockDim.x;
  for (uint64_t i = blockIdx.x * static_cast<uint64_t>(blockDim.x) + threadIdx.x; i < S.n; i += stride) {
    if (S.mode == kXKM) {
      if (S.cnts[i] == 0) continue;
      atomicAdd(&c[2 * dest_of_id(i, S.nranks)], 1ULL);
    } else {
      const Rec r = get_rec(S, i);
      if (r.dest == ~0u) continue;
      atomicAdd(&c[2 * r.dest], 1ULL);
      atomicAdd(&c[2 * r.dest + 1], static_cast<unsigned long long>(r.heap));
    }
  }
  __syncthreads();
  for (uint32_t d = threadIdx.x; d < 2 * S.nranks; d += blockDim.x)
    if (c[d]) atomicAdd(&counts[d], c[d]);
}

// cursors[2R]: next entry index / heap byte of every destination slice (initialised to the
// exclusive prefix of the counts by the host).
__global__ void __launch_bounds__(kXThreads) k_x_scatter(XSource S, unsigned long long* cursors, uint8_t* entries,
                                                       uint8_t* heap) {
  __shared__ unsigned long long lc[2 * kMaxRanks], gb[2 * kMaxRanks];
  const uint64_t tile = static_cast<uint64_t>(blockIdx.x) * kXThreads;
  const uint64_t i = tile + threadIdx.x;
  for (uint32_t d = threadIdx.x; d < 2 * kMaxRanks; d += blockDim.x) lc[d] = 0;
  __syncthreads();
  Rec r{};
  bool live = i < S.n;
  unsigned long long le = 0, lh = 0;
  if (live) {
    if (S.mode == kXKM) {
      live = S.cnts[i] != 0;
      if (live) { r.dest = dest_of_id(i, S.nranks); r.heap = 0; }
    } else {
      r = get_rec(S, i);
      live = r.dest != ~0u;
    }
  }
  if (live) {
    le = atomicAdd(&lc[2 * r.dest], 1ULL);
    lh = atomicAdd(&lc[2 * r.dest + 1], static_cast<unsigned long long>(r.heap));
  }
  __syncthreads();
  if (threadIdx.x < 2 * S.nranks && lc[threadIdx.x]) gb[threadIdx.x] = atomicAdd(&cursors[threadIdx.x], lc[threadIdx.x]);
  __syncthreads();
  if (!live) return;
  const uint64_t e = gb[2 * r.dest] + le;
  if (S.mode == kXKM) {
    XEntryKM* o = reinterpret_cast<XEntryKM*>(entries) + e;
    o->id = i;
    o->cnt = S.cnts[i];
    for (int t = 0; t < 8; ++t) o->sums[t] = S.sums[i * 8 + t];
    return;
  }
  // heap offsets are relative to the destination's heap slice: subtract the slice base
  const uint64_t hoff = gb[2 * r.dest + 1] + lh;
  XEntry* o = reinterpret_cast<XEntry*>(entries) + e;
  o->koff_len = ((hoff - S.heap_base[r.dest]) << 16) | r.klen;
  o->v = r.v;
  uint8_t* hp = heap + hoff;
  for (uint32_t k = 0; k < r.klen; ++k) hp[k] = r.byte(k);
}

// Received entries -> SoA pairs.  src_e / src_h: exclusive prefixes (R + 1) of the entries /
// heap bytes received from each source rank.
__global__ void k_x_ingest(const XEntry* __restrict__ ent, const uint8_t* heap, uint64_t n, const uint64_t* src_e,
                           const uint64_t* src_h, uint32_t R, uint64_t* h, uint64_t* kref, uint64_t* v,
                           uint64_t seed, uint32_t weak, uint32_t key_bits) {
  const uint64_t j = blockIdx.x * static_cast<uint64_t>(blockDim.x) + threadIdx.x;
  if (j >= n) return;
  uint32_t r = 0;
  while (r + 1 < R && j >= src_e[r + 1]) ++r;
  const XEntry x = ent[j];
  const uint32_t klen = static_cast<uint32_t>(x.koff_len & 0xFFFF);
  const uint8_t* kp = heap + src_h[r] + (x.koff_len >> 16);
  const uint64_t key = key_of_bytes(kp, klen, seed, weak != 0, key_bits);
  h[j] = key;
  kref[j] = (reinterpret_cast<uint64_t>(kp) << 16) | klen;
  v[j] = x.v;
}

__global__ void k_x_ingest_km(const XEntryKM* __restrict__ ent, uint64_t n, double* sums, unsigned long long* cnts,
                              uint32_t k) {
  const uint64_t j = blockIdx.x * static_cast<uint64_t>(blockDim.x) + threadIdx.x;
  if (j >= n) return;
  const XEntryKM x = ent[j];
  if (x.id >= k) return;
  atomicAdd(&cnts[x.id], static_cast<unsigned long long>(x.cnt));
  for (int t = 0; t < 8; ++t) atomicAdd(&sums[x.id * 8 + t], x.sums[t]);
}

inline unsigned nblocks(uint64_t n, unsigned t) { return static_cast<unsigned>((n + t - 1) / t); }

}  // namespace

uint32_t km_owner(uint32_t j, uint32_t R) {
  return static_cast<uint32_t>(mix64(static_cast<uint64_t>(j) ^ kPartSeed) % R);
}

cudaError_t launch_x_count(const XSource& S, unsigned long long* counts, int num_sms, cudaStream_t s) {
  cudaError_t e = cudaMemsetAsync(counts, 0, sizeof(unsigned long long) * 2 * S.nranks, s);
  if (e != cudaSuccess || S.n == 0) return e;
  const uint64_t g = std::min<uint64_t>(nblocks(S.n, kXThreads), static_cast<uint64_t>(num_sms) * 8);
  k_x_count<<<static_cast<unsigned>(g), kXThreads, 0, s>>>(S, counts);
  count_launch();
  return cudaGetLastError();
}

cudaError_t launch_x_scatter(const XSource& S, unsigned long long* cursors, uint8_t* entries, uint8_t* heap,
                             cudaStream_t s) {
  if (S.n == 0) return cudaSuccess;
  k_x_scatter<<<nblocks(S.n, kXThreads), kXThreads, 0, s>>>(S, cursors, entries, heap);
  count_launch();
  return cudaGetLastError();
}

cudaError_t launch_x_ingest(const void* entries, const uint8_t* heap, uint64_t n, const uint64_t* src_e,
                            const uint64_t* src_h, uint32_t R, uint64_t* h, uint64_t* kref, uint64_t* v,
                            uint64_t seed, uint32_t weak, uint32_t key_bits, cudaStream_t s) {
  if (n == 0) return cudaSuccess;
  k_x_ingest<<<nblocks(n, 256), 256, 0, s>>>(static_cast<const XEntry*>(entries), heap, n, src_e, src_h, R, h, kref,
                                             v, seed, weak, key_bits);
  count_launch();
  return cudaGetLastError();
}

cudaError_t launch_x_ingest_km(const void* entries, uint64_t n, double* sums, unsigned long long* cnts, uint32_t k,
                               cudaStream_t s) {
  if (n == 0) return cudaSuccess;
  k_x_ingest_km<<<nblocks(n, 256), 256, 0, s>>>(static_cast<const XEntryKM*>(entries), n, sums, cnts, k);
  count_launch();
  return cudaGetLastError();
}

}  // namespace bmr
