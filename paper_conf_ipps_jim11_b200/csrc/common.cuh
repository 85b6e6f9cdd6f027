// common.cuh — device-side building blocks shared by the libbmr kernels (sm_100a only).
//   * PTX wrappers: mbarrier (init / arrive / expect_tx / try_wait.parity) and the 1-D TMA
//     bulk copy cp.async.bulk (global -> shared, completion through an mbarrier).
//   * Key encoding used by the emit step: keys of <= 7 bytes are packed
//     injectively into the 64-bit sort key (length in the top byte, 1..7); longer keys are
//     hashed to 64 bits with the top bit forced to 1, so the two classes never collide.
//     Hashed keys are verified byte-for-byte at segment-boundary time (a8).
#pragma once
#include <cstdint>
#include <cuda_runtime.h>
#include "kernels.h"

namespace bmr {

// ---------------------------------------------------------------- PTX helpers
__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes)
               : "memory");
}
__device__ __forceinline__ bool mbar_try_wait(uint64_t* bar, uint32_t parity) {
  uint32_t ok;
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\t"
      "selp.u32 %0, 1, 0, p;\n\t}"
      : "=r"(ok)
      : "r"(smem_u32(bar)), "r"(parity)
      : "memory");
  return ok != 0;
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
  while (!mbar_try_wait(bar, parity)) {
  }
}
// TMA 1-D bulk copy global -> shared; dst, src and bytes must be multiples of 16.
__device__ __forceinline__ void tma_load_1d(void* smem_dst, const void* gsrc, uint32_t bytes, uint64_t* bar) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
          smem_u32(smem_dst)),
      "l"(gsrc), "r"(bytes), "r"(smem_u32(bar))
      : "memory");
}
__device__ __forceinline__ void fence_proxy_async_shared() {
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}
__device__ __forceinline__ void named_bar_sync(uint32_t id, uint32_t nthreads) {
  asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(nthreads) : "memory");
}
__device__ __forceinline__ uint32_t lanemask_lt() {
  uint32_t m;
  asm("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
  return m;
}
__device__ __forceinline__ uint64_t ld_volatile_u64(const uint64_t* p) {
  uint64_t v;
  asm volatile("ld.volatile.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ uint32_t ld_volatile_u32(const uint32_t* p) {
  uint32_t v;
  asm volatile("ld.volatile.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ uint64_t ld_relaxed_gpu_u64(const uint64_t* p) {
  uint64_t v;
  asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_relaxed_gpu_u64(uint64_t* p, uint64_t v) {
  asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ uint64_t ld_acquire_gpu_u64(const uint64_t* p) {
  uint64_t v;
  asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_release_gpu_u64(uint64_t* p, uint64_t v) {
  asm volatile("st.release.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ void st_volatile_u64(uint64_t* p, uint64_t v) {
  asm volatile("st.volatile.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ void st_volatile_u32(uint32_t* p, uint32_t v) {
  asm volatile("st.volatile.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}

// ---------------------------------------------------------------- key encoding
__host__ __device__ __forceinline__ uint64_t mix64(uint64_t z) {  // murmur3 finaliser
  z ^= z >> 33;
  z *= 0xff51afd7ed558ccdULL;
  z ^= z >> 33;
  z *= 0xc4ceb9fe1a85ec53ULL;
  z ^= z >> 33;
  return z;
}

// 64-bit key hash over 4-byte little-endian words (last word zero-padded): two 32-bit lanes
// (murmur3-style rounds) so that the map warps stay on 32-bit IMAD/LOP3; hash_bytes (generic
// pointer) and the map kernel's SMEM variant feed identical words and agree bit for bit.
struct KeyHash {
  uint32_t h1, h2;
  __device__ __forceinline__ KeyHash(uint64_t seed, uint32_t len)
      : h1(static_cast<uint32_t>(seed) ^ (len * 0x9E3779B1u)), h2(static_cast<uint32_t>(seed >> 32) + len * 0x85EBCA77u) {}
  __device__ __forceinline__ void add(uint32_t w) {
    h1 = __funnelshift_l(h1 ^ (w * 0xCC9E2D51u), h1 ^ (w * 0xCC9E2D51u), 15) * 0x1B873593u;
    h2 = (h2 + w) * 0x27D4EB2Fu;
    h2 ^= h2 >> 15;
  }
  __device__ __forceinline__ static uint32_t fmix(uint32_t h) {
    h ^= h >> 16; h *= 0x85EBCA6Bu; h ^= h >> 13; h *= 0xC2B2AE35u; h ^= h >> 16;
    return h;
  }
  __device__ __forceinline__ uint64_t finish() const {
    return (static_cast<uint64_t>(fmix(h1 + h2)) << 32) | fmix(h2 ^ __funnelshift_l(h1, h1, 7));
  }
};

// Hash of key bytes read through a generic pointer (shared or global).
__device__ __forceinline__ uint64_t hash_bytes(const uint8_t* p, uint32_t len, uint64_t seed) {
  KeyHash hs(seed, len);
  uint32_t i = 0;
  for (; i + 4 <= len; i += 4)
    hs.add(static_cast<uint32_t>(p[i]) | (static_cast<uint32_t>(p[i + 1]) << 8) |
           (static_cast<uint32_t>(p[i + 2]) << 16) | (static_cast<uint32_t>(p[i + 3]) << 24));
  if (i < len) {
    uint32_t w = 0;
    for (uint32_t k = 0; i + k < len; ++k) w |= static_cast<uint32_t>(p[i + k]) << (8 * k);
    hs.add(w);
  }
  return hs.finish();
}
// Sort-key formats.  The key width is 64 bits (II, re-hash slow path) or 48 bits (WC: two LSD
// passes fewer; digits 6 and 7 are then constant and skipped):
//   inline  : keys of <= kInlineMax bytes packed little-endian, length in the 3 bits above them
//             (64: len << 56, <= 7 bytes; 48: len << 40, <= 5 bytes) — injective, top bit clear;
//   alnum   : (48 only) [0-9A-Za-z] keys of 6..7 bytes: 2^43 | 6-bit symbol codes (1..62, so
//             the length is implied) — every exact 48-bit key is < 2^44 (five 9-bit digits);
//   hashed  : longer keys -> hash with the top bit of the width forced to 1 (never collides with
//             an inline key); equal hashes are verified byte-for-byte at segment time;
//   sentinel: all ones in the width — flush filler pairs, sorts after every real key.
__host__ __device__ __forceinline__ uint32_t inline_max(uint32_t bits) { return bits == 48 ? 5u : 7u; }
__host__ __device__ __forceinline__ uint64_t hashed_bit(uint32_t bits) { return 1ULL << (bits - 1); }
__host__ __device__ __forceinline__ uint64_t sentinel_of(uint32_t bits) {
  return bits == 64 ? ~0ULL : ((1ULL << bits) - 1ULL);
}
// WEAK (MR_FLAG_WEAK_HASH_DEBUG) keeps only 4 hash bits so that almost every segment collides
// (tests the verification + re-sort slow path).
__device__ __forceinline__ uint64_t hashed_key(uint64_t h, bool weak, uint32_t bits = 64) {
  const uint64_t hb = hashed_bit(bits);
  const uint64_t k = (weak ? (h & 0xFULL) : (h & (hb - 1ULL))) | hb;
  return k == sentinel_of(bits) ? k - 1ULL : k;
}
__device__ __forceinline__ uint64_t inline_key(uint64_t bytes_le, uint32_t len, uint32_t bits = 64) {
  return (bytes_le & ((1ULL << (8 * len)) - 1ULL)) | (static_cast<uint64_t>(len) << (bits - 8));
}
// 48-bit (WordCount) keys of 6..7 bytes: a WC word is [0-9A-Za-z]+ (C-3 #1), so each symbol
// has a nonzero 6-bit code (1..62); 6 or 7 codes (<= 42 bits, the highest nonzero code gives
// the length) above a 2^43 tag pack injectively — disjoint from the byte-packed keys (< 2^43)
// and from the hashed ones (bit 47).
__device__ __forceinline__ bool alnum_byte(uint32_t c) {
  return (c - '0' < 10u) || (c - 'A' < 26u) || (c - 'a' < 26u);
}
__device__ __forceinline__ uint64_t alnum_key48(uint64_t bytes_le, uint32_t len) {
  // SWAR: per byte code = c - 47 - 7 [c > '9'] - 6 [c > 'Z'], then bytes beyond len cleared and
  // the eight 6-bit codes compressed (byte -> 12-bit pairs -> 24-bit quads -> 48 bits).
  const auto codes = [](uint32_t w) {
    const uint32_t g9 = __vcmpgtu4(w, 0x39393939u) & 0x07070707u;
    const uint32_t gz = __vcmpgtu4(w, 0x5A5A5A5Au) & 0x06060606u;
    return __vsub4(__vsub4(__vsub4(w, 0x2F2F2F2Fu), g9), gz);
  };
  uint64_t x = (static_cast<uint64_t>(codes(static_cast<uint32_t>(bytes_le >> 32))) << 32) |
               codes(static_cast<uint32_t>(bytes_le));
  x &= (1ULL << (8 * len)) - 1ULL;  // len <= 7
  x = (x & 0x003F003F003F003FULL) | ((x >> 2) & 0x0FC00FC00FC00FC0ULL);
  x = (x & 0x00000FFF00000FFFULL) | ((x >> 4) & 0x00FFF00000FFF000ULL);
  x = (x & 0x0000000000FFFFFFULL) | ((x >> 8) & 0x0000FFFFFF000000ULL);
  return x | (1ULL << 43);
}
// Inverse of the 48-bit exact formats (inline <= 5 bytes, alnum 6..7): key bytes little-endian.
__device__ __forceinline__ uint64_t exact_key_bytes48(uint64_t key, uint32_t& len) {
  if (key < (1ULL << 43)) {
    len = static_cast<uint32_t>(key >> 40) & 7u;
    return key & ((1ULL << 40) - 1ULL);
  }
  const uint64_t codes = key & ((1ULL << 42) - 1ULL);
  len = codes ? static_cast<uint32_t>(63 - __clzll(static_cast<long long>(codes))) / 6u + 1u : 0u;
  uint64_t b = 0;
  for (uint32_t i = 0; i < len; ++i) {
    const uint32_t c = static_cast<uint32_t>(key >> (6 * i)) & 63u;
    b |= static_cast<uint64_t>(c <= 10 ? c + 47u : (c <= 36 ? c + 54u : c + 60u)) << (8 * i);
  }
  return b;
}
// key bytes -> sort key (generic pointer)
__device__ __forceinline__ uint64_t key_of_bytes(const uint8_t* p, uint32_t len, uint64_t seed, bool weak,
                                                 uint32_t bits) {
  if (len <= inline_max(bits) || (bits == 48 && len <= 7)) {
    uint64_t b = 0;
    bool alnum = true;
    for (uint32_t k = 0; k < len; ++k) {
      b |= static_cast<uint64_t>(p[k]) << (8 * k);
      alnum = alnum && alnum_byte(p[k]);
    }
    if (len <= inline_max(bits)) return inline_key(b, len, bits);
    if (alnum) return alnum_key48(b, len);
  }
  return hashed_key(hash_bytes(p, len, seed), weak, bits);
}

// ---------------------------------------------------------------- small scans
__device__ __forceinline__ uint32_t warp_inclusive_add(uint32_t v) {
  const uint32_t lane = threadIdx.x & 31;
#pragma unroll
  for (int s = 1; s < 32; s <<= 1) {
    uint32_t t = __shfl_up_sync(0xffffffffu, v, s);
    if (lane >= static_cast<uint32_t>(s)) v += t;
  }
  return v;
}
__device__ __forceinline__ uint64_t warp_inclusive_add64(uint64_t v) {
  const uint32_t lane = threadIdx.x & 31;
#pragma unroll
  for (int s = 1; s < 32; s <<= 1) {
    uint64_t t = __shfl_up_sync(0xffffffffu, v, s);
    if (lane >= static_cast<uint32_t>(s)) v += t;
  }
  return v;
}

}  // namespace bmr
