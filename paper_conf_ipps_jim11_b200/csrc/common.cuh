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
__device__ __forceinline__ void mbar_arrive_cnt(uint64_t* bar, uint32_t cnt) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(cnt) : "memory");
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
// try_wait with an explicit suspend-time hint (ns): the waiting warp stays suspended (instead of
// re-polling and taking issue slots from the compute warps) until the phase completes or the
// hint expires.
__device__ __forceinline__ bool mbar_try_wait_hint(uint64_t* bar, uint32_t parity, uint32_t ns) {
  uint32_t ok;
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2, %3;\n\t"
      "selp.u32 %0, 1, 0, p;\n\t}"
      : "=r"(ok)
      : "r"(smem_u32(bar)), "r"(parity), "r"(ns)
      : "memory");
  return ok != 0;
}
__device__ __forceinline__ void mbar_wait_idle(uint64_t* bar, uint32_t parity, uint32_t ns = 20000) {
  while (!mbar_try_wait_hint(bar, parity, ns)) {
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
// The same with an L2 evict-first policy: streamed input read once (its lines should leave L2
// before the data the kernel revisits, e.g. the WordCount count table)
__device__ __forceinline__ uint64_t l2_policy_evict_first() {
  uint64_t p;
  asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
  return p;
}
__device__ __forceinline__ void tma_load_1d_stream(void* smem_dst, const void* gsrc, uint32_t bytes, uint64_t* bar,
                                                   uint64_t policy) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], %4;" ::"r"(
          smem_u32(smem_dst)),
      "l"(gsrc), "r"(bytes), "r"(smem_u32(bar)), "l"(policy)
      : "memory");
}
__device__ __forceinline__ void fence_proxy_async_shared() {
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}
__device__ __forceinline__ void named_bar_sync(uint32_t id, uint32_t nthreads) {
  asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(nthreads) : "memory");
}
// Fire-and-forget global add (REDG).  A plain atomicAdd whose result is unused was compiled to
// ATOMG with an RZ destination inside the Map's divergent loops, and the loop's next write to the
// address registers then waited on the atomic's long scoreboard (ncu C5 round 2: 22% of the
// WordCount Map's stall samples at one branch).
__device__ __forceinline__ void red_add_u32(uint32_t* p, uint32_t v) {
  asm volatile("red.relaxed.gpu.global.add.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
// shared-window (32-bit address) accessors
__device__ __forceinline__ uint32_t lds_u32(uint32_t a) {   // stage bytes: constant while read
  uint32_t v;
  asm("ld.shared.u32 %0, [%1];" : "=r"(v) : "r"(a));
  return v;
}
__device__ __forceinline__ uint32_t lds_volatile_u32(uint32_t a) {
  uint32_t v;
  asm volatile("ld.volatile.shared.u32 %0, [%1];" : "=r"(v) : "r"(a) : "memory");
  return v;
}
__device__ __forceinline__ uint32_t atom_cas_shared_u32(uint32_t a, uint32_t cmp, uint32_t val) {
  uint32_t old;
  asm volatile("atom.shared.cas.b32 %0, [%1], %2, %3;" : "=r"(old) : "r"(a), "r"(cmp), "r"(val) : "memory");
  return old;
}
__device__ __forceinline__ void red_shared_add_u32(uint32_t a, uint32_t v) {
  asm volatile("red.shared.add.u32 [%0], %1;" ::"r"(a), "r"(v) : "memory");
}
// per-thread asynchronous global -> shared copies (LDGSTS): 8 B through L1, 16 B from L2
__device__ __forceinline__ void cp_async_8(void* sdst, const void* gsrc) {
  asm volatile("cp.async.ca.shared.global [%0], [%1], 8;" ::"r"(smem_u32(sdst)), "l"(gsrc) : "memory");
}
__device__ __forceinline__ void cp_async_16(void* sdst, const void* gsrc) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(smem_u32(sdst)), "l"(gsrc) : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
__device__ __forceinline__ void cp_async_wait_all() { asm volatile("cp.async.wait_all;" ::: "memory"); }
__device__ __forceinline__ uint32_t bfind_u32(uint32_t x) {   // index of the highest set bit (x != 0)
  uint32_t r;
  asm("bfind.u32 %0, %1;" : "=r"(r) : "r"(x));
  return r;
}
__device__ __forceinline__ uint32_t lanemask_lt() {
  uint32_t m;
  asm("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
  return m;
}
// acquire load of a shared-memory flag polled by another warp of the CTA
__device__ __forceinline__ uint32_t ld_acquire_cta_shared_u32(const unsigned int* p) {
  uint32_t v;
  asm volatile("ld.acquire.cta.shared::cta.u32 %0, [%1];" : "=r"(v) : "r"(smem_u32(p)) : "memory");
  return v;
}
__device__ __forceinline__ void st_release_cta_shared_u32(unsigned int* p, uint32_t v) {
  asm volatile("st.release.cta.shared::cta.u32 [%0], %1;" ::"r"(smem_u32(p)), "r"(v) : "memory");
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

// `need` (1..8) bytes at p, little-endian, from 8-byte aligned loads only (never touching an
// 8-byte word that holds none of the needed bytes); bytes beyond `need` are unspecified.
__device__ __forceinline__ uint64_t load8(const uint8_t* p, uint32_t need) {
  const uintptr_t a = reinterpret_cast<uintptr_t>(p) & ~static_cast<uintptr_t>(7);
  const uint32_t sh = static_cast<uint32_t>(reinterpret_cast<uintptr_t>(p) & 7u) * 8;
  const uint64_t w0 = __ldg(reinterpret_cast<const unsigned long long*>(a));
  if (sh == 0) return w0;
  uint64_t v = w0 >> sh;
  if (sh / 8 + need > 8) v |= static_cast<uint64_t>(__ldg(reinterpret_cast<const unsigned long long*>(a + 8))) << (64 - sh);
  return v;
}
// hash_bytes of key bytes in global memory, read 8 bytes at a time (same words, same result).
__device__ __forceinline__ uint64_t hash_bytes_g(const uint8_t* p, uint32_t len, uint64_t seed) {
  KeyHash hs(seed, len);
  for (uint32_t k = 0; k < len; k += 8) {
    const uint32_t need = min(8u, len - k);
    uint64_t v = load8(p + k, need);
    if (need < 8) v &= (1ULL << (8 * need)) - 1ULL;
    hs.add(static_cast<uint32_t>(v));
    if (k + 4 < len) hs.add(static_cast<uint32_t>(v >> 32));
  }
  return hs.finish();
}

// Destination rank of a key in the multi-GPU exchange: from the key BYTES, so it is
// the same on every rank and for every code path (partition pass, fused Map flush).
constexpr uint64_t kPartSeed = 0x9A27D11EB200ULL;
__device__ __forceinline__ uint32_t dest_of_bytes(const uint8_t* p, uint32_t len, uint32_t R) {
  return static_cast<uint32_t>(mix64(hash_bytes(p, len, kPartSeed) ^ 0x51ULL) % R);
}
__device__ __forceinline__ uint32_t dest_of_bytes_g(const uint8_t* p, uint32_t len, uint32_t R) {   // global p
  return static_cast<uint32_t>(mix64(hash_bytes_g(p, len, kPartSeed) ^ 0x51ULL) % R);
}
// Sort-key formats.  The key width is 64 bits (II, re-hash slow path) or 48 bits (WC: two LSD
// passes fewer; digits 6 and 7 are then constant and skipped):
//   inline  : keys of <= kInlineMax bytes packed little-endian, length in the 3 bits above them
//             (64: len << 56, <= 7 bytes; 48: len << 40, <= 5 bytes) — injective, top bit clear;
//   hashed  : longer keys -> hash with the top bit of the width forced to 1 (never collides with
//             an inline key); equal hashes are verified byte-for-byte at segment time;
//   sentinel: all ones in the width — flush filler pairs, sorts after every real key.
// The WordCount exact and mid streams (map.cu) use the 6-bit symbol codes of exact_key below.
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

// WordCount exact keys: a WC word is [0-9A-Za-z]+ (C-3 #1), so every symbol has a nonzero 6-bit
// code: '0'-'9' -> 1..10, 'A'-'Z' -> 11..36, 'a'-'z' -> 37..62.  A word of L <= 8 symbols packs
// injectively into 6L bits (symbol i at bits 6i; the highest nonzero code gives the length):
// <= 5 symbols -> 30 bits (four 8-bit LSD digits), 6..8 symbols -> 48 bits (six digits).  Codes
// of 4 bytes at once, arithmetically: code = c - 47 - 7 [c >= 0x40] - 6 [c >= 0x60] (bits 6 and
// 5 of a word byte give its class; two of the five operations run on the FMA pipe).  Bytes past a
// word's end may borrow into the bytes above them, never below, and are masked off by the callers.
__device__ __forceinline__ uint32_t exact_codes4(uint32_t w) {
  const uint32_t s6 = w >> 6, s5 = w >> 5;
  const uint32_t t6 = s6 & 0x01010101u;                 // [c >= 0x40] per byte
  const uint32_t t65 = s6 & s5 & 0x01010101u;           // [c >= 0x60]
  return (w - 0x2F2F2F2Fu) - 7u * t6 - 6u * t65;        // <= 62 per byte for word bytes
}
__device__ __forceinline__ uint64_t exact_key(uint64_t bytes_le, uint32_t len) {   // len 1..8
  uint64_t x = (static_cast<uint64_t>(exact_codes4(static_cast<uint32_t>(bytes_le >> 32))) << 32) |
               exact_codes4(static_cast<uint32_t>(bytes_le));
  if (len < 8) x &= (1ULL << (8 * len)) - 1ULL;
  x = (x & 0x003F003F003F003FULL) | ((x >> 2) & 0x0FC00FC00FC00FC0ULL);   // byte pairs -> 12 bits
  x = (x & 0x00000FFF00000FFFULL) | ((x >> 4) & 0x00FFF00000FFF000ULL);   // -> 24 bits
  x = (x & 0x0000000000FFFFFFULL) | ((x >> 8) & 0x0000FFFFFF000000ULL);   // -> 48 bits
  return x;
}
// The same key for len 1..5 (the exact stream) on 32-bit operations: codes of bytes 0..3 with
// one table permute, byte 4 with a second one, 4 codes packed to 24 bits, code 4 on top.
__device__ __forceinline__ uint32_t exact_key30(uint64_t bytes_le, uint32_t len) {
  uint32_t c = exact_codes4(static_cast<uint32_t>(bytes_le));
  if (len < 4) c &= (1u << (8 * len)) - 1u;
  uint32_t y = (c & 0x003F003Fu) | ((c >> 2) & 0x0FC00FC0u);   // byte pairs -> 12 bits
  y = (y & 0x00000FFFu) | ((y >> 4) & 0x00FFF000u);            // -> 24 bits
  if (len == 5) y |= (exact_codes4(static_cast<uint32_t>(bytes_le >> 32)) & 0xFFu) << 24;
  return y;
}
// Inverse: key bytes little-endian and the length.
__device__ __forceinline__ uint64_t exact_key_bytes(uint64_t key, uint32_t& len) {
  len = key ? static_cast<uint32_t>(63 - __clzll(static_cast<long long>(key))) / 6u + 1u : 0u;
  uint64_t b = 0;
  for (uint32_t i = 0; i < len; ++i) {
    const uint32_t c = static_cast<uint32_t>(key >> (6 * i)) & 63u;
    b |= static_cast<uint64_t>(c <= 10 ? c + 47u : (c <= 36 ? c + 54u : c + 60u)) << (8 * i);
  }
  return b;
}
// key bytes -> sort key (generic pointer), inline / hashed formats
__device__ __forceinline__ uint64_t key_of_bytes(const uint8_t* p, uint32_t len, uint64_t seed, bool weak,
                                                 uint32_t bits) {
  if (len <= inline_max(bits)) {
    uint64_t b = 0;
    for (uint32_t k = 0; k < len; ++k) b |= static_cast<uint64_t>(p[k]) << (8 * k);
    return inline_key(b, len, bits);
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
