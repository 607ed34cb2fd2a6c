// Common device/host helpers for the sm_100a indexer kernels.
#pragma once
#include <cstdint>
#include <cstdio>
#include <cuda_runtime.h>

namespace wj {

// Table I: 1 special + 10 pure-number + 26 short/special + 26^3 collections.
constexpr uint32_t kCollections = 17613;
constexpr uint32_t kMaxTermLen = 255;
constexpr uint32_t kMiss = 0xFFFFFFFFu;
constexpr int kWarp = 32;

// One B-tree node: Table II field sizes, 512 B in total, degree t = 16 -> at most
// 31 keys and 32 children.  Fields are grouped per 128-byte line by access pattern:
// line 0 {valid term number, 31 x 4-byte cache} is all a descent compares against (one
// coalesced 128 B load per warp, Fig. 7); line 1 {leaf indicator, 31 term-string pointers} is
// read only on a cache tie; line 2 {padding, 31 postings pointers (= termIDs)} on a hit;
// line 3 {32 children} on a miss at an internal node.
struct alignas(128) Node {
  uint32_t count;
  uint32_t cache[31];
  uint32_t leaf;
  uint32_t str[31];
  uint32_t pad;
  uint32_t post[31];
  uint32_t child[32];
};
static_assert(sizeof(Node) == 512, "Table II: a B-tree node is 512 bytes");
static_assert(4 + 31 * 4 + 4 + 31 * 4 + 32 * 4 + 31 * 4 + 4 == 512, "Table II field sizes");

// Chunk-local term table slot (K1 emit): 16 bytes, claimed once by CAS on k0, k1 published after.
//   k0 = len (8 bits) | hash tag (24 bits) << 8 | folded bytes 0-3 << 32      (0 = empty)
//   k1 = folded bytes 4-10 (56 bits) | 1 << 56                                   (0 = unpublished)
// Terms of <= 11 bytes are identified by (k0, k1) alone; longer ones also compare bytes 8.. with
// their first occurrence (offset in a side array written by the inserter before publishing k1).
struct __align__(16) Slot {
  unsigned long long k0;
  unsigned long long k1;
};
constexpr uint32_t kSlotBytes = 11;
// k1 bits 57..63 of a slot seeded with a sampled hot term (k_hot_seed) hold its hot id (1..127)
constexpr int kHotShift = 57;
constexpr unsigned long long kSlotK1Mask = (1ull << kHotShift) - 1ull;

__host__ __device__ inline uint32_t ceil_div32(uint64_t a, uint32_t b) { return (uint32_t)((a + b - 1) / b); }

__device__ __forceinline__ uint32_t lane_id() { return threadIdx.x & 31; }

// ld.acquire.gpu of a 64-bit word: later loads of this thread observe what the releasing writer
// stored before its release (PTX memory model)
__device__ __forceinline__ unsigned long long ld_acquire_u64(const unsigned long long* p) {
  unsigned long long v;
  asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}

// ---- SWAR byte classification (4 bytes per u32, little-endian byte order) -------------------
// Token bytes (reading S1): [0-9] U [A-Z] U [a-z] U [0x80-0xFF].  Returns bit i = byte i.
// a + c as an integer multiply-add: ptxas issues it on the FMA pipe (VIADD / IMAD) instead of the ALU
// pipe's IADD3, and the SWAR classification below is ALU-bound (k_tok_count: ALU 82% of peak)
__device__ __forceinline__ uint32_t fma_add(uint32_t a, uint32_t c) {
  uint32_t r;
  asm("mad.lo.u32 %0, %1, 1, %2;" : "=r"(r) : "r"(a), "r"(c));
  return r;
}
// a * m + c as one multiply-add (FMA pipe)
__device__ __forceinline__ uint32_t fma_mad(uint32_t a, uint32_t m, uint32_t c) {
  uint32_t r;
  asm("mad.lo.u32 %0, %1, %2, %3;" : "=r"(r) : "r"(a), "r"(m), "r"(c));
  return r;
}
__device__ __forceinline__ uint32_t tokmask4(uint32_t x) {
  const uint32_t hi = x & 0x80808080u;
  const uint32_t lo = x & 0x7F7F7F7Fu;
  const uint32_t ge0 = fma_add(lo, 0x50505050u);  // bit7: lo >= '0'
  const uint32_t le9 = ~fma_add(lo, 0x46464646u); // bit7: lo <  ':'
  const uint32_t l = lo | 0x20202020u;
  const uint32_t gea = fma_add(l, 0x1F1F1F1Fu);   // bit7: l >= 'a'
  const uint32_t lez = ~fma_add(l, 0x05050505u);  // bit7: l <  '{'
  const uint32_t t = (hi | ((ge0 & le9) | (gea & lez))) & 0x80808080u;
  // bits 7, 15, 23, 31 -> bits 0..3 in one multiply-high (no carries: the partial products are disjoint)
  return __umulhi(t, (1u << 25) | (1u << 18) | (1u << 11) | (1u << 4)) & 15u;
}
// ASCII A-Z -> a-z (reading S2), other bytes unchanged.
__device__ __forceinline__ uint32_t lower4(uint32_t x) {
  const uint32_t hi = x & 0x80808080u;
  const uint32_t lo = x & 0x7F7F7F7Fu;
  const uint32_t up = (lo + 0x3F3F3F3Fu) & ~(lo + 0x25252525u) & ~hi & 0x80808080u;
  return x | (up >> 2);
}
// bit7 of each byte set iff the byte is '0'..'9'.
__device__ __forceinline__ uint32_t digit4(uint32_t x) {
  const uint32_t hi = x & 0x80808080u;
  const uint32_t lo = x & 0x7F7F7F7Fu;
  return (lo + 0x50505050u) & ~(lo + 0x46464646u) & ~hi & 0x80808080u;
}
__device__ __forceinline__ uint32_t bswap32(uint32_t x) { return __byte_perm(x, 0, 0x0123); }

// Reads the k-th little-endian 4-byte word of the lower-cased term text[s..s+len) (zero-padded past
// len).  Loads aligned words only, so it never touches bytes outside the words holding the term.
struct TermWords {
  const uint32_t* wp;
  uint32_t sh, len, nsrc;
  __device__ __forceinline__ TermWords(const uint8_t* text, uint64_t s, uint32_t len_) {
    const uintptr_t a = (uintptr_t)(text + s);
    wp = (const uint32_t*)(a & ~(uintptr_t)3);
    sh = (uint32_t)(a & 3) * 8;
    len = len_;
    nsrc = ((uint32_t)(a & 3) + len_ + 3) >> 2;
  }
  __device__ __forceinline__ uint32_t word(uint32_t k) const {
    const uint32_t lo = __ldg(wp + k);
    const uint32_t hi = (k + 1 < nsrc) ? __ldg(wp + k + 1) : 0u;
    uint32_t w = __funnelshift_r(lo, hi, sh);
    const uint32_t rem = len - 4 * k;
    if (rem < 4) w &= (1u << (rem * 8)) - 1u;
    return lower4(w);
  }
};

__device__ __forceinline__ uint64_t fmix64(uint64_t k) {
  k ^= k >> 33; k *= 0xff51afd7ed558ccdull; k ^= k >> 33; k *= 0xc4ceb9fe1a85ec53ull; k ^= k >> 33;
  return k;
}

}  // namespace wj

#define WJ_CUDA_CHECK(expr)                                                          \
  do {                                                                               \
    cudaError_t _e = (expr);                                                         \
    if (_e != cudaSuccess) throw ::wj::CudaError(_e, #expr, __FILE__, __LINE__);     \
  } while (0)

namespace wj {
struct CudaError {
  cudaError_t err;
  const char* expr;
  const char* file;
  int line;
  CudaError(cudaError_t e, const char* x, const char* f, int l) : err(e), expr(x), file(f), line(l) {}
};
}  // namespace wj
