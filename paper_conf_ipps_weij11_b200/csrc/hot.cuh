// Sampled popular terms: the paper treats "popular" terms, "the most
// frequently occurring terms", apart from the rest and decides membership on a sample, "1MB out of
// every 1GB".  B200 re-design: per chunk, the first 1 MiB of its documents is
// tokenised with the same kernels and the <= 127 most frequent terms (>= 16 occurrences, <= 11
// bytes) become hot; k_hot_seed claims their slots in the chunk table first, with the hot id in the
// slot's k1 (bits 57..63).  In k_tok_emit the tokens of one hot term that fall in one document of a
// warp's 8 KB window become ONE stream element carrying their count (the other tokens leave holes),
// so the sort and run-length passes see fewer elements (0.75 N on config 2).  The result is unchanged.
#pragma once
#include "common.cuh"
#include "tokenize.cuh"
#include "dict.cuh"

namespace wj {

constexpr uint32_t kHotMax = 127;   // hot ids 1..127
constexpr uint32_t kHotMinCount = 16;

// hash of a term of <= 16 bytes from its folded words: identical to k_tok_emit's
__device__ __forceinline__ uint64_t term_hash16(uint32_t w0, uint32_t w1, uint32_t w2, uint32_t w3, uint32_t len) {
  uint32_t h = hash_init(len);
  h = hash_mix(h, w0);
  h = hash_mix(h, w1);
  h = hash_mix(h, w2);
  h = hash_mix(h, w3);
  return hash_fin(h);
}

// sample documents: doc_off prefix with the last document clipped at S
__global__ void k_sample_docs(const uint64_t* doc_off, uint64_t n_docs, uint64_t S, uint64_t* out, uint64_t* n_out) {
  if (threadIdx.x != 0 || blockIdx.x != 0) return;
  uint64_t lo = 0, hi = n_docs;  // number of documents starting before S
  while (lo < hi) {
    const uint64_t mid = (lo + hi) >> 1;
    if (doc_off[mid] < S) lo = mid + 1; else hi = mid;
  }
  *n_out = lo;
}

__global__ void k_sample_docs_copy(const uint64_t* doc_off, uint64_t nd, uint64_t S, uint64_t* out) {
  const uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i > nd) return;
  out[i] = i == nd ? S : doc_off[i];
}

__global__ void k_sample_count(const uint32_t* key, uint64_t n, uint32_t* cnt) {
  const uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i < n) atomicAdd(&cnt[key[i] & ((1u << 25) - 1u)], 1u);
}

// sampled tokens per trie collection (balanced owner map): hist[bucket(slot term)] += count
__global__ void k_sample_buckets(const Slot* table, const uint32_t* slot_ref, const uint32_t* cnt, uint32_t C,
                                 const uint8_t* text, unsigned long long* hist) {
  const uint32_t i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= C || cnt[i] == 0) return;
  const uint32_t len = (uint32_t)table[i].k0 & 0xFFu;
  const TermInfo ti = term_info(text, slot_ref[i], len);
  atomicAdd(&hist[ti.bucket], (unsigned long long)cnt[i]);
}

// candidates: count if the term is short enough to be identified by its slot bytes, else 0
__global__ void k_sample_cand(const Slot* table, const uint32_t* cnt, uint32_t C, uint32_t* ckey, uint32_t* cval) {
  const uint32_t i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= C) return;
  const uint64_t k0 = table[i].k0;
  const uint32_t len = (uint32_t)k0 & 0xFFu;
  ckey[i] = (k0 != 0 && len <= kSlotBytes) ? cnt[i] : 0u;
  cval[i] = i;
}

__global__ void k_hot_extract(const Slot* table, const uint32_t* slots, uint32_t H, ulonglong2* hk) {
  const uint32_t i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i < H) hk[i] = *(const ulonglong2*)(table + slots[i]);
}

// thread i seeds hot id i + 1: claims the term's slot in the chunk table with the id in k1 bits 57..
__global__ void k_hot_seed(const ulonglong2* hk, uint32_t H, Slot* table, uint32_t* slot_ref, uint32_t cap,
                           uint32_t* hot_slot, uint32_t* overflow) {
  const uint32_t i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= H) return;
  const uint32_t id = i + 1;
  const uint64_t k0 = hk[i].x, k1 = hk[i].y | ((uint64_t)id << kHotShift);
  const uint32_t len = (uint32_t)k0 & 0xFFu;
  const uint32_t w0 = (uint32_t)(k0 >> 32), w1 = (uint32_t)hk[i].y, w2 = (uint32_t)(hk[i].y >> 32) & 0xFFFFFFu;
  const uint64_t h = term_hash16(w0, w1, w2, 0u, len);
  uint32_t hot = 0;
  hot_slot[id] = table_insert(nullptr, table, slot_ref, cap, h, k0, k1, 0u, len, nullptr, 0u, overflow, &hot);
}

}  // namespace wj
