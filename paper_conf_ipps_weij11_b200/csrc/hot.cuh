// Sampled popular terms: the paper splits "popular" trie collections, "containing
// the most frequently occurring terms", from the rest and decides membership on a sample, "1MB out of
// every 1GB".  B200 re-design: per chunk, the first 1 MiB of its documents is
// tokenised with the same kernels, the <= 256 most frequent terms (>= 16 occurrences, <= 11 bytes) are
// "hot"; in k_tok_emit a hot token does not enter the (slot, docID) stream (it leaves a hole) but
// increments a dense (hot term x document) counter; afterwards every nonzero (term, document) counter
// becomes one stream element carrying its count (count <= 127 per element).  The result is unchanged;
// the sort and run-length passes see ~30% fewer elements on Zipf text.
#pragma once
#include "common.cuh"
#include "tokenize.cuh"
#include "dict.cuh"

namespace wj {

constexpr uint32_t kHotMax = 256;
constexpr uint32_t kHotTable = 1024;  // open-addressing slots of the hot lookup table
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

// one thread: insert the hot terms into the chunk table (their slots) and into the hot lookup table
__global__ void k_hot_build(const ulonglong2* hk, uint32_t H, Slot* table, uint32_t* slot_ref, uint32_t cap,
                            HotEntry* hot, uint32_t* hot_slot, uint32_t* overflow) {
  if (threadIdx.x != 0 || blockIdx.x != 0) return;
  for (uint32_t i = 0; i < kHotTable; ++i) hot[i] = HotEntry{0ull, 0ull, 0u, 0u, {0u, 0u}};
  for (uint32_t id = 0; id < H; ++id) {
    const uint64_t k0 = hk[id].x, k1 = hk[id].y;
    const uint32_t len = (uint32_t)k0 & 0xFFu;
    const uint32_t w0 = (uint32_t)(k0 >> 32), w1 = (uint32_t)k1, w2 = (uint32_t)(k1 >> 32) & 0xFFFFFFu;
    const uint64_t h = term_hash16(w0, w1, w2, 0u, len);
    const uint32_t s = table_insert(nullptr, table, slot_ref, cap, h, k0, k1, 0u, len, nullptr, 0u, overflow);
    hot_slot[id] = s;
    uint32_t j = (uint32_t)(h >> 20) & (kHotTable - 1);
    while (hot[j].k0 != 0) j = (j + 1) & (kHotTable - 1);
    hot[j] = HotEntry{k0, k1, id, s, {0u, 0u}};
  }
}

struct HotElemCount {
  const uint32_t* tf;
  __device__ __forceinline__ uint32_t operator()(uint64_t i) const { return (tf[i] + 126u) / 127u; }
};

// nonzero (hot term, document) counters -> stream elements (slot | count << 25, docID), term-major
__global__ void k_hot_elems(const uint32_t* tf, uint64_t n, uint32_t D, const uint32_t* off, const uint32_t* hot_slot,
                            uint32_t doc_base, uint32_t* out_key, uint32_t* out_doc) {
  const uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  uint32_t t = tf[i];
  if (t == 0) return;
  const uint32_t id = (uint32_t)(i / D), d = (uint32_t)(i % D);
  uint32_t p = off[i];
  while (t) {
    const uint32_t c = t < 127u ? t : 127u;
    out_key[p] = hot_slot[id] | (c << 25);
    out_doc[p] = doc_base + d;
    ++p;
    t -= c;
  }
}

}  // namespace wj
