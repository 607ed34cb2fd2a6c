// Sampled popular terms: the paper treats "popular" terms, "the most
// frequently occurring terms", apart from the rest and decides membership on a sample, "1MB out of
// every 1GB".  B200 re-design (opt-in, WJ_FLAG_HOT_TERMS): per chunk, the first
// 1 MiB of its documents is tokenised with the same kernels and the <= 64 most frequent terms
// (>= 16 occurrences, <= 11 bytes) become hot; k_hot_seed claims their slots in the chunk table first,
// with the hot id in the slot's k1 (bits 57..63).  k_tok_emit counts hot tokens in a dense (hot term x
// document) matrix instead of the (slot, docID) stream (they leave holes there), so the sort and
// run-length passes never see them; k_hot_scatter turns each matrix row into the term's partial
// list (docIDs ascending by construction).  The result is unchanged.
#pragma once
#include "common.cuh"
#include "tokenize.cuh"
#include "dict.cuh"
#include "scan.cuh"

namespace wj {

constexpr uint32_t kHotMax = kHotMaxH;  // hot ids 1..64 (tokenize.cuh)
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


// thread i seeds hot id i + 1: claims the term's slot in the chunk table with the id in k1 bits 57..
__global__ void k_hot_seed(const ulonglong2* hk, const uint32_t* H, Slot* table, uint32_t* slot_ref, uint32_t cap,
                           uint32_t* hot_slot, uint32_t* overflow) {
  const uint32_t i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= *H) return;
  const uint32_t id = i + 1;
  const uint64_t k0 = hk[i].x, k1 = hk[i].y | ((uint64_t)id << kHotShift);
  const uint32_t len = (uint32_t)k0 & 0xFFu;
  const uint32_t w0 = (uint32_t)(k0 >> 32), w1 = (uint32_t)hk[i].y, w2 = (uint32_t)(hk[i].y >> 32) & 0xFFFFFFu;
  const uint64_t h = term_hash16(w0, w1, w2, 0u, len);
  uint32_t hot = 0;
  hot_slot[id] = table_insert(nullptr, table, slot_ref, 0u, cap, h, k0, k1, 0u, len, nullptr, 0u, overflow, &hot);
}

// sample token counts per slot; the sample's token count is on the device (*n)
__global__ void k_sample_count_dev(const uint32_t* key, const uint32_t* n, uint32_t* cnt) {
  const uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i < *n) atomicAdd(&cnt[key[i] & ((1u << 25) - 1u)], 1u);
}

// the <= Hmax most frequent sampled terms with >= kHotMinCount occurrences: from the end of the
// (count, slot) pairs sorted by count, in descending count order (ties: descending slot); their slot
// words -> hk[0..H), H -> *H_out.  One block of kHotMax threads.
__global__ void k_hot_pick(const uint32_t* sk, const uint32_t* sv, uint32_t Cs, const Slot* table, uint32_t Hmax,
                           ulonglong2* hk, uint32_t* H_out) {
  const uint32_t i = threadIdx.x;
  const bool ok = i < Hmax && i < Cs && sk[Cs - 1 - i] >= kHotMinCount;
  const uint32_t n = __syncthreads_count(ok);  // counts are non-increasing in i: the kept ones are a prefix
  if (ok) hk[i] = *(const ulonglong2*)(table + sv[Cs - 1 - i]);
  if (i == 0) *H_out = n;
}

struct NonZeroU32 {
  const uint32_t* p;
  __device__ __forceinline__ uint32_t operator()(uint64_t i) const { return p[i] != 0u ? 1u : 0u; }
};

// nonzero matrix entries -> the hot terms' partial lists, appended after the chunk's run-length
// postings (*P_rle of them); pos = exclusive scan of the nonzero flags (row-major: term, document)
__global__ void k_hot_scatter(const uint32_t* mat, uint64_t n, uint32_t D, const uint32_t* pos, const uint32_t* P_rle,
                              uint32_t doc_base, uint2* pp) {
  const uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  const uint32_t c = mat[i];
  if (c == 0) return;
  const uint64_t p = (uint64_t)*P_rle + pos[i];
  pp[p] = make_uint2(doc_base + (uint32_t)(i % D), c);
}

// tokens of each hot term (its cf): one block per matrix row
__global__ void k_hot_rowsum(const uint32_t* mat, uint32_t D, uint32_t* cf) {
  const uint32_t* row = mat + (uint64_t)blockIdx.x * D;
  uint32_t s = 0;
  for (uint32_t d = threadIdx.x; d < D; d += blockDim.x) s += row[d];
  uint32_t tot;
  block_exclusive_sum<uint32_t>(s, tot);
  if (threadIdx.x == 0) cf[blockIdx.x] = tot;
}

// P_rle (run-length postings of the stream) is kept in *p_rle; *P becomes the chunk's total postings
__global__ void k_hot_total(const uint32_t* hot_total, uint32_t* P, uint32_t* p_rle) {
  *p_rle = *P;
  *P += *hot_total;
}

}  // namespace wj
