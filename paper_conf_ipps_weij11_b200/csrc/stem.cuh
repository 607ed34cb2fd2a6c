// Parser Steps 3-4 on the GPU ("stems the tokens using the Porter stemmer",
// P:141 "removes stop words using a stop word list"; reading S20 in DESIGN.md §3).
//
// Placement: a term's stem depends only on the term, so the stemmer runs on the chunk's UNIQUE
// surface terms after K1's dedup (≈3% of the tokens on config 2), never per token:
//   1. k_stem_terms: unique surface term u -> its stem, written into a "stem text" at
//      off[u] = Σ_{v<u} (len_v + 1), padded with spaces to len_u + 1 bytes (a stem is never longer
//      than its term and never empty); a stem that is a stop word (Step 4 after Step 3) writes
//      only spaces and keep[u] = 0, so the stem text holds one token per KEPT unique term, in
//      unique order (token tidx[u] = Σ_{v<u} keep[v]);
//   2. the stem text goes through the same K1 tokenizer/dedup (one document) -> unique stems,
//      which are all the dictionary (K3/K4) or the owner exchange ever sees;
//   3. k_norm_map composes surface slot -> unique surface term -> stem token -> unique stem, with
//      kDropBit for stop words, and k_drop_count / k_drop_write compact those tokens out of the
//      chunk's (slot, docID) stream (dropped tokens do not count in n_tokens, S20).
//
// The stemmer is M.F. Porter, "An algorithm for suffix stripping", Program 14(3):130-137, 1980:
// the rule lists of the 1980 paper (Step 2 "abli"->"able", no "logi"), and the paper's reading of
// each step's list: only the LONGEST matching suffix of a step is a candidate; if its condition
// fails the step does nothing.  Reading S20: only terms of >= 3 bytes made only of a-z are stemmed.
#pragma once
#include "common.cuh"

namespace wj {

constexpr uint32_t kDropBit = 0x80000000u;  // chunk map value flag: the token is a stop word

namespace porter1980 {

__device__ __forceinline__ bool vowel_letter(uint8_t c) {
  return c == 'a' || c == 'e' || c == 'i' || c == 'o' || c == 'u';
}

// Porter's consonant: a letter other than a, e, i, o, u, and other than y preceded by a consonant.
// A run of y's alternates, so walk back over the run instead of recursing.
__device__ __forceinline__ bool is_cons(const uint8_t* b, int i) {
  bool flip = false;
  for (;;) {
    const uint8_t c = b[i];
    if (vowel_letter(c)) return flip;
    if (c != 'y' || i == 0) return !flip;
    flip = !flip;
    --i;
  }
}

// m of [C](VC)^m[V] over b[0, n): the number of vowel-run -> consonant transitions
__device__ __forceinline__ int measure_m(const uint8_t* b, int n) {
  int m = 0;
  bool in_v = false;
  for (int i = 0; i < n; ++i) {
    if (!is_cons(b, i)) in_v = true;
    else if (in_v) { ++m; in_v = false; }
  }
  return m;
}

__device__ __forceinline__ bool contains_vowel(const uint8_t* b, int n) {  // *v*
  for (int i = 0; i < n; ++i)
    if (!is_cons(b, i)) return true;
  return false;
}

__device__ __forceinline__ bool ends_double_cons(const uint8_t* b, int n) {  // *d
  return n >= 2 && b[n - 1] == b[n - 2] && is_cons(b, n - 1);
}

__device__ __forceinline__ bool ends_cvc(const uint8_t* b, int n) {  // *o
  if (n < 3 || !is_cons(b, n - 1) || is_cons(b, n - 2) || !is_cons(b, n - 3)) return false;
  const uint8_t c = b[n - 1];
  return c != 'w' && c != 'x' && c != 'y';
}

// does b[0, n) end with the NUL-terminated s?  returns its length, or 0
__device__ __forceinline__ int suffix_len(const uint8_t* b, int n, const char* s) {
  int l = 0;
  while (s[l]) ++l;
  if (l > n) return 0;
  for (int i = 0; i < l; ++i)
    if (b[n - l + i] != (uint8_t)s[i]) return 0;
  return l;
}

__device__ __forceinline__ int put(uint8_t* b, int n, const char* s) {  // append s, return new length
  while (*s) b[n++] = (uint8_t)*s++;
  return n;
}

struct Repl {
  char from[8];
  char to[6];
};

// Step 2 (condition m > 0), Porter 1980 table
__constant__ Repl kS2[20] = {{"ational", "ate"}, {"tional", "tion"}, {"enci", "ence"},  {"anci", "ance"},
                             {"izer", "ize"},    {"abli", "able"},   {"alli", "al"},    {"entli", "ent"},
                             {"eli", "e"},       {"ousli", "ous"},   {"ization", "ize"}, {"ation", "ate"},
                             {"ator", "ate"},    {"alism", "al"},    {"iveness", "ive"}, {"fulness", "ful"},
                             {"ousness", "ous"}, {"aliti", "al"},    {"iviti", "ive"},  {"biliti", "ble"}};
// Step 3 (condition m > 0)
__constant__ Repl kS3[7] = {{"icate", "ic"}, {"ative", ""}, {"alize", "al"}, {"iciti", "ic"},
                            {"ical", "ic"},  {"ful", ""},   {"ness", ""}};
// Step 4 (condition m > 1; "ion" also needs the stem to end in s or t)
__constant__ char kS4[19][6] = {"al",  "ance", "ence", "er",  "ic",  "able", "ible", "ant", "ement", "ment",
                                "ent", "ion",  "ou",   "ism", "ate", "iti",  "ous",  "ive", "ize"};

// longest matching entry of a replacement list; replaced when m(stem) > 0
template <int N>
__device__ __forceinline__ int replace_longest(uint8_t* b, int n, const Repl (&r)[N]) {
  int best = -1, bl = 0;
  for (int i = 0; i < N; ++i) {
    const int l = suffix_len(b, n, r[i].from);
    if (l > bl) { bl = l; best = i; }
  }
  if (best < 0 || measure_m(b, n - bl) == 0) return n;
  return put(b, n - bl, r[best].to);
}

// Porter (1980), Steps 1a-5b, in place on b[0, n); returns the stem length (1 <= stem <= n)
__device__ int stem(uint8_t* b, int n) {
  // Step 1a
  if (suffix_len(b, n, "sses") || suffix_len(b, n, "ies")) n -= 2;
  else if (suffix_len(b, n, "ss")) {}
  else if (suffix_len(b, n, "s")) n -= 1;
  // Step 1b
  bool again = false;
  if (suffix_len(b, n, "eed")) {
    if (measure_m(b, n - 3) > 0) n -= 1;
  } else if (suffix_len(b, n, "ed")) {
    if (contains_vowel(b, n - 2)) { n -= 2; again = true; }
  } else if (suffix_len(b, n, "ing")) {
    if (contains_vowel(b, n - 3)) { n -= 3; again = true; }
  }
  if (again) {
    if (suffix_len(b, n, "at") || suffix_len(b, n, "bl") || suffix_len(b, n, "iz")) {
      b[n++] = 'e';
    } else if (ends_double_cons(b, n)) {
      const uint8_t c = b[n - 1];
      if (c != 'l' && c != 's' && c != 'z') --n;
    } else if (measure_m(b, n) == 1 && ends_cvc(b, n)) {
      b[n++] = 'e';
    }
  }
  // Step 1c
  if (b[n - 1] == 'y' && contains_vowel(b, n - 1)) b[n - 1] = 'i';
  // Steps 2, 3
  n = replace_longest(b, n, kS2);
  n = replace_longest(b, n, kS3);
  // Step 4
  {
    int best = -1, bl = 0;
    for (int i = 0; i < 19; ++i) {
      const int l = suffix_len(b, n, kS4[i]);
      if (l > bl) { bl = l; best = i; }
    }
    if (best >= 0 && measure_m(b, n - bl) > 1) {
      const bool ion = best == 11;
      if (!ion || (n - bl > 0 && (b[n - bl - 1] == 's' || b[n - bl - 1] == 't'))) n -= bl;
    }
  }
  // Step 5a
  if (b[n - 1] == 'e') {
    const int m = measure_m(b, n - 1);
    if (m > 1 || (m == 1 && !ends_cvc(b, n - 1))) --n;
  }
  // Step 5b
  if (b[n - 1] == 'l' && ends_double_cons(b, n) && measure_m(b, n) > 1) --n;
  return n;
}

__device__ __forceinline__ bool stemmable(const uint8_t* b, int n) {  // reading S20
  if (n < 3) return false;
  for (int i = 0; i < n; ++i)
    if (b[i] < 'a' || b[i] > 'z') return false;
  return true;
}

}  // namespace porter1980

// Stop-word key: bytes 0-7 big-endian in hi, bytes 8-14 big-endian then the length in lo; terms
// longer than 15 bytes are never stop words (the longest listed word has 12 letters).
__host__ __device__ inline void stop_key(const uint8_t* b, uint32_t n, unsigned long long* hi, unsigned long long* lo) {
  unsigned long long h = 0, l = 0;
  for (uint32_t i = 0; i < 8; ++i) h = (h << 8) | (i < n ? b[i] : 0u);
  for (uint32_t i = 8; i < 15; ++i) l = (l << 8) | (i < n ? b[i] : 0u);
  *hi = h;
  *lo = (l << 8) | n;
}

// binary search in the sorted stop keys (ulonglong2 {hi, lo})
__device__ __forceinline__ bool is_stop(const ulonglong2* keys, uint32_t nk, const uint8_t* b, uint32_t n) {
  if (n > 15 || nk == 0) return false;
  unsigned long long hi, lo;
  stop_key(b, n, &hi, &lo);
  uint32_t a = 0, e = nk;
  while (a < e) {
    const uint32_t m = (a + e) >> 1;
    const ulonglong2 k = keys[m];
    if (k.x < hi || (k.x == hi && k.y < lo)) a = m + 1;
    else e = m;
  }
  return a < nk && keys[a].x == hi && keys[a].y == lo;
}

// folded bytes of unique term u into b (u_w holds bytes 0-10 for terms <= 11 bytes)
__device__ __forceinline__ void unique_bytes(const uint4* u_w, const uint32_t* u_ref, const uint8_t* text, uint32_t u,
                                             uint32_t len, uint8_t* b) {
  if (len <= kSlotBytes) {
    const uint4 w = u_w[u];
    const uint32_t ws[3] = {w.x, w.y, w.z};
    for (uint32_t i = 0; i < len; ++i) b[i] = (uint8_t)(ws[i >> 2] >> (8 * (i & 3)));
  } else {
    const TermWords tw(text, u_ref[u], len);
    for (uint32_t k = 0; 4 * k < len; ++k) {
      const uint32_t w = tw.word(k);
      for (uint32_t j = 0; j < 4 && 4 * k + j < len; ++j) b[4 * k + j] = (uint8_t)(w >> (8 * j));
    }
  }
}

constexpr uint32_t kElemSlotMask = (1u << 25) - 1u;  // stream element = slot | count << 25

struct LenPlus1 {
  const uint32_t* len;
  __device__ __forceinline__ uint64_t operator()(uint64_t i) const { return (uint64_t)len[i] + 1; }
};

// 1. unique surface term u -> its stem (stem != 0) at off[u] of the stem text, padded with spaces
//    to len_u + 1 bytes; a stop word (keys != nullptr) leaves only spaces and keep[u] = 0
__global__ void k_stem_terms(const uint4* u_w, const uint32_t* u_ref, const uint32_t* u_len, const uint8_t* text,
                             uint32_t U, const uint64_t* off, uint8_t* out, int do_stem, const ulonglong2* keys,
                             uint32_t nk, uint32_t* keep) {
  const uint32_t u = blockIdx.x * blockDim.x + threadIdx.x;
  if (u >= U) return;
  uint8_t b[kMaxTermLen + 1];
  const uint32_t len = u_len[u];
  unique_bytes(u_w, u_ref, text, u, len, b);
  uint32_t n = len;
  if (do_stem && porter1980::stemmable(b, (int)len)) n = (uint32_t)porter1980::stem(b, (int)len);
  const bool stop = keys && is_stop(keys, nk, b, n);
  uint8_t* o = out + off[u];
  uint32_t i = 0;
  if (!stop)
    for (; i < n; ++i) o[i] = b[i];
  for (; i <= len; ++i) o[i] = ' ';
  keep[u] = stop ? 0u : 1u;
}

// stop list words (packed, offsets) -> keys of their stems (do_stem) or of the words themselves
__global__ void k_stop_keys(const uint8_t* words, const uint32_t* woff, uint32_t nw, int do_stem, ulonglong2* keys) {
  const uint32_t i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= nw) return;
  uint8_t b[32];
  const uint32_t len = min(woff[i + 1] - woff[i], 31u);
  for (uint32_t j = 0; j < len; ++j) b[j] = words[woff[i] + j];
  uint32_t n = len;
  if (do_stem && porter1980::stemmable(b, (int)len)) n = (uint32_t)porter1980::stem(b, (int)len);
  unsigned long long hi, lo;
  stop_key(b, n, &hi, &lo);
  keys[i] = make_ulonglong2(hi, lo);
}

// debug entry (index_debug_stem): word i of a packed list -> its stem at the same offset
__global__ void k_stem_words(const uint8_t* words, const uint32_t* woff, uint32_t nw, uint8_t* out,
                             uint32_t* out_len) {
  const uint32_t i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= nw) return;
  uint8_t b[kMaxTermLen + 1];
  const uint32_t len = woff[i + 1] - woff[i];
  for (uint32_t j = 0; j < len; ++j) b[j] = words[woff[i] + j];
  uint32_t n = len;
  if (porter1980::stemmable(b, (int)len)) n = (uint32_t)porter1980::stem(b, (int)len);
  for (uint32_t j = 0; j < n; ++j) out[woff[i] + j] = b[j];
  out_len[i] = n;
}

// 2. surface slot s -> index of its stem among the chunk's unique stems (kDropBit: stop word;
//    0 for empty slots).  The kept surface term u is token tidx[u] of the stem text, whose slot in
//    the stem table is stem_slot[tidx[u]].
__global__ void k_norm_map(const Slot* table1, const uint32_t* uid1, uint32_t C1, const uint32_t* keep,
                           const uint32_t* tidx, const uint32_t* stem_slot, const uint32_t* uid2, uint32_t* m1) {
  const uint32_t s = blockIdx.x * blockDim.x + threadIdx.x;
  if (s >= C1) return;
  uint32_t v = 0;
  if (table1[s].k0) {
    const uint32_t u = uid1[s];
    v = keep[u] ? uid2[stem_slot[tidx[u]] & kElemSlotMask] : kDropBit;
  }
  m1[s] = v;
}

// 3. surface slot -> termID of its stem (the chunk's postings map)
__global__ void k_norm_tid_map(const uint32_t* m1, uint32_t C1, const uint32_t* u_tid, uint32_t* map) {
  const uint32_t s = blockIdx.x * blockDim.x + threadIdx.x;
  if (s < C1) map[s] = __ldg(&u_tid[m1[s]]);
}

// 4b. stable compaction of the chunk's stream: keep element i iff map[slot[i]] has no kDropBit.
//     Tiles of kDropTile elements, kDropItems consecutive per thread.
constexpr int kDropThreads = 256;
constexpr int kDropItems = 8;
constexpr uint32_t kDropTile = kDropThreads * kDropItems;

__global__ void __launch_bounds__(kDropThreads) k_drop_count(const uint32_t* slot, uint64_t n, const uint32_t* map,
                                                            uint32_t* tile_keep) {
  const uint64_t base = (uint64_t)blockIdx.x * kDropTile + (uint64_t)threadIdx.x * kDropItems;
  uint32_t c = 0;
#pragma unroll
  for (int k = 0; k < kDropItems; ++k)
    if (base + k < n && !(__ldg(&map[slot[base + k] & kElemSlotMask]) & kDropBit)) ++c;
  c = __reduce_add_sync(0xffffffffu, c);
  __shared__ uint32_t ws[kDropThreads / 32];
  if (lane_id() == 0) ws[threadIdx.x >> 5] = c;
  __syncthreads();
  if (threadIdx.x == 0) {
    uint32_t t = 0;
    for (int w = 0; w < kDropThreads / 32; ++w) t += ws[w];
    tile_keep[blockIdx.x] = t;
  }
}

__global__ void __launch_bounds__(kDropThreads) k_drop_write(const uint32_t* slot, const uint32_t* doc, uint64_t n,
                                                            const uint32_t* map, const uint32_t* tile_off,
                                                            uint32_t* slot_out, uint32_t* doc_out) {
  const uint64_t base = (uint64_t)blockIdx.x * kDropTile + (uint64_t)threadIdx.x * kDropItems;
  uint32_t keep = 0, c = 0;
  uint32_t sv[kDropItems], dv[kDropItems];
#pragma unroll
  for (int k = 0; k < kDropItems; ++k) {
    sv[k] = 0;
    dv[k] = 0;
    if (base + k < n) {
      sv[k] = slot[base + k];
      dv[k] = doc[base + k];
      if (!(__ldg(&map[sv[k] & kElemSlotMask]) & kDropBit)) { keep |= 1u << k; ++c; }
    }
  }
  __shared__ uint32_t ws[kDropThreads / 32 + 1];
  uint32_t inc = c;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const uint32_t t = __shfl_up_sync(0xffffffffu, inc, o);
    if ((int)lane_id() >= o) inc += t;
  }
  if (lane_id() == 31) ws[threadIdx.x >> 5] = inc;
  __syncthreads();
  uint32_t wbase = 0;
  for (int w = 0; w < (int)(threadIdx.x >> 5); ++w) wbase += ws[w];
  uint32_t pos = tile_off[blockIdx.x] + wbase + inc - c;
#pragma unroll
  for (int k = 0; k < kDropItems; ++k)
    if (keep >> k & 1u) {
      slot_out[pos] = sv[k];
      doc_out[pos] = dv[k];
      ++pos;
    }
}

// dropped chunk-map entries -> 0 (no kept element refers to them; keeps the rank composition in range)
__global__ void k_clear_drop(uint32_t* map, uint32_t C) {
  const uint32_t s = blockIdx.x * blockDim.x + threadIdx.x;
  if (s < C && (map[s] & kDropBit)) map[s] = 0;
}

}  // namespace wj
