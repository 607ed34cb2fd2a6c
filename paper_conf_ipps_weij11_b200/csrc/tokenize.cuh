// K1: warp-cooperative tokenizer / normaliser + chunk-local term dedup (hash table).
//
// Paper: Step 2 "performs tokenization, that is, parses each document into tokens and determines
// the trie index of each resulting term"; "tokenization scans input document character by
// character and hence a trie index can be calculated as a byproduct".  Readings S1 (token
// bytes), S2 (ASCII folding), S4 (drop > 255 bytes), S16 (empty documents).
//
// B200 design: a warp owns a 512-byte segment (16 B per lane, one coalesced 128-bit load per lane),
// classifies bytes with SWAR, finds token starts/ends with funnel shifts and shuffles, and walks
// the document boundaries (doc_off) with a per-warp cursor.  Pass 1 counts kept tokens per
// segment; a scan gives output offsets; pass 2 re-tokenises and, per token, hashes the folded
// bytes into a chunk-local open-addressing table (one 64-bit CAS claims a slot; equal strings are
// confirmed against the first occurrence in the immutable text), so the dictionary (K3/K4) sees
// each distinct term of the chunk once instead of once per token.
#pragma once
#include "common.cuh"

namespace wj {

constexpr int kSegBytes = 512;
constexpr int kTokThreads = 256;
constexpr int kTokWarps = kTokThreads / 32;
constexpr int kSegsPerWarp = 8;

struct ChunkView {
  const uint8_t* text;     // 16-byte aligned device pointer
  uint64_t n_bytes;        // < 2^32
  const uint64_t* doc_off; // device, n_docs + 1 entries
  uint64_t n_docs;
};

struct EmitOut {
  uint64_t* table;         // chunk hash table (u64 slots, 0 = empty)
  uint32_t mask;           // capacity - 1 (power of two)
  uint32_t doc_base;       // global DocID of local document 0
  uint32_t* slot;          // per kept token: table slot
  uint32_t* doc;           // per kept token: global DocID
  uint32_t* dbg_start;     // optional (debug): token start
  uint32_t* dbg_len;       // optional (debug): token length
  uint32_t* overflow;      // set to 1 if a probe sequence exceeded the limit
};

__device__ __forceinline__ uint64_t lower_bound_u64(const uint64_t* a, uint64_t lo, uint64_t hi, uint64_t x) {
  while (lo < hi) {
    uint64_t mid = (lo + hi) >> 1;
    if (a[mid] < x) lo = mid + 1; else hi = mid;
  }
  return lo;
}

__device__ __forceinline__ uint64_t term_hash(const TermWords& tw, uint32_t len) {
  uint64_t h = 0x9E3779B97F4A7C15ull ^ ((uint64_t)len * 0xA0761D6478BD642Full);
  const uint32_t nw = (len + 3) >> 2;
  for (uint32_t k = 0; k < nw; ++k) {
    h = (h ^ tw.word(k)) * 0xff51afd7ed558ccdull;
    h ^= h >> 29;
  }
  return fmix64(h);
}

__device__ __forceinline__ bool term_equal(const uint8_t* text, uint32_t a, uint32_t b, uint32_t len) {
  if (a == b) return true;
  TermWords A(text, a, len), B(text, b, len);
  const uint32_t nw = (len + 3) >> 2;
  for (uint32_t k = 0; k < nw; ++k)
    if (A.word(k) != B.word(k)) return false;
  return true;
}

// Slot word: bits 0-31 start offset of the first occurrence, 32-39 length, 40-63 hash tag.
__device__ __forceinline__ uint32_t table_insert(const uint8_t* text, uint64_t* table, uint32_t mask, uint64_t h,
                                                 uint32_t s, uint32_t len, uint32_t* overflow) {
  const uint64_t mine = (uint64_t)s | ((uint64_t)len << 32) | (h & 0xFFFFFF0000000000ull);
  uint32_t i = (uint32_t)h & mask;
  for (int probe = 0; probe < 8192; ++probe) {
    uint64_t cur = *(volatile uint64_t*)(table + i);
    if (cur == 0) {
      const unsigned long long prev = atomicCAS((unsigned long long*)(table + i), 0ull, (unsigned long long)mine);
      if (prev == 0) return i;
      cur = prev;
    }
    if ((cur >> 32) == (mine >> 32) && term_equal(text, (uint32_t)cur, s, len)) return i;
    i = (i + 1) & mask;
  }
  atomicExch(overflow, 1u);
  return kMiss;
}

// Per-warp view of one segment after classification.
struct SegState {
  uint32_t startm;   // lane-local 16-bit mask of token starts
  uint32_t termm;    // lane-local 16-bit mask of terminators (non-token byte or doc start)
  uint32_t next_t;   // segment-relative position of the first terminator in a later lane (or 0xFFFF)
  uint32_t far_end;  // absolute end of the token running past the segment (valid in the last-start lane)
  uint64_t k_lo, k_hi;  // doc_off boundary index range for this segment
};

// Classifies segment `seg` for the calling warp; kcur = first doc boundary index >= segment start.
__device__ __forceinline__ SegState classify_segment(const ChunkView& cv, uint64_t seg, uint64_t& kcur,
                                                     uint32_t* bnd_smem /* 32 words, this warp */) {
  const uint32_t lane = lane_id();
  const uint64_t s0 = seg * kSegBytes;
  const uint64_t p0 = s0 + 16 * lane;
  uint32_t wv[4];
  if (p0 + 16 <= cv.n_bytes) {
    const uint4 v = __ldg((const uint4*)(cv.text + p0));
    wv[0] = v.x; wv[1] = v.y; wv[2] = v.z; wv[3] = v.w;
  } else {
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      uint32_t x = 0;
#pragma unroll
      for (int b = 0; b < 4; ++b) {
        const uint64_t p = p0 + 4 * q + b;
        if (p < cv.n_bytes) x |= (uint32_t)cv.text[p] << (8 * b);
      }
      wv[q] = x;
    }
  }
  uint32_t tm = tokmask4(wv[0]) | (tokmask4(wv[1]) << 4) | (tokmask4(wv[2]) << 8) | (tokmask4(wv[3]) << 12);
  if (p0 >= cv.n_bytes) tm = 0;
  else if (p0 + 16 > cv.n_bytes) tm &= (1u << (uint32_t)(cv.n_bytes - p0)) - 1u;

  // document boundaries (doc_off[k], 1 <= k < n_docs) inside [s0, s0+512)
  bnd_smem[lane] = 0;
  __syncwarp();
  const uint64_t s1 = s0 + kSegBytes;
  SegState st;
  st.k_lo = kcur;
  for (;;) {
    const uint64_t k = kcur + lane;
    const uint64_t x = (k < cv.n_docs) ? cv.doc_off[k] : ~0ull;
    const bool in = x < s1;
    if (in) atomicOr(&bnd_smem[(uint32_t)(x - s0) >> 4], 1u << ((uint32_t)(x - s0) & 15u));
    const uint32_t b = __ballot_sync(0xffffffffu, in);
    kcur += __popc(b);
    if (b != 0xffffffffu) break;
  }
  st.k_hi = kcur;
  __syncwarp();
  const uint32_t bm = bnd_smem[lane];

  // previous byte's token bit (for lane 0: last byte of the previous segment)
  uint32_t prev = __shfl_up_sync(0xffffffffu, tm >> 15, 1) & 1u;
  if (lane == 0) prev = (s0 > 0 && s0 - 1 < cv.n_bytes) ? ((tokmask4(cv.text[s0 - 1]) & 1u)) : 0u;
  st.startm = tm & ((~((tm << 1) | prev)) | bm) & 0xFFFFu;
  st.termm = (~tm | bm) & 0xFFFFu;

  // first terminator in any later lane
  uint32_t f = st.termm ? (16 * lane + __ffs(st.termm) - 1) : 0xFFFFu;
  // suffix-min over lanes > lane
  uint32_t m = f;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    uint32_t u = __shfl_down_sync(0xffffffffu, m, o);
    if (lane + o < 32) m = min(m, u);
  }
  uint32_t nt = __shfl_down_sync(0xffffffffu, m, 1);
  if (lane == 31) nt = 0xFFFFu;
  st.next_t = nt;

  // the last start of the segment may run past it: find its end in global memory
  st.far_end = 0;
  const uint32_t has = __ballot_sync(0xffffffffu, st.startm != 0);
  if (has) {
    const int last_lane = 31 - __clz(has);
    if ((int)lane == last_lane) {
      const int j = 31 - __clz(st.startm);
      const uint32_t above = st.termm & ~((2u << j) - 1u);
      if (above == 0 && nt == 0xFFFFu) {
        const uint64_t sabs = p0 + j;
        uint64_t limit = (st.k_hi < cv.n_docs) ? cv.doc_off[st.k_hi] : cv.n_bytes;
        if (limit > cv.n_bytes) limit = cv.n_bytes;
        if (limit > sabs + kMaxTermLen + 1) limit = sabs + kMaxTermLen + 1;
        uint64_t p = s1;
        while (p < limit) {
          uint32_t word = 0;
          if (p + 4 <= cv.n_bytes) word = __ldg((const uint32_t*)(cv.text + p));
          else for (int b = 0; b < 4; ++b) if (p + b < cv.n_bytes) word |= (uint32_t)cv.text[p + b] << (8 * b);
          const uint32_t t4 = tokmask4(word);
          if (t4 != 0xFu) { p += __ffs(~t4) - 1; break; }
          p += 4;
        }
        if (p > limit) p = limit;
        st.far_end = (uint32_t)p;
      }
    }
  }
  return st;
}

// End (absolute) of the token starting at lane-local bit j.
__device__ __forceinline__ uint64_t token_end(const SegState& st, uint64_t p0, uint64_t s0, int j) {
  const uint32_t above = st.termm & ~((2u << j) - 1u);
  if (above) return p0 + (__ffs(above) - 1);
  if (st.next_t != 0xFFFFu) return s0 + st.next_t;
  return st.far_end;
}

template <bool EMIT>
__global__ void __launch_bounds__(kTokThreads) k_tokenize(ChunkView cv, uint64_t n_segs, uint32_t* seg_count,
                                                          const uint32_t* seg_off, EmitOut eo,
                                                          unsigned long long* dropped) {
  __shared__ uint32_t bnd[kTokWarps][32];
  const uint32_t lane = lane_id();
  const int w = threadIdx.x >> 5;
  const uint64_t gw = (uint64_t)blockIdx.x * kTokWarps + w;
  const uint64_t seg_begin = gw * kSegsPerWarp;
  if (seg_begin >= n_segs) return;
  const uint64_t seg_end = min(seg_begin + kSegsPerWarp, n_segs);
  // first boundary index k >= 1 with doc_off[k] >= segment start
  uint64_t kcur = 0;
  if (lane == 0) kcur = lower_bound_u64(cv.doc_off, 1, cv.n_docs > 0 ? cv.n_docs : 1, seg_begin * kSegBytes);
  kcur = __shfl_sync(0xffffffffu, kcur, 0);
  uint32_t drop_acc = 0;
  for (uint64_t seg = seg_begin; seg < seg_end; ++seg) {
    const SegState st = classify_segment(cv, seg, kcur, bnd[w]);
    const uint64_t s0 = seg * kSegBytes;
    const uint64_t p0 = s0 + 16 * lane;
    uint32_t nvalid = 0, ndrop = 0;
    uint32_t sm = st.startm;
    while (sm) {
      const int j = __ffs(sm) - 1;
      sm &= sm - 1;
      const uint64_t e = token_end(st, p0, s0, j);
      if (e - (p0 + j) <= kMaxTermLen) ++nvalid; else ++ndrop;
    }
    drop_acc += ndrop;
    if (!EMIT) {
      uint32_t tot = nvalid;
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) tot += __shfl_xor_sync(0xffffffffu, tot, o);
      if (lane == 0) seg_count[seg] = tot;
    } else {
      // exclusive prefix of nvalid over lanes
      uint32_t inc = nvalid;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        uint32_t u = __shfl_up_sync(0xffffffffu, inc, o);
        if ((int)lane >= o) inc += u;
      }
      uint64_t out = (uint64_t)seg_off[seg] + (inc - nvalid);
      sm = st.startm;
      while (sm) {
        const int j = __ffs(sm) - 1;
        sm &= sm - 1;
        const uint64_t s = p0 + j;
        const uint64_t e = token_end(st, p0, s0, j);
        const uint32_t len = (uint32_t)(e - s);
        if (len > kMaxTermLen) continue;
        // DocID: number of doc_off[k] <= s, k < n_docs, minus one (reading S9/S16)
        uint64_t k = st.k_lo;
        while (k < st.k_hi && cv.doc_off[k] <= s) ++k;
        const uint32_t doc = eo.doc_base + (uint32_t)(k - 1);
        const TermWords tw(cv.text, s, len);
        const uint64_t h = term_hash(tw, len);
        const uint32_t slot = table_insert(cv.text, eo.table, eo.mask, h, (uint32_t)s, len, eo.overflow);
        eo.slot[out] = slot;
        eo.doc[out] = doc;
        if (eo.dbg_start) { eo.dbg_start[out] = (uint32_t)s; eo.dbg_len[out] = len; }
        ++out;
      }
    }
  }
  if (!EMIT) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) drop_acc += __shfl_xor_sync(0xffffffffu, drop_acc, o);
    if (lane == 0 && drop_acc) atomicAdd(dropped, (unsigned long long)drop_acc);
  }
}

}  // namespace wj
