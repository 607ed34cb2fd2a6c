// K1: warp-cooperative tokenizer / normaliser + chunk-local term dedup (hash table).
//
// Paper: Step 2 "performs tokenization, that is, parses each document into tokens and determines
// the trie index of each resulting term"; "tokenization scans input document character by
// character and hence a trie index can be calculated as a byproduct".  Readings S1 (token
// bytes), S2 (ASCII folding), S4 (drop > 255 bytes), S16 (empty documents).
//
// B200 design.  A warp owns a range of 4 x 512-byte segments.  Per segment every lane classifies
// its 16 bytes with SWAR (one 128-bit load per lane), document starts come from doc_off through a
// per-warp cursor (fast path: no boundary in the segment), token starts are `tok & ~prev_tok |
// doc_start`, ends are the next terminator found in-lane, in a later lane (ballot + one shuffle) or
// past the segment (one lane scans forward).
//   * k_tok_count: kept tokens per warp range (a fast path avoids per-token work unless a run of
//     16 token bytes could hide a > 255-byte token).
//   * k_tok_emit: stages the range (+1 segment) in shared memory, queues (start, len) of kept tokens
//     in text order, then processes them one token per lane (full SIMT width): fold, hash, find/claim
//     the term's slot in a chunk-local open-addressing table of 16-byte slots {first-occurrence
//     offset | len | 24-bit tag, first 8 folded bytes}.  A token of <= 8 bytes is resolved from the
//     slot alone; longer ones compare the remaining bytes with the first occurrence in the
//     (immutable) text.  Writes (slot, docID) at the token's scanned position (coalesced).
// The dictionary (K3/K4) then sees each distinct term of the chunk once instead of once per token.
#pragma once
#include "common.cuh"

namespace wj {

constexpr int kSegBytes = 512;
constexpr int kTokThreads = 256;
constexpr int kTokWarps = kTokThreads / 32;
constexpr int kSegsPerWarp = 4;
constexpr int kWinBytes = (kSegsPerWarp + 1) * kSegBytes + 16;  // staged range + 1 segment + pad
#ifndef WJ_QUEUE_CAP
#define WJ_QUEUE_CAP 320
#endif
constexpr int kQueueCap = WJ_QUEUE_CAP;  // a segment with more kept starts is queued in rounds (emit)

struct ChunkView {
  const uint8_t* text;     // 16-byte aligned device pointer
  uint64_t n_bytes;        // < 2^32
  const uint64_t* doc_off; // device, n_docs + 1 entries
  uint64_t n_docs;
};

struct EmitOut {
  uint32_t* hot_mat;       // HOT: (hot term x chunk document) token counts, hot_docs columns
  uint32_t hot_docs;       // documents of the chunk
  Slot* table;             // chunk hash table
  uint32_t* slot_ref;      // per slot: first-occurrence offset (written by the inserter)
  uint32_t cap;            // capacity (slots; any value >= 1)
  uint32_t parts;          // multi-rank: the table is cut into `parts` partitions of part_cap slots,
  uint32_t part_cap;       // partition o holding the terms whose trie collection rank o owns
  const uint32_t* owner_tab;  // collection -> owner (balanced map), or nullptr: b mod parts
  uint32_t doc_base;       // global DocID of local document 0
  uint32_t* slot;          // per kept token: slot | 1 << 25 (key 0 = hole: a hot token, HOT only)
  uint32_t* doc;           // per kept token: global DocID
  unsigned long long* elem;  // or (packed stream, no HOT): per kept token slot << 32 | global DocID
  uint8_t* dig0;           // packed stream: per kept token the first radix pass's digit (slot & 255)
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

// The lane's 16 bytes of segment `seg` (zero past the end of the chunk).  Streaming loads
// (evict-first): the text is read once per pass and must not push the term table out of L2.
__device__ __forceinline__ uint4 load_lane16(const ChunkView& cv, uint32_t seg) {
  const uint64_t p0 = (uint64_t)seg * kSegBytes + 16 * lane_id();
  if (p0 + 16 <= cv.n_bytes) return __ldcs((const uint4*)(cv.text + p0));
  uint32_t wv[4];
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
  return make_uint4(wv[0], wv[1], wv[2], wv[3]);
}

constexpr uint32_t kNone = 0xFFFFu;

// Per-lane view of one segment.
struct SegBits {
  uint32_t tm;      // 16-bit token-byte mask
  uint32_t startm;  // token starts
  uint32_t termm;   // terminators: non-token byte or document start
};

// 16-bit token-byte mask of the lane's 16 bytes of the segment starting at s0
__device__ __forceinline__ uint32_t lane_tm(const ChunkView& cv, uint32_t s0, uint4 v) {
  const uint64_t p0 = (uint64_t)s0 + 16 * lane_id();
  uint32_t tm = tokmask4(v.x) | (tokmask4(v.y) << 4) | (tokmask4(v.z) << 8) | (tokmask4(v.w) << 12);
  if (p0 + 16 > cv.n_bytes) tm = p0 >= cv.n_bytes ? 0u : tm & ((1u << (uint32_t)(cv.n_bytes - p0)) - 1u);
  return tm;
}

// next document boundary doc_off[k] (k < n_docs), else "none" (warp-uniform)
__device__ __forceinline__ uint64_t next_bound(const ChunkView& cv, uint64_t k) {
  return (k < cv.n_docs) ? cv.doc_off[k] : ~0ull;
}

// Document starts inside the segment [s0, s0 + 512) as the lane's 16-bit mask; kcur = first
// boundary index (k >= 1) with doc_off[k] >= s0, advanced past the segment; nb = doc_off[kcur]
// (next_bound), carried in a register so that a segment without a boundary (most of them: documents
// are KBs long) issues no dependent load of doc_off.
__device__ __forceinline__ uint32_t seg_bounds(const ChunkView& cv, uint32_t s0, uint64_t& kcur, uint64_t& nb,
                                               uint32_t* bnd_smem) {
  const uint32_t lane = lane_id();
  const uint64_t s1 = (uint64_t)s0 + kSegBytes;
  uint32_t bm = 0;
  if (nb < s1) {
    bnd_smem[lane] = 0;
    __syncwarp();
    for (;;) {
      const uint64_t k = kcur + lane;
      const uint64_t x = (k < cv.n_docs) ? cv.doc_off[k] : ~0ull;
      const bool in = x < s1;
      if (in) atomicOr(&bnd_smem[(uint32_t)(x - s0) >> 4], 1u << ((uint32_t)(x - s0) & 15u));
      const uint32_t b = __ballot_sync(0xffffffffu, in);
      kcur += __popc(b);
      if (b != 0xffffffffu) {  // doc_off is sorted: lane popc(b) holds the first boundary past s1
        nb = __shfl_sync(0xffffffffu, x, __popc(b));
        break;
      }
    }
    __syncwarp();
    bm = bnd_smem[lane];
    __syncwarp();
  }
  return bm;
}

// token starts of the lane: token byte whose predecessor is not one, or a document start
__device__ __forceinline__ uint32_t start_mask(uint32_t tm, uint32_t bm, uint32_t prev) {
  uint32_t pv = __shfl_up_sync(0xffffffffu, tm >> 15, 1) & 1u;
  if (lane_id() == 0) pv = prev;
  return tm & (~((tm << 1) | pv) | bm) & 0xFFFFu;
}

// Classifies one segment; prev = token bit of the byte before the segment.
__device__ __forceinline__ SegBits seg_bits(const ChunkView& cv, uint32_t s0, uint4 v, uint32_t prev,
                                            uint64_t& kcur, uint64_t& nb, uint32_t* bnd_smem) {
  const uint32_t tm = lane_tm(cv, s0, v);
  const uint32_t bm = seg_bounds(cv, s0, kcur, nb, bnd_smem);
  SegBits sb;
  sb.tm = tm;
  sb.startm = start_mask(tm, bm, prev);
  sb.termm = (~tm | bm) & 0xFFFFu;
  return sb;
}

// Token structure of a segment that needs cross-lane information.
struct SegTok {
  uint32_t anyterm;    // ballot of lanes holding a terminator
  uint32_t nt;         // per lane: first terminator in a later lane (segment-relative) or kNone
  int open_lane;       // lane of the segment's last start if its token runs past the segment, else -1
  uint32_t open_pos;   // its segment-relative position
};

__device__ __forceinline__ SegTok seg_tok(const SegBits& sb) {
  const uint32_t lane = lane_id();
  SegTok t;
  t.anyterm = __ballot_sync(0xffffffffu, sb.termm != 0);
  const uint32_t ft = sb.termm ? 16 * lane + __ffs(sb.termm) - 1 : kNone;
  const uint32_t later = t.anyterm & ~((2u << lane) - 1u);
  const uint32_t v = __shfl_sync(0xffffffffu, ft, later ? __ffs(later) - 1 : lane);
  t.nt = later ? v : kNone;
  t.open_lane = -1;
  t.open_pos = 0;
  const uint32_t hasS = __ballot_sync(0xffffffffu, sb.startm != 0);
  if (hasS) {
    const int H = 31 - __clz(hasS);
    const int j = 31 - __clz(sb.startm | 1u);
    const bool op = ((int)lane == H) && (sb.termm & ~((2u << j) - 1u)) == 0 && t.nt == kNone;
    if (__ballot_sync(0xffffffffu, op)) {
      t.open_lane = H;
      t.open_pos = 16 * H + __shfl_sync(0xffffffffu, (uint32_t)j, H);
    }
  }
  return t;
}

// segment-relative first terminator of the segment (warp-uniform), kNone if none
__device__ __forceinline__ uint32_t first_term(const SegBits& sb, const SegTok& t) {
  const uint32_t lane = lane_id();
  const uint32_t ft = sb.termm ? 16 * lane + __ffs(sb.termm) - 1 : kNone;
  const uint32_t v = __shfl_sync(0xffffffffu, ft, t.anyterm ? __ffs(t.anyterm) - 1 : 0);
  return t.anyterm ? v : kNone;
}

// segment-relative end of the (non-open) token starting at lane bit j
__device__ __forceinline__ uint32_t tok_end_rel(const SegBits& sb, const SegTok& t, int j) {
  const uint32_t above = sb.termm & ~((2u << j) - 1u);
  return above ? 16 * lane_id() + __ffs(above) - 1 : t.nt;
}

// first boundary index k >= 1 with doc_off[k] >= start of each warp's segment range
__global__ void k_warp_kstart(ChunkView cv, uint64_t warps, uint64_t* kstart) {
  const uint64_t gw = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (gw >= warps) return;
  kstart[gw] = lower_bound_u64(cv.doc_off, 1, cv.n_docs > 0 ? cv.n_docs : 1, gw * kSegsPerWarp * kSegBytes);
}

__device__ __forceinline__ uint32_t prev_token_bit(const ChunkView& cv, uint64_t s0) {
  return (s0 > 0 && s0 - 1 < cv.n_bytes) ? (tokmask4(cv.text[s0 - 1]) & 1u) : 0u;
}

// ------------------------------------------------------------------ pass 1: count
// A token that runs past the end of its segment ("open") is resolved by the first terminator of
// the next segment (the warp reads one look-ahead segment past its range), so no lane ever scans
// forward; only a run of 16 token bytes in a lane can hide a > 255-byte token inside a segment.
#ifndef WJ_COUNT_MINB
#define WJ_COUNT_MINB 6  // 40 registers, 6 CTAs/SM: count 0.51 -> 0.43 ms on config 2
#endif
__global__ void __launch_bounds__(kTokThreads, WJ_COUNT_MINB) k_tok_count(ChunkView cv, uint32_t n_segs, const uint64_t* kstart,
                                                           uint32_t* range_count, unsigned long long* dropped) {
  __shared__ uint32_t bnd[kTokWarps][32];
  const uint32_t lane = lane_id();
  const int w = threadIdx.x >> 5;
  const uint32_t gw = blockIdx.x * kTokWarps + w;
  const uint32_t sb0 = gw * kSegsPerWarp;
  if (sb0 >= n_segs) return;
  const uint32_t se = min(sb0 + kSegsPerWarp, n_segs);
  const uint32_t last = se < n_segs ? se : se - 1;  // includes the look-ahead segment
  uint64_t kcur = kstart[gw];
  uint64_t nb = next_bound(cv, kcur);
  uint32_t prev = prev_token_bit(cv, (uint64_t)sb0 * kSegBytes);
  uint32_t cnt = 0, drop = 0;
  bool open = false;
  uint32_t open_start = 0;
  uint4 vr[kSegsPerWarp + 1];
#pragma unroll
  for (int j = 0; j <= kSegsPerWarp; ++j) vr[j] = (sb0 + j <= last) ? load_lane16(cv, sb0 + j) : make_uint4(0, 0, 0, 0);
  // Fast path: no lane of the range or the look-ahead segment holds 16 token bytes, so every token
  // starting in the range is <= 30 bytes long and is kept: the count is the number of token starts.
  uint32_t tmv[kSegsPerWarp + 1];
  bool full = false;
#pragma unroll
  for (int j = 0; j <= kSegsPerWarp; ++j) {
    tmv[j] = (sb0 + j <= last) ? lane_tm(cv, (sb0 + j) * kSegBytes, vr[j]) : 0u;
    full |= tmv[j] == 0xFFFFu;
  }
  if (!__any_sync(0xffffffffu, full)) {
#pragma unroll
    for (int j = 0; j < kSegsPerWarp; ++j) {
      if (sb0 + j >= se) break;
      const uint32_t bm = seg_bounds(cv, (sb0 + j) * kSegBytes, kcur, nb, bnd[w]);
      cnt += __popc(start_mask(tmv[j], bm, prev));
      prev = __shfl_sync(0xffffffffu, tmv[j], 31) >> 15;
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) cnt += __shfl_xor_sync(0xffffffffu, cnt, o);
    if (lane == 0) range_count[gw] = cnt;
    return;
  }
#pragma unroll
  for (int jj = 0; jj <= kSegsPerWarp; ++jj) {
    const uint32_t seg = sb0 + jj;
    if (seg > last) break;
    const uint4 v = vr[jj];
    const uint32_t s0 = seg * kSegBytes;
    const SegBits sb = seg_bits(cv, s0, v, prev, kcur, nb, bnd[w]);
    prev = __shfl_sync(0xffffffffu, sb.tm, 31) >> 15;
    const SegTok tk = seg_tok(sb);
    if (open) {
      const uint32_t ft = first_term(sb, tk);
      if (lane == 0) {
        if (ft != kNone && s0 + ft - open_start <= kMaxTermLen) ++cnt; else ++drop;
      }
      open = false;
    }
    if (seg == se) break;  // look-ahead segment: resolution only
    uint32_t c = __popc(sb.startm);
    if ((int)lane == tk.open_lane) --c;
    if (tk.open_lane >= 0) { open = true; open_start = s0 + tk.open_pos; }
    if (__ballot_sync(0xffffffffu, sb.tm == 0xFFFFu)) {
      for (uint32_t sm = sb.startm; sm; sm &= sm - 1) {
        const int j = __ffs(sm) - 1;
        const uint32_t pos = 16 * lane + j;
        if (tk.open_lane >= 0 && pos == tk.open_pos) continue;
        if (tok_end_rel(sb, tk, j) - pos > kMaxTermLen) { --c; ++drop; }
      }
    }
    cnt += c;
  }
  if (open && lane == 0) {  // chunk end
    if (cv.n_bytes - open_start <= kMaxTermLen) ++cnt; else ++drop;
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    cnt += __shfl_xor_sync(0xffffffffu, cnt, o);
    drop += __shfl_xor_sync(0xffffffffu, drop, o);
  }
  if (lane == 0) {
    range_count[gw] = cnt;
    if (drop) atomicAdd(dropped, (unsigned long long)drop);
  }
}

// ------------------------------------------------------------------ pass 2: emit
// k-th little-endian word of the folded term starting at window byte s (len bytes), zero padded
__device__ __forceinline__ uint32_t win_word(const uint32_t* win32, uint32_t s, uint32_t len, uint32_t k) {
  const uint32_t a = (s >> 2) + k, sh = (s & 3) * 8;
  uint32_t w = __funnelshift_r(win32[a], win32[a + 1], sh);
  const uint32_t rem = len - 4 * k;
  if (rem < 4) w &= (1u << (rem * 8)) - 1u;
  return w;  // the window is staged already folded (reading S2)
}

// 32-bit term hash over the folded, zero-padded little-endian words (cheap integer ops: the emit
// kernel is instruction-bound).  First slot = mulhi(h, capacity) (any capacity, so the table can be
// sized to the expected unique terms instead of the next power of two); the slot tag is a second mix.
__device__ __forceinline__ uint32_t hash_init(uint32_t len) { return len * 0x9E3779B1u + 0x7F4A7C15u; }
// polynomial over the words (one multiply-add per word, FMA pipe; the xor-multiply-xorshift mix per word
// cost 3 ALU instructions each: emit 2.39 -> 2.31 ms) + murmur3's 32-bit finaliser for the slot bits
__device__ __forceinline__ uint32_t hash_mix(uint32_t h, uint32_t w) { return fma_mad(h, 0x85EBCA77u, w); }
__device__ __forceinline__ uint32_t hash_fin(uint32_t h) {
  h ^= h >> 16;
  h *= 0x85EBCA6Bu;
  h ^= h >> 13;
  h *= 0xC2B2AE35u;
  return h ^ (h >> 16);
}
__device__ __forceinline__ uint32_t hash_tag(uint32_t h) { return (h * 0x9E3779B1u) >> 8; }

// Find or claim the slot of a term.  *hot = the sampled hot-term id stored in the slot's k1 (0: none;
// only slots seeded by k_hot_seed carry one).
// The probe sequence stays inside the partition [base, base + cap) (base = 0, cap = capacity for an
// unpartitioned table).
__device__ __forceinline__ uint32_t table_insert(const uint8_t* text, Slot* table, uint32_t* slot_ref, uint32_t base,
                                                 uint32_t cap, uint64_t h, uint64_t k0, uint64_t k1, uint32_t s_abs,
                                                 uint32_t len, const uint32_t* win32, uint32_t s_win, uint32_t* overflow,
                                                 uint32_t* hot) {
  uint32_t i = base + __umulhi((uint32_t)h, cap);
  for (int probe = 0; probe < 4096; ++probe) {
    // Slots are claimed once (CAS on k0) and published once (k1), so a cached read can only be
    // stale-empty: the CAS or the volatile re-read below resolves it.
    ulonglong2 e = *(const ulonglong2*)(table + i);
    if (e.x == 0) {
      const unsigned long long prev = atomicCAS(&table[i].k0, 0ull, (unsigned long long)k0);
      if (prev == 0) {
        slot_ref[i] = s_abs;
        if (len > kSlotBytes) __threadfence();  // only > 11-byte terms are compared via slot_ref
        *(volatile unsigned long long*)&table[i].k1 = k1;
        *hot = 0;
        return i;
      }
      e.x = prev;
      e.y = 0;
    }
    if (e.x == k0) {
      while (e.y == 0) e.y = *(volatile unsigned long long*)&table[i].k1;
      if ((e.y & kSlotK1Mask) == k1) {
        *hot = (uint32_t)(e.y >> kHotShift);
        if (len <= kSlotBytes) return i;
        // acquire: the inserter wrote slot_ref[i] before its release of k1 (__threadfence + store)
        (void)ld_acquire_u64(&table[i].k1);
        const uint32_t r = *(volatile uint32_t*)&slot_ref[i];
        const TermWords other(text, r, len);
        bool eq = true;
        for (uint32_t k = 2; k * 4 < len; ++k)
          if (other.word(k) != win_word(win32, s_win, len, k)) { eq = false; break; }
        if (eq) return i;
      }
    }
    i = i + 1 == base + cap ? base : i + 1;
  }
  atomicExch(overflow, 1u);
  *hot = 0;
  return kMiss;
}

// Table I index (readings S5, S8) of a folded term from its first 16 bytes (wd, zero
// padded) and, past 16 bytes, the staged window (only the all-digits test reads them)
__device__ __forceinline__ uint32_t term_bucket_w(const uint32_t (&wd)[4], uint32_t len, const uint32_t* w32,
                                                  uint32_t s_win) {
  bool digits = true;
#pragma unroll
  for (uint32_t k = 0; k < 4; ++k) {
    if (4 * k >= len) break;
    const uint32_t rem = len - 4 * k;
    const uint32_t valid = rem >= 4 ? 0x80808080u : (0x80808080u & ((1u << (8 * rem)) - 1u));
    if ((digit4(wd[k]) & valid) != valid) digits = false;
  }
  for (uint32_t k = 4; 4 * k < len && digits; ++k) {
    const uint32_t rem = len - 4 * k;
    const uint32_t valid = rem >= 4 ? 0x80808080u : (0x80808080u & ((1u << (8 * rem)) - 1u));
    if ((digit4(win_word(w32, s_win, len, k)) & valid) != valid) digits = false;
  }
  const uint32_t b0 = wd[0] & 0xFFu, b1 = (wd[0] >> 8) & 0xFFu, b2 = (wd[0] >> 16) & 0xFFu;
  if (digits) return 1 + (b0 - '0');
  if (b0 - 'a' < 26u) {
    if (len > 3 && b1 - 'a' < 26u && b2 - 'a' < 26u) return 37 + 676 * (b0 - 'a') + 26 * (b1 - 'a') + (b2 - 'a');
    return 11 + (b0 - 'a');
  }
  return 0;
}

// Launch bounds for 6 CTAs/SM (40 registers) with 320-entry token queues (31 KB of shared memory per
// CTA): emit 2.43 -> 2.34 ms on config 2 vs 48 registers and 512-entry queues.  The L1 share matters as
// much as the warps: with the driver's default carveout the kernel runs at ~66% occupancy; forcing a
// 86-100% shared-memory carveout (more CTAs, less L1 for the table probes) costs ~1 ms, 58-64% costs
// 0.18 ms (profiles/r01_README.md)
#ifndef WJ_EMIT_MINB
#define WJ_EMIT_MINB 6
#endif
// HOT (WJ_FLAG_HOT_TERMS): the <= kHotMaxH sampled hot terms of the chunk (SURVEY 8(f2)(ii),
// P:202-208), recognised by the hot id k_hot_seed stored in their table slot, do not enter the
// (slot, docID) stream (their tokens leave holes, key 0, dropped by the first sort pass) and are
// counted in the dense (hot term x document) matrix eo.hot_mat, through
// per-warp shared-memory counters for the first kHotDocs documents of the warp's range (one global add
// per nonzero counter at the range's end); the matrix rows become the hot terms' partial lists
// (k_hot_scatter).
constexpr uint32_t kHotMaxH = 64;
constexpr uint32_t kHotDocs = 2;
constexpr uint32_t kHotWords = kHotDocs * kHotMaxH;  // u32 counters per warp: [document][hot id]
#ifndef WJ_EMIT_HOT_MINB
#define WJ_EMIT_HOT_MINB 5  // 48 registers: at 40 the hot instance spills (emit 3.84 vs 2.74 ms)
#endif

// PARTS: the table is partitioned by owner rank (multi-rank path); HOT / PARTS are compile-time so that
// the one-GPU instantiation carries neither
template <bool HOT, bool PARTS>
__global__ void __launch_bounds__(kTokThreads, HOT ? WJ_EMIT_HOT_MINB : WJ_EMIT_MINB) k_tok_emit(ChunkView cv, uint32_t n_segs,
                                                          const uint64_t* kstart, const uint32_t* range_off, EmitOut eo) {
  __shared__ __align__(16) uint32_t win[kTokWarps][kWinBytes / 4];
  __shared__ uint32_t queue[kTokWarps][kQueueCap + 1];
  __shared__ uint32_t bnd[kTokWarps][32];
  __shared__ uint32_t hcnt[kTokWarps][HOT ? kHotWords : 1];
  const uint32_t lane = lane_id();
  const int w = threadIdx.x >> 5;
  const uint32_t gw = blockIdx.x * kTokWarps + w;
  const uint32_t sb0 = gw * kSegsPerWarp;
  if (sb0 >= n_segs) return;
  const uint32_t se = min(sb0 + kSegsPerWarp, n_segs);
  const uint32_t last = se < n_segs ? se : se - 1;
  const uint32_t B0 = sb0 * kSegBytes;
  uint32_t* w32 = win[w];
  uint32_t* q = queue[w];
  uint32_t* hc = hcnt[w];
  // stage the range and the look-ahead segment (tokens may run past the range)
  uint4 v[kSegsPerWarp + 1];
#pragma unroll
  for (int j = 0; j <= kSegsPerWarp; ++j) v[j] = load_lane16(cv, sb0 + j);
#pragma unroll
  for (int j = 0; j <= kSegsPerWarp; ++j)  // fold A-Z once here (classification is case-blind)
    *(uint4*)&w32[(j * kSegBytes + 16 * lane) / 4] =
        make_uint4(lower4(v[j].x), lower4(v[j].y), lower4(v[j].z), lower4(v[j].w));
  if (lane < 4) w32[(kWinBytes - 16) / 4 + lane] = 0;
  if (HOT)
    for (uint32_t i = lane; i < kHotWords; i += 32) hc[i] = 0;
  __syncwarp();

  const uint64_t k_range_lo = kstart[gw];
  uint64_t kcur = k_range_lo;
  uint32_t prev = prev_token_bit(cv, B0);
  uint32_t qn = 0;
  uint64_t obase = range_off[gw];
  uint64_t k_range_hi = k_range_lo;
  bool open = false;
  uint32_t open_start = 0;

  auto flush = [&]() {
    for (uint32_t r = 0; r < qn; r += 32) {
      const uint32_t idx = r + lane;
      uint32_t hkey = 0xFFFFFFFFu;  // HOT: [document][hot id] counter of this lane's hot token
      if (idx < qn) {
        const uint32_t e = q[idx];
        const uint32_t s_win = e >> 8, len = e & 255u;
        const uint32_t s_abs = B0 + s_win;
        // first 16 folded bytes: 5 window words, 4 funnel shifts, length masks
        uint32_t wd[4];
        {
          const uint32_t a = s_win >> 2, sh = (s_win & 3) * 8;
          uint32_t x[5];
#pragma unroll
          for (int k = 0; k < 5; ++k) x[k] = w32[a + k];
#pragma unroll
          for (int k = 0; k < 4; ++k) {
            const uint32_t rem = min(max((int)len - 4 * k, 0), 4);
            wd[k] = __funnelshift_r(x[k], x[k + 1], sh) & __funnelshift_lc(0xFFFFFFFFu, 0u, rem * 8);
          }
        }
        uint32_t h32 = hash_init(len);
#pragma unroll
        for (int k = 0; k < 4; ++k) h32 = hash_mix(h32, wd[k]);
        for (uint32_t k = 4; k * 4 < len; ++k) h32 = hash_mix(h32, win_word(w32, s_win, len, k));
        h32 = hash_fin(h32);
        const uint64_t h = h32;
        // DocID = (number of doc_off[k] <= s, k < n_docs) - 1 (readings S9, S16)
        uint64_t lo = k_range_lo, hi = k_range_hi;
        while (lo < hi) {
          const uint64_t mid = (lo + hi) >> 1;
          if (cv.doc_off[mid] <= s_abs) lo = mid + 1; else hi = mid;
        }
        const uint32_t ldoc = (uint32_t)(lo - 1);  // chunk-local document
        const uint64_t k0 = (uint64_t)len | ((uint64_t)hash_tag(h32) << 8) | ((uint64_t)wd[0] << 32);
        const uint64_t k1 = (uint64_t)wd[1] | ((uint64_t)(wd[2] & 0xFFFFFFu) << 32) | (1ull << 56);
        const uint64_t out = obase + idx;
        uint32_t hid = 0, tbase = 0, tcap = eo.cap;
        if (PARTS) {  // multi-rank: the partition of the rank that owns the term's collection
          const uint32_t b = term_bucket_w(wd, len, w32, s_win);
          tbase = (eo.owner_tab ? __ldg(&eo.owner_tab[b]) : b % eo.parts) * eo.part_cap;
          tcap = eo.part_cap;
        }
        // a hot term's slot was seeded with its hot id in k1 (k_hot_seed): table_insert returns it
        const uint32_t slot = table_insert(cv.text, eo.table, eo.slot_ref, tbase, tcap, h, k0, k1, s_abs, len, w32, s_win,
                                           eo.overflow, &hid);
        if (HOT && hid) {  // hot term: counted below (the stream keeps a hole, key 0)
          const uint32_t dd = ldoc - (uint32_t)(k_range_lo - 1), hh = hid - 1;
          if (dd < kHotDocs) hkey = dd * kHotMaxH + hh;
          else atomicAdd(&eo.hot_mat[(uint64_t)hh * eo.hot_docs + ldoc], 1u);
        }
        // branch-free stores: stream element slot | count 1 << 25, or a hole (the docID is not read)
        if (!HOT && eo.elem) {  // one 8-byte store: the sort moves (slot, docID) as one u64 key
          // (a probe-sequence overflow (kMiss) makes the host retry with a larger table; the sort forked
          // early on this stream must still stay in bounds: slot 0 instead)
          const uint32_t ps = slot == kMiss ? 0u : slot;
          __stcs(eo.elem + out, ((unsigned long long)ps << 32) | (eo.doc_base + ldoc));
          eo.dig0[out] = (uint8_t)ps;
        } else {
          __stcs(eo.slot + out, (HOT && hid) ? 0u : (slot | (1u << 25)));
          __stcs(eo.doc + out, eo.doc_base + ldoc);
        }
        if (eo.dbg_start) { eo.dbg_start[out] = s_abs; eo.dbg_len[out] = len; }
      }
      if (HOT && hkey != 0xFFFFFFFFu) atomicAdd(&hc[hkey], 1u);  // (a warp match first was slower)
    }
    obase += qn;
    qn = 0;
    __syncwarp();
  };

  for (uint32_t seg = sb0; seg <= last; ++seg) {
    const uint32_t j = seg - sb0;
    const uint32_t s0 = seg * kSegBytes;
    const uint4 vv = *(const uint4*)&w32[(j * kSegBytes + 16 * lane) / 4];
    // reloaded per segment here: a register carried across the flushes costs the emit kernel more
    // (spills) than the load (count: 0.426 -> 0.408 ms with the carried register, emit +0.025 ms)
    uint64_t nb = next_bound(cv, kcur);
    const SegBits sb = seg_bits(cv, s0, vv, prev, kcur, nb, bnd[w]);
    prev = __shfl_sync(0xffffffffu, sb.tm, 31) >> 15;
    const SegTok tk = seg_tok(sb);
    if (open) {  // the previous segment's last token ends in this one
      const uint32_t ft = first_term(sb, tk);
      if (ft != kNone && s0 + ft - open_start <= kMaxTermLen) {
        if (qn + 1 > (uint32_t)kQueueCap) flush();
        if (lane == 0) q[qn] = ((open_start - B0) << 8) | (s0 + ft - open_start);
        ++qn;
        __syncwarp();
      }
      open = false;
    }
    if (seg == se) break;
    k_range_hi = kcur;
    // kept tokens starting in this lane (a > 255-byte token needs a lane of 16 token bytes)
    uint32_t c = __popc(sb.startm) - ((int)lane == tk.open_lane ? 1u : 0u);
    if (__ballot_sync(0xffffffffu, sb.tm == 0xFFFFu)) {
      c = 0;
      for (uint32_t sm = sb.startm; sm; sm &= sm - 1) {
        const int jb = __ffs(sm) - 1;
        const uint32_t pos = 16 * lane + jb;
        if (tk.open_lane >= 0 && pos == tk.open_pos) continue;
        c += (tok_end_rel(sb, tk, jb) - pos <= kMaxTermLen) ? 1u : 0u;
      }
    }
    uint32_t inc = c;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t u = __shfl_up_sync(0xffffffffu, inc, o);
      if ((int)lane >= o) inc += u;
    }
    const uint32_t tot = __shfl_sync(0xffffffffu, inc, 31);
    if (qn + tot > (uint32_t)kQueueCap) flush();
    if (tot <= (uint32_t)kQueueCap) {
      uint32_t pos_q = qn + inc - c;
      for (uint32_t sm = sb.startm; sm; sm &= sm - 1) {
        const int jb = __ffs(sm) - 1;
        const uint32_t pos = 16 * lane + jb;
        if (tk.open_lane >= 0 && pos == tk.open_pos) continue;
        const uint32_t len = tok_end_rel(sb, tk, jb) - pos;
        if (len <= kMaxTermLen) q[pos_q++] = ((s0 + pos - B0) << 8) | len;
      }
      qn += tot;
    } else {
      // Rare: more kept tokens start in this segment than the queue holds (up to 512: dense
      // document starts, e.g. consecutive 1-byte documents).  Queue them in rounds of kQueueCap,
      // flushing between rounds (the queue is empty here: tot > kQueueCap forced the flush above).
      for (uint32_t r0 = 0; r0 < tot; r0 += (uint32_t)kQueueCap) {
        uint32_t pos_q = inc - c;  // segment-relative index of the lane's first kept token
        for (uint32_t sm = sb.startm; sm; sm &= sm - 1) {
          const int jb = __ffs(sm) - 1;
          const uint32_t pos = 16 * lane + jb;
          if (tk.open_lane >= 0 && pos == tk.open_pos) continue;
          const uint32_t len = tok_end_rel(sb, tk, jb) - pos;
          if (len > kMaxTermLen) continue;
          if (pos_q >= r0 && pos_q < r0 + (uint32_t)kQueueCap) q[pos_q - r0] = ((s0 + pos - B0) << 8) | len;
          ++pos_q;
        }
        qn = min(tot - r0, (uint32_t)kQueueCap);
        __syncwarp();
        flush();
      }
    }
    if (tk.open_lane >= 0) { open = true; open_start = s0 + tk.open_pos; }
    __syncwarp();
  }
  k_range_hi = kcur;
  if (open) {  // chunk end
    if (cv.n_bytes - open_start <= kMaxTermLen) {
      if (qn + 1 > (uint32_t)kQueueCap) flush();
      if (lane == 0) q[qn] = ((open_start - B0) << 8) | (uint32_t)(cv.n_bytes - open_start);
      ++qn;
      __syncwarp();
    }
  }
  flush();
  if (HOT) {  // the range's hot counters -> the (hot term x document) matrix
    const uint32_t d0 = (uint32_t)(k_range_lo - 1);
    for (uint32_t i = lane; i < kHotWords; i += 32) {
      const uint32_t x = hc[i];
      if (x) atomicAdd(&eo.hot_mat[(uint64_t)(i % kHotMaxH) * eo.hot_docs + d0 + i / kHotMaxH], x);
    }
  }
}

}  // namespace wj
