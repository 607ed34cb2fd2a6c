// K2-K4: trie bucket of the chunk's unique terms, B-tree probe, new-term insert, bulk rebuild.
//
// Dictionary = the paper's hybrid structure (§III.B): a trie table of height 3 that maps
// a term to one of 17,613 trie collections (Table I; no trie nodes are built, "we use
// a table to map a trie index directly into the root location of the corresponding B-Tree"), and one
// B-tree of minimum degree 16 per collection (31 keys / 32 children, 512-byte nodes, Table II,
// P:105-127).  The prefix captured by the trie is stripped from stored strings and
// each key keeps a 4-byte cache of the first suffix bytes; strings live in an arena as
// <u8 length><bytes> (Fig. 6).
//
// Probe (Fig. 7): one warp per key; lane j+1 holds key j of the node; a ballot of the
// parallel comparisons gives the child slot (the paper's "parallel comparison ... followed by a
// parallel reduction", re-expressed with __ballot_sync/__popc).  Caches decide almost every compare;
// only equal caches read the arena.
//
// Insert — B200 redesign, documented in DESIGN.md §6: instead of inserting the new terms
// of a collection one at a time with preemptive splits (which serialises a collection on one warp),
// the chunk's new terms are sorted by (collection, suffix), given termIDs with atomics, merged into
// the collection's sorted key order (the probe returns each miss's insertion rank), and every
// collection's B-tree is re-laid bottom-up in parallel with the same node format and B-tree
// invariants (t = 16: every non-root node holds 15..31 keys; all leaves at the same depth).
#pragma once
#include "common.cuh"

namespace wj {

// ------------------------------------------------------------------ term info (Table I)
// New terms are radix-sorted by (collection, first kSortSfxBytes suffix bytes); equal keys are
// ordered by the rest of the suffix (k_tie_fix).  4 bytes = the node cache: 47-bit keys,
// 6 passes; 6 bytes: 63-bit keys, 8 passes.
#ifndef WJ_SORT_SFX_BYTES
#define WJ_SORT_SFX_BYTES 4
#endif
constexpr uint32_t kSortSfxBytes = WJ_SORT_SFX_BYTES;
constexpr int kSortKeyBits = 15 + 8 * kSortSfxBytes;  // 17,613 collections < 2^15
struct TermInfo {
  uint32_t bucket, plen, slen, cache;
  uint64_t key;  // bucket << (8 kSortSfxBytes) | first kSortSfxBytes suffix bytes (big-endian, zero-padded)
};

__device__ __forceinline__ bool is_letter(uint32_t c) { return c - 'a' < 26u; }

// Table I with readings S5 (letters = a-z after folding, "special" = any other byte, pure number =
// all bytes '0'..'9') and S8 (prefix captured: 0 / 1 / 3 bytes).
__device__ __forceinline__ TermInfo term_info(const uint8_t* text, uint64_t ref, uint32_t len) {
  const TermWords tw(text, ref, len);
  const uint32_t nw = (len + 3) >> 2;
  uint32_t w[4] = {0, 0, 0, 0};
  bool digits = true;
  for (uint32_t k = 0; k < nw; ++k) {
    const uint32_t x = tw.word(k);
    if (k < 4) w[k] = x;
    const uint32_t rem = len - 4 * k;
    const uint32_t valid = rem >= 4 ? 0x80808080u : (0x80808080u & ((1u << (8 * rem)) - 1u));
    if ((digit4(x) & valid) != valid) digits = false;
  }
  auto byte = [&](uint32_t i) -> uint32_t { return i < len && i < 16 ? (w[i >> 2] >> (8 * (i & 3))) & 0xFFu : 0u; };
  const uint32_t b0 = byte(0), b1 = byte(1), b2 = byte(2);
  TermInfo ti;
  if (digits) { ti.bucket = 1 + (b0 - '0'); ti.plen = 1; }
  else if (is_letter(b0)) {
    if (len > 3 && is_letter(b1) && is_letter(b2)) { ti.bucket = 37 + 676 * (b0 - 'a') + 26 * (b1 - 'a') + (b2 - 'a'); ti.plen = 3; }
    else { ti.bucket = 11 + (b0 - 'a'); ti.plen = 1; }
  } else { ti.bucket = 0; ti.plen = 0; }
  ti.slen = len - ti.plen;
  uint32_t c = 0;
  uint64_t k6 = 0;
#pragma unroll
  for (uint32_t i = 0; i < 6; ++i) {
    const uint32_t b = byte(ti.plen + i);
    if (i < 4) c |= b << (24 - 8 * i);
    k6 |= (uint64_t)b << (40 - 8 * i);
  }
  ti.cache = c;
  ti.key = kSortSfxBytes == 6 ? (((uint64_t)ti.bucket << 48) | k6) : (((uint64_t)ti.bucket << 32) | c);
  return ti;
}

__host__ __device__ __forceinline__ uint32_t bucket_plen(uint32_t b) { return b == 0 ? 0u : (b <= 36 ? 1u : 3u); }

// Folded byte i of a chunk unique term: the first 16 bytes are held in w (built from its table slot),
// longer terms read the rest from their first occurrence in the chunk text.
__device__ __forceinline__ uint32_t ubyte(const uint4& w, const uint8_t* text, uint32_t ref, uint32_t i) {
  if (i < 16) {
    const uint32_t x = i < 8 ? (i < 4 ? w.x : w.y) : (i < 12 ? w.z : w.w);
    return (x >> (8 * (i & 3))) & 0xFFu;
  }
  const uint32_t c = text[ref + i];
  return (c - 'A' < 26u) ? c + 32 : c;
}

// Table I index etc. of a unique term given its first 16 folded bytes (w) and length.
__device__ __forceinline__ TermInfo term_info_w(const uint4& w, const uint8_t* text, uint32_t ref, uint32_t len) {
  bool digits = true;
  const uint32_t ws[4] = {w.x, w.y, w.z, w.w};
#pragma unroll
  for (uint32_t k = 0; k < 4; ++k) {
    if (4 * k >= len) break;
    const uint32_t rem = len - 4 * k;
    const uint32_t valid = rem >= 4 ? 0x80808080u : (0x80808080u & ((1u << (8 * rem)) - 1u));
    if ((digit4(ws[k]) & valid) != valid) digits = false;
  }
  for (uint32_t i = 16; i < len && digits; ++i) digits = ubyte(w, text, ref, i) - '0' < 10u;
  const uint32_t b0 = ws[0] & 0xFFu, b1 = (ws[0] >> 8) & 0xFFu, b2 = (ws[0] >> 16) & 0xFFu;
  TermInfo ti;
  if (digits) { ti.bucket = 1 + (b0 - '0'); ti.plen = 1; }
  else if (is_letter(b0)) {
    if (len > 3 && is_letter(b1) && is_letter(b2)) { ti.bucket = 37 + 676 * (b0 - 'a') + 26 * (b1 - 'a') + (b2 - 'a'); ti.plen = 3; }
    else { ti.bucket = 11 + (b0 - 'a'); ti.plen = 1; }
  } else { ti.bucket = 0; ti.plen = 0; }
  ti.slen = len - ti.plen;
  uint32_t c = 0;
  uint64_t k6 = 0;
#pragma unroll
  for (uint32_t i = 0; i < 6; ++i) {
    const uint32_t b = (ti.plen + i < len) ? ubyte(w, text, ref, ti.plen + i) : 0u;
    if (i < 4) c |= b << (24 - 8 * i);
    k6 |= (uint64_t)b << (40 - 8 * i);
  }
  ti.cache = c;
  ti.key = kSortSfxBytes == 6 ? (((uint64_t)ti.bucket << 48) | k6) : (((uint64_t)ti.bucket << 32) | c);
  return ti;
}

__host__ __device__ __forceinline__ uint32_t prefix_byte(uint32_t b, uint32_t i) {
  if (b <= 10) return '0' + (b - 1);
  if (b <= 36) return 'a' + (b - 11);
  const uint32_t x = b - 37;
  return i == 0 ? 'a' + x / 676 : (i == 1 ? 'a' + (x / 26) % 26 : 'a' + x % 26);
}

// Folded suffix byte i of a chunk term (text at ref, prefix plen).
__device__ __forceinline__ uint32_t text_sfx_byte(const uint8_t* text, uint64_t ref, uint32_t plen, uint32_t i) {
  uint32_t c = text[ref + plen + i];
  return (c - 'A' < 26u) ? c + 32 : c;
}

// sign(unique term suffix - arena term), given that the first 4 suffix bytes are equal.
__device__ __forceinline__ int cmp_sfx_arena(const uint4& w, const uint8_t* text, uint32_t ref, uint32_t plen,
                                             uint32_t slen, const uint8_t* arena, uint32_t aoff) {
  const uint32_t alen = arena[aoff];
  const uint32_t m = slen < alen ? slen : alen;
  for (uint32_t i = 4; i < m; ++i) {
    const uint32_t x = ubyte(w, text, ref, plen + i), y = arena[aoff + 1 + i];
    if (x != y) return x < y ? -1 : 1;
  }
  return slen == alen ? 0 : (slen < alen ? -1 : 1);
}

// sign(unique a - unique b) on suffixes (same prefix length), starting at suffix byte `from`.
__device__ __forceinline__ int cmp_sfx_sfx(const uint4& wa, uint32_t ra, uint32_t la, const uint4& wb, uint32_t rb,
                                           uint32_t lb, const uint8_t* text, uint32_t plen, uint32_t from) {
  const uint32_t m = la < lb ? la : lb;
  for (uint32_t i = from; i < m; ++i) {
    const uint32_t x = ubyte(wa, text, ra, plen + i), y = ubyte(wb, text, rb, plen + i);
    if (x != y) return x < y ? -1 : 1;
  }
  return la == lb ? 0 : (la < lb ? -1 : 1);
}

// ------------------------------------------------------------------ B-tree layout arithmetic
// Subtree with m keys and height h (h == 1: leaf).  Internal: c = min(32, floor((m+1)/16^(h-1)))
// children, the m-c+1 non-separator keys split evenly (first r children one larger).  With the root
// height minimal (m <= 32^h - 1) this satisfies the B-tree bounds of t = 16.
struct Split {
  uint32_t c, q, r;
};
__host__ __device__ __forceinline__ Split split_of(uint32_t m, uint32_t h) {
  const uint64_t cc = ((uint64_t)m + 1) >> (4 * (h - 1));
  Split s;
  s.c = cc > 32 ? 32u : (uint32_t)cc;
  const uint32_t rest = m - s.c + 1;
  s.q = rest / s.c;
  s.r = rest % s.c;
  return s;
}
__host__ __device__ __forceinline__ uint32_t child_lo(const Split& s, uint32_t lo, uint32_t j) {
  return lo + j * (s.q + 1) + (j < s.r ? j : s.r);
}
__host__ __device__ __forceinline__ uint32_t child_m(const Split& s, uint32_t j) { return s.q + (j < s.r ? 1u : 0u); }
__host__ __device__ __forceinline__ uint32_t height_of(uint32_t n) {
  uint32_t h = 0;
  uint64_t cap = 1;
  while (cap - 1 < n) { cap *= 32; ++h; }
  return h;  // 0 for n == 0
}

struct DictView {
  const Node* nodes;
  const uint32_t* coll_root;
  const uint32_t* coll_n;
  const uint8_t* arena;
};

struct UniqueView {
  const uint8_t* text;
  const uint4* w;
  const uint32_t* ref;
  const uint32_t* len;
  const uint32_t* bucket;
  const uint32_t* cache;
};

// Warp-cooperative descent for one key (retrieval, k_query).  Returns termID (tid) or kMiss with
// *ins_rank set.
__device__ __forceinline__ uint32_t probe_key(const DictView& dv, const uint4& w, const uint8_t* text, uint32_t ref,
                                              uint32_t len, uint32_t bucket, uint32_t cache, uint32_t* ins_rank) {
  const uint32_t lane = lane_id();
  const uint32_t n = dv.coll_n[bucket];
  if (n == 0) { *ins_rank = 0; return kMiss; }
  const uint32_t plen = bucket_plen(bucket), slen = len - plen;
  uint32_t node = dv.coll_root[bucket], lo = 0, m = n, h = height_of(n);
  for (;;) {
    const Node* nd = dv.nodes + node;
    const uint32_t wv = __ldg(((const uint32_t*)nd) + lane);  // line 0: count, cache[0..30]
    const uint32_t cnt = __shfl_sync(0xffffffffu, wv, 0);
    const bool valid = lane >= 1 && lane <= cnt;
    int cmp = 0;
    if (valid) {
      if (cache != wv) cmp = cache < wv ? -1 : 1;
      else if (slen >= 4) cmp = cmp_sfx_arena(w, text, ref, plen, slen, dv.arena, __ldg(&nd->str[lane - 1]));
    }
    const uint32_t eq = __ballot_sync(0xffffffffu, valid && cmp == 0);
    if (eq) {
      const uint32_t j = __ffs(eq) - 2;
      return __ldg(&nd->post[j]);
    }
    const uint32_t pos = __popc(__ballot_sync(0xffffffffu, valid && cmp > 0));
    if (h == 1) { *ins_rank = lo + pos; return kMiss; }
    const Split s = split_of(m, h);
    const uint32_t nlo = child_lo(s, lo, pos), nm = child_m(s, pos);
    node = __ldg(&nd->child[pos]);
    lo = nlo; m = nm; --h;
  }
}

// Probe with four keys per warp (8 lanes per key): a descent is a chain of dependent loads, so the
// probe is latency-bound; four independent descents per warp and the node's key line (caches) and
// child line loaded together halve the dependent loads per level and quadruple the keys in flight.
// Lane gl of a group holds words 4gl..4gl+3 of each line (word 0 of line 0 = count, word j >= 1 =
// cache j-1; line 3 = children).  Same result as probe_key.
constexpr int kProbeKeysPerWarp = 4;
__global__ void __launch_bounds__(256) k_probe4(DictView dv, UniqueView uv, uint32_t U, uint32_t* tid_out,
                                                uint32_t* rank_out) {
  const uint32_t lane = lane_id(), g = lane >> 3, gl = lane & 7;
  const uint32_t warps = gridDim.x * (blockDim.x >> 5);
  for (uint32_t base = (blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5)) * kProbeKeysPerWarp; base < U;
       base += warps * kProbeKeysPerWarp) {
    const uint32_t u = base + g;
    const bool active0 = u < U;
    uint32_t bucket = 0, cache = 0, len = 0, ref = 0, n = 0;
    uint4 w = make_uint4(0, 0, 0, 0);
    if (active0) {
      bucket = uv.bucket[u];
      cache = uv.cache[u];
      len = uv.len[u];
      ref = uv.ref[u];
      w = uv.w[u];
      n = dv.coll_n[bucket];
    }
    const uint32_t plen = bucket_plen(bucket), slen = len - plen;
    uint32_t node = active0 && n ? dv.coll_root[bucket] : 0u, lo = 0, m = n, h = height_of(n);
    bool done = !active0 || n == 0;
    uint32_t res_tid = kMiss, res_rank = 0;
    // every lane of the warp runs the loop until all four descents are done (warp-synchronous ballots)
    while (__any_sync(0xffffffffu, !done)) {
      uint4 c4 = make_uint4(0, 0, 0, 0), ch4 = make_uint4(0, 0, 0, 0);
      const Node* nd = dv.nodes + node;
      if (!done) {
        c4 = __ldg((const uint4*)nd + gl);                 // line 0: count, caches
        if (h > 1) ch4 = __ldg((const uint4*)nd->child + gl);  // line 3: children (same round trip)
      }
      const uint32_t cnt = __shfl_sync(0xffffffffu, c4.x, lane & ~7u);
      const uint32_t cw[4] = {c4.x, c4.y, c4.z, c4.w};
      uint32_t ltm = 0, eqm = 0;  // per lane, bit t: entry 4gl+t-1 is < key / == key
#pragma unroll
      for (int t = 0; t < 4; ++t) {
        const uint32_t j = 4 * gl + t;  // word j = cache j-1
        const bool valid = !done && j >= 1 && j - 1 < cnt;
        int cmp = 0;
        if (valid) {
          if (cache != cw[t]) cmp = cache < cw[t] ? -1 : 1;
          else if (slen >= 4) cmp = cmp_sfx_arena(w, uv.text, ref, plen, slen, dv.arena, __ldg(&nd->str[j - 1]));
        }
        ltm |= (valid && cmp > 0 ? 1u : 0u) << t;
        eqm |= (valid && cmp == 0 ? 1u : 0u) << t;
      }
      // group-wide: number of entries below the key, and the first equal entry
      uint32_t pos = __popc(ltm), eqj = eqm ? 4 * gl + __ffs(eqm) - 2 : 0xFFFFFFFFu;
#pragma unroll
      for (int o = 1; o < 8; o <<= 1) {
        pos += __shfl_xor_sync(0xffffffffu, pos, o);
        eqj = min(eqj, __shfl_xor_sync(0xffffffffu, eqj, o));
      }
      if (!done) {
        if (eqj != 0xFFFFFFFFu) {  // hit
          res_tid = __ldg(&nd->post[eqj]);
          done = true;
        } else if (h == 1) {       // miss at a leaf: insertion rank
          res_rank = lo + pos;
          done = true;
        }
      }
      // child[pos]: word pos of line 3 is in group lane pos / 4, component pos % 4
      const uint32_t chw[4] = {ch4.x, ch4.y, ch4.z, ch4.w};
      uint32_t mine = 0;
#pragma unroll
      for (int t = 0; t < 4; ++t)
        if ((pos & 3u) == (uint32_t)t) mine = chw[t];
      const uint32_t child = __shfl_sync(0xffffffffu, mine, (lane & ~7u) + ((pos >> 2) & 7u));
      if (!done) {
        const Split sp = split_of(m, h);
        lo = child_lo(sp, lo, pos);
        m = child_m(sp, pos);
        node = child;
        --h;
      }
    }
    if (active0 && gl == 0) {
      tid_out[u] = res_tid;
      rank_out[u] = res_rank;
    }
  }
}

// unique gather (slot order, sequential): occupied slot i -> unique index uid[i]; the term's first
// 11 folded bytes come from the slot itself, longer terms read their first occurrence
__global__ void k_unique_gather(const Slot* table, const uint32_t* slot_ref, uint32_t C, const uint32_t* uid,
                                const uint8_t* text, uint4* u_w, uint32_t* u_ref, uint32_t* u_len, uint32_t* u_bucket,
                                uint32_t* u_cache, uint64_t* u_key, uint32_t* u_slot) {
  const uint32_t i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= C) return;
  const ulonglong2 e = *(const ulonglong2*)(table + i);
  if (e.x == 0) return;
  const uint32_t u = uid[i];
  const uint32_t len = (uint32_t)e.x & 0xFFu;
  const uint32_t ref = slot_ref[i];
  uint4 w;
  if (len <= kSlotBytes) {
    w = make_uint4((uint32_t)(e.x >> 32), (uint32_t)e.y, (uint32_t)(e.y >> 32) & 0xFFFFFFu, 0u);
  } else {
    const TermWords tw(text, ref, len);
    w = make_uint4(tw.word(0), tw.word(1), tw.word(2), tw.word(3));
  }
  const TermInfo ti = term_info_w(w, text, ref, len);
  u_w[u] = w; u_ref[u] = ref; u_len[u] = len; u_bucket[u] = ti.bucket; u_cache[u] = ti.cache; u_key[u] = ti.key;
  u_slot[u] = i;
}

// compact the misses: nk_key/nk_val in unique order (radix-sorted next)
__global__ void k_miss_compact(const uint32_t* u_tid, const uint32_t* midx, const uint64_t* u_key, uint32_t U,
                               uint64_t* nk_key, uint32_t* nk_val) {
  const uint32_t u = blockIdx.x * blockDim.x + threadIdx.x;
  if (u >= U || u_tid[u] != kMiss) return;
  const uint32_t k = midx[u];
  nk_key[k] = u_key[u];
  nk_val[k] = u;
}

// Runs of equal (bucket, 6-byte) keys are ordered by the rest of the suffix (insertion sort by the
// run's first thread; runs are rare and short: two new terms sharing bucket + 6 suffix bytes).
__global__ void k_tie_fix(const uint64_t* key, uint32_t* val, uint32_t N, const uint8_t* text, const uint4* u_w,
                          const uint32_t* u_ref, const uint32_t* u_len) {
  const uint32_t i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= N) return;
  if (i > 0 && key[i - 1] == key[i]) return;
  if (i + 1 >= N || key[i + 1] != key[i]) return;
  uint32_t e = i + 1;
  while (e < N && key[e] == key[i]) ++e;
  const uint32_t plen = bucket_plen((uint32_t)(key[i] >> (8 * kSortSfxBytes)));
  for (uint32_t a = i + 1; a < e; ++a) {
    const uint32_t x = val[a];
    const uint4 wx = u_w[x];
    const uint32_t rx = u_ref[x], lx = u_len[x] - plen;
    uint32_t b = a;
    while (b > i) {
      const uint32_t y = val[b - 1];
      if (cmp_sfx_sfx(u_w[y], u_ref[y], u_len[y] - plen, wx, rx, lx, text, plen, kSortSfxBytes) <= 0) break;
      val[b] = y;
      --b;
    }
    val[b] = x;
  }
}

// New terms, in unique order (coalesced column reads): the next termIDs in unique order (V0 + the
// term's index among the chunk's misses; the paper's GPU indexer assigns postings pointers as it
// inserts), arena append <len><suffix> (Fig. 6) at the scanned offset, per-term columns
// (coalesced: consecutive misses get consecutive termIDs).  The sorted-order lists for the merge are
// filled afterwards by k_ns_fill.
__global__ void k_new_terms(uint32_t U, const uint32_t* aoff, uint64_t arena_base, const uint8_t* text,
                            const uint4* u_w, const uint32_t* u_ref, const uint32_t* u_len, const uint32_t* u_bucket,
                            const uint32_t* u_cache, uint32_t* u_tid, const uint32_t* miss_idx, uint32_t V0,
                            uint8_t* arena, uint32_t* t_arena, uint32_t* t_cache, uint32_t* t_bucket,
                            const uint32_t* u_rank, uint4* u_pack) {
  const uint32_t u = blockIdx.x * blockDim.x + threadIdx.x;
  if (u >= U || u_tid[u] != kMiss) return;
  const uint32_t tid = V0 + miss_idx[u];
  const uint32_t b = u_bucket[u], plen = bucket_plen(b), ref = u_ref[u], slen = u_len[u] - plen;
  const uint64_t off = arena_base + aoff[u];
  arena[off] = (uint8_t)slen;
  const uint4 w = u_w[u];
  for (uint32_t i = 0; i < slen; ++i) arena[off + 1 + i] = (uint8_t)ubyte(w, text, ref, plen + i);
  t_arena[tid] = (uint32_t)off;
  t_cache[tid] = u_cache[u];
  t_bucket[tid] = b;
  u_tid[u] = tid;
  // what k_ns_fill gathers in sorted order, as one 16-byte line (one sector per gathered term)
  u_pack[u] = make_uint4(tid, b | u_len[u] << 16, u_rank[u], (uint32_t)off);
}

// E (the per-collection sorted key order) carries, besides termIDs, each term's arena offset and
// "info" = Table I index | full length << 16, so that finalize reads them in E order (k_lexrank)
__host__ __device__ __forceinline__ uint32_t e_info(uint32_t bucket, uint32_t full_len) { return bucket | full_len << 16; }
__host__ __device__ __forceinline__ uint32_t e_info_bucket(uint32_t info) { return info & 0xFFFFu; }

__global__ void k_ns_fill(const uint32_t* sorted_u, uint32_t N, const uint4* __restrict__ u_pack, uint32_t* ns_tid,
                          uint32_t* ns_bucket, uint32_t* ns_rank, uint32_t* ns_info, uint32_t* ns_arena) {
  const uint32_t k = blockIdx.x * blockDim.x + threadIdx.x;
  if (k >= N) return;
  const uint4 x = u_pack[sorted_u[k]];  // {tid, e_info(bucket, full length), insertion rank, arena offset}
  ns_tid[k] = x.x;
  ns_bucket[k] = e_info_bucket(x.y);
  ns_rank[k] = x.z;
  ns_info[k] = x.y;
  ns_arena[k] = x.w;
}

// per-collection [lo, hi) of the sorted new terms
__global__ void k_new_ranges(const uint32_t* ns_bucket, uint32_t N, uint32_t* nlo, uint32_t* nhi) {
  const uint32_t k = blockIdx.x * blockDim.x + threadIdx.x;
  if (k >= N) return;
  const uint32_t b = ns_bucket[k];
  if (k == 0 || ns_bucket[k - 1] != b) nlo[b] = k;
  if (k + 1 == N || ns_bucket[k + 1] != b) nhi[b] = k + 1;
}

struct NewCount {
  const uint32_t* coll_n;
  const uint32_t* nlo;
  const uint32_t* nhi;
  __device__ __forceinline__ uint32_t operator()(uint64_t b) const { return coll_n[b] + (nhi[b] - nlo[b]); }
};

__global__ void k_place_new(const uint32_t* ns_tid, const uint32_t* ns_info, const uint32_t* ns_arena,
                            const uint32_t* ns_rank, uint32_t N, const uint32_t* nlo, const uint32_t* nbase, uint32_t* e_tid,
                            uint32_t* e_inf, uint32_t* e_ar) {
  const uint32_t k = blockIdx.x * blockDim.x + threadIdx.x;
  if (k >= N) return;
  const uint32_t inf = ns_info[k], b = e_info_bucket(inf);
  const uint32_t pos = nbase[b] + ns_rank[k] + (k - nlo[b]);
  e_tid[pos] = ns_tid[k];
  e_inf[pos] = inf;
  e_ar[pos] = ns_arena[k];
}

__global__ void k_place_old(const uint32_t* o_tid, const uint32_t* o_inf, const uint32_t* o_ar, uint32_t V,
                            const uint32_t* obase, const uint32_t* ns_rank, const uint32_t* nlo, const uint32_t* nhi,
                            const uint32_t* nbase, uint32_t* e_tid, uint32_t* e_inf, uint32_t* e_ar) {
  const uint32_t p = blockIdx.x * blockDim.x + threadIdx.x;
  if (p >= V) return;
  const uint32_t inf = o_inf[p], b = e_info_bucket(inf);
  const uint32_t i = p - obase[b];
  // number of new keys of b with insertion rank <= i
  uint32_t lo = nlo[b], hi = nhi[b];
  const uint32_t first = lo;
  while (lo < hi) {
    const uint32_t mid = (lo + hi) >> 1;
    if (ns_rank[mid] <= i) lo = mid + 1; else hi = mid;
  }
  const uint32_t pos = nbase[b] + i + (lo - first);
  e_tid[pos] = o_tid[p];
  e_inf[pos] = inf;
  e_ar[pos] = o_ar[p];
}

// ------------------------------------------------------------------ bulk rebuild, level by level
struct Level {
  uint32_t* b;
  uint32_t* lo;
  uint32_t* m;
  uint32_t* h;
};

__global__ void k_roots(const uint32_t* coll_n, const uint32_t* root_idx, uint32_t* coll_root, Level out) {
  const uint32_t b = blockIdx.x * blockDim.x + threadIdx.x;
  if (b >= kCollections) return;
  const uint32_t n = coll_n[b];
  if (n == 0) { coll_root[b] = kMiss; return; }
  const uint32_t r = root_idx[b];
  coll_root[b] = r;  // level-0 node ids start at 0
  out.b[r] = b; out.lo[r] = 0; out.m[r] = n; out.h[r] = height_of(n);
}

struct ChildCount {
  const uint32_t* m;
  const uint32_t* h;
  __device__ __forceinline__ uint32_t operator()(uint64_t i) const { return h[i] == 1 ? 0u : split_of(m[i], h[i]).c; }
};

struct NonEmpty {
  const uint32_t* n;
  __device__ __forceinline__ uint32_t operator()(uint64_t b) const { return n[b] ? 1u : 0u; }
};

// warp per node record of the level: fill the 512-byte node and emit child records
__global__ void k_build_level(Level cur, uint32_t L, uint32_t cur_base, const uint32_t* child_off, uint32_t next_base,
                              Level nxt, const uint32_t* e_tid, const uint32_t* coll_base, const uint32_t* t_arena,
                              const uint32_t* t_cache, Node* nodes) {
  const uint32_t warps = gridDim.x * (blockDim.x >> 5);
  const uint32_t lane = lane_id();
  for (uint32_t r = blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5); r < L; r += warps) {
    const uint32_t b = cur.b[r], lo = cur.lo[r], m = cur.m[r], h = cur.h[r];
    Node* nd = nodes + cur_base + r;
    const uint32_t eb = coll_base[b];
    uint32_t cnt, key_rank = 0;
    bool has_key;
    if (h == 1) {
      cnt = m;
      has_key = lane < m;
      key_rank = lo + lane;
    } else {
      const Split s = split_of(m, h);
      cnt = s.c - 1;
      has_key = lane < cnt;
      if (has_key) key_rank = child_lo(s, lo, lane) + child_m(s, lane);
      if (lane < s.c) {
        const uint32_t ci = child_off[r] + lane;
        nd->child[lane] = next_base + ci;
        nxt.b[ci] = b; nxt.lo[ci] = child_lo(s, lo, lane); nxt.m[ci] = child_m(s, lane); nxt.h[ci] = h - 1;
      } else {
        nd->child[lane] = kMiss;
      }
    }
    if (h == 1) nd->child[lane] = kMiss;
    if (lane == 0) { nd->count = cnt; nd->leaf = h == 1 ? 1u : 0u; nd->pad = 0; }
    if (lane < 31) {
      if (has_key) {
        const uint32_t tid = e_tid[eb + key_rank];
        nd->cache[lane] = t_cache[tid];
        nd->str[lane] = t_arena[tid];
        nd->post[lane] = tid;
      } else {
        nd->cache[lane] = 0; nd->str[lane] = kMiss; nd->post[lane] = kMiss;
      }
    }
  }
}

// ------------------------------------------------------------------ finalize: lexicographic rank
// Full (unstripped) byte i of term tid.
__device__ __forceinline__ uint32_t full_byte(const uint8_t* arena, uint32_t aoff, uint32_t b, uint32_t plen, uint32_t i) {
  return i < plen ? prefix_byte(b, i) : arena[aoff + 1 + (i - plen)];
}
__device__ __forceinline__ int cmp_full(const uint8_t* arena, const uint32_t* t_arena, const uint32_t* t_bucket,
                                        uint32_t x, uint32_t y) {
  const uint32_t bx = t_bucket[x], by = t_bucket[y], ax = t_arena[x], ay = t_arena[y];
  const uint32_t px = bucket_plen(bx), py = bucket_plen(by);
  const uint32_t lx = px + arena[ax], ly = py + arena[ay];
  const uint32_t m = lx < ly ? lx : ly;
  for (uint32_t i = 0; i < m; ++i) {
    const uint32_t cx = full_byte(arena, ax, bx, px, i), cy = full_byte(arena, ay, by, py, i);
    if (cx != cy) return cx < cy ? -1 : 1;
  }
  return lx == ly ? 0 : (lx < ly ? -1 : 1);
}

// Groups of the global order (reading S12): digits '0'..'9' (bucket 1+k merged with the bucket-0
// terms starting with that digit), letters 'a'..'z' (bucket 11+k merged with buckets
// 37+676k..37+676k+675), then bucket-0 terms starting with a byte >= 0x80.
struct LexGroups {
  uint32_t zlo[11];   // bucket-0 index of the first term with first byte >= '0'+k (k=10: >= 0x80)
  uint32_t gbase[37];
};

// 11 warps (kLexGroupThreads): warp k finds the first bucket-0 index whose first byte is >= '0'+k
// (k = 10: >= 0x80) by a 32-way search (each round probes 32 evenly spaced entries: ~5 dependent rounds
// instead of ~22 for a binary search on one lane); thread 0 then accumulates the group bases.
constexpr int kLexGroupThreads = 11 * 32;
__global__ void k_lex_groups(const uint32_t* e_tid, const uint32_t* coll_base, const uint32_t* coll_n,
                             const uint32_t* t_cache, LexGroups* g) {
  const uint32_t k = threadIdx.x >> 5, lane = lane_id();
  const uint32_t b0 = coll_base[0], n0 = coll_n[0];
  if (k <= 10) {
    const uint32_t target = k < 10 ? '0' + k : 0x80;
    uint32_t lo = 0, hi = n0;  // the answer is in [lo, hi]
    while (lo < hi) {
      const uint32_t pos = lo + (uint32_t)((uint64_t)(hi - lo) * lane / 32u);
      const uint32_t ge = __ballot_sync(0xffffffffu, (t_cache[e_tid[b0 + pos]] >> 24) >= target);
      if (!ge) {
        lo = __shfl_sync(0xffffffffu, pos, 31) + 1;
      } else {
        const int f = __ffs(ge) - 1;
        const uint32_t pf = __shfl_sync(0xffffffffu, pos, f);
        const uint32_t pb = __shfl_sync(0xffffffffu, pos, f > 0 ? f - 1 : 0);
        hi = pf;
        if (f > 0) lo = pb + 1;
      }
    }
    if (lane == 0) g->zlo[k] = lo;
  }
  __syncthreads();
  if (threadIdx.x != 0) return;
  uint32_t acc = 0;
  for (int q = 0; q < 10; ++q) {
    g->gbase[q] = acc;
    const uint32_t zhi = q < 9 ? g->zlo[q + 1] : g->zlo[10];
    acc += coll_n[1 + q] + (zhi - g->zlo[q]);
  }
  for (int q = 0; q < 26; ++q) {
    g->gbase[10 + q] = acc;
    const uint32_t s = coll_base[37 + 676 * q];
    const uint32_t e = (q == 25) ? coll_base[kCollections - 1] + coll_n[kCollections - 1] : coll_base[37 + 676 * (q + 1)];
    acc += coll_n[11 + q] + (e - s);
  }
  g->gbase[36] = acc;
}

// number of entries in E[lo,hi) whose full term is < term x
__device__ __forceinline__ uint32_t count_less(const uint32_t* e_tid, uint32_t lo, uint32_t hi, const uint8_t* arena,
                                               const uint32_t* t_arena, const uint32_t* t_bucket, uint32_t x) {
  const uint32_t first = lo;
  while (lo < hi) {
    const uint32_t mid = (lo + hi) >> 1;
    if (cmp_full(arena, t_arena, t_bucket, e_tid[mid], x) < 0) lo = mid + 1; else hi = mid;
  }
  return lo - first;
}

// term x vs the byte string s[0..sl): <0, 0, >0
__device__ __forceinline__ int cmp_full_str(const uint8_t* arena, const uint32_t* t_arena, const uint32_t* t_bucket,
                                            uint32_t x, const uint8_t* s, uint32_t sl) {
  const uint32_t bx = t_bucket[x], ax = t_arena[x], px = bucket_plen(bx), lx = px + arena[ax];
  const uint32_t m = lx < sl ? lx : sl;
  for (uint32_t i = 0; i < m; ++i) {
    const uint32_t cx = full_byte(arena, ax, bx, px, i);
    if (cx != s[i]) return cx < s[i] ? -1 : 1;
  }
  return lx == sl ? 0 : (lx < sl ? -1 : 1);
}

// Per 3-letter collection b = 37 + 676 k + 26 i + j (prefix c0 c1 c2, terms longer than 3 bytes):
// short_le[b - 37] = terms of the short bucket 11 + k (first letter c0, not in a 3-letter collection)
// that are <= "c0c1c2".  Every term T of collection b compares with a short-bucket term s as
// "c0c1c2" does: s either differs from c0c1c2 within its first min(|s|, 3) bytes, or is a prefix of it
// (< T), and a longer s starting with c0c1c2 would be in collection b itself.  So k_lexrank's count of
// short terms below T is this per-collection constant instead of a binary search per term.
__global__ void k_lex_short(const uint32_t* e_tid, const uint32_t* coll_base, const uint32_t* coll_n,
                            const uint8_t* arena, const uint32_t* t_arena, const uint32_t* t_bucket, uint32_t* short_le) {
  const uint32_t i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= 17576u) return;
  const uint32_t k = i / 676u;
  const uint8_t key[3] = {(uint8_t)('a' + k), (uint8_t)('a' + (i / 26u) % 26u), (uint8_t)('a' + i % 26u)};
  const uint32_t first = coll_base[11 + k];
  uint32_t lo = first, hi = first + coll_n[11 + k];
  while (lo < hi) {  // first entry > key
    const uint32_t mid = (lo + hi) >> 1;
    if (cmp_full_str(arena, t_arena, t_bucket, e_tid[mid], key, 3) <= 0) lo = mid + 1; else hi = mid;
  }
  short_le[i] = lo - first;
}

// Ranks of all terms (rank_of by termID, rank_info by rank), reading E, its arena offsets and infos in
// order.  With rec != nullptr (one run whose records are indexed by termID, engine.cu finalize) the
// run's (list start, df, cf) are gathered here (one 16-byte record per term) and written by rank
// (coalesced) instead of scattered by a separate pass.
__global__ void k_lexrank(const uint32_t* e_tid, const uint32_t* e_inf, const uint32_t* e_ar, uint32_t V,
                          const uint32_t* coll_base, const uint32_t* coll_n, const LexGroups* g, const uint8_t* arena,
                          const uint32_t* t_arena, const uint32_t* t_bucket, const uint32_t* t_cache,
                          const uint32_t* short_le, uint32_t* rank_of, uint2* rank_info, const uint4* rec, uint32_t* df_r,
                          uint64_t* cf_r, uint64_t* start_r) {
  const uint32_t p = blockIdx.x * blockDim.x + threadIdx.x;
  if (p >= V) return;
  const uint32_t tid = e_tid[p], inf = e_inf[p], b = e_info_bucket(inf);
  uint32_t rank;
  if (b == 0) {
    const uint32_t i = p - coll_base[0];
    const uint32_t fb = t_cache[tid] >> 24;
    if (fb - '0' < 10u) {
      const uint32_t k = fb - '0';
      rank = g->gbase[k] + (i - g->zlo[k]) +
             count_less(e_tid, coll_base[1 + k], coll_base[1 + k] + coll_n[1 + k], arena, t_arena, t_bucket, tid);
    } else {
      rank = g->gbase[36] + (i - g->zlo[10]);
    }
  } else if (b <= 10) {
    const uint32_t k = b - 1, i = p - coll_base[b];
    const uint32_t zhi = k < 9 ? g->zlo[k + 1] : g->zlo[10];
    rank = g->gbase[k] + i +
           count_less(e_tid, coll_base[0] + g->zlo[k], coll_base[0] + zhi, arena, t_arena, t_bucket, tid);
  } else if (b <= 36) {
    const uint32_t k = b - 11, i = p - coll_base[b];
    const uint32_t s = coll_base[37 + 676 * k];
    const uint32_t e = (k == 25) ? V : coll_base[37 + 676 * (k + 1)];
    rank = g->gbase[10 + k] + i + count_less(e_tid, s, e, arena, t_arena, t_bucket, tid);
  } else {
    const uint32_t k = (b - 37) / 676;
    const uint32_t j = p - coll_base[37 + 676 * k];
    rank = g->gbase[10 + k] + j + short_le[b - 37];
  }
  rank_of[tid] = rank;
  // by rank, for the final dictionary bytes: arena offset, Table I index | full term length << 16
  rank_info[rank] = make_uint2(e_ar[p], inf);
  if (rec) {
    const uint4 r = rec[tid];  // list start (lo, hi), df, cf
    df_r[rank] = r.z;
    cf_r[rank] = r.w;
    start_r[rank] = (uint64_t)r.x | (uint64_t)r.y << 32;
  }
}

}  // namespace wj
