// K5-K7: postings construction and the final inverted file.
//
// Paper: "All <term, document ID> tuples belonging to the same term are combined together to form
// the postings list of that term"; each posting holds "the ID of the document containing
// the term, term frequency"; lists are "organized in a sorted order of document IDs",
// which the paper gets "intrinsically" from consuming documents in order.  Here the
// device-resident (termID, docID) stream is in submission order, a STABLE radix sort by the term's
// global lexicographic rank groups it term-major while keeping docIDs ascending, and a run-length
// pass turns runs of equal (term, doc) into (docID, tf); df and cf are the dictionary's statistics
// (reading S11).  This single group-by at the end replaces the paper's per-run partial lists
// and their combine step — see DESIGN.md §6.
#pragma once
#include "common.cuh"
#include "dict.cuh"
#include "radix.cuh"
#include "tma.cuh"

namespace wj {

// stream element slot -> term rank (in place; the count bits above bit 25 are kept, holes skipped)
__global__ void k_map_rank(uint32_t* key, uint64_t N, const uint32_t* rank_of) {
  const uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= N) return;
  const uint32_t k = key[i];
  if ((k >> 25) == 0) return;
  key[i] = __ldg(&rank_of[k & ((1u << 25) - 1u)]) | (k & ~((1u << 25) - 1u));
}

// per chunk: table slot -> termID map (the chunk's token stream keeps slot ids; finalize composes
// the map with termID -> rank and the sort's histogram pass gathers through it)
__global__ void k_slot_map(const Slot* table, const uint32_t* slot_uid, const uint32_t* u_tid, uint32_t C,
                           uint32_t* map) {
  const uint32_t i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= C) return;
  map[i] = table[i].k0 ? u_tid[slot_uid[i]] : 0u;
}

// map[i] = rank_of[map[i]] (in place)
__global__ void k_map_compose(uint32_t* map, uint32_t C, const uint32_t* rank_of) {
  const uint32_t i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i < C) map[i] = __ldg(&rank_of[map[i]]);
}

constexpr int kRleThreads = 256;
#ifndef WJ_RLE_ITEMS
#define WJ_RLE_ITEMS 16
#endif
#ifndef WJ_RLE_MINB
#define WJ_RLE_MINB 2
#endif
constexpr int kRleItems = WJ_RLE_ITEMS;
constexpr int kRleTile = kRleThreads * kRleItems;

__device__ __forceinline__ uint32_t block_min_after(uint32_t v, uint32_t* sm /* >= 9 words */) {
  // min over threads with a larger index than the caller
  const uint32_t lane = lane_id();
  const int w = threadIdx.x >> 5;
  uint32_t m = v;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const uint32_t u = __shfl_down_sync(0xffffffffu, m, o);
    if (lane + o < 32) m = min(m, u);
  }
  // m = min over lanes >= lane in this warp
  if (lane == 0) sm[w] = m;
  __syncthreads();
  uint32_t later_warps = 0xFFFFFFFFu;
  for (int x = w + 1; x < kRleThreads / 32; ++x) later_warps = min(later_warps, sm[x]);
  uint32_t after_in_warp = __shfl_down_sync(0xffffffffu, m, 1);
  if (lane == 31) after_in_warp = 0xFFFFFFFFu;
  __syncthreads();
  return min(after_in_warp, later_warps);
}

// ------------------------------------------------------------------ run-length, reduce-then-scan
// Stream elements after the sort: key = rank | count << 25 (count >= 1 tokens of that term in that
// document: 1 for a plain token, the per-document count for an aggregated hot-term element), value =
// docID.  CTA c owns the contiguous element range [c*per, min(N,(c+1)*per)).  k_rle_count counts
// posting starts and tokens per range; scans give each range's first posting index and token offset;
// k_rle_write_tma walks its range tile by tile (TMA-prefetched 2-stage ring), carries the open run
// across tiles and writes docid, tf = sum of counts (coalesced through shared memory; ostride 2 =
// interleaved (docID, tf) pairs, the per-run partial lists), post_off[rank]
// and the token offset cstart[rank] of the term's first element (cf = difference).  Runs that continue
// across ranges are completed by k_rle_fixup (range_lead = tokens before the range's first posting).
// elements per CTA range of the run-length pass (a multiple of its tile); engine.cu rle() cuts the same
__host__ __device__ __forceinline__ uint64_t rle_per(uint64_t N, uint64_t G) {
  const uint64_t per = (N + G - 1) / G;
  return (per + kRleTile - 1) / kRleTile * kRleTile;
}

constexpr uint32_t kCountShift = 25;
constexpr uint32_t kRankMask = (1u << kCountShift) - 1u;

__device__ __forceinline__ void rle_load16(const uint32_t* key, const uint32_t* doc, uint64_t i0, uint64_t hi,
                                           uint32_t* k, uint32_t* d, uint32_t& pk, uint32_t& pd) {
  if (i0 + kRleItems <= hi) {
#pragma unroll
    for (int q = 0; q < kRleItems / 4; ++q) {
      const uint4 a = __ldcs((const uint4*)(key + i0) + q);
      const uint4 b = __ldcs((const uint4*)(doc + i0) + q);
      k[4 * q] = a.x; k[4 * q + 1] = a.y; k[4 * q + 2] = a.z; k[4 * q + 3] = a.w;
      d[4 * q] = b.x; d[4 * q + 1] = b.y; d[4 * q + 2] = b.z; d[4 * q + 3] = b.w;
    }
  } else {
#pragma unroll
    for (int j = 0; j < kRleItems; ++j) {
      const bool v = i0 + j < hi;
      k[j] = v ? key[i0 + j] : 0u;
      d[j] = v ? doc[i0 + j] : 0xFFFFFFFFu;
    }
  }
  pk = 0xFFFFFFFFu;
  pd = 0xFFFFFFFFu;
  if (i0 > 0) { pk = key[i0 - 1]; pd = doc[i0 - 1]; }
}

// posting starts (npm: new rank or new doc) and term starts (ntm: new rank)
__device__ __forceinline__ void rle_flags(const uint32_t* k, const uint32_t* d, uint32_t pk, uint32_t pd, uint64_t i0,
                                          uint64_t hi, uint32_t& npm, uint32_t& ntm) {
  npm = 0;
  ntm = 0;
  uint32_t pr = pk & kRankMask;
#pragma unroll
  for (int j = 0; j < kRleItems; ++j) {
    const bool valid = i0 + j < hi;
    const uint32_t r = k[j] & kRankMask;
    const bool nt = valid && (i0 + j == 0 || r != pr);
    const bool np = valid && (nt || d[j] != pd);
    npm |= (np ? 1u : 0u) << j;
    ntm |= (nt ? 1u : 0u) << j;
    pr = r;
    pd = d[j];
  }
}

template <bool COUNTS>
__global__ void __launch_bounds__(kRleThreads) k_rle_count(const uint32_t* __restrict__ key, const uint32_t* __restrict__ doc,
                                                           uint64_t N, uint64_t per, uint32_t* range_cnt,
                                                           uint64_t* range_tok, const uint32_t* __restrict__ n_dev) {
  if (n_dev) {  // the actual length (N is an upper bound): ranges re-cut for it
    N = min(N, (uint64_t)*n_dev);
    per = rle_per(N, gridDim.x);
  }
  const uint64_t lo = (uint64_t)blockIdx.x * per;
  const uint64_t hi = lo + per < N ? lo + per : N;
  uint32_t c = 0;
  uint64_t tk = 0;
  for (uint64_t i0 = lo + (uint64_t)threadIdx.x * kRleItems; i0 < hi; i0 += (uint64_t)kRleTile) {
    uint32_t k[kRleItems], d[kRleItems], pk, pd, npm, ntm;
    rle_load16(key, doc, i0, hi, k, d, pk, pd);
    rle_flags(k, d, pk, pd, i0, hi, npm, ntm);
    c += __popc(npm);
#pragma unroll
    for (int j = 0; j < kRleItems; ++j)  // invalid items have key 0; without counts every element is 1 token
      tk += COUNTS ? (k[j] >> kCountShift) : (k[j] != 0u ? 1u : 0u);
  }
  uint32_t tot;
  block_exclusive_sum<uint32_t>(c, tot);
  uint64_t ttot;
  block_exclusive_sum<uint64_t>(tk, ttot);
  if (threadIdx.x == 0) {
    range_cnt[blockIdx.x] = tot;
    range_tok[blockIdx.x] = ttot;
  }
}

inline size_t rle_smem_bytes(bool counts = true) {
  return (size_t)4 * kRleTile * 4 /*2 stages x (key, doc)*/ + 2 * kRleTile * 4 /*staged docid, tf*/ +
         (counts ? (kRleTile + 4) * 4 : 0) /*item token-count prefix (COUNTS only)*/;
}

// COUNTS = false: every element is one token (no hot-term elements in the stream), so token prefixes
// are element positions and the second block scan and the prefix array are skipped.
template <bool COUNTS>
#ifndef WJ_RLE_MAXREG
#define WJ_RLE_MAXREG 0
#endif
#if WJ_RLE_MAXREG > 0
#define WJ_RLE_BOUNDS __maxnreg__(WJ_RLE_MAXREG)
#else
#define WJ_RLE_BOUNDS __launch_bounds__(kRleThreads, WJ_RLE_MINB)
#endif
__global__ void WJ_RLE_BOUNDS k_rle_write_tma(const uint32_t* __restrict__ key,
                                                               const uint32_t* __restrict__ doc, uint64_t N,
                                                               uint64_t per, const uint32_t* __restrict__ range_off,
                                                               const uint64_t* __restrict__ range_tok_off,
                                                               uint32_t* out_doc, uint32_t* out_tf, uint32_t ostride,
                                                               uint64_t* post_off,
                                                               uint64_t* cstart, uint32_t* range_lead,
                                                               const uint32_t* __restrict__ n_dev) {
  if (n_dev) {
    N = min(N, (uint64_t)*n_dev);
    per = rle_per(N, gridDim.x);
  }
  extern __shared__ __align__(128) uint32_t rsm[];
  __shared__ __align__(8) uint64_t bar[2];
  __shared__ uint32_t sm[16];
  __shared__ uint32_t s_open_len, s_lead, s_prev_k, s_prev_d;
  __shared__ int s_lead_done;
  auto skey = [&](int s) { return rsm + (size_t)s * 2 * kRleTile; };
  auto sdoc = [&](int s) { return rsm + (size_t)s * 2 * kRleTile + kRleTile; };
  uint32_t* st_doc = rsm + 4 * kRleTile;
  uint32_t* st_tf = rsm + 5 * kRleTile;
  uint32_t* cpi = rsm + 6 * kRleTile;  // exclusive token-count prefix of each tile item (+ total)
  const uint64_t lo = (uint64_t)blockIdx.x * per;
  const uint64_t hi = lo + per < N ? lo + per : N;
  if (lo >= hi) {  // an empty range (N shrank below the launch's upper bound)
    if (threadIdx.x == 0) range_lead[blockIdx.x] = 0;
    return;
  }
  auto issue = [&](int s, uint64_t base) {  // thread 0
    const uint32_t cnt = (uint32_t)min((uint64_t)kRleTile, hi - base);
    const uint32_t b = (cnt * 4 + 15) & ~15u;
    fence_proxy_async_smem();
    mbar_arrive_expect_tx(&bar[s], 2 * b);
    tma_load_1d(skey(s), key + base, b, &bar[s]);
    tma_load_1d(sdoc(s), doc + base, b, &bar[s]);
  };
  if (threadIdx.x == 0) {
    mbar_init(&bar[0], 1);
    mbar_init(&bar[1], 1);
    fence_mbar_init();
    s_open_len = 0;
    s_lead = 0;
    s_lead_done = 0;
    s_prev_k = lo > 0 ? key[lo - 1] : 0xFFFFFFFFu;
    s_prev_d = lo > 0 ? doc[lo - 1] : 0xFFFFFFFFu;
  }
  __syncthreads();
  if (threadIdx.x == 0) issue(0, lo);
  uint32_t p0 = range_off[blockIdx.x];
  uint64_t tokbase = range_tok_off[blockIdx.x];
  bool have_open = false;
  uint32_t open_p = 0;
  uint32_t parity = 0;
  int s = 0;
  for (uint64_t base = lo; base < hi; base += kRleTile) {
    if (threadIdx.x == 0 && base + kRleTile < hi) issue(s ^ 1, base + kRleTile);
    mbar_wait(&bar[s], (parity >> s) & 1u);
    parity ^= 1u << s;
    const uint32_t tile_len = (uint32_t)min((uint64_t)kRleTile, hi - base);
    const uint32_t t0 = threadIdx.x * kRleItems;
    const uint32_t* ks = skey(s);
    const uint32_t* ds = sdoc(s);
    uint32_t k[kRleItems], d[kRleItems];
#pragma unroll
    for (int q = 0; q < kRleItems / 4; ++q) {
      const uint4 a = *(const uint4*)(ks + t0 + 4 * q);
      const uint4 b = *(const uint4*)(ds + t0 + 4 * q);
      k[4 * q] = a.x; k[4 * q + 1] = a.y; k[4 * q + 2] = a.z; k[4 * q + 3] = a.w;
      d[4 * q] = b.x; d[4 * q + 1] = b.y; d[4 * q + 2] = b.z; d[4 * q + 3] = b.w;
    }
#pragma unroll
    for (int j = 0; j < kRleItems; ++j)
      if (t0 + j >= tile_len) k[j] = 0u;  // past the range: no tokens
    const uint32_t pk = t0 ? ks[t0 - 1] : s_prev_k;
    const uint32_t pd = t0 ? ds[t0 - 1] : s_prev_d;
    uint32_t npm, ntm;
    rle_flags(k, d, pk, pd, base + t0, base + tile_len, npm, ntm);
    const uint32_t c = __popc(npm);
    uint32_t tot, ctot = tile_len;
    const uint32_t ex = block_exclusive_sum<uint32_t>(c, tot);
    if (COUNTS) {
      uint32_t ps = 0;
#pragma unroll
      for (int j = 0; j < kRleItems; ++j) ps += k[j] >> kCountShift;
      uint32_t run = block_exclusive_sum<uint32_t>(ps, ctot);
#pragma unroll
      for (int j = 0; j < kRleItems; ++j) {
        cpi[t0 + j] = run;
        run += k[j] >> kCountShift;
      }
    }
    auto cp = [&](uint32_t i) -> uint32_t { return COUNTS ? cpi[i] : i; };
    const uint32_t my_first = npm ? t0 + __ffs(npm) - 1 : 0xFFFFFFFFu;
    const uint32_t next_after = block_min_after(my_first, sm);  // contains __syncthreads: cpi visible
    if (threadIdx.x == 0) {
      const uint32_t first_all = min(my_first, next_after);
      const uint32_t lead = first_all == 0xFFFFFFFFu ? ctot : cp(first_all);
      if (!s_lead_done) {
        s_lead += lead;
        if (first_all != 0xFFFFFFFFu) s_lead_done = 1;
      }
      if (have_open) {
        s_open_len += lead;
        if (first_all != 0xFFFFFFFFu) out_tf[(uint64_t)ostride * open_p] = s_open_len;
      }
    }
    uint32_t lp = ex;
#pragma unroll
    for (int j = 0; j < kRleItems; ++j) {
      if ((npm >> j) & 1u) {
        const uint32_t rest = npm & ~((2u << j) - 1u);
        const uint32_t pos = t0 + j;
        const uint32_t end = rest ? t0 + __ffs(rest) - 1 : min(next_after, tile_len);
        st_doc[lp] = d[j];
        st_tf[lp] = (end < tile_len ? cp(end) : ctot) - cp(pos);
        if ((ntm >> j) & 1u) {
          const uint32_t r = k[j] & kRankMask;
          post_off[r] = p0 + lp;
          cstart[r] = tokbase + cp(pos);
        }
        ++lp;
      }
    }
    __syncthreads();
    for (uint32_t x = threadIdx.x; x < tot; x += kRleThreads) {
      if (ostride == 2) {  // interleaved (docID, tf) pairs (per-run partial lists)
        __stcs((uint2*)out_doc + p0 + x, make_uint2(st_doc[x], st_tf[x]));
      } else {
        __stcs(out_doc + p0 + x, st_doc[x]);
        __stcs(out_tf + p0 + x, st_tf[x]);
      }
    }
    if (threadIdx.x == 0) {
      if (tot) s_open_len = st_tf[tot - 1];
      s_prev_k = ks[tile_len - 1];
      s_prev_d = ds[tile_len - 1];
    }
    if (tot) {
      have_open = true;
      open_p = p0 + tot - 1;
    }
    p0 += tot;
    tokbase += ctot;
    __syncthreads();
    s ^= 1;
  }
  if (threadIdx.x == 0) {
    if (have_open) out_tf[(uint64_t)ostride * open_p] = s_open_len;
    range_lead[blockIdx.x] = s_lead;
  }
}

// ------------------------------------------------------------------ run-length, one warp per range
// Plain streams (every element one token, the element count known on the host): each warp owns a
// contiguous range of `per` elements (a multiple of kRlwStep) and walks it 512 elements per step,
// 16 per lane from registers; head flags, the warp scan of posting counts, the next head after each
// lane (suffix min over lanes) and the staging of (docID, tf) pairs for a coalesced write-out all stay
// inside the warp: no block barriers (the block version stalled ~20% on them at 2 CTAs/SM, 96
// registers).  Posting offsets per warp range come from k_rlw_count + a scan; runs continuing across
// ranges are completed by k_rle_fixup (range_lead = elements before the range's first head).
constexpr int kRlwItems = 16;
constexpr int kRlwStep = 32 * kRlwItems;  // 512
constexpr int kRlwThreads = 256;
constexpr int kRlwWarps = kRlwThreads / 32;

__host__ __device__ __forceinline__ uint64_t rlw_per(uint64_t N, uint64_t W) {
  const uint64_t per = (N + W - 1) / W;
  return (per + kRlwStep - 1) / kRlwStep * kRlwStep;
}

// the lane's 16 elements of the step at i0 (past hi: key 0, doc ~0) and the element before them.
// PACKED: the stream is one u64 array (slot << 32 | docID, the emit kernel's packed output); else
// key[] / doc[] (SoA).
template <bool PACKED>
__device__ __forceinline__ void rlw_load(const uint32_t* key, const uint32_t* doc, const unsigned long long* elem,
                                         uint64_t i0, uint64_t hi, uint32_t (&k)[kRlwItems], uint32_t (&d)[kRlwItems]) {
  const uint64_t b = i0 + (uint64_t)kRlwItems * lane_id();
  if (b + kRlwItems <= hi) {
    if (PACKED) {
#pragma unroll
      for (int q = 0; q < kRlwItems / 2; ++q) {
        const uint4 x = __ldcs((const uint4*)(elem + b) + q);
        d[2 * q] = x.x; k[2 * q] = x.y; d[2 * q + 1] = x.z; k[2 * q + 1] = x.w;
      }
    } else {
#pragma unroll
      for (int q = 0; q < kRlwItems / 4; ++q) {
        const uint4 x = __ldcs((const uint4*)(key + b) + q);
        const uint4 y = __ldcs((const uint4*)(doc + b) + q);
        k[4 * q] = x.x; k[4 * q + 1] = x.y; k[4 * q + 2] = x.z; k[4 * q + 3] = x.w;
        d[4 * q] = y.x; d[4 * q + 1] = y.y; d[4 * q + 2] = y.z; d[4 * q + 3] = y.w;
      }
    }
  } else {
#pragma unroll
    for (int j = 0; j < kRlwItems; ++j) {
      const bool v = b + j < hi;
      if (PACKED) {
        const unsigned long long e = v ? elem[b + j] : 0xFFFFFFFFull;
        k[j] = (uint32_t)(e >> 32);
        d[j] = (uint32_t)e;
      } else {
        k[j] = v ? key[b + j] : 0u;
        d[j] = v ? doc[b + j] : 0xFFFFFFFFu;
      }
    }
  }
}

// (key, doc) of element i
template <bool PACKED>
__device__ __forceinline__ void rlw_at(const uint32_t* key, const uint32_t* doc, const unsigned long long* elem, uint64_t i,
                                       uint32_t& k, uint32_t& d) {
  if (PACKED) {
    const unsigned long long e = elem[i];
    k = (uint32_t)(e >> 32);
    d = (uint32_t)e;
  } else {
    k = key[i];
    d = doc[i];
  }
}

// head (new term or new document) and term-start masks of the lane's items; (pk, pd) = the element
// before the step, carried by the caller (pk = 0xFFFFFFFF before the stream's first element)
__device__ __forceinline__ void rlw_flags(const uint32_t (&k)[kRlwItems], const uint32_t (&d)[kRlwItems], uint32_t pk,
                                          uint32_t pd, uint32_t nvalid, uint32_t& npm, uint32_t& ntm) {
  const uint32_t lane = lane_id();
  uint32_t qk = __shfl_up_sync(0xffffffffu, k[kRlwItems - 1], 1);
  uint32_t qd = __shfl_up_sync(0xffffffffu, d[kRlwItems - 1], 1);
  if (lane == 0) { qk = pk; qd = pd; }
  npm = 0;
  ntm = 0;
  uint32_t pr = qk & kRankMask;
  const uint32_t first = lane * kRlwItems;
#pragma unroll
  for (int j = 0; j < kRlwItems; ++j) {
    const bool valid = first + j < nvalid;
    const uint32_t r = k[j] & kRankMask;
    const bool nt = valid && (qk == 0xFFFFFFFFu || r != pr);
    const bool np = valid && (nt || d[j] != qd);
    npm |= (np ? 1u : 0u) << j;
    ntm |= (nt ? 1u : 0u) << j;
    pr = r;
    qd = d[j];
    qk = 0;
  }
}

template <bool PACKED>
__global__ void __launch_bounds__(kRlwThreads) k_rlw_count(const uint32_t* __restrict__ key,
                                                           const uint32_t* __restrict__ doc,
                                                           const unsigned long long* __restrict__ elem, uint64_t N,
                                                           uint64_t per, uint32_t* wcnt) {
  const uint32_t gw = blockIdx.x * kRlwWarps + (threadIdx.x >> 5);
  const uint64_t lo = (uint64_t)gw * per;
  const uint64_t hi = lo + per < N ? lo + per : N;
  uint32_t c = 0;
  if (lo < hi) {
    uint32_t pk = 0xFFFFFFFFu, pd = 0xFFFFFFFFu;
    if (lo > 0) rlw_at<PACKED>(key, doc, elem, lo - 1, pk, pd);
    for (uint64_t i0 = lo; i0 < hi; i0 += kRlwStep) {
      uint32_t k[kRlwItems], d[kRlwItems], npm, ntm;
      rlw_load<PACKED>(key, doc, elem, i0, hi, k, d);
      const uint32_t nvalid = (uint32_t)min((uint64_t)kRlwStep, hi - i0);
      rlw_flags(k, d, pk, pd, nvalid, npm, ntm);
      c += __popc(npm);
      pk = __shfl_sync(0xffffffffu, k[kRlwItems - 1], 31);
      pd = __shfl_sync(0xffffffffu, d[kRlwItems - 1], 31);
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) c += __shfl_xor_sync(0xffffffffu, c, o);
  }
  if (lane_id() == 0) wcnt[gw] = c;
}

// woff: exclusive posting offset of each warp range (scan of k_rlw_count); writes (docID, tf) at
// out_doc / out_tf [ostride * posting] (ostride 2: interleaved pairs), post_off / cstart at each term's
// key, range_lead[gw] = elements of the range before its first head
template <bool PACKED>
__global__ void __launch_bounds__(kRlwThreads, 3) k_rlw_write(const uint32_t* __restrict__ key,
                                                              const uint32_t* __restrict__ doc,
                                                              const unsigned long long* __restrict__ elem, uint64_t N,
                                                              uint64_t per,
                                                              const uint32_t* __restrict__ woff, uint32_t* out_doc,
                                                              uint32_t* out_tf, uint32_t ostride, uint64_t* post_off,
                                                              uint64_t* cstart, uint32_t* range_lead) {
  __shared__ uint2 stage[kRlwWarps][kRlwStep];
  const uint32_t lane = lane_id();
  const int w = threadIdx.x >> 5;
  const uint32_t gw = blockIdx.x * kRlwWarps + w;
  const uint64_t lo = (uint64_t)gw * per;
  const uint64_t hi = lo + per < N ? lo + per : N;
  if (lo >= hi) {
    if (lane == 0) range_lead[gw] = 0;
    return;
  }
  uint2* sg = stage[w];
  uint32_t pk = 0xFFFFFFFFu, pd = 0xFFFFFFFFu;
  if (lo > 0) rlw_at<PACKED>(key, doc, elem, lo - 1, pk, pd);
  uint32_t p = woff[gw];
  uint32_t lead = 0, open_len = 0, open_p = 0;
  bool lead_done = false, have_open = false;
  const uint32_t lt = (1u << lane) - 1u;
  for (uint64_t i0 = lo; i0 < hi; i0 += kRlwStep) {
    uint32_t k[kRlwItems], d[kRlwItems], npm, ntm;
    rlw_load<PACKED>(key, doc, elem, i0, hi, k, d);
    const uint32_t nvalid = (uint32_t)min((uint64_t)kRlwStep, hi - i0);
    rlw_flags(k, d, pk, pd, nvalid, npm, ntm);
    const uint32_t c = __popc(npm);
    uint32_t inc = c;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t u = __shfl_up_sync(0xffffffffu, inc, o);
      if ((int)lane >= o) inc += u;
    }
    const uint32_t T = __shfl_sync(0xffffffffu, inc, 31);
    const uint32_t base = lane * kRlwItems;
    // first head of each lane; next head after each lane (suffix min over later lanes)
    const uint32_t mine = npm ? base + __ffs(npm) - 1 : 0xFFFFFFFFu;
    uint32_t after = mine;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t u = __shfl_down_sync(0xffffffffu, after, o);
      if (lane + o < 32) after = min(after, u);
    }
    uint32_t next_after = __shfl_down_sync(0xffffffffu, after, 1);
    if (lane == 31) next_after = 0xFFFFFFFFu;
    const uint32_t first_all = __shfl_sync(0xffffffffu, after, 0);
    const uint32_t before = first_all == 0xFFFFFFFFu ? nvalid : first_all;  // elements before the step's first head
    if (!lead_done) {
      lead += before;
      lead_done = first_all != 0xFFFFFFFFu;
    }
    if (have_open) {  // the previous step's last posting runs into this step
      open_len += before;
      if (first_all != 0xFFFFFFFFu) {
        if (lane == 0) out_tf[(uint64_t)ostride * open_p] = open_len;
        have_open = false;
      }
    }
    uint32_t lp = inc - c;
    uint32_t last_tf = 0;
#pragma unroll
    for (int j = 0; j < kRlwItems; ++j) {
      if ((npm >> j) & 1u) {
        const uint32_t pos = base + j;
        const uint32_t rest = npm & ~((2u << j) - 1u);
        const uint32_t end = rest ? base + __ffs(rest) - 1 : min(next_after, nvalid);
        last_tf = end - pos;
        sg[lp] = make_uint2(d[j], last_tf);
        if ((ntm >> j) & 1u) {
          const uint32_t r = k[j] & kRankMask;
          post_off[r] = p + lp;
          cstart[r] = i0 + pos;
        }
        ++lp;
      }
    }
    __syncwarp();
    if (ostride == 2) {
      for (uint32_t x = lane; x < T; x += 32) __stcs((uint2*)out_doc + p + x, sg[x]);
    } else {
      for (uint32_t x = lane; x < T; x += 32) {
        const uint2 v = sg[x];
        __stcs(out_doc + p + x, v.x);
        __stcs(out_tf + p + x, v.y);
      }
    }
    if (T) {  // the step's last posting may continue into the next step
      const uint32_t hl = 31 - __clz(__ballot_sync(0xffffffffu, c != 0));  // lane holding it
      open_len = __shfl_sync(0xffffffffu, last_tf, hl);
      open_p = p + T - 1;
      have_open = true;
    }
    p += T;
    pk = __shfl_sync(0xffffffffu, k[kRlwItems - 1], 31);
    pd = __shfl_sync(0xffffffffu, d[kRlwItems - 1], 31);
    __syncwarp();
  }
  if (lane == 0) {
    if (have_open) out_tf[(uint64_t)ostride * open_p] = open_len;
    range_lead[gw] = lead;
  }
}

// runs that continue across tiles: add each tile's leading items to the preceding posting
__global__ void k_rle_fixup(const uint32_t* tile_p0, const uint32_t* tile_lead, uint32_t tiles, uint32_t* out_tf,
                            uint32_t ostride) {
  const uint32_t t = blockIdx.x * blockDim.x + threadIdx.x;
  if (t == 0 || t >= tiles) return;
  const uint32_t lead = tile_lead[t];
  if (lead) atomicAdd(&out_tf[(uint64_t)ostride * (tile_p0[t] - 1)], lead);
}

__global__ void k_df_cf(uint64_t* post_off, const uint64_t* cstart, uint32_t V, uint64_t P, uint64_t NT, uint32_t* df,
                        uint64_t* cf) {
  const uint32_t r = blockIdx.x * blockDim.x + threadIdx.x;
  if (r > V) return;
  if (r == V) { post_off[V] = P; return; }
  // post_off[r+1] may be written concurrently by another thread only for r+1 == V; read P instead
  const uint64_t a = post_off[r];
  const uint64_t b = (r + 1 < V) ? post_off[r + 1] : P;
  df[r] = (uint32_t)(b - a);
  const uint64_t ta = cstart[r];
  const uint64_t tb = (r + 1 < V) ? cstart[r + 1] : NT;
  cf[r] = tb - ta;
}

struct TermFullLen {  // full length of the term of rank r (rank_info written by k_lexrank)
  const uint2* rank_info;
  __device__ __forceinline__ uint64_t operator()(uint64_t r) const { return rank_info[r].y >> 16; }
};

// final dictionary bytes: trie prefix (restored) + stored suffix
// (grid-stride: launched with a few CTAs per SM, so that the finalize copy of the postings, queued right
// after it on the other stream, runs beside it instead of behind it)
__global__ void k_term_bytes(const uint2* rank_info, uint32_t V, const uint8_t* arena, const uint64_t* term_off,
                             uint8_t* out) {
  for (uint32_t r = blockIdx.x * blockDim.x + threadIdx.x; r < V; r += gridDim.x * blockDim.x) {
    const uint2 ri = rank_info[r];
    const uint32_t b = ri.y & 0xFFFFu, plen = bucket_plen(b), a = ri.x, slen = (ri.y >> 16) - plen;
    uint8_t* o = out + term_off[r];
    for (uint32_t i = 0; i < plen; ++i) o[i] = (uint8_t)prefix_byte(b, i);
    for (uint32_t i = 0; i < slen; ++i) o[plen + i] = arena[a + 1 + i];
  }
}

// ------------------------------------------------------------------ debug token dump
struct DumpSize {
  const uint32_t* len;
  __device__ __forceinline__ uint64_t operator()(uint64_t i) const { return 7 + len[i]; }
};

__global__ void k_dump_tokens(const uint8_t* text, const uint32_t* start, const uint32_t* len, const uint32_t* doc,
                              uint64_t n, const uint64_t* off, uint8_t* out) {
  const uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  const uint32_t s = start[i], l = len[i];
  const TermInfo ti = term_info(text, s, l);
  uint8_t* o = out + off[i];
  const uint32_t d = doc[i];
  o[0] = d & 255; o[1] = (d >> 8) & 255; o[2] = (d >> 16) & 255; o[3] = d >> 24;
  o[4] = ti.bucket & 255; o[5] = ti.bucket >> 8;
  o[6] = (uint8_t)l;
  for (uint32_t k = 0; k < l; ++k) {
    uint32_t c = text[s + k];
    o[7 + k] = (uint8_t)((c - 'A' < 26u) ? c + 32 : c);
  }
}

// ------------------------------------------------------------------ retrieval
struct QueryResult {
  uint32_t tid, rank;
  uint64_t lo, hi;
};

__global__ void k_query(DictView dv, const uint8_t* q, uint32_t len, const uint32_t* rank_of, const uint64_t* post_off,
                        QueryResult* res) {
  const TermInfo ti = term_info(q, 0, len);
  const TermWords tw(q, 0, len);
  const uint4 w = make_uint4(tw.word(0), 4 < len ? tw.word(1) : 0u, 8 < len ? tw.word(2) : 0u, 12 < len ? tw.word(3) : 0u);
  uint32_t r = 0;
  const uint32_t tid = probe_key(dv, w, q, 0, len, ti.bucket, ti.cache, &r);
  if (lane_id() == 0) {
    res->tid = tid;
    if (tid != kMiss) {
      const uint32_t rk = rank_of[tid];
      res->rank = rk;
      res->lo = post_off[rk];
      res->hi = post_off[rk + 1];
    }
  }
}

}  // namespace wj
