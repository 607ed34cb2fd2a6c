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

// stream termID -> term rank (in place)
__global__ void k_map_rank(uint32_t* tid, uint64_t N, const uint32_t* rank_of) {
  const uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i < N) tid[i] = __ldg(&rank_of[tid[i]]);
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

// Fused run-length pass (one read of the sorted (rank, doc) stream): a tile of 4096 tokens flags the
// first token of every posting (new rank or new doc) and of every term, numbers the postings with a
// block scan + decoupled look-back over tiles, and writes docid, tf, post_off[rank], tstart[rank].
// tf of a run that continues past the tile's end is completed by k_rle_fixup (tile_lead).
constexpr int kRleThreads = 256;
constexpr int kRleItems = 16;
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

__global__ void __launch_bounds__(kRleThreads) k_rle_fused(const uint32_t* __restrict__ key, const uint32_t* __restrict__ doc,
                                                           uint64_t N, uint32_t* out_doc, uint32_t* out_tf,
                                                           uint64_t* post_off, uint32_t* tstart, uint64_t* look,
                                                           uint32_t* tile_ctr, uint32_t* tile_p0, uint32_t* tile_lead,
                                                           uint32_t* total_p) {
  __shared__ uint32_t s_tile, s_p0;
  __shared__ uint32_t sm[16];
  __shared__ uint32_t st_doc[kRleTile], st_tf[kRleTile];  // tile postings, written out coalesced
  if (threadIdx.x == 0) s_tile = atomicAdd(tile_ctr, 1u);
  __syncthreads();
  const uint32_t tile = s_tile;
  const uint64_t base = (uint64_t)tile * kRleTile;
  const uint64_t i0 = base + (uint64_t)threadIdx.x * kRleItems;
  const uint32_t tile_len = (uint32_t)min((uint64_t)kRleTile, N - base);
  uint32_t k[kRleItems], d[kRleItems];
  if (i0 + kRleItems <= N) {
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
      const bool v = i0 + j < N;
      k[j] = v ? key[i0 + j] : 0xFFFFFFFFu;
      d[j] = v ? doc[i0 + j] : 0xFFFFFFFFu;
    }
  }
  uint32_t pk = 0xFFFFFFFFu, pd = 0xFFFFFFFFu;
  if (i0 > 0 && i0 <= N) { pk = key[i0 - 1]; pd = doc[i0 - 1]; }
  uint32_t npm = 0, ntm = 0;
#pragma unroll
  for (int j = 0; j < kRleItems; ++j) {
    const bool valid = i0 + j < N;
    const bool nt = valid && (i0 + j == 0 || k[j] != pk);
    const bool np = valid && (nt || d[j] != pd);
    npm |= (np ? 1u : 0u) << j;
    ntm |= (nt ? 1u : 0u) << j;
    pk = k[j];
    pd = d[j];
  }
  const uint32_t c = __popc(npm);
  uint32_t tot;
  const uint32_t ex = block_exclusive_sum<uint32_t>(c, tot);
  // first posting start of this thread (tile-relative) and the next one after this thread
  const uint32_t my_first = npm ? threadIdx.x * kRleItems + __ffs(npm) - 1 : 0xFFFFFFFFu;
  const uint32_t next_after = block_min_after(my_first, sm);
  // tile prefix of postings: decoupled look-back by warp 0, 32 predecessor tiles per step
  if (threadIdx.x < 32) {
    volatile uint64_t* lk = (volatile uint64_t*)look;
    const uint32_t lane = lane_id();
    if (lane == 0) lk[tile] = (tile == 0 ? kLbPre : kLbAgg) | tot;
    uint64_t prefix = 0;
    int64_t hiT = (int64_t)tile - 1;  // next predecessor to examine (window top)
    while (hiT >= 0) {
      const int64_t t = hiT - lane;
      uint64_t v = kLbPre;  // before tile 0: inclusive prefix 0
      if (t >= 0) v = lk[t];
      // wait until every lane of the window (up to the nearest inclusive prefix) is published
      for (;;) {
        const uint32_t notready = __ballot_sync(0xffffffffu, (v & (kLbAgg | kLbPre)) == 0);
        const uint32_t pre = __ballot_sync(0xffffffffu, (v & kLbPre) != 0);
        const uint32_t need = pre ? ((2u << (__ffs(pre) - 1)) - 1u) : 0xffffffffu;  // lanes up to nearest PRE
        if ((notready & need) == 0) break;
        if ((notready >> lane) & 1u) v = lk[t];
      }
      const uint32_t pre = __ballot_sync(0xffffffffu, (v & kLbPre) != 0);
      const int last = pre ? __ffs(pre) - 1 : 31;
      uint64_t x = lane <= (uint32_t)last ? (v & kLbVal) : 0;
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) x += __shfl_xor_sync(0xffffffffu, x, o);
      prefix += x;
      if (pre) break;
      hiT -= 32;
    }
    if (lane == 0) {
      if (tile > 0) lk[tile] = kLbPre | (prefix + tot);
      s_p0 = (uint32_t)prefix;
      tile_p0[tile] = (uint32_t)prefix;
      if (base + tile_len >= N) *total_p = (uint32_t)(prefix + tot);
    }
  }
  // leading continuation of the tile: items before the first posting start
  uint32_t first_all = min(my_first, next_after);
  if (threadIdx.x == 0) tile_lead[tile] = first_all == 0xFFFFFFFFu ? tile_len : first_all;
  __syncthreads();
  const uint32_t p0 = s_p0;
  uint32_t lp = ex;  // tile-local posting index
#pragma unroll
  for (int j = 0; j < kRleItems; ++j) {
    if ((npm >> j) & 1u) {
      const uint32_t rest = npm & ~((2u << j) - 1u);
      const uint32_t pos = threadIdx.x * kRleItems + j;
      const uint32_t end = rest ? threadIdx.x * kRleItems + __ffs(rest) - 1 : min(next_after, tile_len);
      st_doc[lp] = d[j];
      st_tf[lp] = end - pos;
      if ((ntm >> j) & 1u) {
        post_off[k[j]] = p0 + lp;
        tstart[k[j]] = (uint32_t)(i0 + j);
      }
      ++lp;
    }
  }
  __syncthreads();
  for (uint32_t x = threadIdx.x; x < tot; x += kRleThreads) {
    __stcs(out_doc + p0 + x, st_doc[x]);
    __stcs(out_tf + p0 + x, st_tf[x]);
  }
}

// ------------------------------------------------------------------ run-length, reduce-then-scan
// CTA c owns the contiguous token range [c*per, min(N,(c+1)*per)).  k_rle_count counts posting
// starts per range (one streaming read); a scan gives each range's first posting index; k_rle_write
// walks its range tile by tile with a running posting offset, carries the open run across its tiles,
// and writes docid/tf (coalesced through shared memory), post_off[rank], tstart[rank].  Runs that
// continue across ranges are completed by k_rle_fixup (range_lead).
constexpr int kRle2Ctas = 148 * 4;

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
      k[j] = v ? key[i0 + j] : 0xFFFFFFFFu;
      d[j] = v ? doc[i0 + j] : 0xFFFFFFFFu;
    }
  }
  pk = 0xFFFFFFFFu;
  pd = 0xFFFFFFFFu;
  if (i0 > 0) { pk = key[i0 - 1]; pd = doc[i0 - 1]; }
}

__device__ __forceinline__ void rle_flags(const uint32_t* k, const uint32_t* d, uint32_t pk, uint32_t pd, uint64_t i0,
                                          uint64_t hi, uint32_t& npm, uint32_t& ntm) {
  npm = 0;
  ntm = 0;
#pragma unroll
  for (int j = 0; j < kRleItems; ++j) {
    const bool valid = i0 + j < hi;
    const bool nt = valid && (i0 + j == 0 || k[j] != pk);
    const bool np = valid && (nt || d[j] != pd);
    npm |= (np ? 1u : 0u) << j;
    ntm |= (nt ? 1u : 0u) << j;
    pk = k[j];
    pd = d[j];
  }
}

__global__ void __launch_bounds__(kRleThreads) k_rle_count(const uint32_t* __restrict__ key, const uint32_t* __restrict__ doc,
                                                           uint64_t N, uint64_t per, uint32_t* range_cnt) {
  const uint64_t lo = (uint64_t)blockIdx.x * per;
  const uint64_t hi = lo + per < N ? lo + per : N;
  uint32_t c = 0;
  for (uint64_t i0 = lo + (uint64_t)threadIdx.x * kRleItems; i0 < hi; i0 += (uint64_t)kRleTile) {
    uint32_t k[kRleItems], d[kRleItems], pk, pd, npm, ntm;
    rle_load16(key, doc, i0, hi, k, d, pk, pd);
    rle_flags(k, d, pk, pd, i0, hi, npm, ntm);
    c += __popc(npm);
  }
  uint32_t tot;
  block_exclusive_sum<uint32_t>(c, tot);
  if (threadIdx.x == 0) range_cnt[blockIdx.x] = tot;
}

__global__ void __launch_bounds__(kRleThreads) k_rle_write(const uint32_t* __restrict__ key, const uint32_t* __restrict__ doc,
                                                           uint64_t N, uint64_t per, const uint32_t* __restrict__ range_off,
                                                           uint32_t* out_doc, uint32_t* out_tf, uint64_t* post_off,
                                                           uint32_t* tstart, uint32_t* range_lead) {
  __shared__ uint32_t sm[16];
  __shared__ uint32_t st_doc[kRleTile], st_tf[kRleTile];
  __shared__ uint32_t s_open_len, s_lead;
  __shared__ int s_lead_done;
  const uint64_t lo = (uint64_t)blockIdx.x * per;
  const uint64_t hi = lo + per < N ? lo + per : N;
  uint32_t p0 = range_off[blockIdx.x];
  // open run carried from the previous tile: its posting is p0 - 1 (tile-local index tot-1 written
  // as a partial tf into st_tf / global); s_open_len = tokens of it seen so far
  if (threadIdx.x == 0) { s_open_len = 0; s_lead = 0; s_lead_done = 0; }
  bool have_open = false;  // uniform
  uint32_t open_p = 0;
  __syncthreads();
  for (uint64_t base = lo; base < hi; base += kRleTile) {
    const uint32_t tile_len = (uint32_t)min((uint64_t)kRleTile, hi - base);
    const uint64_t i0 = base + (uint64_t)threadIdx.x * kRleItems;
    uint32_t k[kRleItems], d[kRleItems], pk, pd, npm, ntm;
    rle_load16(key, doc, i0, hi, k, d, pk, pd);
    rle_flags(k, d, pk, pd, i0, hi, npm, ntm);
    const uint32_t c = __popc(npm);
    uint32_t tot;
    const uint32_t ex = block_exclusive_sum<uint32_t>(c, tot);
    const uint32_t my_first = npm ? threadIdx.x * kRleItems + __ffs(npm) - 1 : 0xFFFFFFFFu;
    const uint32_t next_after = block_min_after(my_first, sm);
    const uint32_t first_all = min(my_first, next_after);  // valid in thread 0
    if (threadIdx.x == 0) {
      const uint32_t lead = first_all == 0xFFFFFFFFu ? tile_len : first_all;
      if (!s_lead_done) {  // items of the range before its first posting start
        s_lead += lead;
        if (first_all != 0xFFFFFFFFu) s_lead_done = 1;
      }
      if (have_open) {
        s_open_len += lead;
        if (first_all != 0xFFFFFFFFu) out_tf[open_p] = s_open_len;  // the carried run ends here
      }
    }
    uint32_t lp = ex;
#pragma unroll
    for (int j = 0; j < kRleItems; ++j) {
      if ((npm >> j) & 1u) {
        const uint32_t rest = npm & ~((2u << j) - 1u);
        const uint32_t pos = threadIdx.x * kRleItems + j;
        const uint32_t end = rest ? threadIdx.x * kRleItems + __ffs(rest) - 1 : min(next_after, tile_len);
        st_doc[lp] = d[j];
        st_tf[lp] = end - pos;
        if ((ntm >> j) & 1u) {
          post_off[k[j]] = p0 + lp;
          tstart[k[j]] = (uint32_t)(i0 + j);
        }
        ++lp;
      }
    }
    __syncthreads();
    for (uint32_t x = threadIdx.x; x < tot; x += kRleThreads) {
      __stcs(out_doc + p0 + x, st_doc[x]);
      __stcs(out_tf + p0 + x, st_tf[x]);
    }
    if (tot) {
      // the tile's last run may continue into the next tile
      have_open = true;
      open_p = p0 + tot - 1;
      if (threadIdx.x == 0) s_open_len = st_tf[tot - 1];
    } else if (threadIdx.x == 0 && have_open) {
      // whole tile continues the open run (already added as lead)
    }
    p0 += tot;
    __syncthreads();
  }
  if (threadIdx.x == 0) {
    if (have_open) out_tf[open_p] = s_open_len;
    range_lead[blockIdx.x] = s_lead_done ? s_lead : (uint32_t)(hi - lo);
  }
}

// k_rle_write with the next tile's keys/docs prefetched by TMA into a 2-stage shared-memory ring
inline size_t rle_smem_bytes() { return (size_t)4 * kRleTile * 4 /*2 stages x (key, doc)*/ + 2 * kRleTile * 4; }

__global__ void __launch_bounds__(kRleThreads, 2) k_rle_write_tma(const uint32_t* __restrict__ key,
                                                               const uint32_t* __restrict__ doc, uint64_t N,
                                                               uint64_t per, const uint32_t* __restrict__ range_off,
                                                               uint32_t* out_doc, uint32_t* out_tf, uint64_t* post_off,
                                                               uint32_t* tstart, uint32_t* range_lead) {
  extern __shared__ __align__(128) uint32_t rsm[];
  __shared__ __align__(8) uint64_t bar[2];
  __shared__ uint32_t sm[16];
  __shared__ uint32_t s_open_len, s_lead, s_prev_k, s_prev_d;
  __shared__ int s_lead_done;
  auto skey = [&](int s) { return rsm + (size_t)s * 2 * kRleTile; };
  auto sdoc = [&](int s) { return rsm + (size_t)s * 2 * kRleTile + kRleTile; };
  uint32_t* st_doc = rsm + 4 * kRleTile;
  uint32_t* st_tf = rsm + 5 * kRleTile;
  const uint64_t lo = (uint64_t)blockIdx.x * per;
  const uint64_t hi = lo + per < N ? lo + per : N;
  if (lo >= hi) return;
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
    const uint32_t pk = t0 ? ks[t0 - 1] : s_prev_k;
    const uint32_t pd = t0 ? ds[t0 - 1] : s_prev_d;
    uint32_t npm, ntm;
    rle_flags(k, d, pk, pd, base + t0, base + tile_len, npm, ntm);
    const uint32_t c = __popc(npm);
    uint32_t tot;
    const uint32_t ex = block_exclusive_sum<uint32_t>(c, tot);
    const uint32_t my_first = npm ? t0 + __ffs(npm) - 1 : 0xFFFFFFFFu;
    const uint32_t next_after = block_min_after(my_first, sm);
    if (threadIdx.x == 0) {
      const uint32_t first_all = min(my_first, next_after);
      const uint32_t lead = first_all == 0xFFFFFFFFu ? tile_len : first_all;
      if (!s_lead_done) {
        s_lead += lead;
        if (first_all != 0xFFFFFFFFu) s_lead_done = 1;
      }
      if (have_open) {
        s_open_len += lead;
        if (first_all != 0xFFFFFFFFu) out_tf[open_p] = s_open_len;
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
        st_tf[lp] = end - pos;
        if ((ntm >> j) & 1u) {
          post_off[k[j]] = p0 + lp;
          tstart[k[j]] = (uint32_t)(base + pos);
        }
        ++lp;
      }
    }
    __syncthreads();
    for (uint32_t x = threadIdx.x; x < tot; x += kRleThreads) {
      __stcs(out_doc + p0 + x, st_doc[x]);
      __stcs(out_tf + p0 + x, st_tf[x]);
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
    __syncthreads();
    s ^= 1;
  }
  if (threadIdx.x == 0) {
    if (have_open) out_tf[open_p] = s_open_len;
    range_lead[blockIdx.x] = s_lead_done ? s_lead : (uint32_t)(hi - lo);
  }
}

// runs that continue across tiles: add each tile's leading items to the preceding posting
__global__ void k_rle_fixup(const uint32_t* tile_p0, const uint32_t* tile_lead, uint32_t tiles, uint32_t* out_tf) {
  const uint32_t t = blockIdx.x * blockDim.x + threadIdx.x;
  if (t == 0 || t >= tiles) return;
  const uint32_t lead = tile_lead[t];
  if (lead) atomicAdd(&out_tf[tile_p0[t] - 1], lead);
}

__global__ void k_df_cf(uint64_t* post_off, const uint32_t* tstart, uint32_t V, uint64_t P, uint64_t N, uint32_t* df,
                        uint64_t* cf) {
  const uint32_t r = blockIdx.x * blockDim.x + threadIdx.x;
  if (r > V) return;
  if (r == V) { post_off[V] = P; return; }
  // post_off[r+1] may be written concurrently by another thread only for r+1 == V; read P instead
  const uint64_t a = post_off[r];
  const uint64_t b = (r + 1 < V) ? post_off[r + 1] : P;
  df[r] = (uint32_t)(b - a);
  const uint64_t ta = tstart[r];
  const uint64_t tb = (r + 1 < V) ? (uint64_t)tstart[r + 1] : N;
  cf[r] = tb - ta;
}

struct TermFullLen {
  const uint32_t* term_at;
  const uint32_t* t_bucket;
  const uint32_t* t_arena;
  const uint8_t* arena;
  __device__ __forceinline__ uint64_t operator()(uint64_t r) const {
    const uint32_t tid = term_at[r];
    return bucket_plen(t_bucket[tid]) + arena[t_arena[tid]];
  }
};

// final dictionary bytes: trie prefix (restored) + stored suffix
__global__ void k_term_bytes(const uint32_t* term_at, uint32_t V, const uint32_t* t_bucket, const uint32_t* t_arena,
                             const uint8_t* arena, const uint64_t* term_off, uint8_t* out) {
  const uint32_t r = blockIdx.x * blockDim.x + threadIdx.x;
  if (r >= V) return;
  const uint32_t tid = term_at[r];
  const uint32_t b = t_bucket[tid], plen = bucket_plen(b), a = t_arena[tid], slen = arena[a];
  uint8_t* o = out + term_off[r];
  for (uint32_t i = 0; i < plen; ++i) o[i] = (uint8_t)prefix_byte(b, i);
  for (uint32_t i = 0; i < slen; ++i) o[plen + i] = arena[a + 1 + i];
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
