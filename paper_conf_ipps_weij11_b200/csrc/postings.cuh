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
  // tile prefix of postings (decoupled look-back, thread 0)
  if (threadIdx.x == 0) {
    volatile uint64_t* lk = (volatile uint64_t*)look;
    uint64_t prefix = 0;
    if (tile == 0) {
      lk[0] = kLbPre | tot;
    } else {
      lk[tile] = kLbAgg | tot;
      int64_t t = (int64_t)tile - 1;
      for (;;) {
        const uint64_t v = lk[t];
        if ((v & (kLbAgg | kLbPre)) == 0) continue;
        prefix += v & kLbVal;
        if (v & kLbPre) break;
        --t;
      }
      lk[tile] = kLbPre | (prefix + tot);
    }
    s_p0 = (uint32_t)prefix;
    tile_p0[tile] = (uint32_t)prefix;
    if (base + tile_len >= N) *total_p = (uint32_t)(prefix + tot);
  }
  // leading continuation of the tile: items before the first posting start
  uint32_t first_all = min(my_first, next_after);
  if (threadIdx.x == 0) tile_lead[tile] = first_all == 0xFFFFFFFFu ? tile_len : first_all;
  __syncthreads();
  uint32_t p = s_p0 + ex;
#pragma unroll
  for (int j = 0; j < kRleItems; ++j) {
    if ((npm >> j) & 1u) {
      const uint32_t rest = npm & ~((2u << j) - 1u);
      const uint32_t pos = threadIdx.x * kRleItems + j;
      const uint32_t end = rest ? threadIdx.x * kRleItems + __ffs(rest) - 1 : min(next_after, tile_len);
      out_doc[p] = d[j];
      out_tf[p] = end - pos;
      if ((ntm >> j) & 1u) {
        post_off[k[j]] = p;
        tstart[k[j]] = (uint32_t)(i0 + j);
      }
      ++p;
    }
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
  uint32_t r = 0;
  const uint32_t tid = probe_key(dv, q, 0, len, ti.bucket, ti.cache, &r);
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
