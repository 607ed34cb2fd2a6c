// Partial postings lists per run, combined at finalize.
//
// The paper's indexer appends each run's postings to partial lists and post-processing combines the
// partial lists of a term in run order (docIDs ascend across runs).  Here a run is one
// index_add_stream chunk: its (slot, docID) stream is sorted by chunk slot and run-length encoded on
// a side stream while the dictionary update of the same chunk runs on the main stream, giving per
// chunk a CSR by slot.  Once the chunk's slots are mapped to termIDs, one record per unique term
// (termID, start, df, cf) describes the term's partial list.  Finalize accumulates df / cf per term
// over the chunks (in chunk order, which also gives each partial its offset inside the term's final
// list), scans df in lexicographic rank order into post_off, and copies every partial list to its
// final place.
#pragma once
#include "common.cuh"

namespace wj {

// Per unique term u of a chunk (u ascending = slot ascending = the order of the sorted runs):
// start / df / cf of its partial list from the run-length output (post_off / cstart indexed by slot).
// With hot terms (hot_pos != nullptr) a hot slot (k1 hot id) has no stream elements: its list is row
// h of the hot matrix, appended after the *P_rle run-length postings; a non-hot term's list ends where
// the next non-hot term's begins (at most kHotMax hot terms lie in between).  NT = stream tokens.
// With hot terms the records are ordered like the partial lists: non-hot terms in slot order at their
// rank among the non-hot ones (nh_pos), then the H hot terms in hot-id order.
__global__ void k_chunk_records(const uint32_t* __restrict__ u_slot, uint32_t U, const uint64_t* __restrict__ post_off,
                                const uint64_t* __restrict__ cstart, const uint32_t* __restrict__ P_rle, uint64_t NT,
                                const uint32_t* __restrict__ NT_dev, const uint32_t* __restrict__ u_tid, uint64_t pbase,
                                uint32_t* rec_tid,
                                uint64_t* rec_start, uint32_t* rec_df, uint32_t* rec_cf, const Slot* __restrict__ table,
                                const uint32_t* __restrict__ hot_pos, const uint32_t* __restrict__ hot_cf, uint32_t D,
                                const uint32_t* __restrict__ nh_pos, const uint32_t* __restrict__ H_dev,
                                uint4* rec_aos) {
  const uint32_t u = blockIdx.x * blockDim.x + threadIdx.x;
  if (u >= U) return;
  auto hot_of = [&](uint32_t slot) -> uint32_t {
    return hot_pos ? (uint32_t)(table[slot].k1 >> kHotShift) : 0u;
  };
  const uint32_t s = u_slot[u];
  const uint32_t h = hot_of(s);
  const uint32_t r = h ? U - *H_dev + (h - 1) : (hot_pos ? nh_pos[u] : u);
  rec_tid[r] = u_tid[u];
  if (h) {
    const uint64_t a = hot_pos[(uint64_t)(h - 1) * D], b = hot_pos[(uint64_t)h * D];
    rec_start[r] = pbase + *P_rle + a;
    rec_df[r] = (uint32_t)(b - a);
    rec_cf[r] = hot_cf[h - 1];
    return;
  }
  const uint64_t a = post_off[s], ta = cstart[s];
  uint64_t b = *P_rle, tb = NT_dev ? *NT_dev : NT;  // NT_dev: stream tokens left after the hot holes
  for (uint32_t v = u + 1; v < U; ++v) {
    const uint32_t s2 = u_slot[v];
    if (hot_of(s2)) continue;
    b = post_off[s2];
    tb = cstart[s2];
    break;
  }
  rec_start[r] = pbase + a;
  rec_df[r] = (uint32_t)(b - a);
  rec_cf[r] = (uint32_t)(tb - ta);
  if (rec_aos)  // the same record as one 16-byte line (finalize of a run indexed by termID, k_lexrank)
    rec_aos[r] = make_uint4((uint32_t)(pbase + a), (uint32_t)((pbase + a) >> 32), (uint32_t)(b - a), (uint32_t)(tb - ta));
}

struct NotHotSlot {  // 1 for a unique term whose slot carries no hot id
  const uint32_t* u_slot;
  const Slot* table;
  __device__ __forceinline__ uint32_t operator()(uint64_t u) const {
    return (table[u_slot[u]].k1 >> kHotShift) ? 0u : 1u;
  }
};

// One chunk's records, in chunk order: offset of the partial inside its term's list = postings of
// the term in earlier chunks; termIDs are distinct within a chunk, so there is no conflict.
__global__ void k_rec_accum(const uint32_t* __restrict__ rec_tid, const uint32_t* __restrict__ rec_df,
                            const uint32_t* __restrict__ rec_cf, uint64_t lo, uint64_t hi, uint32_t* df_tot,
                            uint64_t* cf_tot, uint32_t* before) {
  const uint64_t i = lo + (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= hi) return;
  const uint32_t t = rec_tid[i];
  before[i] = df_tot[t];
  df_tot[t] += rec_df[i];
  cf_tot[t] += rec_cf[i];
}

// termID-indexed totals -> rank order (df, cf of the final dictionary)
__global__ void k_rank_scatter(const uint32_t* __restrict__ rank_of, uint32_t V, const uint32_t* __restrict__ df_tot,
                               const uint64_t* __restrict__ cf_tot, uint32_t* df, uint64_t* cf) {
  const uint32_t t = blockIdx.x * blockDim.x + threadIdx.x;
  if (t >= V) return;
  const uint32_t r = rank_of[t];
  df[r] = df_tot[t];
  cf[r] = cf_tot[t];
}

// a single run: the records are the terms, df / cf straight to rank order, and the start of each rank's list
__global__ void k_rank_scatter_rec(const uint32_t* __restrict__ rec_tid, const uint32_t* __restrict__ rec_df,
                                   const uint32_t* __restrict__ rec_cf, uint64_t R, const uint32_t* __restrict__ rank_of,
                                   uint32_t* df, uint64_t* cf, const uint64_t* __restrict__ rec_start,
                                   uint64_t* src_of_rank) {
  const uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= R) return;
  const uint32_t r = rank_of[rec_tid[i]];
  df[r] = rec_df[i];
  cf[r] = rec_cf[i];
  src_of_rank[r] = rec_start[i];  // sequential read here, so the copy reads its sources in rank order
}

// Single run: the same copy walked in destination (rank) order -- warp w writes the final postings
// [w * kCopyChunk, (w + 1) * kCopyChunk) coalesced and gathers them from the partial lists (each
// term's list is contiguous in both).
__global__ void __launch_bounds__(256) k_copy_by_rank(const uint64_t* __restrict__ src_of_rank, uint32_t V, uint64_t P,
                                                      const uint64_t* __restrict__ post_off,
                                                      const uint2* __restrict__ pp,
                                                      uint32_t* __restrict__ out_doc, uint32_t* __restrict__ out_tf);

// several runs: each record's (rank of its term) as the key of a stable sort that puts the records in
// destination order (rank, then run), and its index as the value
__global__ void k_rec_rank_key(const uint32_t* __restrict__ rec_tid, uint64_t R, const uint32_t* __restrict__ rank_of,
                               uint32_t* key, uint32_t* idx) {
  const uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= R) return;
  key[i] = rank_of[rec_tid[i]];
  idx[i] = (uint32_t)i;
}

// records in destination order -> (destination start, source start) of each partial list; the
// destination starts increase strictly (df >= 1), so k_copy_by_rank copies them like one run's lists
__global__ void k_rec_dest(const uint32_t* __restrict__ sorted, uint64_t R, const uint32_t* __restrict__ rec_tid,
                           const uint32_t* __restrict__ before, const uint64_t* __restrict__ rec_start,
                           const uint32_t* __restrict__ rank_of, const uint64_t* __restrict__ post_off,
                           uint64_t* dst_start, uint64_t* src_start) {
  const uint64_t j = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (j >= R) return;
  const uint32_t i = sorted[j];
  dst_start[j] = post_off[rank_of[rec_tid[i]]] + before[i];
  src_start[j] = rec_start[i];
}

struct U32AsU64 {
  const uint32_t* p;
  __device__ __forceinline__ uint64_t operator()(uint64_t i) const { return p[i]; }
};

constexpr uint32_t kCopyChunk = 1024;  // postings per warp of the copy

__global__ void __launch_bounds__(256) k_copy_by_rank(const uint64_t* __restrict__ src_of_rank, uint32_t V, uint64_t P,
                                                      const uint64_t* __restrict__ post_off,
                                                      const uint2* __restrict__ pp,
                                                      uint32_t* __restrict__ out_doc, uint32_t* __restrict__ out_tf) {
  const uint64_t w = ((uint64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const uint32_t lane = threadIdx.x & 31;
  uint64_t lo = w * kCopyChunk;
  if (lo >= P) return;
  const uint64_t hi = lo + kCopyChunk < P ? lo + kCopyChunk : P;
  uint64_t r = 0;  // last rank with post_off <= lo
  if (lane == 0) {
    uint64_t a = 0, b = V;
    while (b - a > 1) {
      const uint64_t m = (a + b) >> 1;
      if (post_off[m] <= lo) a = m; else b = m;
    }
    r = a;
  }
  r = __shfl_sync(0xffffffffu, r, 0);
  for (;;) {
    const uint64_t i = r + lane;
    const bool v = i < V;
    const uint64_t d0 = v ? post_off[i] : ~0ull;
    const uint64_t src = v ? src_of_rank[i] : 0ull;
    const uint64_t wend = (r + 32 < V) ? post_off[r + 32] : P;  // first posting after the window
    const uint64_t e = wend < hi ? wend : hi;
    const uint64_t ws = __shfl_sync(0xffffffffu, d0, 0);
    const uint32_t drel = v ? (uint32_t)(d0 - ws) : 0xFFFFFFFFu;
    constexpr int Q = 4;  // gathers in flight per lane (8: 0.54 -> 0.65 ms, profiles/r02_README.md)
    for (uint64_t base = lo; base < e; base += 32 * Q) {  // warp-uniform trip count
      uint32_t dv[Q], tv[Q];
#pragma unroll
      for (int q = 0; q < Q; ++q) {
        const uint64_t p = base + 32 * q + lane;
        const uint32_t pr = (uint32_t)(p - ws);
        uint32_t j = 0;  // last lane of the window whose list starts at or before p
#pragma unroll
        for (int b = 16; b > 0; b >>= 1) {
          const uint32_t dj = __shfl_sync(0xffffffffu, drel, j + b);
          if (dj <= pr) j += b;
        }
        const uint32_t dj = __shfl_sync(0xffffffffu, drel, j);
        const uint64_t sp = __shfl_sync(0xffffffffu, src, j) + (pr - dj);
        if (p < e) {
          const uint2 x = __ldg(pp + sp);
          dv[q] = x.x;
          tv[q] = x.y;
        }
      }
#pragma unroll
      for (int q = 0; q < Q; ++q) {
        const uint64_t p = base + 32 * q + lane;
        if (p < e) {
          __stcs(out_doc + p, dv[q]);
          __stcs(out_tf + p, tv[q]);
        }
      }
    }
    if (e >= hi) break;
    lo = e;
    r += 32;
  }
}

}  // namespace wj
