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

namespace wj {

// stream termID -> term rank (in place)
__global__ void k_map_rank(uint32_t* tid, uint64_t N, const uint32_t* rank_of) {
  const uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i < N) tid[i] = __ldg(&rank_of[tid[i]]);
}

// per token of the chunk: slot -> termID (in place into the global stream)
__global__ void k_slot_to_tid(uint32_t* stream, uint64_t n, const uint32_t* slot_uid, const uint32_t* u_tid) {
  const uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i < n) stream[i] = __ldg(&u_tid[__ldg(&slot_uid[stream[i]])]);
}

struct NewPosting {
  const uint32_t* key;
  const uint32_t* doc;
  __device__ __forceinline__ uint32_t operator()(uint64_t i) const {
    return (i == 0 || key[i] != key[i - 1] || doc[i] != doc[i - 1]) ? 1u : 0u;
  }
};

// for each first token of a posting: docid, posting start; for each first token of a term: post_off, tstart
__global__ void k_rle_emit(const uint32_t* key, const uint32_t* doc, uint64_t N, const uint32_t* pidx,
                           uint32_t* out_doc, uint32_t* pstart, uint64_t* post_off, uint32_t* tstart) {
  const uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= N) return;
  const uint32_t k = key[i], d = doc[i];
  const bool new_term = i == 0 || key[i - 1] != k;
  if (new_term || doc[i - 1] != d) {
    const uint32_t p = pidx[i];
    out_doc[p] = d;
    pstart[p] = (uint32_t)i;
    if (new_term) { post_off[k] = p; tstart[k] = (uint32_t)i; }
  }
}

__global__ void k_rle_tf(const uint32_t* pstart, uint64_t P, uint64_t N, uint32_t* tf) {
  const uint64_t p = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (p >= P) return;
  const uint64_t nx = (p + 1 < P) ? pstart[p + 1] : N;
  tf[p] = (uint32_t)(nx - pstart[p]);
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
