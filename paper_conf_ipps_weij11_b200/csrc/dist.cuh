// Multi-GPU pack / unpack kernels.
//
// Ownership: trie collection b belongs to rank b mod K — the paper's static split of collections
// over GPUs, "assigning the trie collection TC_i with index i to the GPU whose index is given by
// i mod N_2" — or, with WJ_FLAG_BALANCED_OWNERS, to the rank a sampled
// bin-packing picked (engine.cu build_owner_map).  Each rank owns an exclusive slice of the
// dictionary.
//
// Per chunk, rank r has tokenised its own document range into a chunk table (unique terms) and a
// (slot, docID) stream.  For every owner o it sends
//   * the folded bytes of the unique terms it saw whose collection o owns, each followed by ' '
//     (so the owner can run the received bytes through the same tokenizer/dedup kernels), and
//   * one record (xid, docID) per token of those terms, in stream (= docID) order, xid = the
//     term's index in the list sent to o.
// The owner appends the records in source-rank order, so postings stay docID-sorted.
#pragma once
#include "common.cuh"
#include "dict.cuh"

namespace wj {

// per-owner counts: block histogram in shared memory, one global atomic per (block, owner)
constexpr int kMaxRanks = 1024;

__global__ void k_owner(const uint32_t* u_bucket, uint32_t U, uint32_t K, const uint32_t* owner_tab, uint32_t* owner,
                        uint32_t* iota, uint32_t* owner_cnt) {
  __shared__ uint32_t h[kMaxRanks];
  for (uint32_t i = threadIdx.x; i < K; i += blockDim.x) h[i] = 0;
  __syncthreads();
  const uint32_t u = blockIdx.x * blockDim.x + threadIdx.x;
  if (u < U) {
    const uint32_t b = u_bucket[u];
    const uint32_t o = owner_tab ? owner_tab[b] : b % K;
    owner[u] = o;
    iota[u] = u;
    atomicAdd(&h[o], 1u);
  }
  __syncthreads();
  for (uint32_t i = threadIdx.x; i < K; i += blockDim.x)
    if (h[i]) atomicAdd(&owner_cnt[i], h[i]);
}

// xid = index of the unique term in the list sent to its owner (terms sorted stably by owner)
__global__ void k_xid(const uint32_t* sorted_u, uint32_t U, const uint32_t* u_owner, const uint64_t* t_off,
                      uint32_t* xid) {
  const uint32_t j = blockIdx.x * blockDim.x + threadIdx.x;
  if (j >= U) return;
  const uint32_t u = sorted_u[j];
  xid[u] = j - (uint32_t)t_off[u_owner[u]];
}

struct PackTermSize {
  const uint32_t* sorted_u;  // nullptr: identity (unique terms already in owner order)
  const uint32_t* u_len;
  __device__ __forceinline__ uint64_t operator()(uint64_t j) const {
    return (uint64_t)u_len[sorted_u ? sorted_u[j] : (uint32_t)j] + 1;
  }
};

__global__ void k_pack_terms(const uint32_t* sorted_u, uint32_t U, const uint64_t* boff, const uint4* u_w,
                             const uint8_t* text, const uint32_t* u_ref, const uint32_t* u_len, uint8_t* out) {
  const uint32_t j = blockIdx.x * blockDim.x + threadIdx.x;
  if (j >= U) return;
  const uint32_t u = sorted_u ? sorted_u[j] : j;
  const uint4 w = u_w[u];
  const uint32_t len = u_len[u], ref = u_ref[u];
  uint8_t* o = out + boff[j];
  for (uint32_t i = 0; i < len; ++i) o[i] = (uint8_t)ubyte(w, text, ref, i);
  o[len] = ' ';
}

__global__ void k_tok_owner(const uint32_t* slot, uint64_t n, const uint32_t* slot_uid, const uint32_t* u_owner,
                            uint32_t K, uint32_t* tkey, uint32_t* tidx, uint32_t* tok_cnt) {
  __shared__ uint32_t h[kMaxRanks];
  for (uint32_t i = threadIdx.x; i < K; i += blockDim.x) h[i] = 0;
  __syncthreads();
  const uint64_t t = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (t < n) {
    const uint32_t o = u_owner[slot_uid[slot[t] & ((1u << 25) - 1u)]];
    tkey[t] = o;
    tidx[t] = (uint32_t)t;
    atomicAdd(&h[o], 1u);
  }
  __syncthreads();
  for (uint32_t i = threadIdx.x; i < K; i += blockDim.x)
    if (h[i]) atomicAdd(&tok_cnt[i], h[i]);
}

// K > 64 path: records gathered in owner order from the sorted token indices
__global__ void k_pack_tok(const uint32_t* sorted_t, uint64_t n, const uint32_t* slot, const uint32_t* doc,
                           const uint32_t* slot_uid, const uint32_t* xid, uint32_t* rkey, uint32_t* rdoc) {
  const uint64_t j = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (j >= n) return;
  const uint32_t t = sorted_t[j];
  rkey[j] = xid[slot_uid[slot[t] & ((1u << 25) - 1u)]];
  rdoc[j] = doc[t];
}

// K <= 64 path: per table slot, the token's record key owner << 26 | xid (bit 25 stays the stream
// element's count flag); one radix pass over the (slot, docID) stream with this map applied in the
// histogram pass partitions the records by owner, stably (docID order kept per owner).
constexpr uint32_t kXidMask = (1u << 25) - 1u;
constexpr int kOwnerShift = 26;
__global__ void k_slot_xkey(const Slot* table, uint32_t C, const uint32_t* slot_uid, const uint32_t* u_owner,
                            const uint32_t* xid, uint32_t* km) {
  const uint32_t i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= C || table[i].k0 == 0) return;
  const uint32_t u = slot_uid[i];
  km[i] = (u_owner[u] << kOwnerShift) | xid[u];
}

// owner side: the records of source s carry xid = index of the term in the text s sent; the
// received text was tokenised as one synthetic document, so term j has token j and slot syn_slot[j].
// map[xid] = termID of term (base + xid); registered as the stream segment's map.
__global__ void k_xid_map(const uint32_t* syn_slot, uint32_t n, const Slot* table, const uint32_t* slot_uid,
                          const uint32_t* u_tid, uint32_t* map) {
  const uint32_t x = blockIdx.x * blockDim.x + threadIdx.x;
  if (x >= n) return;
  const uint32_t sl = syn_slot[x] & kXidMask;
  map[x] = table[sl].k0 ? u_tid[slot_uid[sl]] : 0u;
}

// ------------------------------------------------------------------ sender-side partial lists
// (SURVEY 8(e)): every rank's chunk table is partitioned by owner, so sorting and
// run-length encoding its stream by slot makes the postings it sends to owner o one contiguous range
// of (docID, tf) pairs, grouped per term (P:160-162's per-term grouping, aggregated to one posting per
// (term, document)); a header (df, cf) per term and the folded term bytes go with them.

// per unique term u (slot order = owner order: the chunk table is partitioned by owner): df, cf of
// its local partial list from the run-length output (post_off / cstart indexed by slot; every unique
// term occurs); P_dev = postings of the chunk, NT = its tokens
__global__ void k_term_hdr(const uint32_t* u_slot, uint32_t U, const uint64_t* post_off, const uint64_t* cstart,
                           const uint32_t* P_dev, uint64_t NT, uint32_t* df, uint32_t* cf) {
  const uint32_t u = blockIdx.x * blockDim.x + threadIdx.x;
  if (u >= U) return;
  const uint32_t s = u_slot[u];
  const uint64_t b = u + 1 < U ? post_off[u_slot[u + 1]] : (uint64_t)*P_dev;
  const uint64_t tb = u + 1 < U ? cstart[u_slot[u + 1]] : NT;
  df[u] = (uint32_t)(b - post_off[s]);
  cf[u] = (uint32_t)(tb - cstart[s]);
}

// per owner o (o <= K): postings / tokens before its first term (t_off[o] = its first unique term)
__global__ void k_owner_bounds(const uint32_t* u_slot, const uint64_t* post_off, const uint64_t* cstart,
                               const uint64_t* t_off, uint32_t K, uint32_t U, const uint32_t* P_dev, uint64_t NT,
                               uint64_t* p_off, uint64_t* c_off) {
  const uint32_t o = blockIdx.x * blockDim.x + threadIdx.x;
  if (o > K) return;
  const uint64_t u = t_off[o];
  p_off[o] = u < U ? post_off[u_slot[u]] : (uint64_t)*P_dev;
  c_off[o] = u < U ? cstart[u_slot[u]] : NT;
}

// first unique term of each table partition: t_off[o] = uid of slot o * Cp (exclusive scan), t_off[K] = U
__global__ void k_part_bounds(const uint32_t* uid, uint32_t K, uint64_t Cp, const uint32_t* U_dev, uint64_t* t_off) {
  const uint32_t o = blockIdx.x * blockDim.x + threadIdx.x;
  if (o > K) return;
  t_off[o] = o < K ? uid[(uint64_t)o * Cp] : *U_dev;
}

// owner side: the records of source s's terms (xid order = the order s sent them): termID from the
// owner's dictionary, start = base + exclusive prefix of df, df, cf
__global__ void k_recv_records(const uint32_t* syn_slot, uint32_t n, const Slot* table, const uint32_t* slot_uid,
                               const uint32_t* u_tid, const uint32_t* hdf, const uint32_t* hcf, const uint64_t* dprefix,
                               uint64_t base, uint32_t* rec_tid, uint64_t* rec_start, uint32_t* rec_df,
                               uint32_t* rec_cf) {
  const uint32_t x = blockIdx.x * blockDim.x + threadIdx.x;
  if (x >= n) return;
  const uint32_t sl = syn_slot[x] & kXidMask;
  rec_tid[x] = u_tid[slot_uid[sl]];
  rec_start[x] = base + dprefix[x];
  rec_df[x] = hdf[x];
  rec_cf[x] = hcf[x];
}

}  // namespace wj
