// Per-document pre-aggregation of the (term, docID) stream ("doc combine"), before the finalize sort.
//
// P:196 updates the postings list of a term on every occurrence; a posting is (DocID, tf).
// All occurrences of a term inside one document collapse into one posting, so the stream elements
// of one (term, docID) pair can be merged before the group-by: the stream shrinks from N tokens to
// ~0.68 N elements on config 2 (4096-element tiles), which every radix pass and the run-length pass
// then move once less per merged token.
//
// Element format (postings.cuh): key = id | count << 25 (id = key & kRankMask: a chunk slot, or a
// rank once the chunk maps are applied; count 1..127 tokens), value = docID.  Input elements are
// single tokens (bits above kRankMask are ignored).
//
// Layout: CTA c owns the contiguous range [c*per, min(n, (c+1)*per)) of the stream -- the same ranges
// as the first radix pass -- walks it in 4096-element tiles, and writes the tile's merged elements
// compacted at the front of its range (in place: the write cursor never passes the read cursor).
// range_len[c] = elements kept; the first radix pass reads only [c*per, c*per + range_len[c]).
//
// Per tile (no shared-memory CAS: 64-bit CAS runs at ~2 cycles/lane on sm_100a):
//  1. docs are numbered inside the tile (block scan of "docID changes"), key = (id, local doc);
//  2. round-based insertion into a shared open-addressing table with plain 64-bit loads/stores: a
//     pending item reads its slot; empty -> it stores (key | own item index) and becomes a candidate,
//     its own key -> candidate, another key -> next slot; after a barrier every candidate re-reads:
//     only empty slots are stored to and the last store won, so a key holds exactly one slot with
//     one stored item index (its leader), and all items of the key resolve to it (equal keys probe
//     identical sequences);
//  3. every item adds 1 to its leader's counter (shared atomic add, no return value);
//  4. leaders, in item order, emit ceil(count / 127) elements, so for one id the elements keep
//     ascending docIDs and the stable sort downstream still yields docID-sorted postings;
//     a pair split across tiles yields one element per tile and the run-length pass sums them.
#pragma once
#include "common.cuh"
#include "postings.cuh"
#include "scan.cuh"

namespace wj {

constexpr int kDcThreads = 256;  // block_exclusive_sum is a 256-thread scan
constexpr int kDcItems = 16;
constexpr int kDcTile = kDcThreads * kDcItems;  // 4096 (the radix tile: ranges are multiples of it)
constexpr int kDcHashBits = 13;
constexpr int kDcHash = 1 << kDcHashBits;  // load factor <= 0.5
constexpr uint32_t kDcMaxCount = (1u << (32 - kCountShift)) - 1u;  // 127
// table entry: bit 63 valid | item index (12 bits) << 37 | local doc (12 bits) << 25 | id (25 bits)
constexpr uint64_t kDcValid = 1ull << 63;
constexpr uint64_t kDcKeyMask = kDcValid | ((1ull << 37) - 1);

inline size_t dc_smem_bytes() {
  return (size_t)kDcHash * 8 /*table*/ + (size_t)kDcTile * 4 /*leader counts*/ + (size_t)kDcTile * 8 /*staged out*/;
}

__device__ __forceinline__ uint32_t dc_hash(uint32_t id, uint32_t dl) {
  uint32_t h = id * 0x9E3779B1u ^ (dl + 1u) * 0x85EBCA77u;
  h ^= h >> 15;
  h *= 0x2C1B3C6Du;
  return h >> (32 - kDcHashBits);
}

__global__ void __launch_bounds__(kDcThreads, 2) k_doc_combine(uint32_t* key, uint32_t* doc, uint64_t n, uint64_t per,
                                                               uint32_t* range_len) {
  extern __shared__ __align__(16) unsigned char dc_smem[];
  uint64_t* hk = (uint64_t*)dc_smem;
  uint32_t* hc = (uint32_t*)(dc_smem + (size_t)kDcHash * 8);
  uint32_t* st_k = hc + kDcTile;
  uint32_t* st_d = st_k + kDcTile;
  __shared__ uint32_t s_lastdoc[kDcThreads];
  const uint64_t lo = (uint64_t)blockIdx.x * per;
  const uint64_t hi = lo + per < n ? lo + per : n;
  if (lo >= hi) {
    if (threadIdx.x == 0) range_len[blockIdx.x] = 0;
    return;
  }
  for (int i = threadIdx.x; i < kDcHash; i += kDcThreads) hk[i] = 0ull;
  for (int i = threadIdx.x; i < kDcTile; i += kDcThreads) hc[i] = 0u;
  __syncthreads();
  const uint32_t t0 = threadIdx.x * kDcItems;
  uint64_t out = lo;
  for (uint64_t base = lo; base < hi; base += kDcTile) {
    const uint32_t tn = (uint32_t)min((uint64_t)kDcTile, hi - base);
    uint32_t k[kDcItems], d[kDcItems];
    if (t0 + kDcItems <= tn) {  // tiles start 16 KB aligned in the stream: vector loads
#pragma unroll
      for (int q = 0; q < kDcItems / 4; ++q) {
        const uint4 a = *(const uint4*)(key + base + t0 + 4 * q);
        const uint4 b = *(const uint4*)(doc + base + t0 + 4 * q);
        k[4 * q] = a.x; k[4 * q + 1] = a.y; k[4 * q + 2] = a.z; k[4 * q + 3] = a.w;
        d[4 * q] = b.x; d[4 * q + 1] = b.y; d[4 * q + 2] = b.z; d[4 * q + 3] = b.w;
      }
    } else {
#pragma unroll
      for (int j = 0; j < kDcItems; ++j) {
        const bool v = t0 + j < tn;
        k[j] = v ? key[base + t0 + j] : 0u;
        d[j] = v ? doc[base + t0 + j] : 0xFFFFFFFFu;
      }
    }
    const uint32_t nv = tn > t0 ? min(tn - t0, (uint32_t)kDcItems) : 0u;
    const uint32_t valid = (1u << nv) - 1u;  // nv <= 16
    // 1. local document numbers: changes of docID in item order (docIDs are non-decreasing)
    s_lastdoc[threadIdx.x] = d[kDcItems - 1];
    __syncthreads();
    const uint32_t d_before = threadIdx.x ? s_lastdoc[threadIdx.x - 1] : d[0];
    uint32_t prevd = d_before, chg = 0;
#pragma unroll
    for (int j = 0; j < kDcItems; ++j) {
      chg += ((valid >> j) & 1u) && d[j] != prevd ? 1u : 0u;
      prevd = d[j];
    }
    uint32_t tot_chg;
    uint32_t dl = block_exclusive_sum<uint32_t>(chg, tot_chg);  // barriers: s_lastdoc reads done
    uint64_t ek[kDcItems];  // entry key (without the item index)
    uint32_t hs[kDcItems];  // probe slot
    prevd = d_before;
#pragma unroll
    for (int j = 0; j < kDcItems; ++j) {
      if (((valid >> j) & 1u) && d[j] != prevd) ++dl;
      prevd = d[j];
      const uint32_t id = k[j] & kRankMask;
      ek[j] = kDcValid | ((uint64_t)(dl & 0xFFFu) << 25) | id;
      hs[j] = dc_hash(id, dl);
    }
    // 2. round-based insertion (plain loads/stores, two barriers per round)
    uint32_t pend = valid, lead = 0;
    uint32_t own[kDcItems];
    while (__syncthreads_or(pend)) {
      uint32_t cand = 0;
#pragma unroll
      for (int j = 0; j < kDcItems; ++j) {
        if ((pend >> j) & 1u) {
          const uint64_t v = hk[hs[j]];
          if (v == 0ull) {
            hk[hs[j]] = ek[j] | ((uint64_t)(t0 + j) << 37);
            cand |= 1u << j;
          } else if ((v & kDcKeyMask) == ek[j]) {
            cand |= 1u << j;  // may be a store of this phase that a later store replaces: verify
          } else {
            hs[j] = (hs[j] + 1u) & (kDcHash - 1);
          }
        }
      }
      __syncthreads();
#pragma unroll
      for (int j = 0; j < kDcItems; ++j) {
        if ((cand >> j) & 1u) {
          const uint64_t v = hk[hs[j]];
          if ((v & kDcKeyMask) == ek[j]) {
            own[j] = (uint32_t)(v >> 37) & 0xFFFu;
            pend &= ~(1u << j);
          } else {
            hs[j] = (hs[j] + 1u) & (kDcHash - 1);
          }
        }
      }
    }
    // 3. counts at the leaders (the loop's final __syncthreads_or separates the reads above)
#pragma unroll
    for (int j = 0; j < kDcItems; ++j) {
      if ((valid >> j) & 1u) {
        atomicAdd(&hc[own[j]], 1u);
        if (own[j] == t0 + j) lead |= 1u << j;
      }
    }
    __syncthreads();
    // 4. leaders emit in item order; they also clear their table slot and counter
    uint32_t ne = 0;
    uint32_t cnt[kDcItems];
#pragma unroll
    for (int j = 0; j < kDcItems; ++j) {
      cnt[j] = 0;
      if ((lead >> j) & 1u) {
        cnt[j] = hc[t0 + j];
        ne += (cnt[j] + kDcMaxCount - 1) / kDcMaxCount;
        hc[t0 + j] = 0u;
        hk[hs[j]] = 0ull;
      }
    }
    uint32_t tot;
    uint32_t p = block_exclusive_sum<uint32_t>(ne, tot);
#pragma unroll
    for (int j = 0; j < kDcItems; ++j) {
      uint32_t c = cnt[j];
      while (c > 0) {  // m tokens of a pair give ceil(m / 127) <= m elements
        const uint32_t e = min(c, kDcMaxCount);
        st_k[p] = (k[j] & kRankMask) | (e << kCountShift);
        st_d[p] = d[j];
        ++p;
        c -= e;
      }
    }
    __syncthreads();
    for (uint32_t x = threadIdx.x; x < tot; x += kDcThreads) {
      key[out + x] = st_k[x];
      doc[out + x] = st_d[x];
    }
    out += tot;
    __syncthreads();
  }
  if (threadIdx.x == 0) range_len[blockIdx.x] = (uint32_t)(out - lo);
}

}  // namespace wj
