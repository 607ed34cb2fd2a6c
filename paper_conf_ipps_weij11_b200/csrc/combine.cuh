// Per-document pre-aggregation of the (term, docID) stream ("doc combine").
//
// P:196 updates the postings list of a term on every occurrence; a posting is (DocID, tf).
// All occurrences of a term inside one document collapse into one posting, so the stream elements
// of one (slot, docID) pair can be merged before the finalize group-by: the stream shrinks from N
// tokens to ~P postings (0.68 N on config 2 with 4096-token tiles), which every radix pass and the
// run-length pass then read and write once less per merged token.
//
// Element format (postings.cuh): key = slot | count << 25 (count 1..127 tokens), value = docID.
// CTA = one 4096-element tile of the stream, claimed in order by an atomic ticket.  Every element
// is inserted into a shared-memory hash table keyed by (docID, slot) (64-bit CAS); the CAS winner is
// the pair's leader and counts add up with shared atomics.  Leaders emit ceil(count / 127)
// elements, in token order of the leaders, so for one slot the elements keep ascending docIDs and
// the stable sort downstream still yields docID-sorted postings.  A pair split across tiles
// (a document crossing a tile boundary) yields one element per tile; the run-length pass sums them
// (tf = sum of counts over equal (rank, docID) runs).
//
// The output is written in place, compacted: tile t's elements go to [prefix_t, prefix_t + A_t)
// with prefix_t from a decoupled look-back over the tile aggregates.  prefix_t + A_t <= the end of
// tile t's input, and prefix_t is known only after every earlier tile has published (i.e. loaded
// its input), so no tile overwrites input that has not been read.
#pragma once
#include "common.cuh"
#include "postings.cuh"
#include "scan.cuh"

#ifndef DC_VARIANT
#define DC_VARIANT 0  // microbenchmark switches (tools/micro/dc_bench.cu): 1 no look-back, 2 no hash
#endif

namespace wj {

constexpr int kDcThreads = 256;  // block_exclusive_sum is a 256-thread scan
constexpr int kDcItems = 16;
constexpr int kDcTile = kDcThreads * kDcItems;  // 4096
constexpr int kDcHash = 2 * kDcTile;            // load factor <= 0.5
constexpr uint32_t kDcMaxCount = (1u << (32 - kCountShift)) - 1u;  // 127
constexpr uint64_t kDcEmpty = ~0ull;
constexpr uint64_t kDcAgg = 1ull << 62;
constexpr uint64_t kDcPre = 2ull << 62;
constexpr uint64_t kDcVal = (1ull << 62) - 1;

inline size_t dc_smem_bytes() { return (size_t)kDcHash * (sizeof(uint64_t) + sizeof(uint32_t)); }

__device__ __forceinline__ uint32_t dc_hash(uint32_t slot, uint32_t doc) {
  uint32_t h = slot * 0x9E3779B1u ^ doc * 0x85EBCA77u;
  h ^= h >> 15;
  h *= 0x2C1B3C6Du;
  return h >> (32 - 13);
}
static_assert(kDcHash == 1 << 13, "dc_hash returns 13 bits");

// look[ntiles] and *tile_ctr zeroed by the caller; *n_out = elements after the combine.
__global__ void __launch_bounds__(kDcThreads, 2) k_doc_combine(uint32_t* key, uint32_t* doc, uint64_t n,
                                                               uint32_t ntiles, uint64_t* look, uint32_t* tile_ctr,
                                                               uint32_t* n_out) {
  extern __shared__ __align__(16) unsigned char dc_smem[];
  uint64_t* hk = (uint64_t*)dc_smem;
  uint32_t* hc = (uint32_t*)(dc_smem + (size_t)kDcHash * sizeof(uint64_t));
  __shared__ uint32_t s_tile;
  __shared__ uint64_t s_prefix;
  if (threadIdx.x == 0) s_tile = atomicAdd(tile_ctr, 1u);
  {
    uint4* z = (uint4*)dc_smem;
    const uint4 e8 = make_uint4(~0u, ~0u, ~0u, ~0u), z4 = make_uint4(0, 0, 0, 0);
    for (int i = threadIdx.x; i < kDcHash / 2; i += kDcThreads) z[i] = e8;
    for (int i = threadIdx.x; i < kDcHash / 4; i += kDcThreads) z[kDcHash / 2 + i] = z4;
  }
  __syncthreads();
  const uint32_t tile = s_tile;
  if (tile >= ntiles) return;
  const uint64_t base = (uint64_t)tile * kDcTile;
  const uint32_t tn = (uint32_t)min((uint64_t)kDcTile, n - base);
  const uint32_t t0 = threadIdx.x * kDcItems;
  uint32_t k[kDcItems], d[kDcItems];
  if (t0 + kDcItems <= tn) {  // stream segments start 16-byte aligned only by chance: scalar loads
#pragma unroll
    for (int j = 0; j < kDcItems; ++j) {
      k[j] = key[base + t0 + j];
      d[j] = doc[base + t0 + j];
    }
  } else {
#pragma unroll
    for (int j = 0; j < kDcItems; ++j) {
      const bool v = t0 + j < tn;
      k[j] = v ? key[base + t0 + j] : 0u;
      d[j] = v ? doc[base + t0 + j] : 0u;
    }
  }
  uint32_t idx[kDcItems];  // hash index, then the pair's token count (leaders)
  uint32_t lead = 0;
#pragma unroll
  for (int j = 0; j < kDcItems; ++j) {
    idx[j] = 0;
    if (DC_VARIANT & 2) { if (t0 + j < tn) { lead |= 1u << j; idx[j] = 0; } continue; }
    if (t0 + j < tn) {
      const uint32_t slot = k[j] & kRankMask;
      const uint64_t pk = ((uint64_t)d[j] << 32) | slot;
      uint32_t h = dc_hash(slot, d[j]);
      for (;;) {
        const unsigned long long old = atomicCAS((unsigned long long*)&hk[h], (unsigned long long)kDcEmpty,
                                                 (unsigned long long)pk);
        if (old == kDcEmpty) { lead |= 1u << j; break; }
        if (old == pk) break;
        h = (h + 1) & (kDcHash - 1);
      }
      atomicAdd(&hc[h], k[j] >> kCountShift);
      idx[j] = h;
    }
  }
  __syncthreads();
  uint32_t ne = 0;
#pragma unroll
  for (int j = 0; j < kDcItems; ++j) {
    if ((lead >> j) & 1u) {
      const uint32_t c = (DC_VARIANT & 2) ? 1u : hc[idx[j]];
      idx[j] = c;
      k[j] &= kRankMask;
      ne += (c + kDcMaxCount - 1) / kDcMaxCount;
    }
  }
  uint32_t tot;
  const uint32_t ex = block_exclusive_sum<uint32_t>(ne, tot);  // contains barriers: hash reads done
  // stage the tile's output in the (now unused) hash table: keys, then docIDs
  uint32_t* st_k = (uint32_t*)dc_smem;
  uint32_t* st_d = st_k + kDcTile;
  uint32_t p = ex;
#pragma unroll
  for (int j = 0; j < kDcItems; ++j) {
    if ((lead >> j) & 1u) {
      uint32_t c = idx[j];  // m input elements of count <= 127 give <= m output elements
      while (c > 0) {
        const uint32_t e = min(c, kDcMaxCount);
        st_k[p] = k[j] | (e << kCountShift);
        st_d[p] = d[j];
        ++p;
        c -= e;
      }
    }
  }
  // decoupled look-back over the tile aggregates (tiles are claimed in order), one warp reading 32
  // predecessors per step
  if ((DC_VARIANT & 1) && threadIdx.x == 0) s_prefix = base;
  if (!(DC_VARIANT & 1) && threadIdx.x < 32) {
    const uint32_t lane = threadIdx.x;
    volatile uint64_t* lk = (volatile uint64_t*)look;
    if (lane == 0) lk[tile] = (tile == 0 ? kDcPre : kDcAgg) | tot;
    uint64_t prefix = 0;
    int64_t end = (int64_t)tile;  // look at tiles [end - 32, end)
    while (end > 0) {
      const int64_t t = end - 1 - (int64_t)lane;
      uint64_t v = kDcPre;  // before tile 0: an inclusive prefix of 0
      if (t >= 0) {
        do { v = lk[t]; } while ((v & (kDcAgg | kDcPre)) == 0);
      }
      const uint32_t pre = __ballot_sync(0xffffffffu, (v & kDcPre) != 0);
      const uint32_t upto = pre ? (uint32_t)(__ffs(pre) - 1) : 31u;  // nearest inclusive prefix
      uint64_t x = lane <= upto ? (v & kDcVal) : 0ull;
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) x += __shfl_xor_sync(0xffffffffu, x, o);
      prefix += x;
      if (pre) break;
      end -= 32;
    }
    if (lane == 0) {
      if (tile > 0) lk[tile] = kDcPre | (prefix + tot);
      s_prefix = prefix;
      if (tile == ntiles - 1) *n_out = (uint32_t)(prefix + tot);
    }
  }
  __syncthreads();
  const uint64_t ob = s_prefix;
  for (uint32_t x = threadIdx.x; x < tot; x += kDcThreads) {
    key[ob + x] = st_k[x];
    doc[ob + x] = st_d[x];
  }
}

}  // namespace wj
