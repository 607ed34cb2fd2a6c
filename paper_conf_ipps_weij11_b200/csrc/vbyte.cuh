// f1: compressed postings, d-gaps + variable-byte code.
//
// Paper: "Because document IDs are stored in sorted order in each postings list, a basic idea used
// is to encode the gap between two neighbor document IDs instead of their absolute values combined
// with a compression strategy such as variable byte encoding"; post-processing "compress[es]
// them with variable bytes encoding".  Byte layout (reading S19): per posting vbyte(gap)
// then vbyte(tf), gap = docID for a list's first posting, else docID - previous docID; vbyte = 7-bit
// groups, least significant first, high bit set iff more bytes follow.
//
// B200 design (HBM-bound, three light passes over the (docID, tf) arrays the run-length pass wrote):
//   k_vb_first   one bit per posting marks the first posting of every term (from post_off);
//   k_vb_tile    per tile of 4096 postings: encoded bytes (block reduce) -> scanned on the device;
//   k_vb_encode  per tile: block scan of (bytes, list starts) per thread, encode 16 postings per
//                thread into shared memory, byte offsets of the tile's lists, one coalesced copy of
//                the tile's code to HBM.
#pragma once
#include "common.cuh"
#include "scan.cuh"

namespace wj {

constexpr int kVbThreads = 256;
constexpr int kVbItems = 16;
constexpr int kVbTile = kVbThreads * kVbItems;  // 4096 postings
constexpr int kVbMaxTileBytes = kVbTile * 10 + 16;  // <= 5 + 5 bytes per posting, + alignment

__device__ __forceinline__ uint32_t vb_len(uint32_t v) { return 1u + (31u - __clz(v | 1u)) / 7u; }

__global__ void k_vb_first(const uint64_t* post_off, uint32_t V, uint32_t* first_bits) {
  const uint32_t t = blockIdx.x * blockDim.x + threadIdx.x;
  if (t >= V) return;
  const uint64_t p = post_off[t];
  atomicOr(&first_bits[p >> 5], 1u << (p & 31));
}

// The thread's 16 consecutive postings [i0, i0+16): docIDs, tfs, list-start bits (16-byte vector
// loads when the group is complete; i0 is a multiple of 16).  dprev = docID before i0.
struct VbGroup {
  uint32_t d[kVbItems], f[kVbItems];
  uint32_t fm;     // bit k: posting i0+k starts a list
  uint32_t n;      // valid postings (< 16 only in the last group)
  uint32_t dprev;
};

__device__ __forceinline__ void vb_load(const uint32_t* doc, const uint32_t* tf, const uint32_t* first_bits,
                                        uint64_t P, uint64_t i0, VbGroup& g) {
  g.n = i0 >= P ? 0u : (uint32_t)min((uint64_t)kVbItems, P - i0);
  g.dprev = (i0 > 0 && i0 < P) ? doc[i0 - 1] : 0u;
  if (g.n == kVbItems) {
#pragma unroll
    for (int q = 0; q < kVbItems / 4; ++q) {
      const uint4 x = *(const uint4*)(doc + i0 + 4 * q);
      const uint4 y = *(const uint4*)(tf + i0 + 4 * q);
      g.d[4 * q] = x.x; g.d[4 * q + 1] = x.y; g.d[4 * q + 2] = x.z; g.d[4 * q + 3] = x.w;
      g.f[4 * q] = y.x; g.f[4 * q + 1] = y.y; g.f[4 * q + 2] = y.z; g.f[4 * q + 3] = y.w;
    }
  } else {
#pragma unroll
    for (int k = 0; k < kVbItems; ++k) {
      g.d[k] = k < (int)g.n ? doc[i0 + k] : 0u;
      g.f[k] = k < (int)g.n ? tf[i0 + k] : 0u;
    }
  }
  g.fm = g.n ? (first_bits[i0 >> 5] >> (i0 & 31)) & ((g.n == 32 ? 0u : (1u << g.n)) - 1u) : 0u;
  if (g.n == kVbItems) g.fm &= 0xFFFFu;
}

__device__ __forceinline__ uint32_t vb_gap(const VbGroup& g, int k) {
  return ((g.fm >> k) & 1u) ? g.d[k] : g.d[k] - (k ? g.d[k - 1] : g.dprev);
}

__device__ __forceinline__ uint32_t vb_group_bytes(const VbGroup& g) {
  uint32_t b = 0;
#pragma unroll
  for (int k = 0; k < kVbItems; ++k)
    if (k < (int)g.n) b += vb_len(vb_gap(g, k)) + vb_len(g.f[k]);
  return b;
}

__global__ void __launch_bounds__(kVbThreads) k_vb_tile(const uint32_t* doc, const uint32_t* tf,
                                                        const uint32_t* first_bits, uint64_t P, uint64_t* tile_bytes) {
  VbGroup g;
  vb_load(doc, tf, first_bits, P, (uint64_t)blockIdx.x * kVbTile + (uint64_t)threadIdx.x * kVbItems, g);
  uint32_t tot;
  block_exclusive_sum<uint32_t>(vb_group_bytes(g), tot);
  if (threadIdx.x == 0) tile_bytes[blockIdx.x] = tot;
}

__device__ __forceinline__ uint32_t vb_put(uint8_t* o, uint32_t v) {
  uint32_t n = 0;
  while (v >= 128u) {
    o[n++] = (uint8_t)(0x80u | (v & 127u));
    v >>= 7;
  }
  o[n++] = (uint8_t)v;
  return n;
}

// tile_off: exclusive byte offset of every tile (scanned k_vb_tile output).  post_boff[t] = byte
// offset of term t's list (t < V; the caller writes post_boff[V] = total).
__global__ void __launch_bounds__(kVbThreads) k_vb_encode(const uint32_t* doc, const uint32_t* tf,
                                                          const uint32_t* first_bits, uint64_t P,
                                                          const uint64_t* post_off, uint32_t V,
                                                          const uint64_t* tile_off, uint8_t* out, uint64_t* post_boff) {
  extern __shared__ __align__(16) uint8_t vb_smem[];
  __shared__ uint32_t s_t0;
  const uint64_t tile0 = (uint64_t)blockIdx.x * kVbTile;
  if (threadIdx.x == 0) {  // terms whose list starts before the tile
    uint32_t lo = 0, hi = V;
    while (lo < hi) {
      const uint32_t mid = (lo + hi) >> 1;
      if (post_off[mid] < tile0) lo = mid + 1; else hi = mid;
    }
    s_t0 = lo;
  }
  VbGroup g;
  vb_load(doc, tf, first_bits, P, tile0 + (uint64_t)threadIdx.x * kVbItems, g);
  uint32_t tot;
  const uint32_t ex = block_exclusive_sum<uint32_t>((vb_group_bytes(g) << 16) | (uint32_t)__popc(g.fm), tot);
  const uint64_t base = tile_off[blockIdx.x];
  // stage at smem byte (base & 3) + pos: smem word k <-> global word (base & ~3) / 4 + k
  const uint32_t a = (uint32_t)(base & 3u);
  uint32_t pos = a + (ex >> 16), t = s_t0 + (ex & 0xFFFFu);
#pragma unroll
  for (int k = 0; k < kVbItems; ++k) {
    if (k >= (int)g.n) break;
    if ((g.fm >> k) & 1u) post_boff[t++] = base + pos - a;
    pos += vb_put(vb_smem + pos, vb_gap(g, k));
    pos += vb_put(vb_smem + pos, g.f[k]);
  }
  __syncthreads();
  const uint32_t n = tot >> 16;
  if (n == 0) return;
  const uint32_t e = a + n;                  // smem end
  const uint32_t wb = (a + 3u) >> 2, we = e >> 2;  // whole words [wb, we)
  uint8_t* gw = out + (base - a);
  for (uint32_t j = threadIdx.x; j < 8; j += kVbThreads) {  // partial head / tail bytes
    const uint32_t h = a + j;
    if (j < 4 && h < 4u * wb && h < e) gw[h] = vb_smem[h];
    const uint32_t tl = 4u * max(we, wb) + (j - 4u);
    if (j >= 4 && tl < e) gw[tl] = vb_smem[tl];
  }
  for (uint32_t k = wb + threadIdx.x; k < we; k += kVbThreads) ((uint32_t*)gw)[k] = ((const uint32_t*)vb_smem)[k];
}

}  // namespace wj
