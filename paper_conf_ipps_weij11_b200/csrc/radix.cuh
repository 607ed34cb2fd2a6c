// Stable LSD radix sort of (key, u32 value) pairs, 8-bit digits, reduce-then-scan per digit.
// Stability (equal keys keep input order) is what turns the docID-ordered token stream into
// docID-sorted postings: within one term, tokens stay in submission order.
#pragma once
#include "common.cuh"
#include "scan.cuh"

namespace wj {

constexpr int kRsThreads = 256;
constexpr int kRsWarps = kRsThreads / 32;
constexpr int kRsItems = 8;
constexpr int kRsTile = kRsThreads * kRsItems;  // 2048 elements per sub-tile
constexpr int kRsBins = 256;

// Histogram of one digit for the CTA's contiguous range [c*per, min(n,(c+1)*per)).
template <typename K>
__global__ void __launch_bounds__(kRsThreads) k_radix_hist(const K* __restrict__ keys, uint64_t n, uint64_t per,
                                                           int shift, uint32_t* __restrict__ hist) {
  __shared__ uint32_t h[kRsBins];
  for (int i = threadIdx.x; i < kRsBins; i += kRsThreads) h[i] = 0;
  __syncthreads();
  const uint64_t lo = (uint64_t)blockIdx.x * per;
  const uint64_t hi = lo + per < n ? lo + per : n;
  const uint32_t lane = lane_id();
  for (uint64_t b = lo; b < hi; b += kRsThreads) {
    const uint64_t i = b + threadIdx.x;
    const bool valid = i < hi;
    const uint32_t d = valid ? (uint32_t)((keys[i] >> shift) & 255u) : 256u + lane;
    const uint32_t peers = __match_any_sync(0xffffffffu, d);
    if (valid && lane == (uint32_t)(__ffs(peers) - 1)) atomicAdd(&h[d], (uint32_t)__popc(peers));
  }
  __syncthreads();
  for (int i = threadIdx.x; i < kRsBins; i += kRsThreads) hist[(uint64_t)i * gridDim.x + blockIdx.x] = h[i];
}

// Stable scatter: warp w of a sub-tile owns elements sub + w*256 + k*32 + lane (k < 8), so the
// (warp, round, lane) order is the input order; ranks = CTA offset + earlier warps + running count.
template <typename K>
__global__ void __launch_bounds__(kRsThreads) k_radix_scatter(const K* __restrict__ kin, const uint32_t* __restrict__ vin,
                                                              K* __restrict__ kout, uint32_t* __restrict__ vout,
                                                              uint64_t n, uint64_t per, int shift,
                                                              const uint32_t* __restrict__ offs) {
  __shared__ uint32_t wcnt[kRsWarps][kRsBins];
  __shared__ uint32_t base[kRsBins];
  const uint32_t lane = lane_id();
  const int w = threadIdx.x >> 5;
  for (int i = threadIdx.x; i < kRsBins; i += kRsThreads) {
    base[i] = offs[(uint64_t)i * gridDim.x + blockIdx.x];
#pragma unroll
    for (int x = 0; x < kRsWarps; ++x) wcnt[x][i] = 0;
  }
  __syncthreads();
  const uint64_t lo = (uint64_t)blockIdx.x * per;
  const uint64_t hi = lo + per < n ? lo + per : n;
  const uint32_t lt = (1u << lane) - 1u;
  for (uint64_t sub = lo; sub < hi; sub += kRsTile) {
    K key[kRsItems];
    uint32_t val[kRsItems], rank[kRsItems], dig[kRsItems];
#pragma unroll
    for (int k = 0; k < kRsItems; ++k) {
      const uint64_t i = sub + (uint64_t)w * (32 * kRsItems) + k * 32 + lane;
      const bool valid = i < hi;
      key[k] = valid ? kin[i] : K(0);
      val[k] = valid ? vin[i] : 0u;
      const uint32_t d = valid ? (uint32_t)((key[k] >> shift) & 255u) : 256u;
      const uint32_t peers = __match_any_sync(0xffffffffu, d);
      const int leader = __ffs(peers) - 1;
      uint32_t old = 0;
      if (valid && (int)lane == leader) {
        old = wcnt[w][d];
        wcnt[w][d] = old + __popc(peers);
      }
      old = __shfl_sync(0xffffffffu, old, leader);
      rank[k] = old + __popc(peers & lt);
      dig[k] = d;
      __syncwarp();
    }
    __syncthreads();
    for (int i = threadIdx.x; i < kRsBins; i += kRsThreads) {
      uint32_t run = base[i];
#pragma unroll
      for (int x = 0; x < kRsWarps; ++x) {
        const uint32_t t = wcnt[x][i];
        wcnt[x][i] = run;
        run += t;
      }
      base[i] = run;
    }
    __syncthreads();
#pragma unroll
    for (int k = 0; k < kRsItems; ++k) {
      if (dig[k] < 256u) {
        const uint32_t pos = wcnt[w][dig[k]] + rank[k];
        kout[pos] = key[k];
        vout[pos] = val[k];
      }
    }
    __syncthreads();
    for (int i = threadIdx.x; i < kRsBins; i += kRsThreads) {
#pragma unroll
      for (int x = 0; x < kRsWarps; ++x) wcnt[x][i] = 0;
    }
    __syncthreads();
  }
}

// ------------------------------------------------------------------ onesweep (decoupled look-back)
// One histogram pass computes every digit's global counts (fused with an optional key map); each
// digit pass is then a single kernel: dynamic tile id, stable in-tile rank (match_any + per-warp
// running counters), publish the tile's digit counts, look back over predecessor tiles for the
// exclusive prefix, stage the tile in shared memory in digit order and write it out so that
// consecutive threads write consecutive addresses inside each digit run.
constexpr int kOsThreads = 256;
constexpr int kOsWarps = kOsThreads / 32;
constexpr int kOsItems = 16;
constexpr int kOsTile = kOsThreads * kOsItems;  // 4096
constexpr uint64_t kLbAgg = 1ull << 62;
constexpr uint64_t kLbPre = 2ull << 62;
constexpr uint64_t kLbVal = (1ull << 62) - 1;

template <typename K>
inline size_t os_smem_bytes() { return (size_t)kOsTile * (sizeof(K) + sizeof(uint32_t)); }

// Global digit histograms of `passes` 8-bit digits starting at begin_bit.  If rank_of != nullptr the
// keys are first mapped in place: key = rank_of[key] (termID -> lexicographic rank).
template <typename K>
__global__ void __launch_bounds__(256) k_os_hist(K* keys, uint64_t n, int begin_bit, int passes,
                                                 const uint32_t* __restrict__ rank_of, uint32_t* ghist) {
  __shared__ uint32_t h[sizeof(K)][256];
  for (int i = threadIdx.x; i < (int)sizeof(K) * 256; i += blockDim.x) (&h[0][0])[i] = 0;
  __syncthreads();
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += stride) {
    K k = keys[i];
    if (rank_of) {
      k = (K)__ldg(&rank_of[(uint32_t)k]);
      keys[i] = k;
    }
    for (int p = 0; p < passes; ++p) atomicAdd(&h[p][(uint32_t)(k >> (begin_bit + 8 * p)) & 255u], 1u);
  }
  __syncthreads();
  for (int i = threadIdx.x; i < passes * 256; i += blockDim.x) {
    const uint32_t v = (&h[0][0])[i];
    if (v) atomicAdd(&ghist[i], v);
  }
}

// exclusive scan of each pass's 256 counts (one CTA of 256 threads per pass)
__global__ void __launch_bounds__(256) k_os_hist_scan(uint32_t* ghist) {
  uint32_t* h = ghist + blockIdx.x * 256;
  const uint32_t v = h[threadIdx.x];
  uint32_t tot;
  const uint32_t ex = block_exclusive_sum<uint32_t>(v, tot);
  h[threadIdx.x] = ex;
}

template <typename K>
__global__ void __launch_bounds__(kOsThreads, 3) k_os_pass(const K* __restrict__ kin, const uint32_t* __restrict__ vin,
                                                        K* __restrict__ kout, uint32_t* __restrict__ vout, uint64_t n,
                                                        int shift, const uint32_t* __restrict__ gofs,
                                                        uint64_t* look, uint32_t* tile_ctr) {
  extern __shared__ __align__(16) unsigned char os_smem[];
  K* sk = (K*)os_smem;
  uint32_t* sv = (uint32_t*)(os_smem + (size_t)kOsTile * sizeof(K));
  __shared__ uint32_t wcnt[kOsWarps][256];
  __shared__ uint32_t dig_off[256];
  __shared__ uint32_t dig_glob[256];
  __shared__ uint32_t s_tile;
  const uint32_t lane = lane_id();
  const int w = threadIdx.x >> 5;
  if (threadIdx.x == 0) s_tile = atomicAdd(tile_ctr, 1u);
  for (int x = 0; x < kOsWarps; ++x) wcnt[x][threadIdx.x] = 0;
  __syncthreads();
  const uint32_t tile = s_tile;
  const uint64_t base = (uint64_t)tile * kOsTile;
  const uint32_t lt = (1u << lane) - 1u;
  K key[kOsItems];
  uint32_t rank[kOsItems];
#pragma unroll
  for (int k = 0; k < kOsItems; ++k) {
    const uint64_t i = base + (uint64_t)w * (32 * kOsItems) + k * 32 + lane;
    key[k] = i < n ? kin[i] : K(0);
  }
#pragma unroll
  for (int k = 0; k < kOsItems; ++k) {
    const uint64_t i = base + (uint64_t)w * (32 * kOsItems) + k * 32 + lane;
    const bool valid = i < n;
    const uint32_t d = valid ? (uint32_t)((key[k] >> shift) & 255u) : 256u;
    const uint32_t peers = __match_any_sync(0xffffffffu, d);
    const int leader = __ffs(peers) - 1;
    uint32_t old = 0;
    if (valid && (int)lane == leader) {
      old = wcnt[w][d];
      wcnt[w][d] = old + __popc(peers);
    }
    old = __shfl_sync(0xffffffffu, old, leader);
    rank[k] = old + __popc(peers & lt);
    __syncwarp();
  }
  __syncthreads();
  // per digit: exclusive offsets across warps, tile count
  const uint32_t d = threadIdx.x;
  uint32_t cnt = 0;
#pragma unroll
  for (int x = 0; x < kOsWarps; ++x) {
    const uint32_t t = wcnt[x][d];
    wcnt[x][d] = cnt;
    cnt += t;
  }
  // publish this tile's aggregate (or inclusive prefix for tile 0)
  volatile uint64_t* lk = (volatile uint64_t*)look;
  if (tile == 0) lk[d] = kLbPre | cnt;
  else lk[(uint64_t)tile * 256 + d] = kLbAgg | cnt;
  uint32_t tot;
  const uint32_t toff = block_exclusive_sum<uint32_t>(cnt, tot);
  dig_off[d] = toff;
  uint64_t prefix = 0;
  if (tile > 0) {
    int64_t t = (int64_t)tile - 1;
    for (;;) {
      const uint64_t v = lk[(uint64_t)t * 256 + d];
      if ((v & (kLbAgg | kLbPre)) == 0) continue;
      prefix += v & kLbVal;
      if (v & kLbPre) break;
      --t;
    }
    lk[(uint64_t)tile * 256 + d] = kLbPre | (prefix + cnt);
  }
  dig_glob[d] = gofs[d] + (uint32_t)prefix - toff;
  __syncthreads();
#pragma unroll
  for (int k = 0; k < kOsItems; ++k) {
    const uint64_t i = base + (uint64_t)w * (32 * kOsItems) + k * 32 + lane;
    if (i < n) {
      const uint32_t dk = (uint32_t)((key[k] >> shift) & 255u);
      const uint32_t p = dig_off[dk] + wcnt[w][dk] + rank[k];
      sk[p] = key[k];
      sv[p] = vin[i];  // values are read only now (coalesced), keeping registers for occupancy
    }
  }
  __syncthreads();
  const uint32_t tn = (uint32_t)((n - base) < (uint64_t)kOsTile ? (n - base) : (uint64_t)kOsTile);
  for (uint32_t j = threadIdx.x; j < tn; j += kOsThreads) {
    const K kk = sk[j];
    const uint32_t pos = dig_glob[(uint32_t)((kk >> shift) & 255u)] + j;
    kout[pos] = kk;
    vout[pos] = sv[j];
  }
}

struct RadixPlan {
  uint64_t per;
  uint32_t ctas;
};

inline RadixPlan radix_plan(uint64_t n) {
  const uint64_t target = 148 * 8;
  uint64_t per = (n + target - 1) / target;
  per = ((per + kRsTile - 1) / kRsTile) * kRsTile;
  if (per == 0) per = kRsTile;
  return RadixPlan{per, (uint32_t)((n + per - 1) / per)};
}

inline size_t radix_hist_bytes(uint64_t n) { return (size_t)radix_plan(n).ctas * kRsBins * 4 + 256; }

// Sorts bits [begin_bit, end_bit) of the keys.  (k0,v0) is the input; (k1,v1) scratch of equal
// size.  Returns true if the result ended in (k1,v1).  hist: radix_hist_bytes(n) bytes (x2 for
// the scanned copy); scan_scratch: scan_scratch_bytes<uint32_t>(256*ctas).  *launches += count.
template <typename K>
inline bool radix_sort_pairs(K* k0, uint32_t* v0, K* k1, uint32_t* v1, uint64_t n, int begin_bit, int end_bit,
                             uint32_t* hist, uint32_t* hist_scan, void* scan_scratch, cudaStream_t st,
                             uint64_t* launches) {
  if (n <= 1 || end_bit <= begin_bit) return false;
  const RadixPlan p = radix_plan(n);
  bool in1 = false;
  for (int shift = begin_bit; shift < end_bit; shift += 8) {
    K* ki = in1 ? k1 : k0;
    uint32_t* vi = in1 ? v1 : v0;
    K* ko = in1 ? k0 : k1;
    uint32_t* vo = in1 ? v0 : v1;
    k_radix_hist<K><<<p.ctas, kRsThreads, 0, st>>>(ki, n, p.per, shift, hist);
    *launches += 1;
    *launches += exclusive_scan<uint32_t>(ArrayIn<uint32_t>{hist}, (uint64_t)kRsBins * p.ctas, hist_scan,
                                          (uint32_t*)nullptr, scan_scratch, st);
    k_radix_scatter<K><<<p.ctas, kRsThreads, 0, st>>>(ki, vi, ko, vo, n, p.per, shift, hist_scan);
    *launches += 1;
    in1 = !in1;
  }
  return in1;
}

}  // namespace wj
