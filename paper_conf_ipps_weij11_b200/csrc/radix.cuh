// Stable LSD radix sort of (key, u32 value) pairs, 8-bit digits, reduce-then-scan per digit.
// Stability (equal keys keep input order) is what turns the docID-ordered token stream into
// docID-sorted postings: within one term, tokens stay in submission order.
#pragma once
#include <type_traits>
#include "common.cuh"
#include "scan.cuh"
#include "tma.cuh"

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

// Lanes holding the same 8-bit digit (a warp-wide multi-split with 8 ballots: cheaper than
// MATCH.ANY on sm_100a); `valid` lanes only.
__device__ __forceinline__ uint32_t digit_peers(uint32_t d, bool valid) {
  uint32_t peers = __ballot_sync(0xffffffffu, valid);
#pragma unroll
  for (int b = 0; b < 8; ++b) {
    const bool bit = (d >> b) & 1u;
    const uint32_t m = __ballot_sync(0xffffffffu, bit);
    peers &= bit ? m : ~m;
  }
  return peers;
}

// Same result through a per-warp table of 256 lane masks in shared memory (all zero on entry and
// on exit): one shared atomic OR per lane instead of 8 ballots.
__device__ __forceinline__ uint32_t digit_peers_smem(uint32_t* bins, uint32_t d, bool valid) {
  const uint32_t lane = lane_id();
  if (valid) atomicOr(&bins[d], 1u << lane);
  __syncwarp();
  const uint32_t peers = valid ? bins[d] : 0u;
  __syncwarp();
  if (valid && (peers & ((1u << lane) - 1u)) == 0) bins[d] = 0u;  // the lowest peer clears
  __syncwarp();
  return peers;
}

template <typename K>
__global__ void __launch_bounds__(kOsThreads, 4) k_os_pass(const K* __restrict__ kin, const uint32_t* __restrict__ vin,
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
    const uint32_t d = (uint32_t)((key[k] >> shift) & 255u);
    const uint32_t peers = digit_peers(d, valid);
    const int leader = valid ? __ffs(peers) - 1 : (int)lane;
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

// Persistent onesweep pass with TMA: each CTA claims tiles in order (atomic counter), prefetches the
// next tile's keys and values into the other half of a 2-stage shared-memory ring with one
// cp.async.bulk each (completion on an mbarrier), ranks the current tile from shared memory,
// publishes / looks back, stages the tile in digit order in the same buffer and writes it out.
template <typename K>
inline size_t os_tma_smem_bytes() { return 2 * (size_t)kOsTile * (sizeof(K) + sizeof(uint32_t)); }

template <typename K>
__global__ void __launch_bounds__(kOsThreads, 2) k_os_pass_tma(const K* __restrict__ kin, const uint32_t* __restrict__ vin,
                                                            K* __restrict__ kout, uint32_t* __restrict__ vout, uint64_t n,
                                                            int shift, const uint32_t* __restrict__ gofs, uint64_t* look,
                                                            uint32_t* tile_ctr, uint32_t ntiles) {
  extern __shared__ __align__(128) unsigned char os_smem[];
  __shared__ __align__(8) uint64_t bar[2];
  __shared__ uint32_t wcnt[kOsWarps][256];
  __shared__ uint32_t dig_off[256];
  __shared__ uint32_t dig_glob[256];
  __shared__ uint32_t s_tile[2];
  const size_t stage_bytes = (size_t)kOsTile * (sizeof(K) + sizeof(uint32_t));
  auto skey = [&](int s) { return (K*)(os_smem + s * stage_bytes); };
  auto sval = [&](int s) { return (uint32_t*)(os_smem + s * stage_bytes + (size_t)kOsTile * sizeof(K)); };
  const uint32_t lane = lane_id();
  const int w = threadIdx.x >> 5;
  const uint32_t lt = (1u << lane) - 1u;

  auto issue = [&](int s, uint32_t tile) {  // thread 0
    const uint64_t base = (uint64_t)tile * kOsTile;
    const uint32_t cnt = (uint32_t)((n - base) < (uint64_t)kOsTile ? (n - base) : (uint64_t)kOsTile);
    const uint32_t bk = (uint32_t)((cnt * sizeof(K) + 15) & ~(size_t)15);
    const uint32_t bv = (cnt * 4 + 15) & ~15u;
    fence_proxy_async_smem();
    mbar_arrive_expect_tx(&bar[s], bk + bv);
    tma_load_1d(skey(s), kin + base, bk, &bar[s]);
    tma_load_1d(sval(s), vin + base, bv, &bar[s]);
  };

  if (threadIdx.x == 0) {
    mbar_init(&bar[0], 1);
    mbar_init(&bar[1], 1);
    fence_mbar_init();
  }
  for (int x = 0; x < kOsWarps; ++x) wcnt[x][threadIdx.x] = 0;
  __syncthreads();
  if (threadIdx.x == 0) {
    const uint32_t t = atomicAdd(tile_ctr, 1u);
    s_tile[0] = t;
    if (t < ntiles) issue(0, t);
  }
  __syncthreads();
  uint32_t parity = 0u;  // bit s: phase of stage s
  int s = 0;
  for (;;) {
    const uint32_t tile = s_tile[s];
    if (tile >= ntiles) break;
    if (threadIdx.x == 0) {  // prefetch the next tile into the other stage
      const uint32_t t2 = atomicAdd(tile_ctr, 1u);
      s_tile[s ^ 1] = t2;
      if (t2 < ntiles) issue(s ^ 1, t2);
    }
    mbar_wait(&bar[s], (parity >> s) & 1u);
    parity ^= 1u << s;
    const uint64_t base = (uint64_t)tile * kOsTile;
    const K* sk = skey(s);
    uint32_t* sv = sval(s);
    K key[kOsItems];
    uint32_t val[kOsItems], rank[kOsItems];
#pragma unroll
    for (int k = 0; k < kOsItems; ++k) {
      const uint32_t li = w * (32 * kOsItems) + k * 32 + lane;
      key[k] = sk[li];
      val[k] = sv[li];
    }
#pragma unroll
    for (int k = 0; k < kOsItems; ++k) {
      const uint64_t i = base + (uint64_t)w * (32 * kOsItems) + k * 32 + lane;
      const bool valid = i < n;
      const uint32_t d = (uint32_t)((key[k] >> shift) & 255u);
      const uint32_t peers = digit_peers(d, valid);
      const int leader = valid ? __ffs(peers) - 1 : (int)lane;
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
    const uint32_t d = threadIdx.x;
    uint32_t cnt = 0;
#pragma unroll
    for (int x = 0; x < kOsWarps; ++x) {
      const uint32_t t = wcnt[x][d];
      wcnt[x][d] = cnt;
      cnt += t;
    }
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
    // stage in digit order (same buffer: every thread already holds its keys and values)
    K* sko = (K*)sk;
#pragma unroll
    for (int k = 0; k < kOsItems; ++k) {
      const uint64_t i = base + (uint64_t)w * (32 * kOsItems) + k * 32 + lane;
      if (i < n) {
        const uint32_t dk = (uint32_t)((key[k] >> shift) & 255u);
        const uint32_t p = dig_off[dk] + wcnt[w][dk] + rank[k];
        sko[p] = key[k];
        sv[p] = val[k];
      }
    }
    __syncthreads();
    const uint32_t tn = (uint32_t)((n - base) < (uint64_t)kOsTile ? (n - base) : (uint64_t)kOsTile);
    for (uint32_t j = threadIdx.x; j < tn; j += kOsThreads) {
      const K kk = sko[j];
      const uint32_t pos = dig_glob[(uint32_t)((kk >> shift) & 255u)] + j;
      kout[pos] = kk;
      vout[pos] = sv[j];
    }
#pragma unroll
    for (int x = 0; x < kOsWarps; ++x) wcnt[x][threadIdx.x] = 0;
    __syncthreads();
    s ^= 1;
  }
}

// ------------------------------------------------------------------ reduce-then-scan, TMA ring
// Pass = upsweep (per-CTA-range digit histogram) + scan of the 256 x G counts (digit-major) +
// downsweep: CTA c walks its contiguous range tile by tile with exact running digit offsets (no
// look-back), the next tile's keys/values streaming into the other half of a 2-stage smem ring by
// cp.async.bulk while the current tile is ranked, staged in digit order and written out.
constexpr int kRsCtas = 148 * 2;

// Digits come from (key & kmask) (the count bits of a stream element ride along unsorted); with skip0
// the elements whose bits above kmask are 0 are holes (not counted, dropped by the downsweep).  A map
// (slot -> rank) is applied in place to the masked part: key = map[key & kmask] | (key & ~kmask).
// HOLES / MASK are compile-time so the common path (no holes, digits below the count bits) is the
// plain branch-free kernel.
template <typename K, bool HOLES>
__device__ __forceinline__ bool rs_hole(K k, K kmask) { return HOLES && (k & ~kmask) == 0; }
template <typename K, bool MASK>
__device__ __forceinline__ K rs_dkey(K k, K kmask) { return MASK ? (k & kmask) : k; }

// kRsUpSplit CTAs share one downsweep range (each a contiguous quarter), adding their counts to the
// range's histogram column with global atomics (hist zeroed by the caller): 4x the warps in flight for
// the map gather of the first pass, which is L2-latency bound at 2 CTAs/SM.
constexpr int kRsUpSplit = 4;

template <typename K, bool HOLES, bool MASK>
__global__ void __launch_bounds__(256) k_rs_up(K* keys, uint64_t n, uint64_t per, int shift,
                                               const uint32_t* __restrict__ map, uint32_t* hist, K kmask,
                                               const uint32_t* __restrict__ rlen) {
  __shared__ uint32_t h[kOsWarps][256];
  const int w = threadIdx.x >> 5;
  for (int x = 0; x < kOsWarps; ++x) h[x][threadIdx.x] = 0;
  __syncthreads();
  const uint32_t range = blockIdx.x / kRsUpSplit, part = blockIdx.x % kRsUpSplit;
  const uint32_t n_ranges = gridDim.x / kRsUpSplit;
  const uint64_t sub = per / kRsUpSplit;  // per is a multiple of the 4096-element tile
  // rlen (optional): range r holds only its first rlen[r] elements (doc combine, combine.cuh)
  const uint64_t rhi = rlen ? (uint64_t)range * per + rlen[range]
                            : ((uint64_t)range * per + per < n ? (uint64_t)range * per + per : n);
  const uint64_t lo0 = (uint64_t)range * per + part * sub;  // 16-byte aligned
  const uint64_t lo = lo0 < rhi ? lo0 : rhi;
  const uint64_t hi = (part + 1 == kRsUpSplit) ? rhi : (lo0 + sub < rhi ? lo0 + sub : rhi);
  constexpr int V = 16 / sizeof(K);  // keys per 16-byte vector
  const uint64_t nvec = (hi - lo) / V;
  typedef typename std::conditional<sizeof(K) == 4, uint4, ulonglong2>::type Vec;
  Vec* vp = (Vec*)(keys + lo);
  constexpr int U = 4;  // vectors in flight per thread
  uint64_t v0 = threadIdx.x;
  for (; v0 + (U - 1) * 256 < nvec; v0 += U * 256) {
    Vec x[U];
#pragma unroll
    for (int u = 0; u < U; ++u) x[u] = vp[v0 + u * 256];
    // all U * V map gathers are issued before any histogram update (the gathers are L2-latency
    // bound; interleaving them with shared atomics serialised them)
    if (map) {
#pragma unroll
      for (int u = 0; u < U; ++u) {
        K* kk = (K*)&x[u];
#pragma unroll
        for (int j = 0; j < V; ++j)
          if (!rs_hole<K, HOLES>(kk[j], kmask)) kk[j] = (K)__ldg(&map[(uint32_t)(kk[j] & kmask)]) | (kk[j] & ~kmask);
      }
    }
#pragma unroll
    for (int u = 0; u < U; ++u) {
      K* kk = (K*)&x[u];
#pragma unroll
      for (int j = 0; j < V; ++j) {
        // a mapped hole stays a hole: map values keep the bits above kmask of a non-hole
        const bool hole = rs_hole<K, HOLES>(kk[j], kmask);
        if (!hole) atomicAdd(&h[w][(uint32_t)(rs_dkey<K, MASK>(kk[j], kmask) >> shift) & 255u], 1u);
      }
      if (map) vp[v0 + u * 256] = x[u];
    }
  }
  for (uint64_t v = v0; v < nvec; v += 256) {
    Vec x = vp[v];
    K* kk = (K*)&x;
#pragma unroll
    for (int j = 0; j < V; ++j) {
      const bool hole = rs_hole<K, HOLES>(kk[j], kmask);
      if (map && !hole) kk[j] = (K)__ldg(&map[(uint32_t)(kk[j] & kmask)]) | (kk[j] & ~kmask);
      if (!hole) atomicAdd(&h[w][(uint32_t)(rs_dkey<K, MASK>(kk[j], kmask) >> shift) & 255u], 1u);
    }
    if (map) vp[v] = x;
  }
  for (uint64_t i = lo + nvec * V + threadIdx.x; i < hi; i += 256) {
    K k = keys[i];
    if (rs_hole<K, HOLES>(k, kmask)) continue;
    if (map) {
      k = (K)__ldg(&map[(uint32_t)(k & kmask)]) | (k & ~kmask);
      keys[i] = k;
    }
    atomicAdd(&h[w][(uint32_t)(rs_dkey<K, MASK>(k, kmask) >> shift) & 255u], 1u);
  }
  __syncthreads();
  uint32_t t = 0;
#pragma unroll
  for (int x = 0; x < kOsWarps; ++x) t += h[x][threadIdx.x];
  if (t) atomicAdd(&hist[(uint64_t)threadIdx.x * n_ranges + range], t);
}

template <typename K>
__global__ void __launch_bounds__(kOsThreads, 2) k_rs_down(const K* __restrict__ kin, const uint32_t* __restrict__ vin,
                                                        K* __restrict__ kout, uint32_t* __restrict__ vout, uint64_t n,
                                                        uint64_t per, int shift, const uint32_t* __restrict__ offs) {
  extern __shared__ __align__(128) unsigned char os_smem[];
  __shared__ __align__(8) uint64_t bar[2];
  __shared__ uint32_t wcnt[kOsWarps][256];
  __shared__ uint32_t dig_off[256];
  __shared__ uint32_t dig_glob[256];
  __shared__ uint32_t run_base[256];
  const size_t stage_bytes = (size_t)kOsTile * (sizeof(K) + sizeof(uint32_t));
  auto skey = [&](int s) { return (K*)(os_smem + s * stage_bytes); };
  auto sval = [&](int s) { return (uint32_t*)(os_smem + s * stage_bytes + (size_t)kOsTile * sizeof(K)); };
  const uint32_t lane = lane_id();
  const int w = threadIdx.x >> 5;
  const uint32_t lt = (1u << lane) - 1u;
  const uint64_t lo = (uint64_t)blockIdx.x * per;
  const uint64_t hi = lo + per < n ? lo + per : n;
  if (lo >= hi) return;

  auto issue = [&](int s, uint64_t base) {  // thread 0
    const uint32_t cnt = (uint32_t)((hi - base) < (uint64_t)kOsTile ? (hi - base) : (uint64_t)kOsTile);
    const uint32_t bk = (uint32_t)((cnt * sizeof(K) + 15) & ~(size_t)15);
    const uint32_t bv = (cnt * 4 + 15) & ~15u;
    fence_proxy_async_smem();
    mbar_arrive_expect_tx(&bar[s], bk + bv);
    tma_load_1d(skey(s), kin + base, bk, &bar[s]);
    tma_load_1d(sval(s), vin + base, bv, &bar[s]);
  };

  if (threadIdx.x == 0) {
    mbar_init(&bar[0], 1);
    mbar_init(&bar[1], 1);
    fence_mbar_init();
  }
  for (int x = 0; x < kOsWarps; ++x) wcnt[x][threadIdx.x] = 0;
  run_base[threadIdx.x] = offs[(uint64_t)threadIdx.x * gridDim.x + blockIdx.x];
  __syncthreads();
  if (threadIdx.x == 0) issue(0, lo);
  uint32_t parity = 0u;
  int s = 0;
  for (uint64_t base = lo; base < hi; base += kOsTile) {
    if (threadIdx.x == 0 && base + kOsTile < hi) issue(s ^ 1, base + kOsTile);
    mbar_wait(&bar[s], (parity >> s) & 1u);
    parity ^= 1u << s;
    const uint32_t tn = (uint32_t)((hi - base) < (uint64_t)kOsTile ? (hi - base) : (uint64_t)kOsTile);
    K* sk = skey(s);
    uint32_t* sv = sval(s);
    K key[kOsItems];
    uint32_t val[kOsItems], rank[kOsItems];
#pragma unroll
    for (int k = 0; k < kOsItems; ++k) {
      const uint32_t li = w * (32 * kOsItems) + k * 32 + lane;
      key[k] = sk[li];
      val[k] = sv[li];
    }
    // peer masks by 8-ballot multisplit (no MATCH.ANY), then the per-warp running counters
#pragma unroll
    for (int k = 0; k < kOsItems; ++k) {
      const uint32_t li = w * (32 * kOsItems) + k * 32 + lane;
      rank[k] = digit_peers((uint32_t)((key[k] >> shift) & 255u), li < tn);
    }
#pragma unroll
    for (int k = 0; k < kOsItems; ++k) {
      const uint32_t li = w * (32 * kOsItems) + k * 32 + lane;
      const bool valid = li < tn;
      const uint32_t d = (uint32_t)((key[k] >> shift) & 255u);
      const uint32_t peers = rank[k];
      const int leader = valid ? __ffs(peers) - 1 : (int)lane;
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
    const uint32_t d = threadIdx.x;
    uint32_t cnt = 0;
#pragma unroll
    for (int x = 0; x < kOsWarps; ++x) {
      const uint32_t t = wcnt[x][d];
      wcnt[x][d] = cnt;
      cnt += t;
    }
    uint32_t tot;
    const uint32_t toff = block_exclusive_sum<uint32_t>(cnt, tot);
    dig_off[d] = toff;
    const uint32_t rb = run_base[d];
    dig_glob[d] = rb - toff;
    run_base[d] = rb + cnt;
    __syncthreads();
#pragma unroll
    for (int k = 0; k < kOsItems; ++k) {
      const uint32_t li = w * (32 * kOsItems) + k * 32 + lane;
      if (li < tn) {
        const uint32_t dk = (uint32_t)((key[k] >> shift) & 255u);
        const uint32_t p = dig_off[dk] + wcnt[w][dk] + rank[k];
        sk[p] = key[k];
        sv[p] = val[k];
      }
    }
    __syncthreads();
    for (uint32_t j = threadIdx.x; j < tn; j += kOsThreads) {
      const K kk = sk[j];
      const uint32_t pos = dig_glob[(uint32_t)((kk >> shift) & 255u)] + j;
      kout[pos] = kk;
      vout[pos] = sv[j];
    }
#pragma unroll
    for (int x = 0; x < kOsWarps; ++x) wcnt[x][threadIdx.x] = 0;
    __syncthreads();
    s ^= 1;
  }
}

// Downsweep v2: 512 threads x 8 items (tile 4096); the tile is never copied inside shared memory:
// ranks produce an inverse permutation (u16) and the write-out gathers keys/values from the TMA
// stage through it, so keys/values need no registers across barriers (occupancy: 32 warps/SM).
constexpr int kDsThreads = 512;
constexpr int kDsWarps = kDsThreads / 32;
constexpr int kDsItems = 8;
static_assert(kDsThreads * kDsItems == kOsTile, "tile");

template <typename K>
inline size_t ds_smem_bytes() { return 2 * (size_t)kOsTile * (sizeof(K) + sizeof(uint32_t)) + kOsTile * 2; }

template <typename K, bool HOLES, bool MASK>
// 48 registers (no spills): two CTAs use 48K of the 64K registers and 183 KB of shared memory, so
// small CTAs of another stream (the dictionary update next to the partials path's side-stream sort)
// can run beside the persistent downsweep: step 9.36 -> 9.27 ms on config 2, although the pass
// itself is ~4% slower than at 64 registers (WJ_DS_MAXREG=0: __launch_bounds__(512, 2) only)
#ifndef WJ_DS_MAXREG
#define WJ_DS_MAXREG 48
#endif
#if WJ_DS_MAXREG > 0
#define WJ_DS_BOUNDS __maxnreg__(WJ_DS_MAXREG)
#else
#define WJ_DS_BOUNDS __launch_bounds__(kDsThreads, 2)
#endif
__global__ void WJ_DS_BOUNDS k_rs_down2(const K* __restrict__ kin, const uint32_t* __restrict__ vin,
                                                         K* __restrict__ kout, uint32_t* __restrict__ vout, uint64_t n,
                                                         uint64_t per, int shift, const uint32_t* __restrict__ offs,
                                                         K kmask, const uint32_t* __restrict__ rlen) {
  extern __shared__ __align__(128) unsigned char os_smem[];
  __shared__ __align__(8) uint64_t bar[2];
  __shared__ uint32_t wcnt[kDsWarps][256];
  __shared__ uint32_t wbins[kDsWarps][256];
  __shared__ uint32_t dig_off[256];
  __shared__ uint32_t dig_glob[256];
  __shared__ uint32_t run_base[256];
  __shared__ uint32_t wtot[8];
  __shared__ uint32_t s_tvalid;
  const size_t stage_bytes = (size_t)kOsTile * (sizeof(K) + sizeof(uint32_t));
  auto skey = [&](int s) { return (K*)(os_smem + s * stage_bytes); };
  auto sval = [&](int s) { return (uint32_t*)(os_smem + s * stage_bytes + (size_t)kOsTile * sizeof(K)); };
  uint16_t* inv = (uint16_t*)(os_smem + 2 * stage_bytes);
  const uint32_t lane = lane_id();
  const int w = threadIdx.x >> 5;
  const uint32_t lt = (1u << lane) - 1u;
  const uint64_t lo = (uint64_t)blockIdx.x * per;
  const uint64_t hi = rlen ? lo + rlen[blockIdx.x] : (lo + per < n ? lo + per : n);
  if (lo >= hi) return;

  auto issue = [&](int s, uint64_t base) {  // thread 0
    const uint32_t cnt = (uint32_t)((hi - base) < (uint64_t)kOsTile ? (hi - base) : (uint64_t)kOsTile);
    const uint32_t bk = (uint32_t)((cnt * sizeof(K) + 15) & ~(size_t)15);
    const uint32_t bv = (cnt * 4 + 15) & ~15u;
    fence_proxy_async_smem();
    mbar_arrive_expect_tx(&bar[s], bk + bv);
    tma_load_1d(skey(s), kin + base, bk, &bar[s]);
    tma_load_1d(sval(s), vin + base, bv, &bar[s]);
  };

  if (threadIdx.x == 0) {
    mbar_init(&bar[0], 1);
    mbar_init(&bar[1], 1);
    fence_mbar_init();
  }
  for (int i = threadIdx.x; i < kDsWarps * 256; i += kDsThreads) (&wcnt[0][0])[i] = (&wbins[0][0])[i] = 0;
  if (threadIdx.x < 256) run_base[threadIdx.x] = offs[(uint64_t)threadIdx.x * gridDim.x + blockIdx.x];
  __syncthreads();
  if (threadIdx.x == 0) issue(0, lo);
  uint32_t parity = 0u;
  int s = 0;
  for (uint64_t base = lo; base < hi; base += kOsTile) {
    if (threadIdx.x == 0 && base + kOsTile < hi) issue(s ^ 1, base + kOsTile);
    mbar_wait(&bar[s], (parity >> s) & 1u);
    parity ^= 1u << s;
    const uint32_t tn = (uint32_t)((hi - base) < (uint64_t)kOsTile ? (hi - base) : (uint64_t)kOsTile);
    const K* sk = skey(s);
    const uint32_t* sv = sval(s);
    uint32_t dg[kDsItems], rank[kDsItems];
    uint32_t vmask = 0;  // valid items of this thread (in range, not a hole)
#pragma unroll
    for (int k = 0; k < kDsItems; ++k) {
      const uint32_t li = w * (32 * kDsItems) + k * 32 + lane;
      const K kv = sk[li];
      const bool valid = li < tn && !rs_hole<K, HOLES>(kv, kmask);
      vmask |= (valid ? 1u : 0u) << k;
      dg[k] = (uint32_t)((rs_dkey<K, MASK>(kv, kmask) >> shift) & 255u);
      // 64-bit keys (all distinct: new-term sort): shared-memory masks; 32-bit keys (Zipf-skewed
      // ranks, many equal digits per warp -> atomic conflicts): ballots
      rank[k] = sizeof(K) == 8 ? digit_peers_smem(wbins[w], dg[k], valid) : digit_peers(dg[k], valid);
    }
#pragma unroll
    for (int k = 0; k < kDsItems; ++k) {
      const bool valid = (vmask >> k) & 1u;
      const uint32_t peers = rank[k];
      const int leader = valid ? __ffs(peers) - 1 : (int)lane;
      uint32_t old = 0;
      if (valid && (int)lane == leader) {
        old = wcnt[w][dg[k]];
        wcnt[w][dg[k]] = old + __popc(peers);
      }
      old = __shfl_sync(0xffffffffu, old, leader);
      rank[k] = old + __popc(peers & lt);
      __syncwarp();
    }
    __syncthreads();
    // per digit (threads 0..255): offsets across warps, tile count, tile-exclusive digit offset
    uint32_t cnt = 0, inc = 0;
    if (threadIdx.x < 256) {
      const uint32_t d = threadIdx.x;
#pragma unroll
      for (int x = 0; x < kDsWarps; ++x) {
        const uint32_t t = wcnt[x][d];
        wcnt[x][d] = cnt;
        cnt += t;
      }
      inc = warp_inclusive_sum<uint32_t>(cnt);
      if (lane == 31) wtot[w] = inc;
    }
    __syncthreads();
    if (threadIdx.x < 256) {
      const uint32_t d = threadIdx.x;
      uint32_t wp = 0;
      for (int x = 0; x < w; ++x) wp += wtot[x];
      const uint32_t toff = wp + inc - cnt;
      dig_off[d] = toff;
      const uint32_t rb = run_base[d];
      dig_glob[d] = rb - toff;
      run_base[d] = rb + cnt;
      if (d == 255) s_tvalid = toff + cnt;
    }
    __syncthreads();
#pragma unroll
    for (int k = 0; k < kDsItems; ++k) {
      const uint32_t li = w * (32 * kDsItems) + k * 32 + lane;
      if ((vmask >> k) & 1u) inv[dig_off[dg[k]] + wcnt[w][dg[k]] + rank[k]] = (uint16_t)li;
    }
    __syncthreads();
    const uint32_t tvalid = HOLES ? s_tvalid : tn;  // valid (non-hole) items of the tile
    for (uint32_t j = threadIdx.x; j < tvalid; j += kDsThreads) {
      const uint32_t li = inv[j];
      const K kk = sk[li];
      const uint32_t pos = dig_glob[(uint32_t)((rs_dkey<K, MASK>(kk, kmask) >> shift) & 255u)] + j;
      kout[pos] = kk;
      vout[pos] = sv[li];
    }
    for (int i = threadIdx.x; i < kDsWarps * 256; i += kDsThreads) (&wcnt[0][0])[i] = 0;
    __syncthreads();
    s ^= 1;
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
