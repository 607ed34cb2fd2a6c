// Device-wide exclusive prefix sum (reduce-then-scan), input given by a device functor so that
// flags / counts are computed on the fly instead of being materialised.
#pragma once
#include "common.cuh"

namespace wj {

constexpr int kScanThreads = 256;
constexpr int kScanItems = 16;
constexpr int kScanTile = kScanThreads * kScanItems;  // 4096

template <typename T>
struct ArrayIn {
  const T* p;
  __device__ __forceinline__ T operator()(uint64_t i) const { return p[i]; }
};

__device__ __forceinline__ int scan_pad(int i) { return i + (i >> 5); }

template <typename T>
__device__ __forceinline__ T warp_inclusive_sum(T v) {
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    T u = __shfl_up_sync(0xffffffffu, v, o);
    if ((int)lane_id() >= o) v += u;
  }
  return v;
}

// 256-thread block exclusive scan; returns exclusive prefix, sets total for all threads.
template <typename T>
__device__ __forceinline__ T block_exclusive_sum(T v, T& total) {
  __shared__ T wsum[kScanThreads / 32 + 1];
  const int w = threadIdx.x >> 5;
  T inc = warp_inclusive_sum(v);
  if (lane_id() == 31) wsum[w] = inc;
  __syncthreads();
  if (w == 0) {
    T x = lane_id() < kScanThreads / 32 ? wsum[lane_id()] : T(0);
    T xi = warp_inclusive_sum(x);
    if (lane_id() < kScanThreads / 32) wsum[lane_id()] = xi - x;
    if (lane_id() == kScanThreads / 32 - 1) wsum[kScanThreads / 32] = xi;  // uses slot 8
  }
  __syncthreads();
  T r = wsum[w] + inc - v;
  total = wsum[kScanThreads / 32];
  __syncthreads();
  return r;
}

template <typename T, typename F>
__global__ void __launch_bounds__(kScanThreads) k_scan_reduce(F in, uint64_t n, T* partials) {
  const uint64_t base = (uint64_t)blockIdx.x * kScanTile;
  T s = 0;
#pragma unroll 4
  for (int k = 0; k < kScanItems; ++k) {
    uint64_t i = base + (uint64_t)k * kScanThreads + threadIdx.x;
    if (i < n) s += in(i);
  }
  T tot;
  block_exclusive_sum<T>(s, tot);
  if (threadIdx.x == 0) partials[blockIdx.x] = tot;
}

// Scans one tile of `in` with a starting offset; writes exclusive results to out.
template <typename T, typename F>
__device__ __forceinline__ void scan_tile(F in, uint64_t n, uint64_t base, T offset, T* out, T* total_out,
                                          bool last) {
  __shared__ T buf[kScanTile + kScanTile / 32];
#pragma unroll 4
  for (int k = 0; k < kScanItems; ++k) {
    int j = k * kScanThreads + threadIdx.x;
    uint64_t i = base + j;
    buf[scan_pad(j)] = (i < n) ? in(i) : T(0);
  }
  __syncthreads();
  T v[kScanItems];
  T s = 0;
#pragma unroll
  for (int k = 0; k < kScanItems; ++k) {
    v[k] = buf[scan_pad(threadIdx.x * kScanItems + k)];
    s += v[k];
  }
  T tot;
  T ex = block_exclusive_sum<T>(s, tot) + offset;
#pragma unroll
  for (int k = 0; k < kScanItems; ++k) {
    buf[scan_pad(threadIdx.x * kScanItems + k)] = ex;
    ex += v[k];
  }
  __syncthreads();
#pragma unroll 4
  for (int k = 0; k < kScanItems; ++k) {
    int j = k * kScanThreads + threadIdx.x;
    uint64_t i = base + j;
    if (i < n) out[i] = buf[scan_pad(j)];
  }
  if (last && total_out && threadIdx.x == 0) *total_out = offset + tot;
}

template <typename T, typename F>
__global__ void __launch_bounds__(kScanThreads) k_scan_down(F in, uint64_t n, const T* offsets, T* out, T* total_out) {
  scan_tile<T, F>(in, n, (uint64_t)blockIdx.x * kScanTile, offsets ? offsets[blockIdx.x] : T(0), out, total_out,
                  blockIdx.x == gridDim.x - 1);
}

// Single CTA, any n: in-place-safe exclusive scan of an array (sequential over tiles).
template <typename T>
__global__ void __launch_bounds__(kScanThreads) k_scan_single(const T* in, uint64_t n, T* out, T* total_out) {
  T off = 0;
  const uint64_t tiles = (n + kScanTile - 1) / kScanTile;
  for (uint64_t t = 0; t < tiles; ++t) {
    T s = 0;
    for (int k = 0; k < kScanItems; ++k) {
      uint64_t i = t * kScanTile + (uint64_t)k * kScanThreads + threadIdx.x;
      if (i < n) s += in[i];
    }
    T tot;
    block_exclusive_sum<T>(s, tot);
    scan_tile<T, ArrayIn<T>>(ArrayIn<T>{in}, n, t * kScanTile, off, out, nullptr, false);
    __syncthreads();
    off += tot;
  }
  if (threadIdx.x == 0 && total_out) *total_out = off;
}

struct ScanScratch {
  // device buffers for partial sums (grown on demand by the caller)
  void* p = nullptr;
  size_t bytes = 0;
};

// Launch helper.  scratch must hold >= scan_scratch_bytes<T>(n) bytes.
template <typename T>
inline size_t scan_scratch_bytes(uint64_t n) {
  uint64_t tiles = (n + kScanTile - 1) / kScanTile;
  return (size_t)(tiles + 1) * sizeof(T) * 2 + 256;
}

// exclusive scan of in(0..n) into out; *d_total (device) = sum.  Returns number of launches.
template <typename T, typename F>
inline int exclusive_scan(F in, uint64_t n, T* out, T* d_total, void* scratch, cudaStream_t st) {
  if (n == 0) {
    if (d_total) cudaMemsetAsync(d_total, 0, sizeof(T), st);
    return 0;
  }
  const uint64_t tiles = (n + kScanTile - 1) / kScanTile;
  if (tiles == 1) {
    k_scan_down<T, F><<<1, kScanThreads, 0, st>>>(in, n, (const T*)nullptr, out, d_total);
    return 1;
  }
  T* partials = (T*)scratch;
  T* poff = partials + tiles + 1;
  k_scan_reduce<T, F><<<(unsigned)tiles, kScanThreads, 0, st>>>(in, n, partials);
  k_scan_single<T><<<1, kScanThreads, 0, st>>>(partials, tiles, poff, nullptr);
  k_scan_down<T, F><<<(unsigned)tiles, kScanThreads, 0, st>>>(in, n, poff, out, d_total);
  return 3;
}

}  // namespace wj
