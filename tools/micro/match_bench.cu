// Microbenchmark: 8-ballot multisplit vs __match_any_sync peer masks (sm_100a).
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
#include <cmath>
__device__ __forceinline__ uint32_t peers_ballot(uint32_t d) {
  uint32_t p = 0xffffffffu;
#pragma unroll
  for (int b = 0; b < 8; ++b) { const bool bit = (d >> b) & 1u; const uint32_t m = __ballot_sync(0xffffffffu, bit); p &= bit ? m : ~m; }
  return p;
}
__device__ __forceinline__ uint32_t peers_smem(uint32_t* bins, uint32_t d) {
  const uint32_t lane = threadIdx.x & 31;
  atomicOr(&bins[d], 1u << lane);
  __syncwarp();
  const uint32_t p = bins[d];
  __syncwarp();
  if ((p & ((1u << lane) - 1u)) == 0) bins[d] = 0u;
  __syncwarp();
  return p;
}
template <int MODE>
__global__ void k(const uint32_t* in, uint32_t n, uint32_t* out) {
  __shared__ uint32_t bins[8][256];
  for (int i = threadIdx.x; i < 8 * 256; i += 256) (&bins[0][0])[i] = 0;
  __syncthreads();
  uint32_t acc = 0;
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) {
    const uint32_t d = in[i] & 255u;
    uint32_t p;
    if (MODE == 0) p = peers_ballot(d);
    else if (MODE == 1) p = __match_any_sync(0xffffffffu, d);
    else p = peers_smem(bins[threadIdx.x >> 5], d);
    acc += __popc(p & ((1u << (threadIdx.x & 31)) - 1u));
  }
  out[blockIdx.x * blockDim.x + threadIdx.x] = acc;
}
int main() {
  const uint32_t n = 1u << 27;
  uint32_t *in, *out;
  cudaMalloc(&in, n * 4ull); cudaMalloc(&out, 148 * 8 * 256 * 4);
  uint32_t* h = new uint32_t[n];
  for (int dist = 0; dist < 4; ++dist) {
    uint64_t x = 88172645463325252ull;
    for (uint32_t i = 0; i < n; ++i) {
      x ^= x << 13; x ^= x >> 7; x ^= x << 17;
      if (dist == 0) h[i] = (uint32_t)x;                    // uniform
      else if (dist == 1) h[i] = (uint32_t)(x % 1000) < 300 ? 7 : (uint32_t)x;   // 30% one value
      else if (dist == 2) h[i] = (uint32_t)(x % 8);                        // 8 values
      else {  // Zipf(1)-like ranks over 4.7M terms, hashed (lexicographic rank is not frequency order)
        double u = (double)(x >> 11) / 9007199254740992.0;
        uint32_t r = (uint32_t)exp(u * log(4.7e6));
        r *= 0x9E3779B1u; h[i] = r >> 9;
      }
    }
    cudaMemcpy(in, h, n * 4ull, cudaMemcpyHostToDevice);
    for (int mode = 0; mode < 3; ++mode) {
      cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
      for (int r = 0; r < 2; ++r) {
        cudaEventRecord(a);
        if (mode == 0) k<0><<<148 * 8, 256>>>(in, n, out); else if (mode == 1) k<1><<<148 * 8, 256>>>(in, n, out); else k<2><<<148 * 8, 256>>>(in, n, out);
        cudaEventRecord(b); cudaEventSynchronize(b);
        float ms; cudaEventElapsedTime(&ms, a, b);
        if (r) printf("dist %d mode %s: %.3f ms (%.1f Gelem/s)\n", dist, mode == 2 ? "smem_or" : mode ? "match" : "ballot8", ms, n / ms / 1e6);
      }
    }
  }
  return 0;
}
