// Yardstick (not product code): CUB DeviceRadixSort::SortPairs on a Zipf-like (rank, docID) stream
// of config-2 size, to compare against the library's own LSD radix passes.
#include <cub/cub.cuh>
#include <cstdio>
#include <cstdint>
#include <vector>
#include <cmath>
#include <random>
#include <algorithm>
int main(int argc, char** argv) {
  const uint64_t n = argc > 1 ? strtoull(argv[1], 0, 10) : 141059477ull;
  const uint32_t V = 4764143;
  std::vector<uint32_t> hk(n), hv(n);
  std::mt19937_64 g(1);
  // Zipf(1) by inverse CDF on log scale; keys = lexicographic rank ~ random permutation of Zipf rank
  std::vector<uint32_t> perm(V);
  for (uint32_t i = 0; i < V; ++i) perm[i] = i;
  std::shuffle(perm.begin(), perm.end(), g);
  const double H = std::log((double)V) + 0.5772;
  std::uniform_real_distribution<double> u(0, 1);
  for (uint64_t i = 0; i < n; ++i) {
    double r = std::exp(u(g) * H - 0.5772);
    uint32_t z = r < 1 ? 0 : (uint32_t)r; if (z >= V) z = V - 1;
    hk[i] = perm[z]; hv[i] = (uint32_t)(i / 2600);
  }
  uint32_t *k0, *k1, *v0, *v1;
  cudaMalloc(&k0, n * 4); cudaMalloc(&k1, n * 4); cudaMalloc(&v0, n * 4); cudaMalloc(&v1, n * 4);
  cudaMemcpy(k0, hk.data(), n * 4, cudaMemcpyHostToDevice);
  cudaMemcpy(v0, hv.data(), n * 4, cudaMemcpyHostToDevice);
  uint32_t *kk, *vv; cudaMalloc(&kk, n * 4); cudaMalloc(&vv, n * 4);
  cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
  for (int bits : {23, 24, 32}) {
    size_t tmp = 0;
    cub::DoubleBuffer<uint32_t> dk(kk, k1), dv(vv, v1);
    cub::DeviceRadixSort::SortPairs(nullptr, tmp, dk, dv, (int)n, 0, bits);
    void* t; cudaMalloc(&t, tmp);
    float best = 1e9;
    for (int it = 0; it < 6; ++it) {
      cudaMemcpy(kk, k0, n * 4, cudaMemcpyDeviceToDevice);
      cudaMemcpy(vv, v0, n * 4, cudaMemcpyDeviceToDevice);
      cub::DoubleBuffer<uint32_t> ek(kk, k1), ev(vv, v1);
      cudaEventRecord(a);
      cub::DeviceRadixSort::SortPairs(t, tmp, ek, ev, (int)n, 0, bits);
      cudaEventRecord(b); cudaEventSynchronize(b);
      float ms; cudaEventElapsedTime(&ms, a, b); if (it) best = ms < best ? ms : best;
    }
    printf("cub SortPairs u32/u32 n=%llu bits=%d: %.3f ms\n", (unsigned long long)n, bits, best);
    cudaFree(t);
  }
  float best = 1e9;
  for (int it = 0; it < 6; ++it) {
    cudaEventRecord(a);
    cudaMemcpy(k1, k0, n * 4, cudaMemcpyDeviceToDevice);
    cudaMemcpy(v1, v0, n * 4, cudaMemcpyDeviceToDevice);
    cudaEventRecord(b); cudaEventSynchronize(b);
    float ms; cudaEventElapsedTime(&ms, a, b); if (it) best = ms < best ? ms : best;
  }
  printf("copy of keys+values (%.2f GB moved): %.3f ms\n", n * 16 / 1e9, best);
  return 0;
}
