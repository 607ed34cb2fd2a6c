// Microbenchmark (not product code): k_doc_combine on a synthetic Zipf (slot, doc) stream of
// config-2 size; variants selected by -DDC_VARIANT in combine.cuh experiments.
#include <cstdio>
#include <cstdint>
#include <vector>
#include <cmath>
#include <random>
#include <algorithm>
#include "../../paper_conf_ipps_weij11_b200/csrc/combine.cuh"
using namespace wj;
int main(int argc, char** argv) {
  const uint64_t n = argc > 1 ? strtoull(argv[1], 0, 10) : 141059477ull;
  const uint32_t V = 4764143;
  std::vector<uint32_t> hk(n), hv(n);
  std::mt19937_64 g(1);
  std::vector<uint32_t> perm(V);
  for (uint32_t i = 0; i < V; ++i) perm[i] = i;
  std::shuffle(perm.begin(), perm.end(), g);
  const double H = std::log((double)V) + 0.5772;
  std::uniform_real_distribution<double> u(0, 1);
  std::lognormal_distribution<double> ln(std::log(2600.0) - 0.5, 1.0);
  uint32_t doc = 0; uint64_t left = (uint64_t)ln(g) + 1;
  for (uint64_t i = 0; i < n; ++i) {
    double r = std::exp(u(g) * H - 0.5772);
    uint32_t z = r < 1 ? 0 : (uint32_t)r; if (z >= V) z = V - 1;
    if (left-- == 0) { ++doc; left = (uint64_t)ln(g); }
    hk[i] = perm[z] | (1u << 25); hv[i] = doc;
  }
  uint32_t *k0, *v0, *k, *v;
  cudaMalloc(&k0, n * 4); cudaMalloc(&v0, n * 4); cudaMalloc(&k, n * 4 + 64); cudaMalloc(&v, n * 4 + 64);
  cudaMemcpy(k0, hk.data(), n * 4, cudaMemcpyHostToDevice);
  cudaMemcpy(v0, hv.data(), n * 4, cudaMemcpyHostToDevice);
  const uint32_t ntiles = (uint32_t)((n + kDcTile - 1) / kDcTile);
  uint64_t* lk; cudaMalloc(&lk, (ntiles + 2) * 8);
  uint32_t* nout; cudaMalloc(&nout, 4);
  cudaFuncSetAttribute(k_doc_combine, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)dc_smem_bytes());
  cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
  float best = 1e9; uint32_t m = 0;
  for (int it = 0; it < 5; ++it) {
    cudaMemcpy(k, k0, n * 4, cudaMemcpyDeviceToDevice);
    cudaMemcpy(v, v0, n * 4, cudaMemcpyDeviceToDevice);
    cudaMemset(lk, 0, (ntiles + 2) * 8);
    cudaEventRecord(a);
    k_doc_combine<<<ntiles, kDcThreads, dc_smem_bytes()>>>(k, v, n, ntiles, lk, (uint32_t*)(lk + ntiles), nout);
    cudaEventRecord(b); cudaEventSynchronize(b);
    float ms; cudaEventElapsedTime(&ms, a, b); if (it) best = std::min(best, ms);
  }
  cudaMemcpy(&m, nout, 4, cudaMemcpyDeviceToHost);
  printf("doc_combine n=%llu -> %u elements (%.3f): %.3f ms  err=%s\n", (unsigned long long)n, m, (double)m / n, best,
         cudaGetErrorString(cudaGetLastError()));
  return 0;
}
