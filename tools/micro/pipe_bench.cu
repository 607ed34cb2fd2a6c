// Microbenchmark: issue throughput of integer SASS ops on sm_100a (which pipe VIADD / IADD3 use).
// Each thread runs 8 independent chains; reports warp-instructions per cycle per SM.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
template <int MODE>
__global__ void k(uint32_t* out, int iters) {
  uint32_t a[8];
  for (int i = 0; i < 8; ++i) a[i] = threadIdx.x * (i + 3);
  uint32_t c = out[0] | 0x13579bdu;
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int i = 0; i < 8; ++i) {
      const int m = MODE == 2 ? (i & 1) : MODE == 3 ? (i & 1) * 2 : MODE == 5 ? (i & 1) * 3 : MODE;
      if (m == 0) asm volatile("lop3.b32 %0, %0, %1, 0x5a5a5a5a, 0x96;" : "+r"(a[i]) : "r"(c));
      else if (m == 1) asm volatile("add.u32 %0, %0, 0x31313131;" : "+r"(a[i]));
      else if (m == 2) asm volatile("mad.lo.u32 %0, %0, 0x1003, %1;" : "+r"(a[i]) : "r"(c));
      else if (m == 3) asm volatile("add.u32 %0, %0, %1;" : "+r"(a[i]) : "r"(c));
      else if (m == 4) asm volatile("shr.u32 %0, %0, 3;" : "+r"(a[i]));
    }
  }
  uint32_t s = 0;
  for (int i = 0; i < 8; ++i) s ^= a[i];
  if (s == 0x12345678u) out[1] = s;
}
int main() {
  uint32_t* out; cudaMalloc(&out, 64); cudaMemset(out, 0, 64);
  int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  int clk; cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
  const char* names[] = {"lop3 x8", "add-imm x8", "lop3+add-imm", "lop3+mad", "shr x8", "lop3+add-reg"};
  const int iters = 20000;
  for (int mode = 0; mode < 6; ++mode) {
    cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
    for (int r = 0; r < 2; ++r) {
      cudaEventRecord(e0);
      switch (mode) {
        case 0: k<0><<<sms * 4, 512>>>(out, iters); break;
        case 1: k<1><<<sms * 4, 512>>>(out, iters); break;
        case 2: k<2><<<sms * 4, 512>>>(out, iters); break;
        case 3: k<3><<<sms * 4, 512>>>(out, iters); break;
        case 4: k<4><<<sms * 4, 512>>>(out, iters); break;
        case 5: k<5><<<sms * 4, 512>>>(out, iters); break;
      }
      cudaEventRecord(e1); cudaEventSynchronize(e1);
    }
    float ms; cudaEventElapsedTime(&ms, e0, e1);
    const double winst = (double)sms * 4 * 512 / 32 * iters * 8;
    const double cyc = ms * 1e-3 * clk * 1e3;  // rough: nominal clock
    printf("%-16s %.3f ms  %.2f warp-inst/cycle/SM (nominal clock)\n", names[mode], ms, winst / cyc / sms);
  }
  return 0;
}
