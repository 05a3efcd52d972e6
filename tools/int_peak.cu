// INT-issue roofline microbenchmark: warp-instructions per
// second of a dependency-light LOP3 / IADD3 / SHF mix on every SM, the
// denominator for the issue-bound configs (the JIT kernels are straight-line
// integer code). nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o int_peak tools/int_peak.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

template <int MIX>
__global__ void int_mix(uint32_t *out, uint32_t iters, uint32_t seed) {
  uint32_t a[8];
#pragma unroll
  for (int k = 0; k < 8; k++) a[k] = seed * (threadIdx.x + 1 + k) + blockIdx.x;
  for (uint32_t i = 0; i < iters; i++) {
#pragma unroll
    for (int k = 0; k < 8; k++) {   // 8 independent chains, 3 instructions each
      if (MIX == 0) {
        uint32_t t;
        asm volatile("lop3.b32 %0, %1, %2, %3, 0x96;" : "=r"(t) : "r"(a[k]), "r"(a[(k + 1) & 7]), "r"(i));
        asm volatile("add.u32 %0, %1, %2;" : "=r"(a[k]) : "r"(t), "r"(a[(k + 3) & 7]));
        asm volatile("shf.l.wrap.b32 %0, %1, %1, 5;" : "=r"(a[k]) : "r"(a[k]));
      } else {   // LOP3 only
        asm volatile("lop3.b32 %0, %1, %2, %3, 0x96;" : "=r"(a[k]) : "r"(a[k]), "r"(a[(k + 1) & 7]), "r"(i));
        asm volatile("lop3.b32 %0, %1, %2, %3, 0xe8;" : "=r"(a[k]) : "r"(a[k]), "r"(a[(k + 2) & 7]), "r"(i));
        asm volatile("lop3.b32 %0, %1, %2, %3, 0x6a;" : "=r"(a[k]) : "r"(a[k]), "r"(a[(k + 5) & 7]), "r"(i));
      }
    }
  }
  uint32_t r = 0;
#pragma unroll
  for (int k = 0; k < 8; k++) r ^= a[k];
  if (r == 0x12345678u) out[blockIdx.x] = r;
}

int main() {
  int dev = 0, sms = 0, clk = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, dev);
  uint32_t *out;
  cudaMalloc(&out, 1 << 20);
  const uint32_t iters = 20000;
  for (int mix = 0; mix < 2; mix++) {
    for (int warps : {16, 32}) {
      dim3 grid(sms * (64 / warps)), block(32 * warps);
      cudaEvent_t e0, e1;
      cudaEventCreate(&e0);
      cudaEventCreate(&e1);
      for (int rep = 0; rep < 2; rep++) {
        cudaEventRecord(e0);
        if (mix == 0) int_mix<0><<<grid, block>>>(out, iters, 12345u);
        else int_mix<1><<<grid, block>>>(out, iters, 12345u);
        cudaEventRecord(e1);
        cudaEventSynchronize(e1);
      }
      float ms = 0;
      cudaEventElapsedTime(&ms, e0, e1);
      const double winst = (double)grid.x * block.x / 32.0 * iters * 8.0 * 3.0;   // warp-instructions in the loop
      printf("{\"mix\": \"%s\", \"warps_per_cta\": %d, \"ctas\": %u, \"ms\": %.3f, \"warp_inst_per_s\": %.4g, "
             "\"per_sm_per_clk_at_rated\": %.3f, \"sms\": %d, \"rated_khz\": %d}\n",
             mix ? "lop3" : "lop3+iadd+shf", warps, grid.x, ms, winst / (ms * 1e-3),
             winst / (ms * 1e-3) / sms / (clk * 1e3), sms, clk);
    }
  }
  return 0;
}
