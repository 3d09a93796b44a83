// MUFU exp2 throughput probe: f32 vs f16x2 vs bf16x2 (results per SM per clock).
#include <cstdio>
#include <cuda_fp16.h>
#include <cuda_bf16.h>
template <int MODE>
__global__ void k(float* out, int iters) {
  float a0 = -threadIdx.x * 1e-3f, a1 = a0 - 0.1f, a2 = a0 - 0.2f, a3 = a0 - 0.3f;
  unsigned u0, u1, u2, u3;
  {
    __half2 h0 = __floats2half2_rn(a0, a1), h1 = __floats2half2_rn(a2, a3);
    u0 = *(unsigned*)&h0; u1 = *(unsigned*)&h1; u2 = u0 ^ 1; u3 = u1 ^ 1;
  }
  for (int i = 0; i < iters; ++i) {
#pragma unroll
    for (int j = 0; j < 16; ++j) {
      if (MODE == 0) {
        asm volatile("ex2.approx.ftz.f32 %0, %0;" : "+f"(a0)); asm volatile("ex2.approx.ftz.f32 %0, %0;" : "+f"(a1));
        asm volatile("ex2.approx.ftz.f32 %0, %0;" : "+f"(a2)); asm volatile("ex2.approx.ftz.f32 %0, %0;" : "+f"(a3));
      } else if (MODE == 1) {
        asm volatile("ex2.approx.f16x2 %0, %0;" : "+r"(u0)); asm volatile("ex2.approx.f16x2 %0, %0;" : "+r"(u1));
        asm volatile("ex2.approx.f16x2 %0, %0;" : "+r"(u2)); asm volatile("ex2.approx.f16x2 %0, %0;" : "+r"(u3));
      } else {
        asm volatile("ex2.approx.ftz.bf16x2 %0, %0;" : "+r"(u0)); asm volatile("ex2.approx.ftz.bf16x2 %0, %0;" : "+r"(u1));
        asm volatile("ex2.approx.ftz.bf16x2 %0, %0;" : "+r"(u2)); asm volatile("ex2.approx.ftz.bf16x2 %0, %0;" : "+r"(u3));
      }
    }
  }
  out[blockIdx.x * blockDim.x + threadIdx.x] = a0 + a1 + a2 + a3 + __uint_as_float(u0 ^ u1 ^ u2 ^ u3);
}
int main() {
  int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  int clk; cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
  float* out; cudaMalloc(&out, sms * 8 * 1024 * 4);
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  const int iters = 4096;
  const char* names[3] = {"f32", "f16x2", "bf16x2"};
  for (int m = 0; m < 3; ++m) {
    for (int rep = 0; rep < 2; ++rep) {
      cudaEventRecord(e0);
      if (m == 0) k<0><<<sms * 4, 512>>>(out, iters);
      if (m == 1) k<1><<<sms * 4, 512>>>(out, iters);
      if (m == 2) k<2><<<sms * 4, 512>>>(out, iters);
      cudaEventRecord(e1); cudaEventSynchronize(e1);
      float ms; cudaEventElapsedTime(&ms, e0, e1);
      double instr = (double)sms * 4 * 512 * iters * 64;
      double per_ns = instr / (ms * 1e6);
      printf("%s: %.3f ms  %.1f instr/ns total  %.2f instr/clk/SM at max clk %d MHz (results x%d)\n", names[m], ms, per_ns,
             per_ns / sms / (clk / 1e6), clk / 1000, m ? 2 : 1);
    }
  }
  printf("err %s\n", cudaGetErrorString(cudaGetLastError()));
}
