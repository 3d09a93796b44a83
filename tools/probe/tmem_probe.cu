// TMEM read/write bandwidth probe: W warps per CTA (one CTA per SM) stream tcgen05.ld 32x32b.x32
// (4 in flight, then wait) or tcgen05.st over a 512-column allocation; bytes per SM clock.
#include <cstdio>
#include <cstdint>
#include "../../paper_conf_asplos_luhtlwm0c26_b200/csrc/ptx.cuh"
using namespace tsv;
__device__ __forceinline__ void st32(uint32_t taddr, const uint32_t (&r)[32]) {
  asm volatile(
      "tcgen05.st.sync.aligned.32x32b.x32.b32 [%0], "
      "{%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16,"
      "%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31,%32};" ::"r"(taddr),
      "r"(r[0]), "r"(r[1]), "r"(r[2]), "r"(r[3]), "r"(r[4]), "r"(r[5]), "r"(r[6]), "r"(r[7]), "r"(r[8]),
      "r"(r[9]), "r"(r[10]), "r"(r[11]), "r"(r[12]), "r"(r[13]), "r"(r[14]), "r"(r[15]), "r"(r[16]), "r"(r[17]),
      "r"(r[18]), "r"(r[19]), "r"(r[20]), "r"(r[21]), "r"(r[22]), "r"(r[23]), "r"(r[24]), "r"(r[25]), "r"(r[26]),
      "r"(r[27]), "r"(r[28]), "r"(r[29]), "r"(r[30]), "r"(r[31]));
}
template <bool STORE>
__global__ void k(unsigned long long* cyc, uint32_t* sink, int iters) {
  __shared__ uint32_t slot;
  const int warp = threadIdx.x >> 5;
  if (warp == 0) tmem_alloc<512>(&slot);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = slot + ((uint32_t)((warp & 3) * 32) << 16);
  const int nw = blockDim.x >> 5;
  const int colbase = (warp >> 2) * 128 % 512;
  uint32_t acc = 0;
  uint32_t r0[32], r1[32], r2[32], r3[32];
  for (int i = 0; i < 32; ++i) r0[i] = r1[i] = r2[i] = r3[i] = i + threadIdx.x;
  __syncthreads();
  unsigned long long t0 = clock64();
  for (int it = 0; it < iters; ++it) {
    const uint32_t c = (colbase + (it & 1) * 0) % 512;
    if (STORE) {
      st32(tmem + c, r0); st32(tmem + c + 32, r1); st32(tmem + c + 64, r2); st32(tmem + c + 96, r3);
      asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
    } else {
      tmem_ld32(tmem + c, r0); tmem_ld32(tmem + c + 32, r1); tmem_ld32(tmem + c + 64, r2); tmem_ld32(tmem + c + 96, r3);
      tmem_ld_wait();
      acc += r0[0] ^ r1[7] ^ r2[19] ^ r3[31];
    }
  }
  unsigned long long t1 = clock64();
  __syncthreads();
  if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
  sink[blockIdx.x * blockDim.x + threadIdx.x] = acc;
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  if (warp == 0) tmem_dealloc<512>(slot);
  (void)nw;
}
int main() {
  int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  unsigned long long* cyc; uint32_t* sink;
  cudaMalloc(&cyc, sms * 8); cudaMalloc(&sink, sms * 1024 * 4);
  const int iters = 20000;
  for (int store = 0; store < 2; ++store)
    for (int nw : {1, 4, 8, 16}) {
      if (store) k<true><<<sms, nw * 32>>>(cyc, sink, iters); else k<false><<<sms, nw * 32>>>(cyc, sink, iters);
      cudaDeviceSynchronize();
      unsigned long long h[256];
      cudaMemcpy(h, cyc, sms * 8, cudaMemcpyDeviceToHost);
      double avg = 0; for (int i = 0; i < sms; ++i) avg += h[i]; avg /= sms;
      const double bytes = (double)nw * iters * 4 * 32 * 32 * 4;   // per SM
      printf("%s warps=%2d: %.1f B/clk/SM (%.0f cycles per 16 KB warp batch)\n", store ? "st" : "ld", nw, bytes / avg,
             avg / iters);
    }
  printf("err %s\n", cudaGetErrorString(cudaGetLastError()));
}
