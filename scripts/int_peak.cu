// int_peak.cu -- measured integer / bitwise issue rates of the B200 (sm_100a)
// for the instruction mix of the bitstream kernels:
// LOP3 (every AND/OR/NOT/class node), IADD3 (MatchStar adds), SHF (funnel
// shifts = Advance), PRMT (byte transpose), SHFL (cross-lane shifts), VOTE
// (ballots / zero-block guards), POPC (epilogue).
//
// Each thread runs 8 independent dependency chains of one instruction kind,
// so the rate is the pipe's throughput, not its latency.  Result: thread-ops
// per clock per SM and aggregate Tops/s at the clock the GPU ran at.
//   nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o int_peak int_peak.cu
//   ./int_peak > profiles/int_peak.json
#include <cstdio>
#include <cuda_runtime.h>

#define CH 8
#define ITERS 4096

template <int KIND>
__global__ void __launch_bounds__(1024) kern(unsigned *out, unsigned seed) {
  unsigned a[CH];
#pragma unroll
  for (int j = 0; j < CH; ++j) a[j] = seed * (threadIdx.x + 1) + j * 0x9E3779B9u;
  const unsigned b = seed ^ 0x5bd1e995u, c = seed + 0x27d4eb2fu;
  for (int it = 0; it < ITERS; ++it) {
#pragma unroll
    for (int j = 0; j < CH; ++j) {
      if (KIND == 0) asm volatile("lop3.b32 %0, %0, %1, %2, 0x96;" : "+r"(a[j]) : "r"(b), "r"(c));
      if (KIND == 1) asm volatile("add.u32 %0, %0, %1;\n\tadd.u32 %0, %0, %2;" : "+r"(a[j]) : "r"(b), "r"(c));  // one IADD3
      if (KIND == 2) asm volatile("shf.l.wrap.b32 %0, %0, %1, %2;" : "+r"(a[j]) : "r"(b), "r"(c));
      if (KIND == 3) asm volatile("prmt.b32 %0, %0, %1, %2;" : "+r"(a[j]) : "r"(b), "r"(c));
      if (KIND == 4) a[j] = __shfl_xor_sync(0xffffffffu, a[j], 1) + 1u;
      if (KIND == 5) a[j] = __ballot_sync(0xffffffffu, a[j] & 1u) ^ b;
      if (KIND == 6) asm volatile("popc.b32 %0, %0;" : "+r"(a[j]));
    }
  }
  unsigned s = 0;
#pragma unroll
  for (int j = 0; j < CH; ++j) s ^= a[j];
  if (s == 0x12345678u) out[0] = s;
}

template <int KIND>
double rate(int blocks, int threads, float &ms) {
  unsigned *o;
  cudaMalloc(&o, 4);
  kern<KIND><<<blocks, threads>>>(o, 1u);  // warm-up
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  cudaEventRecord(e0);
  for (int r = 0; r < 5; ++r) kern<KIND><<<blocks, threads>>>(o, 1u + r);
  cudaEventRecord(e1);
  cudaEventSynchronize(e1);
  cudaEventElapsedTime(&ms, e0, e1);
  ms /= 5;
  cudaFree(o);
  return (double)blocks * threads * ITERS * CH / (ms * 1e-3);  // thread-ops/s
}

int main() {
  cudaDeviceProp pr;
  cudaGetDeviceProperties(&pr, 0);
  int clk_khz = 0;
  cudaDeviceGetAttribute(&clk_khz, cudaDevAttrClockRate, 0);
  const int sms = pr.multiProcessorCount, threads = 1024, blocks = sms * 2;
  const char *names[] = {"lop3", "iadd", "shf", "prmt", "shfl", "vote", "popc"};
  double r[7];
  float ms[7];
  r[0] = rate<0>(blocks, threads, ms[0]);
  r[1] = rate<1>(blocks, threads, ms[1]);
  r[2] = rate<2>(blocks, threads, ms[2]);
  r[3] = rate<3>(blocks, threads, ms[3]);
  r[4] = rate<4>(blocks, threads, ms[4]);
  r[5] = rate<5>(blocks, threads, ms[5]);
  r[6] = rate<6>(blocks, threads, ms[6]);
  printf("{\"device\": \"%s\", \"sms\": %d, \"clock_mhz_attr\": %.0f, \"threads\": %d, \"chains\": %d, \"rates\": {", pr.name,
         sms, clk_khz / 1e3, blocks * threads, CH);
  for (int k = 0; k < 7; ++k)
    printf("%s\"%s\": {\"tops\": %.2f, \"ms\": %.3f, \"per_sm_per_clk_at_attr_clock\": %.1f}", k ? ", " : "", names[k],
           r[k] / 1e12, ms[k], r[k] / sms / (clk_khz * 1e3));
  printf("}}\n");
  return 0;
}
