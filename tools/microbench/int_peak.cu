// int_peak.cu -- measured integer peak of the B200 for the join's roofline
// (bench.py roofline_join.peak).  Every thread runs 8 independent chains of
// LOP3 (3-input logic, alu pipe), IMAD (integer multiply-add, fma pipe) or
// both interleaved; lane-ops/s = threads x chains x iterations / time, timed
// with CUDA events (best of 5) over 148 SMs x 8 CTAs x 256 threads.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 int_peak.cu -o int_peak
#include <cstdio>
#include <cuda_runtime.h>

template <int OP>
__global__ void k_ops(unsigned *out, unsigned seed, int iters) {
  unsigned x0 = seed ^ threadIdx.x, x1 = x0 * 3u, x2 = x0 * 5u, x3 = x0 * 7u, x4 = x0 * 11u, x5 = x0 * 13u,
           x6 = x0 * 17u, x7 = x0 * 19u;
  const unsigned y = seed * 0x9e3779b9u, z = blockIdx.x | 1u;
  for (int i = 0; i < iters; i++) {
#pragma unroll
    for (int k = 0; k < 16; k++) {
      if (OP == 0) {  // LOP3: one 3-input logic op per chain step
        asm volatile("lop3.b32 %0, %0, %1, %2, 0x96;" : "+r"(x0) : "r"(y), "r"(z));
        asm volatile("lop3.b32 %0, %0, %1, %2, 0x96;" : "+r"(x1) : "r"(y), "r"(z));
        asm volatile("lop3.b32 %0, %0, %1, %2, 0x96;" : "+r"(x2) : "r"(y), "r"(z));
        asm volatile("lop3.b32 %0, %0, %1, %2, 0x96;" : "+r"(x3) : "r"(y), "r"(z));
        asm volatile("lop3.b32 %0, %0, %1, %2, 0x96;" : "+r"(x4) : "r"(y), "r"(z));
        asm volatile("lop3.b32 %0, %0, %1, %2, 0x96;" : "+r"(x5) : "r"(y), "r"(z));
        asm volatile("lop3.b32 %0, %0, %1, %2, 0x96;" : "+r"(x6) : "r"(y), "r"(z));
        asm volatile("lop3.b32 %0, %0, %1, %2, 0x96;" : "+r"(x7) : "r"(y), "r"(z));
      } else if (OP == 1) {  // IMAD (the fma pipe's integer op)
        asm volatile("mad.lo.u32 %0, %0, %1, %2;" : "+r"(x0) : "r"(y), "r"(z));
        asm volatile("mad.lo.u32 %0, %0, %1, %2;" : "+r"(x1) : "r"(y), "r"(z));
        asm volatile("mad.lo.u32 %0, %0, %1, %2;" : "+r"(x2) : "r"(y), "r"(z));
        asm volatile("mad.lo.u32 %0, %0, %1, %2;" : "+r"(x3) : "r"(y), "r"(z));
        asm volatile("mad.lo.u32 %0, %0, %1, %2;" : "+r"(x4) : "r"(y), "r"(z));
        asm volatile("mad.lo.u32 %0, %0, %1, %2;" : "+r"(x5) : "r"(y), "r"(z));
        asm volatile("mad.lo.u32 %0, %0, %1, %2;" : "+r"(x6) : "r"(y), "r"(z));
        asm volatile("mad.lo.u32 %0, %0, %1, %2;" : "+r"(x7) : "r"(y), "r"(z));
      } else {  // mixed: 4 LOP3 (alu pipe) + 4 IMAD (fma pipe) chains
        asm volatile("lop3.b32 %0, %0, %1, %2, 0x96;" : "+r"(x0) : "r"(y), "r"(z));
        asm volatile("mad.lo.u32 %0, %0, %1, %2;" : "+r"(x1) : "r"(y), "r"(z));
        asm volatile("lop3.b32 %0, %0, %1, %2, 0x96;" : "+r"(x2) : "r"(y), "r"(z));
        asm volatile("mad.lo.u32 %0, %0, %1, %2;" : "+r"(x3) : "r"(y), "r"(z));
        asm volatile("lop3.b32 %0, %0, %1, %2, 0x96;" : "+r"(x4) : "r"(y), "r"(z));
        asm volatile("mad.lo.u32 %0, %0, %1, %2;" : "+r"(x5) : "r"(y), "r"(z));
        asm volatile("lop3.b32 %0, %0, %1, %2, 0x96;" : "+r"(x6) : "r"(y), "r"(z));
        asm volatile("mad.lo.u32 %0, %0, %1, %2;" : "+r"(x7) : "r"(y), "r"(z));
      }
    }
  }
  out[blockIdx.x * blockDim.x + threadIdx.x] = x0 ^ x1 ^ x2 ^ x3 ^ x4 ^ x5 ^ x6 ^ x7;
}

template <int OP>
double run(int sms, int iters) {
  const int blocks = sms * 8, threads = 256;
  unsigned *out;
  cudaMalloc(&out, sizeof(unsigned) * blocks * threads);
  k_ops<OP><<<blocks, threads>>>(out, 1u, 16);
  cudaDeviceSynchronize();
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  float best = 1e30f;
  for (int r = 0; r < 5; r++) {
    cudaEventRecord(a);
    k_ops<OP><<<blocks, threads>>>(out, 2u + r, iters);
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms = 0;
    cudaEventElapsedTime(&ms, a, b);
    if (ms < best) best = ms;
  }
  cudaFree(out);
  const double ops = (double)blocks * threads * iters * 16.0 * 8.0;
  return ops / (best * 1e-3);
}

int main() {
  int dev = 0, sms = 0, clk = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, dev);  // kHz (max)
  const int iters = 4096;
  const double lop = run<0>(sms, iters), mad = run<1>(sms, iters), mix = run<2>(sms, iters);
  const double per = sms * clk * 1e3;
  printf("{\"sms\": %d, \"max_clock_mhz\": %.0f, \"lop3_lane_ops_per_s\": %.4e, \"imad_lane_ops_per_s\": %.4e, "
         "\"mixed_lane_ops_per_s\": %.4e, \"lop3_lanes_per_sm_per_clk\": %.1f, \"imad_lanes_per_sm_per_clk\": %.1f, "
         "\"mixed_lanes_per_sm_per_clk\": %.1f}\n",
         sms, clk / 1e3, lop, mad, mix, lop / per, mad / per, mix / per);
  return 0;
}
