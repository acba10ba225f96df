// MUFU (XU pipe) throughput on this GPU: ex2 / lg2 / rsqrt per SM per clock, 8 independent
// chains per thread, full occupancy.  usage: tools/mufu_bench
#include <cstdio>
#include <cuda_runtime.h>
template <int OP>
__global__ void k(float* out, int iters) {
  float v[8];
#pragma unroll
  for (int j = 0; j < 8; ++j) v[j] = 1.0f + 1e-3f * (threadIdx.x + j);
  for (int i = 0; i < iters; ++i) {
#pragma unroll
    for (int j = 0; j < 8; ++j) {
      if (OP == 0) asm volatile("ex2.approx.ftz.f32 %0, %0;" : "+f"(v[j]));
      if (OP == 1) asm volatile("lg2.approx.ftz.f32 %0, %0;" : "+f"(v[j]));
      if (OP == 2) asm volatile("rsqrt.approx.ftz.f32 %0, %0;" : "+f"(v[j]));
      if (OP == 3) asm volatile("fma.rn.f32 %0, %0, %0, %0;" : "+f"(v[j]));
      // packed half2 ex2: one instruction, two results (counted as 2 lane-ops)
      if (OP == 4) asm volatile("ex2.approx.f16x2 %0, %0;" : "+r"(*reinterpret_cast<unsigned*>(&v[j])));
      if (OP == 5) asm volatile("sqrt.approx.ftz.f32 %0, %0;" : "+f"(v[j]));
      if (OP == 6) asm volatile("tanh.approx.f32 %0, %0;" : "+f"(v[j]));
    }
  }
  float s = 0;
#pragma unroll
  for (int j = 0; j < 8; ++j) s += v[j];
  if (s == 12345.f) out[0] = s;
}
int main() {
  float* o;
  cudaMalloc(&o, 4);
  int sms;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  int clk;
  cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
  const int iters = 4096, blocks = sms * 8, threads = 256;
  const char* names[] = {"ex2", "lg2", "rsqrt", "ffma", "ex2h2", "sqrt", "tanh"};
  for (int op = 0; op < 7; ++op) {
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    for (int rep = 0; rep < 2; ++rep) {
      cudaEventRecord(a);
      if (op == 0) k<0><<<blocks, threads>>>(o, iters);
      if (op == 1) k<1><<<blocks, threads>>>(o, iters);
      if (op == 2) k<2><<<blocks, threads>>>(o, iters);
      if (op == 3) k<3><<<blocks, threads>>>(o, iters);
      if (op == 4) k<4><<<blocks, threads>>>(o, iters);
      if (op == 5) k<5><<<blocks, threads>>>(o, iters);
      if (op == 6) k<6><<<blocks, threads>>>(o, iters);
      cudaEventRecord(b);
      cudaEventSynchronize(b);
    }
    float ms;
    cudaEventElapsedTime(&ms, a, b);
    const double ops = (double)blocks * threads * iters * 8 * (op == 4 ? 2 : 1);
    printf("%-6s %.3f ms  %.2f lane-ops/clk/SM (at %d MHz nominal)\n", names[op], ms,
           ops / (ms * 1e-3) / sms / (clk * 1e3), clk / 1000);
  }
  return 0;
}
