// Microbenchmark: issue/pipe throughput of the FP32 instruction forms K6 uses
// (scalar FFMA/FADD/FMUL, packed FFMA2/FADD2/FMUL2, MUFU.RSQ) on one SM and
// on the whole chip.  nvcc -gencode arch=compute_100a,code=sm_100a -O3 pipe_rates.cu
#include <cstdio>
#include <cuda_runtime.h>

constexpr int kIters = 4096;

template <int OP>
__global__ void k(float* out, float a0, float b0, long long* cyc) {
  float2 x[8], y = make_float2(a0, b0), z = make_float2(b0, a0);
  float s[8];
  double d[8], dy = a0, dz = b0;
#pragma unroll
  for (int i = 0; i < 8; ++i) { x[i] = make_float2(a0 + i, b0 - i); s[i] = a0 * i; d[i] = b0 * i; }
  __syncthreads();
  long long t0 = clock64();
  for (int it = 0; it < kIters; ++it) {
#pragma unroll
    for (int i = 0; i < 8; ++i) {
      if (OP == 0) s[i] = fmaf(s[i], y.x, z.x);                       // FFMA 3-reg
      if (OP == 1) x[i] = __ffma2_rn(x[i], y, z);                    // FFMA2
      if (OP == 2) x[i] = __fadd2_rn(x[i], y);                       // FADD2
      if (OP == 3) x[i] = __fmul2_rn(x[i], y);                       // FMUL2
      if (OP == 4) s[i] = s[i] + y.x;                                // FADD
      if (OP == 5) { float r; asm volatile("rsqrt.approx.ftz.f32 %0, %1;" : "=f"(r) : "f"(s[i])); s[i] = r; }
      if (OP == 6) { s[i] = fmaf(s[i], y.x, z.x); x[i] = __ffma2_rn(x[i], y, z); }  // mix
      if (OP == 7) { x[i] = __ffma2_rn(x[i], x[i], z); }  // FFMA2 with a repeated operand
      if (OP == 8) { d[i] = fma(d[i], dy, dz); }           // DFMA
    }
  }
  long long t1 = clock64();
  float acc = 0.f;
#pragma unroll
  for (int i = 0; i < 8; ++i) acc += x[i].x + x[i].y + s[i] + float(d[i]);
  out[blockIdx.x * blockDim.x + threadIdx.x] = acc;
  if (threadIdx.x == 0 && blockIdx.x == 0) *cyc = t1 - t0;
}

template <int OP>
void run(const char* name, int blocks, int threads) {
  float* out;
  long long* cyc;
  cudaMalloc(&out, sizeof(float) * blocks * threads);
  cudaMalloc(&cyc, 8);
  k<OP><<<blocks, threads>>>(out, 1.0001f, 0.9999f, cyc);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  cudaEventRecord(e0);
  k<OP><<<blocks, threads>>>(out, 1.0001f, 0.9999f, cyc);
  cudaEventRecord(e1);
  cudaEventSynchronize(e1);
  float ms;
  cudaEventElapsedTime(&ms, e0, e1);
  long long c;
  cudaMemcpy(&c, cyc, 8, cudaMemcpyDeviceToHost);
  const double warp_inst = double(blocks) * threads / 32 * kIters * 8 * (OP == 6 ? 2 : 1);
  int sms;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  const double per_sm_per_cyc = warp_inst / (blocks < sms ? blocks : sms) / double(c);
  printf("%-28s blocks=%4d thr=%4d  %8.3f ms  cycles(block0)=%lld  warp-inst/SM/clk=%.3f  lane-ops/SM/clk=%.1f\n", name,
         blocks, threads, ms, c, per_sm_per_cyc, per_sm_per_cyc * 32 * ((OP == 1 || OP == 2 || OP == 3 || OP == 7) ? 2 : 1));
  cudaFree(out);
  cudaFree(cyc);
}

int main() {
  int sms;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  for (int thr : {256, 512, 1024}) {
    run<0>("FFMA (3 reg)", sms, thr);
    run<4>("FADD", sms, thr);
    run<1>("FFMA2", sms, thr);
    run<2>("FADD2", sms, thr);
    run<3>("FMUL2", sms, thr);
    run<7>("FFMA2 repeated operand", sms, thr);
    run<5>("MUFU.RSQ", sms, thr);
    run<6>("FFMA + FFMA2 mix (2 inst)", sms, thr);
    run<8>("DFMA", sms, thr);
  }
  return 0;
}
