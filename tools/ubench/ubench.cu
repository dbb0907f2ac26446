// Microbenchmarks of the sm_100a pipes the FMHA softmax uses (run on a B200 via gpurun).
// Each test: 1 CTA per SM, W warps per SMSP, every thread runs ITERS iterations of 8 independent
// chains; reports cycles per warp-instruction per SMSP.
#include <cstdio>
#include <cstdint>
#include <cuda_fp16.h>

#define ITERS 2048

__device__ __forceinline__ float ex2(float x) { float y; asm volatile("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x)); return y; }

template <int OP>
__global__ void bench(float* out, long long* cyc, float seed) {
  float v[8];
#pragma unroll
  for (int i = 0; i < 8; ++i) v[i] = seed * (threadIdx.x + i) * 1e-3f;
  uint32_t h[8] = {0};
  __syncthreads();
  long long t0 = clock64();
  for (int it = 0; it < ITERS; ++it) {
#pragma unroll
    for (int i = 0; i < 8; ++i) {
      if (OP == 0) v[i] = ex2(v[i]);                                      // MUFU.EX2
      if (OP == 1) {                                                        // FFMA2 (2 lanes of work)
        uint64_t a; asm volatile("mov.b64 %0, {%1, %2};" : "=l"(a) : "f"(v[i]), "f"(v[(i+1)&7]));
        asm volatile("fma.rn.f32x2 %0, %0, %0, %0;" : "+l"(a));
        asm volatile("mov.b64 {%0, %1}, %2;" : "=f"(v[i]), "=f"(v[(i+1)&7]) : "l"(a));
      }
      if (OP == 2) { __half2 t = __floats2half2_rn(v[i], v[(i + 3) & 7]); h[i] ^= *(uint32_t*)&t; v[i] += 1e-7f; }
      if (OP == 3) v[i] = fmaf(v[i], 1.0001f, 0.5f);                      // FFMA
    }
  }
  long long t1 = clock64();
  float acc = 0;
#pragma unroll
  for (int i = 0; i < 8; ++i) acc += v[i] + h[i];
  out[blockIdx.x * blockDim.x + threadIdx.x] = acc;
  if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
}

// polynomial exp2 on the FMA pipe: 2^x = 2^floor(x) * p(frac), p degree 3 (minimax-ish)
__device__ __forceinline__ float exp2_poly(float x) {
  x = fmaxf(x, -127.f);
  float fl = floorf(x);
  float f = x - fl;
  float p = fmaf(fmaf(fmaf(0.0555041086648216f, f, 0.2402264923172690f), f, 0.6931471805599453f), f, 1.0f);
  int e = __float2int_rn(fl);
  return __int_as_float(__float_as_int(p) + (e << 23));
}
__global__ void bench_poly(float* out, long long* cyc, float seed) {
  float v[8];
#pragma unroll
  for (int i = 0; i < 8; ++i) v[i] = -seed * (threadIdx.x + i) * 1e-3f;
  __syncthreads();
  long long t0 = clock64();
  for (int it = 0; it < ITERS; ++it) {
#pragma unroll
    for (int i = 0; i < 8; ++i) v[i] = exp2_poly(v[i]) - 1.5f;
  }
  long long t1 = clock64();
  float acc = 0;
#pragma unroll
  for (int i = 0; i < 8; ++i) acc += v[i];
  out[blockIdx.x * blockDim.x + threadIdx.x] = acc;
  if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
}

int main() {
  float* out; long long* cyc; cudaMalloc(&out, 148 * 1024 * 4); cudaMalloc(&cyc, 148 * 8);
  long long h[148];
  const char* names[] = {"MUFU.EX2", "FFMA2", "F2FP(cvt f16x2)", "FFMA"};
  for (int w = 1; w <= 4; w *= 2) {
    for (int op = 0; op < 5; ++op) {
      int threads = 128 * w;
      for (int rep = 0; rep < 2; ++rep) {
        if (op == 0) bench<0><<<148, threads>>>(out, cyc, 1.f);
        if (op == 1) bench<1><<<148, threads>>>(out, cyc, 1.f);
        if (op == 2) bench<2><<<148, threads>>>(out, cyc, 1.f);
        if (op == 3) bench<3><<<148, threads>>>(out, cyc, 1.f);
        if (op == 4) bench_poly<<<148, threads>>>(out, cyc, 1.f);
      }
      cudaMemcpy(h, cyc, sizeof(h), cudaMemcpyDeviceToHost);
      double per = (double)h[0] / (ITERS * 8.0 * w);  // cycles per warp-op per SMSP
      printf("%-18s warps/SMSP=%d  cycles per warp-op per SMSP = %.2f  (lanes/clk/SM = %.1f)\n",
             op < 4 ? names[op] : "exp2_poly(~8 ops)", w, per, 128.0 / per);
    }
  }
  cudaError_t e = cudaDeviceSynchronize();
  printf("status %s\n", cudaGetErrorString(e));
  return 0;
}
