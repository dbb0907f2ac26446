// Microbenchmark 6: which instructions share the MUFU (XU) pipe with ex2.approx.f32?
// 16 warps per CTA (4 per SMSP), one CTA per SM; each thread runs R rounds of 8 independent chains of
// one op mix; reports SMSP cycles per warp-instruction of each mix.
#include <cstdio>
#include <cstdint>
#include <cuda_fp16.h>
#define R 256

__device__ __forceinline__ float ex2(float x) { float y; asm volatile("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x)); return y; }
__device__ __forceinline__ uint32_t f2fp(float a, float b) { uint32_t r; asm volatile("cvt.rn.f16x2.f32 %0, %1, %2;" : "=r"(r) : "f"(b), "f"(a)); return r; }
__device__ __forceinline__ float fmx3(float a, float b, float c) { float d; asm volatile("max.f32 %0, %1, %2, %3;" : "=f"(d) : "f"(a), "f"(b), "f"(c)); return d; }
__device__ __forceinline__ uint64_t ffma2(uint64_t a, uint64_t b, uint64_t c) { uint64_t r; asm volatile("fma.rn.f32x2 %0, %1, %2, %3;" : "=l"(r) : "l"(a), "l"(b), "l"(c)); return r; }
__device__ __forceinline__ int imad(int a, int b, int c) { int d; asm volatile("mad.lo.s32 %0, %1, %2, %3;" : "=r"(d) : "r"(a), "r"(b), "r"(c)); return d; }

template <int MIX>
__global__ void __launch_bounds__(512, 1) k(float* out, long long* cyc, float seed) {
  float x[8]; uint32_t u[8]; uint64_t v[8]; int iv[8];
  for (int i = 0; i < 8; ++i) { x[i] = seed * (i + 1) * 1e-3f + threadIdx.x * 1e-6f; u[i] = i; v[i] = 0x3f8000003f800000ull + i; iv[i] = i + threadIdx.x; }
  __syncthreads();
  long long t0 = clock64();
  for (int r = 0; r < R; ++r) {
#pragma unroll
    for (int i = 0; i < 8; ++i) {
      if (MIX == 0) { x[i] = ex2(x[i]); }
      if (MIX == 1) { u[i] ^= f2fp(x[i], x[(i + 1) & 7]); x[i] += 1e-7f; }
      if (MIX == 2) { x[i] = ex2(x[i]); u[i] ^= f2fp(x[(i + 3) & 7], x[(i + 5) & 7]); }
      if (MIX == 3) { x[i] = ex2(x[i]); v[i] = ffma2(v[i], v[(i + 1) & 7], v[(i + 2) & 7]); }
      if (MIX == 4) { x[i] = ex2(x[i]); x[(i + 4) & 7] = fmx3(x[(i + 4) & 7], x[(i + 5) & 7], x[(i + 6) & 7]); }
      if (MIX == 5) { x[i] = ex2(x[i]); iv[i] = imad(iv[i], iv[(i + 1) & 7], iv[(i + 2) & 7]); }
      if (MIX == 6) { v[i] = ffma2(v[i], v[(i + 1) & 7], v[(i + 2) & 7]); }
      if (MIX == 7) { u[i] ^= f2fp(x[i], x[(i + 1) & 7]); v[i] = ffma2(v[i], v[(i + 1) & 7], v[(i + 2) & 7]); x[i] += 1e-7f; }
      if (MIX == 8) { x[i] = fmx3(x[i], x[(i + 1) & 7], x[(i + 2) & 7]); }
      if (MIX == 9) { iv[i] = imad(iv[i], iv[(i + 1) & 7], iv[(i + 2) & 7]); }
    }
  }
  long long t1 = clock64();
  float acc = 0.f;
  for (int i = 0; i < 8; ++i) acc += x[i] + (float)u[i] + (float)(v[i] & 0xff) + (float)iv[i];
  out[blockIdx.x * blockDim.x + threadIdx.x] = acc;
  if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
}

template <int MIX>
void run(const char* name, int ops_per_iter, float* out, long long* cyc) {
  k<MIX><<<148, 512>>>(out, cyc, 0.5f);
  k<MIX><<<148, 512>>>(out, cyc, 0.5f);
  cudaDeviceSynchronize();
  long long h[148];
  cudaMemcpy(h, cyc, sizeof(h), cudaMemcpyDeviceToHost);
  double avg = 0; for (int i = 0; i < 148; ++i) avg += h[i]; avg /= 148;
  // per SMSP: 4 warps x R x 8 x ops_per_iter warp-instructions
  printf("%-28s cycles per warp-instr per SMSP = %.2f\n", name, avg / (4.0 * R * 8 * ops_per_iter));
}

int main() {
  float* out; long long* cyc;
  cudaMalloc(&out, 148 * 512 * 4); cudaMalloc(&cyc, 148 * 8);
  run<0>("MUFU.EX2", 1, out, cyc);
  run<1>("F2FP (+FADD)", 1, out, cyc);
  run<2>("EX2 + F2FP (per pair)", 1, out, cyc);
  run<3>("EX2 + FFMA2 (per pair)", 1, out, cyc);
  run<4>("EX2 + FMNMX3 (per pair)", 1, out, cyc);
  run<5>("EX2 + IMAD (per pair)", 1, out, cyc);
  run<6>("FFMA2", 1, out, cyc);
  run<7>("F2FP + FFMA2 (+FADD) per grp", 1, out, cyc);
  run<8>("FMNMX3", 1, out, cyc);
  run<9>("IMAD", 1, out, cyc);
  printf("status %s\n", cudaGetErrorString(cudaGetLastError()));
}
