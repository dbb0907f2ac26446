// Microbenchmark, part 5: the kernel's exact exp phase (64 scores/thread, half the pairs on the FMA
// pipe via exp2_poly2, FADD2 row sum, F2FP pack, 2 x tcgen05.st.32x32b.x16 + wait::st), with 1, 2
// and 4 warps per SMSP.  Reports cycles per 64-element half-row per warp.
#include <cstdio>
#include <cstdint>
#include "../../paper_conf_asplos_hagedornfccgg23_b200/csrc/sm100.cuh"
using namespace b200;

template <int POLY_CNT>
__global__ void __launch_bounds__(512, 1) phase(float* out, long long* cyc, float seed, int iters) {
  __shared__ uint32_t holder;
  if (threadIdx.x < 32) { tmem_alloc(smem_u32(&holder), 512); tmem_relinquish(); }
  tc_fence_before(); __syncthreads(); tc_fence_after();
  const uint32_t tmem = holder;
  const int warp = threadIdx.x >> 5, quad = warp & 3;
  const uint32_t tP = tmem + ((uint32_t)(quad * 32) << 16) + 32 * (warp >> 2);
  float s[64];
#pragma unroll
  for (int k = 0; k < 64; ++k) s[k] = seed * (k - 32) * 0.05f + threadIdx.x * 1e-4f;
  const float c = 0.18f, mc = 0.5f;
  float l = 0.f;
  __syncthreads();
  long long t0 = clock64();
  for (int it = 0; it < iters; ++it) {
    float2 acc0 = make_float2(0.f, 0.f), acc1 = make_float2(0.f, 0.f);
#pragma unroll
    for (int hh = 0; hh < 2; ++hh) {
      uint32_t pk[16];
#pragma unroll
      for (int u = 0; u < 16; u += 2) {
        const int k = 32 * hh + 2 * u;
        float2 x0 = ffma2(make_float2(s[k], s[k + 1]), c, -mc);
        float2 x1 = ffma2(make_float2(s[k + 2], s[k + 3]), c, -mc);
        if (((16 * hh + u) % 8) < POLY_CNT) x0 = exp2_poly2(x0);
        else { x0.x = ex2(x0.x); x0.y = ex2(x0.y); }
        if (((16 * hh + u + 1) % 8) < POLY_CNT) x1 = exp2_poly2(x1);
        else { x1.x = ex2(x1.x); x1.y = ex2(x1.y); }
        acc0 = fadd2(acc0, x0);
        acc1 = fadd2(acc1, x1);
        pk[u] = pack2<false>(x0.x, x0.y);
        pk[u + 1] = pack2<false>(x1.x, x1.y);
      }
      tmem_st_32x32b_x16(tP + 16 * hh, pk);
    }
    tmem_wait_st();
    l = l * 0.999f + ((acc0.x + acc0.y) + (acc1.x + acc1.y));
    s[it & 63] += l * 1e-12f;
  }
  long long t1 = clock64();
  out[blockIdx.x * blockDim.x + threadIdx.x] = l;
  if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
  tc_fence_before(); __syncthreads(); tc_fence_after();
  if (threadIdx.x < 32) tmem_dealloc(tmem, 512);
}

int main() {
  float* out; long long* cyc; cudaMalloc(&out, 148 * 1024 * 4); cudaMalloc(&cyc, 148 * 8);
  long long h[148];
  for (int pc : {0, 2, 4}) {
    for (int w = 1; w <= 4; w *= 2) {
      for (int r = 0; r < 2; ++r) {
        if (pc == 0) phase<0><<<148, 128 * w>>>(out, cyc, 1.f, 64);
        if (pc == 2) phase<2><<<148, 128 * w>>>(out, cyc, 1.f, 64);
        if (pc == 4) phase<4><<<148, 128 * w>>>(out, cyc, 1.f, 64);
      }
      cudaMemcpy(h, cyc, 8 * 148, cudaMemcpyDeviceToHost);
      printf("poly %d/8  warps/SMSP=%d: %.1f cycles per half-row per warp; SMSP busy %.1f cycles per half-row-set\n",
             pc, w, h[0] / (64.0 * w), h[0] / 64.0);
    }
  }
  printf("status %s\n", cudaGetErrorString(cudaDeviceSynchronize()));
  return 0;
}
