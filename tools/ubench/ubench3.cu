// Microbenchmarks, part 3: variants of the softmax exp phase (128 fp32 scores per thread ->
// 128 16-bit P values + row sum), 1 and 2 warps per SMSP, plus tcgen05.ld/st costs.
#include <cstdio>
#include <cstdint>
#include "../../paper_conf_asplos_hagedornfccgg23_b200/csrc/sm100.cuh"
using namespace b200;

// 2^x on the FMA/ALU pipes for x <= 0 (x >= -126 clamp): Cody-Waite split with a round-to-nearest
// magic constant, degree-3 polynomial on f in [-0.5, 0.5], exponent add in the integer pipe.
__device__ __forceinline__ float2 exp2_poly2(float2 x) {
  const float2 mg = make_float2(12582912.f, 12582912.f);  // 1.5 * 2^23
  x.x = fmaxf(x.x, -126.f); x.y = fmaxf(x.y, -126.f);
  float2 t = fadd2(x, mg);                                  // round(x) in the low mantissa bits
  float2 j = fadd2(t, make_float2(-12582912.f, -12582912.f));
  float2 f = fadd2(x, make_float2(-j.x, -j.y));             // f in [-0.5, 0.5]
  float2 p = ffma2(f, make_float2(0.0555041f, 0.0555041f), make_float2(0.2402265f, 0.2402265f));
  p = ffma2(p, f, make_float2(0.6931472f, 0.6931472f));
  p = ffma2(p, f, make_float2(1.0f, 1.0f));
  const int ex = __float_as_int(t.x) << 23, ey = __float_as_int(t.y) << 23;
  return make_float2(__int_as_float(__float_as_int(p.x) + ex), __int_as_float(__float_as_int(p.y) + ey));
}

template <int V, int POLY_EVERY>
__global__ void exp_phase(float* out, long long* cyc, float seed) {
  float s[128];
#pragma unroll
  for (int k = 0; k < 128; ++k) s[k] = seed * (k - 64) * 0.01f + threadIdx.x * 1e-4f;
  const float c = 0.18f, mc = 0.5f;
  uint32_t sink = 0;
  float lsum = 0.f;
  __syncthreads();
  long long t0 = clock64();
  for (int it = 0; it < 32; ++it) {
    float2 acc0 = make_float2(0.f, 0.f), acc1 = make_float2(0.f, 0.f);
    uint32_t pk[64];
    if (V == 0) {  // current kernel: FFMA2, 2 MUFU, FADD2, F2FP per pair
#pragma unroll
      for (int k = 0; k < 128; k += 4) {
        float2 x0 = ffma2(make_float2(s[k], s[k + 1]), c, -mc);
        float2 x1 = ffma2(make_float2(s[k + 2], s[k + 3]), c, -mc);
        if (POLY_EVERY && (k / 4) % (POLY_EVERY ? POLY_EVERY : 1) == POLY_EVERY - 1) x0 = exp2_poly2(x0);
        else { x0.x = ex2(x0.x); x0.y = ex2(x0.y); }
        x1.x = ex2(x1.x); x1.y = ex2(x1.y);
        acc0 = fadd2(acc0, x0); acc1 = fadd2(acc1, x1);
        pk[k / 2] = pack2<false>(x0.x, x0.y); pk[k / 2 + 1] = pack2<false>(x1.x, x1.y);
      }
    } else if (V == 1) {  // scalar FFMA / FADD
      float a0 = 0, a1 = 0, a2 = 0, a3 = 0;
#pragma unroll
      for (int k = 0; k < 128; k += 4) {
        float e0 = ex2(fmaf(s[k], c, -mc)), e1 = ex2(fmaf(s[k + 1], c, -mc));
        float e2 = ex2(fmaf(s[k + 2], c, -mc)), e3 = ex2(fmaf(s[k + 3], c, -mc));
        a0 += e0; a1 += e1; a2 += e2; a3 += e3;
        pk[k / 2] = pack2<false>(e0, e1); pk[k / 2 + 1] = pack2<false>(e2, e3);
      }
      acc0 = make_float2(a0 + a1, a2 + a3);
    } else {  // batched in groups of 16 elements: all FFMA2, then all MUFU, then FADD2 + F2FP
#pragma unroll
      for (int g = 0; g < 128; g += 16) {
        float2 x[8];
#pragma unroll
        for (int u = 0; u < 8; ++u) x[u] = ffma2(make_float2(s[g + 2 * u], s[g + 2 * u + 1]), c, -mc);
#pragma unroll
        for (int u = 0; u < 8; ++u) {
          if (POLY_EVERY && u % (POLY_EVERY ? POLY_EVERY : 1) == POLY_EVERY - 1) x[u] = exp2_poly2(x[u]);
          else { x[u].x = ex2(x[u].x); x[u].y = ex2(x[u].y); }
        }
#pragma unroll
        for (int u = 0; u < 8; u += 2) { acc0 = fadd2(acc0, x[u]); acc1 = fadd2(acc1, x[u + 1]); }
#pragma unroll
        for (int u = 0; u < 8; ++u) pk[g / 2 + u] = pack2<false>(x[u].x, x[u].y);
      }
    }
#pragma unroll
    for (int u = 0; u < 64; ++u) sink ^= pk[u];
    lsum += acc0.x + acc0.y + acc1.x + acc1.y;
    s[it & 127] += lsum * 1e-9f;
  }
  long long t1 = clock64();
  out[blockIdx.x * blockDim.x + threadIdx.x] = s[5] + sink + lsum;
  if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
}

// TMEM: 4 x tcgen05.ld.32x32b.x32 (128 columns) + wait, and 2 x st.x32 + wait, per warp
__global__ void __launch_bounds__(256, 1) tmem_bench(long long* cyc, int warps_active) {
  __shared__ uint32_t holder;
  if (threadIdx.x < 32) { tmem_alloc(smem_u32(&holder), 512); tmem_relinquish(); }
  tc_fence_before(); __syncthreads(); tc_fence_after();
  const uint32_t tmem = holder;
  const int warp = threadIdx.x >> 5;
  const uint32_t base = tmem + ((uint32_t)((warp & 3) * 32) << 16) + (warp >> 2) * 128;
  long long tl = 0, ts = 0;
  if (warp < warps_active) {
    uint32_t acc = 0;
    long long t0 = clock64();
    for (int it = 0; it < 16; ++it) {
      uint32_t r[128];
#pragma unroll
      for (int q = 0; q < 4; ++q) tmem_ld_32x32b_x32(base + 32 * q, *reinterpret_cast<uint32_t(*)[32]>(&r[32 * q]));
      tmem_wait_ld();
      reg_fence(r);
#pragma unroll
      for (int q = 0; q < 128; ++q) acc += r[q];
    }
    long long t1 = clock64();
    for (int it = 0; it < 16; ++it) {
      uint32_t r[32];
#pragma unroll
      for (int q = 0; q < 32; ++q) r[q] = acc + q + it;
      tmem_st_32x32b_x32(base + 256, r);
      tmem_st_32x32b_x32(base + 288, r);
      tmem_wait_st();
    }
    long long t2 = clock64();
    tl = (t1 - t0) / 16; ts = (t2 - t1) / 16;
    if (acc == 12345) tl = 0;
  }
  tc_fence_before(); __syncthreads(); tc_fence_after();
  if (threadIdx.x == 0) { cyc[2 * blockIdx.x] = tl; cyc[2 * blockIdx.x + 1] = ts; }
  if (threadIdx.x < 32) tmem_dealloc(tmem, 512);
}

int main() {
  float* out; long long* cyc; cudaMalloc(&out, 148 * 1024 * 4); cudaMalloc(&cyc, 148 * 8 * 2);
  long long h[2 * 148];
  auto run = [&](const char* name, void (*k)(float*, long long*, float)) {
    for (int w = 1; w <= 2; ++w) {
      for (int rep = 0; rep < 2; ++rep) k<<<148, 128 * w>>>(out, cyc, 1.f);
      cudaMemcpy(h, cyc, 8 * 148, cudaMemcpyDeviceToHost);
      printf("%-40s warps/SMSP=%d : %7.1f cycles per 128-element row per warp\n", name, w, h[0] / (32.0 * w));
    }
  };
  run("packed (kernel today)", exp_phase<0, 0>);
  run("scalar FFMA/FADD", exp_phase<1, 0>);
  run("batched x16", exp_phase<2, 0>);
  run("packed, 1/8 pairs poly", exp_phase<0, 8>);
  run("packed, 1/4 pairs poly", exp_phase<0, 4>);
  run("batched, 1/4 pairs poly", exp_phase<2, 4>);
  run("batched, 1/2 pairs poly", exp_phase<2, 2>);
  run("batched, 3/8 pairs poly", exp_phase<2, 3>);
  for (int wa : {4, 8}) {
    tmem_bench<<<148, 256>>>(cyc, wa);
    tmem_bench<<<148, 256>>>(cyc, wa);
    cudaMemcpy(h, cyc, 16 * 148, cudaMemcpyDeviceToHost);
    printf("TMEM %d warps: ld 128 cols + wait %lld cycles; st 64 cols + wait %lld cycles\n", wa, h[0], h[1]);
  }
  cudaError_t e = cudaDeviceSynchronize();
  printf("status %s\n", cudaGetErrorString(e));
  return 0;
}
