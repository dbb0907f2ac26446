// Microbenchmarks, part 2: packed fp32x2 pipes, the softmax inner-loop mix, and tcgen05.mma
// issue cost / latency (SS N=128 and TS N=64, M=128, K=16) from one elected lane of a converged warp.
#include <cstdio>
#include <cstdint>
#include <cuda_fp16.h>
#include "../../paper_conf_asplos_hagedornfccgg23_b200/csrc/sm100.cuh"
using namespace b200;
#define ITERS 1024

template <int OP>
__global__ void packed(float* out, long long* cyc, float seed) {
  uint64_t a[8];
#pragma unroll
  for (int i = 0; i < 8; ++i) a[i] = f2_as_u64(make_float2(seed * i, seed * (threadIdx.x + 1)));
  const uint64_t c = f2_as_u64(make_float2(0.999f, 0.999f)), d = f2_as_u64(make_float2(1e-3f, 1e-3f));
  __syncthreads();
  long long t0 = clock64();
  for (int it = 0; it < ITERS; ++it) {
#pragma unroll
    for (int i = 0; i < 8; ++i) {
      if (OP == 0) asm volatile("fma.rn.f32x2 %0, %0, %1, %2;" : "+l"(a[i]) : "l"(c), "l"(d));
      if (OP == 1) asm volatile("add.f32x2 %0, %0, %1;" : "+l"(a[i]) : "l"(d));
      if (OP == 2) asm volatile("mul.f32x2 %0, %0, %1;" : "+l"(a[i]) : "l"(c));
    }
  }
  long long t1 = clock64();
  float acc = 0;
#pragma unroll
  for (int i = 0; i < 8; ++i) { float2 v = u64_as_f2(a[i]); acc += v.x + v.y; }
  out[blockIdx.x * blockDim.x + threadIdx.x] = acc;
  if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
}

// the softmax exp phase on 128 values held in registers: FFMA2, 2x MUFU, FADD2, F2FP per pair
__global__ void smix(float* out, long long* cyc, float seed) {
  float s[128];
#pragma unroll
  for (int k = 0; k < 128; ++k) s[k] = seed * (k - 64) * 0.01f + threadIdx.x * 1e-4f;
  const float c = 0.18f, mc = 0.5f;
  uint32_t sink = 0;
  __syncthreads();
  long long t0 = clock64();
  for (int it = 0; it < 64; ++it) {
    float2 acc0 = make_float2(0.f, 0.f), acc1 = make_float2(0.f, 0.f);
#pragma unroll
    for (int k = 0; k < 128; k += 4) {
      float2 x0 = ffma2(make_float2(s[k], s[k + 1]), c, -mc);
      float2 x1 = ffma2(make_float2(s[k + 2], s[k + 3]), c, -mc);
      x0.x = ex2(x0.x); x0.y = ex2(x0.y); x1.x = ex2(x1.x); x1.y = ex2(x1.y);
      acc0 = fadd2(acc0, x0); acc1 = fadd2(acc1, x1);
      sink ^= pack2<false>(x0.x, x0.y) + pack2<false>(x1.x, x1.y);
    }
    s[it & 127] += acc0.x + acc1.y;
  }
  long long t1 = clock64();
  out[blockIdx.x * blockDim.x + threadIdx.x] = s[5] + sink;
  if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
}

// tcgen05.mma issue: one warp issues NM MMAs back to back (elected lane), then commit + wait.
template <int MODE>  // 0: SS M128 N128 K16; 1: TS M128 N64 K16
__global__ void __launch_bounds__(128, 1) mma_issue(long long* cyc, int nm) {
  extern __shared__ __align__(1024) uint8_t smem[];
  const uint32_t sbase = smem_u32(smem);
  __shared__ uint32_t holder;
  __shared__ __align__(8) uint64_t barm;
  const uint32_t bar = smem_u32(&barm);
  if (threadIdx.x == 0) { mbar_init(bar, 1); fence_mbar_init(); }
  if (threadIdx.x < 32) { tmem_alloc(smem_u32(&holder), 512); tmem_relinquish(); }
  tc_fence_before(); __syncthreads(); tc_fence_after();
  const uint32_t tmem = holder;
  long long t0 = 0, t1 = 0, t2 = 0;
  if (threadIdx.x < 32) {
    const uint64_t desc0 = sdesc_sw128(sbase, 16, 1024);
    const uint64_t vdesc0 = sdesc_sw128(sbase, 16384, 1024);
    constexpr uint32_t IQK = idesc_f16(false, 128, 128, false, false);
    constexpr uint32_t IPV = idesc_f16(false, 128, 64, false, true);
    __syncwarp();
    t0 = clock64();
    for (int i = 0; i < nm; ++i) {
      if (MODE == 0) umma_ss_elect(tmem, desc0 + ((i & 3) * 2), desc0 + 1024 + ((i & 3) * 2), IQK, i > 0);
      else umma_ts_elect(tmem + 256, tmem + 128 + (i & 7) * 8, vdesc0 + 2048 + (i & 7) * 128, IPV, i > 0);
    }
    umma_commit_elect(bar);
    t1 = clock64();
    mbar_wait(bar, 0);
    t2 = clock64();
  }
  tc_fence_before(); __syncthreads(); tc_fence_after();
  if (threadIdx.x == 0) { cyc[3 * blockIdx.x] = t1 - t0; cyc[3 * blockIdx.x + 1] = t2 - t0; }
  if (threadIdx.x < 32) tmem_dealloc(tmem, 512);
}

int main() {
  float* out; long long* cyc; cudaMalloc(&out, 148 * 1024 * 4); cudaMalloc(&cyc, 148 * 8 * 3);
  long long h[3 * 148];
  const char* pn[] = {"FFMA2", "FADD2", "FMUL2"};
  for (int w = 1; w <= 2; ++w)
    for (int op = 0; op < 3; ++op) {
      for (int rep = 0; rep < 2; ++rep) {
        if (op == 0) packed<0><<<148, 128 * w>>>(out, cyc, 1.f);
        if (op == 1) packed<1><<<148, 128 * w>>>(out, cyc, 1.f);
        if (op == 2) packed<2><<<148, 128 * w>>>(out, cyc, 1.f);
      }
      cudaMemcpy(h, cyc, 8 * 148, cudaMemcpyDeviceToHost);
      printf("%-6s warps/SMSP=%d  cycles per warp-op per SMSP = %.2f\n", pn[op], w, h[0] / (ITERS * 8.0 * w));
    }
  for (int w = 1; w <= 2; ++w) {
    for (int rep = 0; rep < 2; ++rep) smix<<<148, 128 * w>>>(out, cyc, 1.f);
    cudaMemcpy(h, cyc, 8 * 148, cudaMemcpyDeviceToHost);
    printf("softmax mix (128 elem/thread) warps/SMSP=%d: %.1f cycles per 128-element row per warp (MUFU floor 1024)\n",
           w, h[0] / (64.0 * w));
  }
  cudaFuncSetAttribute(mma_issue<0>, cudaFuncAttributeMaxDynamicSharedMemorySize, 64 * 1024);
  cudaFuncSetAttribute(mma_issue<1>, cudaFuncAttributeMaxDynamicSharedMemorySize, 64 * 1024);
  for (int nm : {1, 4, 8, 32, 128}) {
    for (int rep = 0; rep < 2; ++rep) mma_issue<0><<<148, 128, 64 * 1024>>>(cyc, nm);
    cudaMemcpy(h, cyc, 8 * 3 * 148, cudaMemcpyDeviceToHost);
    printf("SS M128N128K16 x%-3d: issue %6lld cyc (%.1f/mma), issue->done %6lld cyc (%.1f/mma; TC floor 64)\n", nm,
           h[0], (double)h[0] / nm, h[1], (double)h[1] / nm);
    for (int rep = 0; rep < 2; ++rep) mma_issue<1><<<148, 128, 64 * 1024>>>(cyc, nm);
    cudaMemcpy(h, cyc, 8 * 3 * 148, cudaMemcpyDeviceToHost);
    printf("TS M128N64K16  x%-3d: issue %6lld cyc (%.1f/mma), issue->done %6lld cyc (%.1f/mma; TC floor 32)\n", nm,
           h[0], (double)h[0] / nm, h[1], (double)h[1] / nm);
  }
  cudaError_t e = cudaDeviceSynchronize();
  printf("status %s\n", cudaGetErrorString(e));
  return 0;
}
