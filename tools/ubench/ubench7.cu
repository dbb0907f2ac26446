// Microbenchmark 7: latency of mbarrier waits on an already-completed phase (try_wait vs test_wait),
// a shared-memory load, and a 64-column TMEM load, for one warp alone and with 3 other warps of the
// SMSP running an ex2/FFMA2 loop.
#include <cstdio>
#include <cstdint>
#include "../../paper_conf_asplos_hagedornfccgg23_b200/csrc/sm100.cuh"
using namespace b200;

__device__ __forceinline__ bool test_wait(uint32_t bar, uint32_t parity) {
  uint32_t ok;
  asm volatile("{\n\t.reg .pred p;\n\tmbarrier.test_wait.parity.shared::cta.b64 p, [%1], %2;\n\tselp.u32 %0, 1, 0, p;\n\t}"
               : "=r"(ok) : "r"(bar), "r"(parity) : "memory");
  return ok != 0;
}

__global__ void __launch_bounds__(512, 1) k(long long* out, int busy) {
  __shared__ __align__(8) uint64_t mb[2];
  __shared__ uint32_t holder;
  __shared__ float sm[1024];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (threadIdx.x == 0) { mbar_init(smem_u32(&mb[0]), 1); fence_mbar_init(); }
  if (warp == 0) { tmem_alloc(smem_u32(&holder), 512); tmem_relinquish(); }
  sm[threadIdx.x] = threadIdx.x; sm[threadIdx.x + 512] = 1.f;
  tc_fence_before(); __syncthreads(); tc_fence_after();
  if (threadIdx.x == 0) mbar_arrive(smem_u32(&mb[0]));  // phase 0 completes
  __syncthreads();
  const uint32_t bar = smem_u32(&mb[0]);
  const uint32_t tmem = holder;
  if (warp == 0) {
    long long t[6];
    uint32_t acc = 0;
    // try_wait on the completed phase 0
    long long a = clock64();
    for (int i = 0; i < 64; ++i) acc += mbar_try_wait(bar, 0) ? 1 : 0;
    long long b = clock64();
    for (int i = 0; i < 64; ++i) acc += test_wait(bar, 0) ? 1 : 0;
    long long c = clock64();
    float f = 0.f;
    for (int i = 0; i < 64; ++i) { f += sm[(lane + (int)f) & 1023]; }
    long long d = clock64();
    uint32_t r[64];
    for (int i = 0; i < 16; ++i) {
      tmem_ld_32x32b_x32(tmem + 64 * (i & 3), *reinterpret_cast<uint32_t(*)[32]>(&r[0]));
      tmem_ld_32x32b_x32(tmem + 64 * (i & 3) + 32, *reinterpret_cast<uint32_t(*)[32]>(&r[32]));
      tmem_wait_ld();
      reg_fence(r);
      acc += r[i & 63];
    }
    long long e = clock64();
    if (lane == 0) {
      out[blockIdx.x * 8 + 0] = (b - a) / 64;
      out[blockIdx.x * 8 + 1] = (c - b) / 64;
      out[blockIdx.x * 8 + 2] = (d - c) / 64;
      out[blockIdx.x * 8 + 3] = (e - d) / 16;
      out[blockIdx.x * 8 + 4] = acc + (long long)f;
    }
  } else if (busy && (warp & 3) == 0) {  // same SMSP as warp 0: an exp-phase-like loop
    float x = threadIdx.x * 1e-3f;
    for (int i = 0; i < 4000; ++i) { x = ex2(x * 0.5f - 1.f); }
    sm[threadIdx.x] = x;
  }
  tc_fence_before(); __syncthreads(); tc_fence_after();
  if (warp == 0) tmem_dealloc(tmem, 512);
}

int main() {
  long long* d; cudaMalloc(&d, 148 * 8 * 8);
  long long h[8];
  for (int busy = 0; busy < 2; ++busy) {
    for (int r = 0; r < 2; ++r) k<<<148, 512>>>(d, busy);
    cudaMemcpy(h, d, 64, cudaMemcpyDeviceToHost);
    printf("busy=%d: try_wait(done) %lld cyc, test_wait(done) %lld cyc, LDS dep %lld cyc, TMEM ld 64 cols+wait %lld cyc\n",
           busy, h[0], h[1], h[2], h[3]);
  }
  printf("status %s\n", cudaGetErrorString(cudaDeviceSynchronize()));
}
