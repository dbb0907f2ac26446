// gemm_kernel.cuh — C = act(A W^T + bias) on sm_100a: the MLP building block of the paper
// ("GEMM kernels with fused pointwise operations, like addition of a bias tensor
// or applying the Rectified Linear Unit (ReLU) activation function"; L453 MLP layer = GEMM +
// bias-add + activation).  SURVEY §8(a) a10.
//
//   tile         128 x 256 output tile per CTA, K streamed in 64-wide blocks
//   warp 0       TMA producer: A [128 x 64] and W [256 x 64] boxes into a 4-stage smem ring
//   warp 1       MMA issuer: tcgen05.mma M=128 N=256 K=16, fp32 accumulator in TMEM (256 columns)
//   warps 2-5    epilogue: tcgen05.ld (thread = output row), + bias, activation in fp32, one RNE
//                rounding to fp16, swizzled st.shared into the drained ring, TMA store
#pragma once
#include <cstdio>
#include <cstring>

#include "sm100.cuh"

namespace b200 {

struct GemmParams {
  CUtensorMap tmA;  // {K, M, 1} box {64, 128, 1}
  CUtensorMap tmW;  // {K, N, 1} box {64, 256, 1}
  CUtensorMap tmC;  // {N, M, 1} box {64, 128, 1}
  const __half* bias;
  int M, N, K;
  int act;
};

struct GemmCfg {
  static constexpr int BM = 128, BN = 256, BK = 64;
  static constexpr int STAGES = 4;
  static constexpr int A_BYTES = BM * BK * 2;  // 16 KB
  static constexpr int B_BYTES = BN * BK * 2;  // 32 KB
  static constexpr int STAGE_BYTES = A_BYTES + B_BYTES;
  static constexpr int OFF_BAR = STAGES * STAGE_BYTES;
  static constexpr int NUM_BARS = 2 * STAGES + 1;
  static constexpr int OFF_TMEMPTR = OFF_BAR + NUM_BARS * 8;
  static constexpr int SMEM_ALLOC = OFF_TMEMPTR + 16 + 1024;
  static constexpr int TMEM_COLS = 256;
  static constexpr int THREADS = 192;
  static constexpr int C_BOX = BM * 64 * 2;  // 16 KB output staging box (128 rows x 64 cols)
};

__device__ __forceinline__ float apply_act(float x, int act) {
  switch (act) {
    case 1: return fmaxf(x, 0.f);
    case 2: return 0.5f * x * (1.f + erff(x * 0.70710678118654752f));
    case 3: return 0.5f * x * (1.f + tanhf(0.7978845608028654f * (x + 0.044715f * x * x * x)));
    default: return x;
  }
}

__global__ void __launch_bounds__(192, 1) gemm_bias_act_kernel(const __grid_constant__ GemmParams p) {
  using C = GemmCfg;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  const uint32_t sbase = smem_u32(smem);
  const uint32_t bar = sbase + C::OFF_BAR;
  auto BAR_FULL = [&](int s) { return bar + 8 * s; };
  auto BAR_EMPTY = [&](int s) { return bar + 8 * C::STAGES + 8 * s; };
  const uint32_t BAR_ACC = bar + 16 * C::STAGES;
  uint32_t* tmem_holder = reinterpret_cast<uint32_t*>(smem + C::OFF_TMEMPTR);
  const int warp = warp_id(), lane = lane_id();
  const int n0 = blockIdx.x * C::BN, m0 = blockIdx.y * C::BM;
  const int nk = (p.K + C::BK - 1) / C::BK;

  if (threadIdx.x == 0) {
    for (int s = 0; s < C::STAGES; ++s) {
      mbar_init(BAR_FULL(s), 1);
      mbar_init(BAR_EMPTY(s), 1);
    }
    mbar_init(BAR_ACC, 1);
    fence_mbar_init();
  }
  if (warp == 0 && lane == 0) {
    tma_prefetch_desc(&p.tmA);
    tma_prefetch_desc(&p.tmW);
    tma_prefetch_desc(&p.tmC);
  }
  if (warp == 1) {
    tmem_alloc(smem_u32(tmem_holder), C::TMEM_COLS);
    tmem_relinquish();
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = *tmem_holder;

  if (warp == 0) {
    if (lane == 0) {
      for (int kb = 0; kb < nk; ++kb) {
        const int s = kb % C::STAGES;
        mbar_wait(BAR_EMPTY(s), ((kb / C::STAGES) & 1) ^ 1);
        mbar_arrive_expect_tx(BAR_FULL(s), C::STAGE_BYTES);
        const uint32_t sA = sbase + s * C::STAGE_BYTES;
        tma_load_3d(sA, &p.tmA, BAR_FULL(s), kb * C::BK, m0, 0);
        tma_load_3d(sA + C::A_BYTES, &p.tmW, BAR_FULL(s), kb * C::BK, n0, 0);
      }
    }
  } else if (warp == 1) {
    if (lane == 0) {
      constexpr uint32_t IDESC = idesc_f16(false, C::BM, C::BN, false, false);
      for (int kb = 0; kb < nk; ++kb) {
        const int s = kb % C::STAGES;
        mbar_wait(BAR_FULL(s), (kb / C::STAGES) & 1);
        tc_fence_after();
        const uint32_t sA = sbase + s * C::STAGE_BYTES;
        const uint32_t sB = sA + C::A_BYTES;
#pragma unroll
        for (int kk = 0; kk < C::BK / 16; ++kk)
          umma_ss(tmem, sdesc_sw128(sA + kk * 32, 16, 1024), sdesc_sw128(sB + kk * 32, 16, 1024), IDESC,
                  (kb > 0 || kk > 0));
        umma_commit(BAR_EMPTY(s));
      }
      umma_commit(BAR_ACC);
    }
  } else {
    const int quad = warp & 3;
    const int row = quad * 32 + lane;
    const uint32_t taddr = tmem + (static_cast<uint32_t>(quad * 32) << 16);
    mbar_wait(BAR_ACC, 0);
    tc_fence_after();
    // The ring is drained (every MMA completed), so its smem stages out the C tile:
    // 4 boxes of [128 rows x 64 cols] fp16, SWIZZLE_128B.
#pragma unroll 1
    for (int q = 0; q < C::BN / 32; ++q) {
      uint32_t v[32];
      tmem_ld_32x32b_x32(taddr + 32 * q, v);
      tmem_wait_ld();
      reg_fence(v);
      const int col0 = 32 * q;
      float f[32];
#pragma unroll
      for (int k = 0; k < 32; ++k) {
        const int n = n0 + col0 + k;
        float x = __uint_as_float(v[k]);
        if (p.bias) x += (n < p.N) ? __half2float(p.bias[n]) : 0.f;
        f[k] = apply_act(x, p.act);
      }
      const uint32_t box = sbase + (col0 / 64) * C::C_BOX + row * 128;
#pragma unroll
      for (int u = 0; u < 4; ++u) {
        const int unit = ((col0 % 64) / 8) + u;
        st_shared_v4(box + ((unit ^ (row & 7)) << 4), pack2<false>(f[8 * u + 0], f[8 * u + 1]),
                     pack2<false>(f[8 * u + 2], f[8 * u + 3]), pack2<false>(f[8 * u + 4], f[8 * u + 5]),
                     pack2<false>(f[8 * u + 6], f[8 * u + 7]));
      }
    }
    fence_proxy_async_smem();
    named_bar_sync(1, 128);
    if (row == 0) {
#pragma unroll
      for (int c = 0; c < C::BN / 64; ++c)
        if (n0 + c * 64 < p.N) tma_store_3d(&p.tmC, sbase + c * C::C_BOX, n0 + c * 64, m0, 0);
      tma_store_commit();
      tma_store_wait_read0();
    }
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 1) {
    tc_fence_after();
    tmem_dealloc(tmem, C::TMEM_COLS);
  }
}

// Host launcher (defined here so the ABI file stays thin).
int make_map_2d_rows(CUtensorMap* m, const void* base, uint64_t cols, uint64_t rows, uint32_t box_rows,
                     char* err, size_t errlen);

inline int launch_gemm_bias_act(const void* A, const void* W, const void* bias, void* Cm, int M, int N, int K,
                                int act, int /*sms*/, cudaStream_t stream, char* err, size_t errlen) {
  GemmParams prm;
  memset(&prm, 0, sizeof(prm));
  int st;
  if ((st = make_map_2d_rows(&prm.tmA, A, K, M, GemmCfg::BM, err, errlen)) != 0) return st;
  if ((st = make_map_2d_rows(&prm.tmW, W, K, N, GemmCfg::BN, err, errlen)) != 0) return st;
  if ((st = make_map_2d_rows(&prm.tmC, Cm, N, M, GemmCfg::BM, err, errlen)) != 0) return st;
  prm.bias = static_cast<const __half*>(bias);
  prm.M = M;
  prm.N = N;
  prm.K = K;
  prm.act = act;
  static bool attr_done[64];
  int dev = 0;
  cudaGetDevice(&dev);
  if (dev >= 64 || !attr_done[dev]) {
    cudaError_t e =
        cudaFuncSetAttribute(gemm_bias_act_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, GemmCfg::SMEM_ALLOC);
    if (e != cudaSuccess) {
      snprintf(err, errlen, "cudaFuncSetAttribute(gemm): %s", cudaGetErrorString(e));
      return 4;
    }
    if (dev < 64) attr_done[dev] = true;
  }
  dim3 grid((N + GemmCfg::BN - 1) / GemmCfg::BN, (M + GemmCfg::BM - 1) / GemmCfg::BM, 1);
  gemm_bias_act_kernel<<<grid, GemmCfg::THREADS, GemmCfg::SMEM_ALLOC, stream>>>(prm);
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) {
    snprintf(err, errlen, "gemm_bias_act_kernel launch: %s", cudaGetErrorString(e));
    return 4;
  }
  return 0;
}

}  // namespace b200
