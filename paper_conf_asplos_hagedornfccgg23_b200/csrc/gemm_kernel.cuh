// gemm_kernel.cuh — C = act(A W^T + bias) on sm_100a: the MLP building block of the paper
// ("GEMM kernels with fused pointwise operations, like addition of a bias tensor
// or applying the Rectified Linear Unit (ReLU) activation function"; L453 MLP layer = GEMM +
// bias-add + activation).  SURVEY §8(a) a10.
//
// Persistent: one CTA (384 threads) per SM walks 128 x 256 output tiles (static round-robin).
//   warp 0       TMA producer: A [128 x 64] and W [256 x 64] boxes into an S-stage smem ring
//   warp 1       MMA issuer: tcgen05.mma M=128 N=256 K=16, fp32 accumulator in TMEM; two
//                accumulator buffers (2 x 256 columns) so tile i+1's mainloop runs under tile i's
//                epilogue
//   warps 4-11   epilogue: warp (g, q) = 4 + 4g + q takes TMEM lanes 32q.. (output rows) and columns
//                128g..128g+127; tcgen05.ld -> + bias, activation in fp32 -> one RNE rounding to fp16
//                -> swizzled st.shared -> TMA store (rows >= M / cols >= N clipped)
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
  int tiles_m, tiles_n;
};

struct GemmCfg {
  static constexpr int BM = 128, BN = 256, BK = 64;
  static constexpr int STAGES = 3;
  static constexpr int A_BYTES = BM * BK * 2;  // 16 KB
  static constexpr int B_BYTES = BN * BK * 2;  // 32 KB
  static constexpr int STAGE_BYTES = A_BYTES + B_BYTES;
  static constexpr int C_BOX = BM * 64 * 2;  // 16 KB output staging box (128 rows x 64 cols)
  static constexpr int OFF_STG = STAGES * STAGE_BYTES;
  static constexpr int OFF_BAR = OFF_STG + 4 * C_BOX;
  // barriers: full[S], empty[S], acc_full[2], acc_empty[2]
  static constexpr int NUM_BARS = 2 * STAGES + 4;
  static constexpr int OFF_TMEMPTR = OFF_BAR + NUM_BARS * 8;
  static constexpr int SMEM_ALLOC = OFF_TMEMPTR + 16;
  static constexpr int TMEM_COLS = 512;
  static constexpr int THREADS = 384;
  static_assert(SMEM_ALLOC <= 232448, "shared memory budget");
};

template <int ACT>
__device__ __forceinline__ float apply_act(float x) {
  if (ACT == 1) return fmaxf(x, 0.f);
  if (ACT == 2) return 0.5f * x * (1.f + erff(x * 0.70710678118654752f));
  if (ACT == 3) return 0.5f * x * (1.f + tanhf(0.7978845608028654f * (x + 0.044715f * x * x * x)));
  return x;
}

template <int ACT>
__global__ void __launch_bounds__(384, 1) gemm_bias_act_kernel(const __grid_constant__ GemmParams p) {
  using C = GemmCfg;
  extern __shared__ __align__(1024) uint8_t smem[];
  const uint32_t sbase = smem_u32(smem);
  const uint32_t bar = sbase + C::OFF_BAR;
  auto FULL = [&](int s) { return bar + 8 * s; };
  auto EMPTY = [&](int s) { return bar + 8 * (C::STAGES + s); };
  auto ACC_FULL = [&](int b) { return bar + 8 * (2 * C::STAGES + b); };
  auto ACC_EMPTY = [&](int b) { return bar + 8 * (2 * C::STAGES + 2 + b); };
  uint32_t* tmem_holder = reinterpret_cast<uint32_t*>(smem + C::OFF_TMEMPTR);
  const int warp = warp_id(), lane = lane_id();
  const int nk = (p.K + C::BK - 1) / C::BK;
  const int num_tiles = p.tiles_m * p.tiles_n;

  if (threadIdx.x == 0) {
    if (sbase & 1023u) __trap();
    for (int s = 0; s < C::STAGES; ++s) {
      mbar_init(FULL(s), 1);
      mbar_init(EMPTY(s), 1);
    }
    for (int b = 0; b < 2; ++b) {
      mbar_init(ACC_FULL(b), 1);
      mbar_init(ACC_EMPTY(b), 256);  // all epilogue threads
    }
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
    // ---------------------------------------------------------------- TMA producer
    uint32_t it = 0;
    const uint64_t keep = policy_evict_last();  // A rows and W are re-read by other tiles (all fit in L2)
    for (int tile = blockIdx.x; tile < num_tiles; tile += gridDim.x) {
      const int m0 = (tile / p.tiles_n) * C::BM, n0 = (tile % p.tiles_n) * C::BN;
      for (int kb = 0; kb < nk; ++kb, ++it) {
        const int s = it % C::STAGES;
        mbar_wait(EMPTY(s), ((it / C::STAGES) & 1) ^ 1);
        mbar_arrive_expect_tx_elect(FULL(s), C::STAGE_BYTES);
        const uint32_t sA = sbase + s * C::STAGE_BYTES;
        tma_load_3d_hint_elect(sA, &p.tmA, FULL(s), kb * C::BK, m0, 0, keep);
        tma_load_3d_hint_elect(sA + C::A_BYTES, &p.tmW, FULL(s), kb * C::BK, n0, 0, keep);
      }
    }
  } else if (warp == 1) {
    // ---------------------------------------------------------------- MMA issuer
    constexpr uint32_t IDESC = idesc_f16(false, C::BM, C::BN, false, false);
    const uint64_t desc0 = sdesc_sw128(sbase, 16, 1024);
    uint32_t it = 0, tc = 0;
    for (int tile = blockIdx.x; tile < num_tiles; tile += gridDim.x, ++tc) {
      const int b = tc & 1;
      mbar_wait(ACC_EMPTY(b), ((tc >> 1) & 1) ^ 1);  // epilogue drained this accumulator
      tc_fence_after();
      const uint32_t tacc = tmem + 256 * b;
      for (int kb = 0; kb < nk; ++kb, ++it) {
        const int s = it % C::STAGES;
        mbar_wait(FULL(s), (it / C::STAGES) & 1);
        tc_fence_after();
        const uint32_t aoff = s * C::STAGE_BYTES, boff = aoff + C::A_BYTES;
#pragma unroll
        for (int kk = 0; kk < C::BK / 16; ++kk)
          umma_ss_elect(tacc, desc0 + ((aoff + kk * 32) >> 4), desc0 + ((boff + kk * 32) >> 4), IDESC,
                        (kb > 0 || kk > 0));
        umma_commit_elect(EMPTY(s));
      }
      umma_commit_elect(ACC_FULL(b));
    }
  } else if (warp >= 4) {
    // ---------------------------------------------------------------- epilogue
    const int g = (warp - 4) >> 2, quad = warp & 3;
    const int row = quad * 32 + lane;
    const uint32_t lane_off = static_cast<uint32_t>(quad * 32) << 16;
    const uint32_t bar_id = 1 + g;  // named barrier per column half (128 threads)
    uint32_t tc = 0;
    for (int tile = blockIdx.x; tile < num_tiles; tile += gridDim.x, ++tc) {
      const int m0 = (tile / p.tiles_n) * C::BM, n0 = (tile % p.tiles_n) * C::BN;
      const int b = tc & 1;
      mbar_wait(ACC_FULL(b), (tc >> 1) & 1);
      tc_fence_after();
      if (row == 0) tma_store_wait_read0();  // this half's staging boxes are free again
      named_bar_sync(bar_id, 128);
      const uint32_t tacc = tmem + lane_off + 256 * b + 128 * g;
#pragma unroll 1
      for (int q = 0; q < 4; ++q) {
        uint32_t v[32];
        tmem_ld_32x32b_x32(tacc + 32 * q, v);
        tmem_wait_ld();
        reg_fence(v);
        const int col0 = 128 * g + 32 * q;  // column within the tile
        // bias for these 32 columns: four 16-byte loads (N % 8 == 0, so a group is all in or all out)
        float bv[32];
#pragma unroll
        for (int u = 0; u < 4; ++u) {
          const int n = n0 + col0 + 8 * u;
          uint4 raw = make_uint4(0u, 0u, 0u, 0u);
          if (p.bias && n < p.N) raw = __ldg(reinterpret_cast<const uint4*>(p.bias + n));
          const __half2* h2 = reinterpret_cast<const __half2*>(&raw);
#pragma unroll
          for (int e = 0; e < 4; ++e) {
            const float2 f2 = __half22float2(h2[e]);
            bv[8 * u + 2 * e] = f2.x;
            bv[8 * u + 2 * e + 1] = f2.y;
          }
        }
        float f[32];
#pragma unroll
        for (int k = 0; k < 32; ++k) f[k] = apply_act<ACT>(__uint_as_float(v[k]) + bv[k]);
        const uint32_t box = sbase + C::OFF_STG + (col0 / 64) * C::C_BOX + row * 128;
#pragma unroll
        for (int u = 0; u < 4; ++u) {
          const int unit = ((col0 % 64) / 8) + u;
          st_shared_v4(box + ((unit ^ (row & 7)) << 4), pack2<false>(f[8 * u + 0], f[8 * u + 1]),
                       pack2<false>(f[8 * u + 2], f[8 * u + 3]), pack2<false>(f[8 * u + 4], f[8 * u + 5]),
                       pack2<false>(f[8 * u + 6], f[8 * u + 7]));
        }
      }
      // accumulator b fully read: the MMA warp may start the tile after next into it
      tc_fence_before();
      mbar_arrive(ACC_EMPTY(b));
      fence_proxy_async_smem();
      named_bar_sync(bar_id, 128);
      if (row == 0) {
#pragma unroll
        for (int c = 2 * g; c < 2 * g + 2; ++c)
          if (n0 + c * 64 < p.N) tma_store_3d(&p.tmC, sbase + C::OFF_STG + c * C::C_BOX, n0 + c * 64, m0, 0);
        tma_store_commit();
      }
    }
    if (row == 0) tma_store_wait0();
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
                                int act, int sms, cudaStream_t stream, char* err, size_t errlen) {
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
  prm.tiles_m = (M + GemmCfg::BM - 1) / GemmCfg::BM;
  prm.tiles_n = (N + GemmCfg::BN - 1) / GemmCfg::BN;
  void (*kern)(GemmParams) = act == 1 ? gemm_bias_act_kernel<1>
                            : act == 2 ? gemm_bias_act_kernel<2>
                            : act == 3 ? gemm_bias_act_kernel<3>
                                       : gemm_bias_act_kernel<0>;
  static bool attr_done[64][4];
  int dev = 0;
  cudaGetDevice(&dev);
  if (dev >= 64 || !attr_done[dev][act]) {
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, GemmCfg::SMEM_ALLOC);
    if (e != cudaSuccess) {
      snprintf(err, errlen, "cudaFuncSetAttribute(gemm): %s", cudaGetErrorString(e));
      return 4;
    }
    if (dev < 64) attr_done[dev][act] = true;
  }
  const long long tiles = static_cast<long long>(prm.tiles_m) * prm.tiles_n;
  dim3 grid(static_cast<unsigned>(tiles < sms ? tiles : sms), 1, 1);
  kern<<<grid, GemmCfg::THREADS, GemmCfg::SMEM_ALLOC, stream>>>(prm);
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) {
    snprintf(err, errlen, "gemm_bias_act_kernel launch: %s", cudaGetErrorString(e));
    return 4;
  }
  return 0;
}

}  // namespace b200
