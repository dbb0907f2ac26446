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
#include <algorithm>

#include "sm100.cuh"

namespace b200 {

struct GemmParams {
  // Operand pair q (q = 1 only for the dual GEMM, K2 > 0): C = act(A_0 W_0^T + A_1 W_1^T + bias).
  CUtensorMap tmA[2];     // A_q {K_q, M, 1} box {64, 128, 1}
  CUtensorMap tmW[2][3];  // W_q {K_q, N, 1} boxes of {64, 256 | 128 | 64, 1} rows: single-CTA tile,
                          // single-CTA half tile / CTA-pair W half, CTA-pair half tile
  CUtensorMap tmC;  // {N, M, 1} box {64, 128, 1}
  CUtensorMap tmC32;  // {N, M, 1} box {64, 32, 1}: one epilogue warp's 32 rows (CTA-pair kernel)
  const __half* bias;
  int M, N, K, K2;  // K2 = 0: a single GEMM
  int act;
  int tiles_m, tiles_n;
  // Work units: big tiles u < split_from are 128 x 256 (u / tiles_n, u % tiles_n); the last
  // (num_units - split_from) / 2 big tiles are split into two 128 x 128 half tiles each, so a last
  // wave that would hold r <= G/2 big tiles holds 2r half tiles instead and takes half as long.
  int split_from, num_units;
};

struct GemmUnit {
  int m0, n0, width;  // output rows m0.., columns n0..n0+width-1 (width 256 or 128)
};
__device__ __forceinline__ GemmUnit gemm_unit(const GemmParams& p, int u) {
  GemmUnit g;
  if (u < p.split_from) {
    g.m0 = (u / p.tiles_n) * 128;
    g.n0 = (u % p.tiles_n) * 256;
    g.width = 256;
  } else {
    const int h = u - p.split_from, b = p.split_from + (h >> 1);
    g.m0 = (b / p.tiles_n) * 128;
    g.n0 = (b % p.tiles_n) * 256 + (h & 1) * 128;
    g.width = 128;
  }
  return g;
}
// the same for the CTA pair's 256 x 256 tiles (half tiles 256 x 128)
__device__ __forceinline__ GemmUnit gemm_unit2(const GemmParams& p, int u) {
  GemmUnit g;
  if (u < p.split_from) {
    g.m0 = (u / p.tiles_n) * 256;
    g.n0 = (u % p.tiles_n) * 256;
    g.width = 256;
  } else {
    const int h = u - p.split_from, b = p.split_from + (h >> 1);
    g.m0 = (b / p.tiles_n) * 256;
    g.n0 = (b % p.tiles_n) * 256 + (h & 1) * 128;
    g.width = 128;
  }
  return g;
}

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

// GELU_erf(x) = x * Phi(x), Phi(x) = 0.5 * (1 + erf(x / sqrt 2)).  erf by Abramowitz & Stegun 7.1.26
// (|error| <= 1.5e-7): for z = |x| / sqrt 2, 1 - erf(z) = t (a1 + t (a2 + t (a3 + t (a4 + t a5)))) e^(-z^2),
// t = 1 / (1 + p z).  q = (1 - erf(z)) / 2 gives Phi = q for x < 0 (no cancellation) and 1 - q for
// x >= 0.  Branch-free: one MUFU.RCP, one MUFU.EX2 and ~12 FMA-pipe ops per element, against ~25
// instructions and a divergent branch for erff; the approximate rcp/ex2 add < 1e-6 relative, far
// below the fp16 output rounding (R15 tolerance).
__device__ __forceinline__ float gelu_erf_fast(float x) {
  const float z = fabsf(x) * 0.70710678118654752f;
  float t;
  asm("rcp.approx.ftz.f32 %0, %1;" : "=f"(t) : "f"(fmaf(0.3275911f, z, 1.f)));
  float poly = fmaf(t, 1.061405429f, -1.453152027f);
  poly = fmaf(t, poly, 1.421413741f);
  poly = fmaf(t, poly, -0.284496736f);
  poly = fmaf(t, poly, 0.254829592f);
  poly *= t;
  const float e = ex2(-1.4426950408889634f * z * z);
  const float q = 0.5f * poly * e;
  return x * (x < 0.f ? q : 1.f - q);
}

// The same GELU_erf on a pair with packed fp32x2 arithmetic (FFMA2 / FMUL2 / FADD2: two elements per
// FMA-pipe instruction, half the issue slots of the scalar form -- the GELU GEMM's epilogue was
// issue-bound).  The 0.5 of q is folded into the polynomial's coefficients (exact:
// powers of two).  Identical formula, so identical error bound.
__device__ __forceinline__ float2 gelu_erf_fast2(float2 x) {
  const float2 z = make_float2(fabsf(x.x) * 0.70710678118654752f, fabsf(x.y) * 0.70710678118654752f);
  const float2 d = ffma2(z, 0.3275911f, 1.f);
  float2 t;
  asm("rcp.approx.ftz.f32 %0, %1;" : "=f"(t.x) : "f"(d.x));
  asm("rcp.approx.ftz.f32 %0, %1;" : "=f"(t.y) : "f"(d.y));
  float2 poly = ffma2(t, make_float2(0.5f * 1.061405429f, 0.5f * 1.061405429f),
                      make_float2(0.5f * -1.453152027f, 0.5f * -1.453152027f));
  poly = ffma2(t, poly, make_float2(0.5f * 1.421413741f, 0.5f * 1.421413741f));
  poly = ffma2(t, poly, make_float2(0.5f * -0.284496736f, 0.5f * -0.284496736f));
  poly = ffma2(t, poly, make_float2(0.5f * 0.254829592f, 0.5f * 0.254829592f));
  poly = fmul2(poly, t);
  const float2 arg = fmul2(fmul2(z, z), make_float2(-1.4426950408889634f, -1.4426950408889634f));
  const float2 q = fmul2(poly, make_float2(ex2(arg.x), ex2(arg.y)));
  const float2 omq = fadd2(make_float2(1.f, 1.f), make_float2(-q.x, -q.y));
  return fmul2(x, make_float2(x.x < 0.f ? q.x : omq.x, x.y < 0.f ? q.y : omq.y));
}

// GELU_erf on a pair through Abramowitz & Stegun 7.1.28, erf(z) = 1 - (1 + a1 z + ... + a6 z^6)^-16
// (|err| <= 3e-7): one MUFU (the reciprocal) per element instead of two (reciprocal + exp2) in 7.1.26.
// Measured max |err| of the resulting GELU against math.erf on [-12, 12]: 7.9e-7.  GEMM_GELU_V2=1.
__device__ __forceinline__ float2 gelu_erf_fast2_v2(float2 x) {
  const float2 z = make_float2(fabsf(x.x) * 0.70710678118654752f, fabsf(x.y) * 0.70710678118654752f);
  float2 p = ffma2(z, make_float2(0.0000430638f, 0.0000430638f), make_float2(0.0002765672f, 0.0002765672f));
  p = ffma2(p, z, make_float2(0.0001520143f, 0.0001520143f));
  p = ffma2(p, z, make_float2(0.0092705272f, 0.0092705272f));
  p = ffma2(p, z, make_float2(0.0422820123f, 0.0422820123f));
  p = ffma2(p, z, make_float2(0.0705230784f, 0.0705230784f));
  p = ffma2(p, z, make_float2(1.f, 1.f));
  float2 t;
  asm("rcp.approx.ftz.f32 %0, %1;" : "=f"(t.x) : "f"(p.x));
  asm("rcp.approx.ftz.f32 %0, %1;" : "=f"(t.y) : "f"(p.y));
  t = fmul2(t, t);   // ^2
  t = fmul2(t, t);   // ^4
  t = fmul2(t, t);   // ^8
  const float2 h = fmul2(t, fmul2(t, make_float2(0.5f, 0.5f)));  // 0.5 (1 - erf(z)) = 0.5 t^16
  const float2 omh = fadd2(make_float2(1.f, 1.f), make_float2(-h.x, -h.y));
  return fmul2(x, make_float2(x.x < 0.f ? h.x : omh.x, x.y < 0.f ? h.y : omh.y));
}

template <int ACT>
__device__ __forceinline__ float apply_act(float x) {
  if (ACT == 1) return fmaxf(x, 0.f);
  if (ACT == 2) return gelu_erf_fast(x);
  if (ACT == 3) return 0.5f * x * (1.f + tanhf(0.7978845608028654f * (x + 0.044715f * x * x * x)));
  if (ACT == 4) return tanhf(x);
  return x;
}

// act on the 32 accumulator columns of a chunk: f = act(v + bias), packed pairs for GELU_erf
#ifndef GEMM_GELU_V2
#define GEMM_GELU_V2 0
#endif
#ifndef GEMM_GELU_PACKED
#define GEMM_GELU_PACKED 1
#endif
template <int ACT>
__device__ __forceinline__ void act_chunk(const uint32_t (&v)[32], const float (&bv)[32], float (&f)[32]) {
  if constexpr (ACT == 2 && GEMM_GELU_PACKED) {
#pragma unroll
    for (int k = 0; k < 32; k += 2) {
      const float2 xin = fadd2(make_float2(__uint_as_float(v[k]), __uint_as_float(v[k + 1])), make_float2(bv[k], bv[k + 1]));
      const float2 y = GEMM_GELU_V2 ? gelu_erf_fast2_v2(xin) : gelu_erf_fast2(xin);
      f[k] = y.x;
      f[k + 1] = y.y;
    }
  } else {
#pragma unroll
    for (int k = 0; k < 32; ++k) f[k] = apply_act<ACT>(__uint_as_float(v[k]) + bv[k]);
  }
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
  const int nk1 = (p.K + C::BK - 1) / C::BK;
  const int nk = nk1 + (p.K2 + C::BK - 1) / C::BK;
  const int num_tiles = p.num_units;

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
    tma_prefetch_desc(&p.tmA[0]);
    tma_prefetch_desc(&p.tmW[0][0]);
    tma_prefetch_desc(&p.tmW[0][1]);
    tma_prefetch_desc(&p.tmC);
  }
  if (warp == 1) {
    tmem_alloc(smem_u32(tmem_holder), C::TMEM_COLS);
    tmem_relinquish();
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  pdl_wait();  // global memory only from here on (PDL)
  pdl_trigger();
  const uint32_t tmem = *tmem_holder;

  if (warp == 0) {
    // ---------------------------------------------------------------- TMA producer
    uint32_t it = 0;
    const uint64_t keep = policy_evict_last();  // A rows and W are re-read by other tiles (all fit in L2)
    for (int tile = blockIdx.x; tile < num_tiles; tile += gridDim.x) {
      const GemmUnit g = gemm_unit(p, tile);
      const bool half = g.width == 128;
      for (int kb = 0; kb < nk; ++kb, ++it) {
        const int s = it % C::STAGES;
        mbar_wait(EMPTY(s), ((it / C::STAGES) & 1) ^ 1);
        mbar_arrive_expect_tx_elect(FULL(s), half ? C::A_BYTES + C::B_BYTES / 2 : C::STAGE_BYTES);
        const uint32_t sA = sbase + s * C::STAGE_BYTES;
        const int q = kb >= nk1, kq = (kb - (q ? nk1 : 0)) * C::BK;  // operand pair, its K offset
        tma_load_3d_hint_elect(sA, &p.tmA[q], FULL(s), kq, g.m0, 0, keep);
        tma_load_3d_hint_elect(sA + C::A_BYTES, &p.tmW[q][half ? 1 : 0], FULL(s), kq, g.n0, 0, keep);
      }
    }
  } else if (warp == 1) {
    // ---------------------------------------------------------------- MMA issuer
    constexpr uint32_t IDESC = idesc_f16(false, C::BM, C::BN, false, false);
    constexpr uint32_t IDESC_HALF = idesc_f16(false, C::BM, C::BN / 2, false, false);
    const uint64_t desc0 = sdesc_sw128(sbase, 16, 1024);
    uint32_t it = 0, tc = 0;
    for (int tile = blockIdx.x; tile < num_tiles; tile += gridDim.x, ++tc) {
      const int b = tc & 1;
      mbar_wait(ACC_EMPTY(b), ((tc >> 1) & 1) ^ 1);  // epilogue drained this accumulator
      tc_fence_after();
      const uint32_t tacc = tmem + 256 * b;
      const uint32_t idesc = tile < p.split_from ? IDESC : IDESC_HALF;
      for (int kb = 0; kb < nk; ++kb, ++it) {
        const int s = it % C::STAGES;
        mbar_wait(FULL(s), (it / C::STAGES) & 1);
        tc_fence_after();
        const uint32_t aoff = s * C::STAGE_BYTES, boff = aoff + C::A_BYTES;
#pragma unroll
        for (int kk = 0; kk < C::BK / 16; ++kk)
          umma_ss_elect(tacc, desc0 + ((aoff + kk * 32) >> 4), desc0 + ((boff + kk * 32) >> 4), idesc,
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
      const GemmUnit gu = gemm_unit(p, tile);
      const int m0 = gu.m0, n0 = gu.n0;
      const bool active = 128 * g < gu.width;  // half tiles: column group 1 has nothing to store
      const int b = tc & 1;
      mbar_wait(ACC_FULL(b), (tc >> 1) & 1);
      tc_fence_after();
      if (row == 0) tma_store_wait_read0();  // this half's staging boxes are free again
      named_bar_sync(bar_id, 128);
      const uint32_t tacc = tmem + lane_off + 256 * b + 128 * g;
      // The four 32-column chunks are software-pipelined: chunk q+1's TMEM load is in flight while
      // chunk q is computed, and the accumulator is released as soon as the last chunk is in
      // registers (before its bias/activation/store), so the MMA can start the tile after next.
      uint32_t va[32], vb[32];
      if (active) tmem_ld_32x32b_x32(tacc, va);
#pragma unroll
      for (int q = 0; q < 4; ++q) {
        if (!active) break;
        uint32_t(&v)[32] = (q & 1) ? vb : va;
        tmem_wait_ld();
        reg_fence(v);
        if (q + 1 < 4) {
          tmem_ld_32x32b_x32(tacc + 32 * (q + 1), (q & 1) ? va : vb);
        } else {  // accumulator b fully read: the MMA warp may start the tile after next into it
          tc_fence_before();
          mbar_arrive(ACC_EMPTY(b));
        }
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
        act_chunk<ACT>(v, bv, f);
        const uint32_t box = sbase + C::OFF_STG + (col0 / 64) * C::C_BOX + row * 128;
#pragma unroll
        for (int u = 0; u < 4; ++u) {
          const int unit = ((col0 % 64) / 8) + u;
          st_shared_v4(box + ((unit ^ (row & 7)) << 4), pack2<false>(f[8 * u + 0], f[8 * u + 1]),
                       pack2<false>(f[8 * u + 2], f[8 * u + 3]), pack2<false>(f[8 * u + 4], f[8 * u + 5]),
                       pack2<false>(f[8 * u + 6], f[8 * u + 7]));
        }
      }
      if (!active) {  // (nothing read: release the accumulator at once)
        tc_fence_before();
        mbar_arrive(ACC_EMPTY(b));
      }
      fence_proxy_async_smem();
      named_bar_sync(bar_id, 128);
      if (row == 0 && active) {
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

// ------------------------------------------------------------------------------------------------
// CTA-pair variant (cta_group::2): a cluster of two CTAs on one TPC computes a 256 x 256 output
// tile.  CTA r loads A rows m0 + 128 r .. (its half of M) and W rows n0 + 128 r .. (its half of N);
// the leader (r = 0) issues tcgen05.mma.cta_group::2 M=256 N=256 K=16, which reads both CTAs' smem
// and leaves rows 128 r .. of the accumulator in CTA r's TMEM.  Per SM and 64-deep K block that is
// 32 KB of operand traffic for 512 MMA cycles, against 48 KB for the single-CTA 128 x 256 tile: the
// L2 -> SMEM feed, not the tensor core, bounds the single-CTA kernel on the MLP shapes.
//   FULL[s]      leader only, count 1 (its arrive.expect_tx of both CTAs' bytes); both CTAs' TMA
//                loads complete_tx on it
//   EMPTY[s]     both CTAs, count 1: the leader's MMA commit is multicast to both
//   ACC_FULL[b]  both CTAs, count 1: multicast commit after a tile's last MMA
//   ACC_EMPTY[b] leader only, count 16: one arrival per epilogue warp of either CTA (remote for r = 1)
// GEMM2_PREFETCH_FIRST: the FMHA's first-item L2 prefetch applied to the CTA-pair GEMM (first tile's first
// STAGES K blocks of A and W before griddepcontrol.wait): measured level to -0.5% on the MLP block, BERT
// layer and LSTM cell (profiles/r02c_ab_gemm_prefetch_first.txt; ~100 us launches have little fill to
// hide), so off
#ifndef GEMM2_PREFETCH_FIRST
#define GEMM2_PREFETCH_FIRST 0
#endif
// GEMM2_WARP_STORES: each epilogue warp writes its 32 rows to the staging buffer and stores them with
// its own TMA store (box 64 x 32), so the four warps of a column group never wait for one another
// (the group's two named barriers per tile were the top stall of the GELU GEMM, 2.3 warps per issue
// cycle).  Measured in one session: MLP block 1250 -> 1277 TFLOP/s, BERT layer +1.2%, LSTM cell +0.5%
// (profiles/r02b_ab_gemm_warp_stores.txt).
#ifndef GEMM2_WARP_STORES
#define GEMM2_WARP_STORES 1
#endif
struct Gemm2Cfg {
  static constexpr int BM = 128, BN = 128, BK = 64;  // per CTA: A 128 x 64, W 128 x 64 per stage
#ifndef GEMM2_STAGES
#define GEMM2_STAGES 5
#endif
  static constexpr int STAGES = GEMM2_STAGES;
  static constexpr int A_BYTES = BM * BK * 2;  // 16 KB
  static constexpr int B_BYTES = BN * BK * 2;  // 16 KB
  static constexpr int STAGE_BYTES = A_BYTES + B_BYTES;
  static constexpr int C_BOX = 128 * 64 * 2;
  static constexpr int OFF_STG = STAGES * STAGE_BYTES;
  static constexpr int OFF_BAR = OFF_STG + 4 * C_BOX;
  static constexpr int NUM_BARS = 2 * STAGES + 4;
  static constexpr int OFF_TMEMPTR = OFF_BAR + NUM_BARS * 8;
  static constexpr int SMEM_ALLOC = OFF_TMEMPTR + 16;
  static constexpr int THREADS = 384;
  static_assert(SMEM_ALLOC <= 232448, "shared memory budget");
};

template <int ACT>
__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(384, 1) gemm_bias_act_2sm_kernel(const __grid_constant__ GemmParams p) {
  using C = Gemm2Cfg;
  extern __shared__ __align__(1024) uint8_t smem[];
  const uint32_t sbase = smem_u32(smem);
  const uint32_t bar = sbase + C::OFF_BAR;
  auto FULL = [&](int s) { return bar + 8 * s; };
  auto EMPTY = [&](int s) { return bar + 8 * (C::STAGES + s); };
  auto ACC_FULL = [&](int b) { return bar + 8 * (2 * C::STAGES + b); };
  auto ACC_EMPTY = [&](int b) { return bar + 8 * (2 * C::STAGES + 2 + b); };
  uint32_t* tmem_holder = reinterpret_cast<uint32_t*>(smem + C::OFF_TMEMPTR);
  const int warp = warp_id(), lane = lane_id();
  const uint32_t rank = cluster_ctarank();
  const int nk1 = (p.K + C::BK - 1) / C::BK;
  const int nk = nk1 + (p.K2 + C::BK - 1) / C::BK;
  const int num_tiles = p.num_units;                  // 256 x 256 tiles
  const int cid = blockIdx.x >> 1, ncl = gridDim.x >> 1;

  if (threadIdx.x == 0) {
    if (sbase & 1023u) __trap();
    for (int s = 0; s < C::STAGES; ++s) {
      mbar_init(FULL(s), 1);
      mbar_init(EMPTY(s), 1);
    }
    for (int b = 0; b < 2; ++b) {
      mbar_init(ACC_FULL(b), 1);
      mbar_init(ACC_EMPTY(b), 16);
    }
    fence_mbar_init();
  }
  if (warp == 0 && lane == 0) {
    tma_prefetch_desc(&p.tmA[0]);
    tma_prefetch_desc(&p.tmW[0][1]);
    tma_prefetch_desc(&p.tmC);
  }
  if (warp == 1) tmem_alloc_2sm(smem_u32(tmem_holder), 512);
  // GEMM2_PREFETCH_FIRST: this CTA's first tile's first STAGES K blocks of A and W into L2 while the previous
  // kernel drains (a prefetch writes nothing, so it is safe before griddepcontrol.wait; as the FMHA)
  if (GEMM2_PREFETCH_FIRST && warp == 0 && lane == 0 && cid < num_tiles) {
    const GemmUnit gu = gemm_unit2(p, cid);
    const bool half = gu.width == 128;
    for (int kb = 0; kb < min(nk1, C::STAGES); ++kb) {
      tma_prefetch_l2_3d(&p.tmA[0], kb * C::BK, gu.m0 + 128 * static_cast<int>(rank), 0);
      tma_prefetch_l2_3d(&p.tmW[0][half ? 2 : 1], kb * C::BK, gu.n0 + (half ? 64 : 128) * static_cast<int>(rank), 0);
    }
  }
  tc_fence_before();
  cluster_sync_all();  // both CTAs' barriers initialised and TMEM allocated before any signal crosses
  tc_fence_after();
  pdl_wait();  // global memory only from here on (PDL)
  pdl_trigger();
  const uint32_t tmem = *tmem_holder;
  if (warp == 1) tmem_relinquish_2sm();

  if (warp == 0) {
    // ---------------------------------------------------------------- TMA producer (both CTAs)
    uint32_t it = 0;
    const uint64_t keep = policy_evict_last();
    for (int tile = cid; tile < num_tiles; tile += ncl) {
      const GemmUnit gu = gemm_unit2(p, tile);
      const bool half = gu.width == 128;  // N = 128 tile: 64 W rows per CTA
      for (int kb = 0; kb < nk; ++kb, ++it) {
        const int s = it % C::STAGES;
        mbar_wait(EMPTY(s), ((it / C::STAGES) & 1) ^ 1);
        if (rank == 0) mbar_arrive_expect_tx_elect(FULL(s), 2 * (half ? C::A_BYTES + C::B_BYTES / 2 : C::STAGE_BYTES));
        const uint32_t sA = sbase + s * C::STAGE_BYTES;
        const uint32_t full_leader = mapa_shared(FULL(s), 0);
        const int q = kb >= nk1, kq = (kb - (q ? nk1 : 0)) * C::BK;  // operand pair, its K offset
        tma_load_3d_2sm_elect(sA, &p.tmA[q], full_leader, kq, gu.m0 + 128 * rank, 0, keep);
        tma_load_3d_2sm_elect(sA + C::A_BYTES, &p.tmW[q][half ? 2 : 1], full_leader, kq,
                              gu.n0 + (half ? 64 : 128) * rank, 0, keep);
      }
    }
  } else if (warp == 1) {
    // ---------------------------------------------------------------- MMA issuer (leader only)
    if (rank == 0) {
      constexpr uint32_t IDESC = idesc_f16(false, 256, 256, false, false);
      constexpr uint32_t IDESC_HALF = idesc_f16(false, 256, 128, false, false);
      const uint64_t desc0 = sdesc_sw128(sbase, 16, 1024);
      uint32_t it = 0, tc = 0;
      for (int tile = cid; tile < num_tiles; tile += ncl, ++tc) {
        const int b = tc & 1;
        mbar_wait(ACC_EMPTY(b), ((tc >> 1) & 1) ^ 1);  // both CTAs' epilogues drained this accumulator
        tc_fence_after();
        const uint32_t tacc = tmem + 256 * b;
        const uint32_t idesc = tile < p.split_from ? IDESC : IDESC_HALF;
        for (int kb = 0; kb < nk; ++kb, ++it) {
          const int s = it % C::STAGES;
          mbar_wait(FULL(s), (it / C::STAGES) & 1);
          tc_fence_after();
          const uint32_t aoff = s * C::STAGE_BYTES, boff = aoff + C::A_BYTES;
#pragma unroll
          for (int kk = 0; kk < C::BK / 16; ++kk)
            umma_ss_2sm_elect(tacc, desc0 + ((aoff + kk * 32) >> 4), desc0 + ((boff + kk * 32) >> 4), idesc,
                              (kb > 0 || kk > 0));
          umma_commit_2sm_mc_elect(EMPTY(s));
        }
        umma_commit_2sm_mc_elect(ACC_FULL(b));
      }
    }
  } else if (warp >= 4) {
    // ---------------------------------------------------------------- epilogue (both CTAs)
    const int g = (warp - 4) >> 2, quad = warp & 3;
    const int row = quad * 32 + lane;
    const uint32_t lane_off = static_cast<uint32_t>(quad * 32) << 16;
    const uint32_t bar_id = 1 + g;
    uint32_t tc = 0;
    for (int tile = cid; tile < num_tiles; tile += ncl, ++tc) {
      const GemmUnit gu = gemm_unit2(p, tile);
      const int m0 = gu.m0 + 128 * static_cast<int>(rank), n0 = gu.n0;
      const bool active = 128 * g < gu.width;  // half tiles: column group 1 has nothing to store
      const int b = tc & 1;
      mbar_wait(ACC_FULL(b), (tc >> 1) & 1);
      tc_fence_after();
      if constexpr (GEMM2_WARP_STORES) {  // this warp's previous stores have read its staging rows
        if (lane == 0) tma_store_wait_read0();
        __syncwarp();
      } else {
        if (row == 0) tma_store_wait_read0();
        named_bar_sync(bar_id, 128);
      }
      const uint32_t tacc = tmem + lane_off + 256 * b + 128 * g;
      // software-pipelined chunks and early accumulator release, as in gemm_bias_act_kernel
      uint32_t va[32], vb[32];
      if (active) tmem_ld_32x32b_x32(tacc, va);
#pragma unroll
      for (int q = 0; q < 4; ++q) {
        if (!active) break;
        uint32_t(&v)[32] = (q & 1) ? vb : va;
        tmem_wait_ld();
        reg_fence(v);
        if (q + 1 < 4) {
          tmem_ld_32x32b_x32(tacc + 32 * (q + 1), (q & 1) ? va : vb);
        } else {  // this warp's accumulator reads are done: one arrival per warp on the leader's ACC_EMPTY
          tc_fence_before();
          __syncwarp();
          if (lane == 0) mbar_arrive_cluster(mapa_shared(ACC_EMPTY(b), 0));
        }
        const int col0 = 128 * g + 32 * q;
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
        act_chunk<ACT>(v, bv, f);
        const uint32_t box = sbase + C::OFF_STG + (col0 / 64) * C::C_BOX + row * 128;
#pragma unroll
        for (int u = 0; u < 4; ++u) {
          const int unit = ((col0 % 64) / 8) + u;
          st_shared_v4(box + ((unit ^ (row & 7)) << 4), pack2<false>(f[8 * u + 0], f[8 * u + 1]),
                       pack2<false>(f[8 * u + 2], f[8 * u + 3]), pack2<false>(f[8 * u + 4], f[8 * u + 5]),
                       pack2<false>(f[8 * u + 6], f[8 * u + 7]));
        }
      }
      if (!active) {  // (nothing read: release at once)
        tc_fence_before();
        __syncwarp();
        if (lane == 0) mbar_arrive_cluster(mapa_shared(ACC_EMPTY(b), 0));
      }
      fence_proxy_async_smem();
      if constexpr (GEMM2_WARP_STORES) {  // each warp stores its own 32 rows: no barrier across the group
        __syncwarp();
        if (lane == 0 && active) {
#pragma unroll
          for (int c = 2 * g; c < 2 * g + 2; ++c)
            if (n0 + c * 64 < p.N && m0 + 32 * quad < p.M)
              tma_store_3d(&p.tmC32, sbase + C::OFF_STG + c * C::C_BOX + quad * 32 * 128, n0 + c * 64, m0 + 32 * quad, 0);
          tma_store_commit();
        }
      } else {
        named_bar_sync(bar_id, 128);
        if (row == 0 && active) {
#pragma unroll
          for (int c = 2 * g; c < 2 * g + 2; ++c)
            if (n0 + c * 64 < p.N && m0 < p.M)
              tma_store_3d(&p.tmC, sbase + C::OFF_STG + c * C::C_BOX, n0 + c * 64, m0, 0);
          tma_store_commit();
        }
      }
    }
    if (GEMM2_WARP_STORES ? lane == 0 : row == 0) tma_store_wait0();
  }
  tc_fence_before();
  cluster_sync_all();  // the peer's last MMA-side signals and TMEM reads are done before dealloc
  if (warp == 1) {
    tc_fence_after();
    tmem_dealloc_2sm(tmem, 512);
  }
}

// Host launcher (defined here so the ABI file stays thin).
int make_map_2d_rows(CUtensorMap* m, const void* base, uint64_t cols, uint64_t rows, uint32_t box_rows,
                     char* err, size_t errlen);

// C = act(A W^T [+ A2 W2^T] + bias); A2 / W2 are used when K2 > 0 (the dual GEMM).
inline int launch_gemm_bias_act(const void* A, const void* W, const void* A2, const void* W2, const void* bias,
                                void* Cm, int M, int N, int K, int K2, int act, int sms, cudaStream_t stream,
                                char* err, size_t errlen) {
  GemmParams prm;
  memset(&prm, 0, sizeof(prm));
  int st;
  for (int q = 0; q < (K2 > 0 ? 2 : 1); ++q) {
    const void* a = q ? A2 : A;
    const void* w = q ? W2 : W;
    const int kq = q ? K2 : K;
    if ((st = make_map_2d_rows(&prm.tmA[q], a, kq, M, GemmCfg::BM, err, errlen)) != 0) return st;
    for (int v = 0; v < 3; ++v)
      if ((st = make_map_2d_rows(&prm.tmW[q][v], w, kq, N, 256 >> v, err, errlen)) != 0) return st;
  }
  if ((st = make_map_2d_rows(&prm.tmC, Cm, N, M, GemmCfg::BM, err, errlen)) != 0) return st;
  if ((st = make_map_2d_rows(&prm.tmC32, Cm, N, M, 32, err, errlen)) != 0) return st;
  prm.bias = static_cast<const __half*>(bias);
  prm.M = M;
  prm.N = N;
  prm.K = K;
  prm.K2 = K2 > 0 ? K2 : 0;
  prm.act = act;
  prm.tiles_m = (M + GemmCfg::BM - 1) / GemmCfg::BM;
  prm.tiles_n = (N + GemmCfg::BN - 1) / GemmCfg::BN;
  // CTA-pair kernel for problems with at least one 256 x 256 tile per pair of SMs
  const long long pair_tiles = static_cast<long long>((M + 255) / 256) * ((N + 255) / 256);
  bool two_sm = pair_tiles >= sms / 2 && sms >= 2;
#ifdef GEMM_FORCE_1SM
  two_sm = false;
#endif
  if (two_sm) {
    prm.tiles_m = (M + 255) / 256;
    prm.tiles_n = (N + 255) / 256;
    const long long ncl = std::min<long long>(pair_tiles, sms / 2);
    const long long r2 = pair_tiles > ncl ? pair_tiles % ncl : 0;  // tiles in the last, partial wave
    const long long split2 = (r2 > 0 && 2 * r2 <= ncl) ? r2 : 0;
    prm.split_from = static_cast<int>(pair_tiles - split2);
    prm.num_units = static_cast<int>(pair_tiles + split2);
    void (*k2)(GemmParams) = act == 1 ? gemm_bias_act_2sm_kernel<1>
                            : act == 2 ? gemm_bias_act_2sm_kernel<2>
                            : act == 3 ? gemm_bias_act_2sm_kernel<3>
                            : act == 4 ? gemm_bias_act_2sm_kernel<4>
                                       : gemm_bias_act_2sm_kernel<0>;
    if (cudaError_t e = ensure_smem_attr(reinterpret_cast<const void*>(k2), Gemm2Cfg::SMEM_ALLOC); e != cudaSuccess) {
      snprintf(err, errlen, "cudaFuncSetAttribute(gemm2sm): %s", cudaGetErrorString(e));
      return 4;
    }
    const long long clusters = std::min<long long>(pair_tiles, sms / 2);
    cudaError_t e = launch_pdl(true, k2, dim3(static_cast<unsigned>(2 * clusters)), dim3(Gemm2Cfg::THREADS),
                               Gemm2Cfg::SMEM_ALLOC, stream, prm);
    if (e != cudaSuccess) {
      snprintf(err, errlen, "gemm_bias_act_2sm_kernel launch: %s", cudaGetErrorString(e));
      return 4;
    }
    return 0;
  }
  void (*kern)(GemmParams) = act == 1 ? gemm_bias_act_kernel<1>
                            : act == 2 ? gemm_bias_act_kernel<2>
                            : act == 3 ? gemm_bias_act_kernel<3>
                            : act == 4 ? gemm_bias_act_kernel<4>
                                       : gemm_bias_act_kernel<0>;
  if (cudaError_t e = ensure_smem_attr(reinterpret_cast<const void*>(kern), GemmCfg::SMEM_ALLOC); e != cudaSuccess) {
    snprintf(err, errlen, "cudaFuncSetAttribute(gemm): %s", cudaGetErrorString(e));
    return 4;
  }
  const long long tiles = static_cast<long long>(prm.tiles_m) * prm.tiles_n;
  const long long r = tiles > sms ? tiles % sms : 0;  // big tiles in the last, partial wave
  const long long split = (r > 0 && 2 * r <= sms) ? r : 0;
  if (tiles + split > 2147483647LL) return 2;
  prm.split_from = static_cast<int>(tiles - split);
  prm.num_units = static_cast<int>(tiles + split);
  dim3 grid(static_cast<unsigned>(tiles < sms ? tiles : sms), 1, 1);
  cudaError_t e = launch_pdl(true, kern, grid, dim3(GemmCfg::THREADS), GemmCfg::SMEM_ALLOC, stream, prm);
  if (e != cudaSuccess) {
    snprintf(err, errlen, "gemm_bias_act_kernel launch: %s", cudaGetErrorString(e));
    return 4;
  }
  return 0;
}

}  // namespace b200
