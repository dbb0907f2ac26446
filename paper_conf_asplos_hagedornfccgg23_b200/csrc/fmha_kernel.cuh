// fmha_kernel.cuh — FMHA forward for sm_100a.
//
// The operation is the paper's fused multi-head attention (§6): two back-to-back
// GEMMs with a softmax between, per (batch, head).  This kernel is the B200-native design:
//
//   unit of work     one 128-row query tile of one (b, h)                        [SURVEY §8(a) a1]
//   warp roles       warp 0: TMA producer      (Q once, then K_j / V_j through a smem ring) [a2, a3]
//                    warp 1: MMA issuer        (one thread issues tcgen05.mma)              [a4, a8]
//                    warps 2-5: softmax group  (thread = query row; online softmax,
//                                               O correction, epilogue)                     [a5-a7, a9]
//   S = Q K^T        tcgen05.mma SS, M=128 N=128 K=D, fp32 accumulator in TMEM cols [0,128)
//   P                exp2 of the scaled, max-shifted scores, rounded to fp16/bf16 and written
//                    back into TMEM over S (cols [0,64)), so it never touches shared memory
//   O += P V         tcgen05.mma TS (A = P from TMEM, B = V from smem, MN-major), fp32 in TMEM
//                    cols [128, 128+D)
//   epilogue         O / l, RNE to fp16/bf16, 128-bit swizzled st.shared into the (dead) Q
//                    buffer, one TMA store per 64-column box (rows >= seq_q are clipped)
//
// Because tcgen05.ld hands each thread one full TMEM lane (= one query row), the row max and row
// sum are thread-local: no warp-shuffle reduction is needed.
//
// Ordering facts the pipeline relies on:
//   * tcgen05.mma ops issued by one thread execute in issue order, so QK_{j+1} may be issued into
//     the S columns right after PV_j (which reads P_j from the same columns).
//   * tcgen05.commit arrives once every earlier tcgen05 op of the issuing thread has completed.
#pragma once
#include "sm100.cuh"

namespace b200 {

enum : int { MASK_NONE = 0, MASK_KEY_PADDING = 1, MASK_CAUSAL = 2 };

struct FmhaParams {
  CUtensorMap tmQ;  // 3-D {D, seq_q, B*H}, box {64, 128, 1}, SWIZZLE_128B
  CUtensorMap tmK;  // 3-D {D, seq_kv, B*H}
  CUtensorMap tmV;
  CUtensorMap tmO;  // same geometry as Q
  const int32_t* kv_len;
  int seq_q;
  int seq_kv;
  int heads;
  int num_q_tiles;
  int num_units;  // B*H
  int mask_kind;
  float scale_log2;  // scale * log2(e)
};

template <int D>
struct FmhaCfg {
  static constexpr int BM = 128;                  // query rows per tile (UMMA M)
  static constexpr int BN = 128;                  // keys per KV tile (UMMA N of QK^T, K of PV)
  static constexpr int CHUNK = 128 * 64 * 2;      // one SW128 TMA box: 128 rows x 64 halves
  static constexpr int TILE = BM * D * 2;         // bytes of a Q / K / V / O tile
  static constexpr int NSLOT = (D == 64) ? 4 : 2; // K,V ring slots (K_j and V_j alternate)
  static constexpr int OFF_Q = 0;
  static constexpr int OFF_KV = TILE;
  static constexpr int OFF_BAR = OFF_KV + NSLOT * TILE;
  static constexpr int NUM_BARS = 4 + 2 * NSLOT;
  static constexpr int OFF_TMEMPTR = OFF_BAR + NUM_BARS * 8;
  static constexpr int SMEM_BYTES = OFF_TMEMPTR + 16;
  static constexpr int SMEM_ALLOC = SMEM_BYTES + 1024;  // slack for manual 1024-B alignment
  static constexpr int TMEM_COLS = 256;
  static constexpr int TMEM_S = 0;    // S (fp32, 128 cols); P (packed 16-bit, cols 0..63) aliases it
  static constexpr int TMEM_O = 128;  // O accumulator (fp32, D cols)
  static constexpr int THREADS = 192;
};

template <int D, bool BF16>
__global__ void __launch_bounds__(192, 2) fmha_fwd_kernel(const __grid_constant__ FmhaParams p) {
  using C = FmhaCfg<D>;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  const uint32_t sbase = smem_u32(smem);
  const uint32_t sQ = sbase + C::OFF_Q;
  const uint32_t sKV = sbase + C::OFF_KV;
  const uint32_t bar = sbase + C::OFF_BAR;
  const uint32_t BAR_Q = bar, BAR_S = bar + 8, BAR_P = bar + 16, BAR_O = bar + 24;
  auto BAR_FULL = [&](int s) { return bar + 32 + 8 * s; };
  auto BAR_EMPTY = [&](int s) { return bar + 32 + 8 * C::NSLOT + 8 * s; };
  uint32_t* tmem_holder = reinterpret_cast<uint32_t*>(smem + C::OFF_TMEMPTR);

  const int warp = warp_id();
  const int lane = lane_id();

  // ---- work unit.  Causal: longest (last) q-tiles first, across all heads.
  int qtile, bh;
  if (p.mask_kind == MASK_CAUSAL) {
    bh = blockIdx.x;
    qtile = p.num_q_tiles - 1 - static_cast<int>(blockIdx.y);
  } else {
    qtile = blockIdx.x;
    bh = blockIdx.y;
  }
  const int b = bh / p.heads;
  const int q0 = qtile * C::BM;
  int kv_valid = p.seq_kv;
  if (p.mask_kind == MASK_KEY_PADDING) kv_valid = min(max(__ldg(p.kv_len + b), 0), p.seq_kv);
  const int causal_off = p.seq_kv - p.seq_q;
  int kv_end = kv_valid;  // keys [kv_end, seq_kv) are invisible to every row of this tile
  if (p.mask_kind == MASK_CAUSAL) kv_end = min(kv_end, max(0, q0 + C::BM + causal_off));
  const int n_tiles = (kv_end + C::BN - 1) / C::BN;  // fully masked KV tiles are skipped (a5)

  // ---- one-time setup
  if (threadIdx.x == 0) {
    mbar_init(BAR_Q, 1);
    mbar_init(BAR_S, 1);
    mbar_init(BAR_P, 128);
    mbar_init(BAR_O, 1);
    for (int s = 0; s < C::NSLOT; ++s) {
      mbar_init(BAR_FULL(s), 1);
      mbar_init(BAR_EMPTY(s), 1);
    }
    fence_mbar_init();
  }
  if (warp == 0 && lane == 0) {
    tma_prefetch_desc(&p.tmQ);
    tma_prefetch_desc(&p.tmK);
    tma_prefetch_desc(&p.tmV);
    tma_prefetch_desc(&p.tmO);
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
    // ================================================================ TMA producer (a2, a3)
    if (lane == 0 && n_tiles > 0) {
      const uint64_t keep = policy_evict_last();   // K/V are re-read by the other q-tiles of (b,h)
      const uint64_t once = policy_evict_first();  // Q is read exactly once
      mbar_arrive_expect_tx(BAR_Q, C::TILE);
#pragma unroll
      for (int c = 0; c < D / 64; ++c) tma_load_3d_hint(sQ + c * C::CHUNK, &p.tmQ, BAR_Q, c * 64, q0, bh, once);
      for (int j = 0; j < n_tiles; ++j) {
#pragma unroll
        for (int w = 0; w < 2; ++w) {  // w = 0: K_j, w = 1: V_j
          const int t = 2 * j + w;
          const int slot = t % C::NSLOT;
          const uint32_t ph = (t / C::NSLOT) & 1;
          mbar_wait(BAR_EMPTY(slot), ph ^ 1);
          mbar_arrive_expect_tx(BAR_FULL(slot), C::TILE);
          const CUtensorMap* m = w ? &p.tmV : &p.tmK;
#pragma unroll
          for (int c = 0; c < D / 64; ++c)
            tma_load_3d_hint(sKV + slot * C::TILE + c * C::CHUNK, m, BAR_FULL(slot), c * 64, j * C::BN, bh, keep);
        }
      }
    }
  } else if (warp == 1) {
    // ================================================================ MMA issuer (a4, a8)
    if (lane == 0 && n_tiles > 0) {
      constexpr uint32_t IDESC_QK = idesc_f16(BF16, 128, 128, false, false);  // Q, K both K-major
      constexpr uint32_t IDESC_PV = idesc_f16(BF16, 128, D, false, true);     // P K-major, V MN-major
      const uint32_t tS = tmem + C::TMEM_S;
      const uint32_t tO = tmem + C::TMEM_O;
      mbar_wait(BAR_Q, 0);
      tc_fence_after();
      auto issue_qk = [&](int j) {
        const int t = 2 * j;
        const int slot = t % C::NSLOT;
        mbar_wait(BAR_FULL(slot), (t / C::NSLOT) & 1);
        tc_fence_after();
        const uint32_t sK = sKV + slot * C::TILE;
#pragma unroll
        for (int kk = 0; kk < D / 16; ++kk) {
          const uint32_t off = (kk / 4) * C::CHUNK + (kk % 4) * 32;
          umma_ss(tS, sdesc_sw128(sQ + off, 16, 1024), sdesc_sw128(sK + off, 16, 1024), IDESC_QK, kk > 0);
        }
        umma_commit(BAR_EMPTY(slot));  // K_j slot free once this QK completes
        umma_commit(BAR_S);            // S_j ready for the softmax group
      };
      issue_qk(0);
      for (int j = 0; j < n_tiles; ++j) {
        mbar_wait(BAR_P, j & 1);  // P_j written into TMEM, O rescaled
        tc_fence_after();
        const int t = 2 * j + 1;
        const int slot = t % C::NSLOT;
        mbar_wait(BAR_FULL(slot), (t / C::NSLOT) & 1);
        tc_fence_after();
        const uint32_t sV = sKV + slot * C::TILE;
#pragma unroll
        for (int kk = 0; kk < C::BN / 16; ++kk)
          umma_ts(tO, tS + kk * 8, sdesc_sw128(sV + kk * 2048, C::CHUNK, 1024), IDESC_PV, (j > 0 || kk > 0));
        umma_commit(BAR_EMPTY(slot));  // V_j slot free
        umma_commit(BAR_O);            // O holds sum_{<=j} P V
        if (j + 1 < n_tiles) issue_qk(j + 1);
      }
    }
  } else {
    // ================================================================ softmax group (a5, a6, a7, a9)
    const int quad = warp & 3;  // TMEM lane quadrant this warp may access
    const int row = quad * 32 + lane;
    const uint32_t lane_off = static_cast<uint32_t>(quad * 32) << 16;
    const uint32_t tS = tmem + lane_off + C::TMEM_S;
    const uint32_t tO = tmem + lane_off + C::TMEM_O;
    const int qi = q0 + row;
    int lim = kv_valid;  // keys j < lim are visible to this row
    if (p.mask_kind == MASK_CAUSAL) lim = min(lim, qi + causal_off + 1);
    const float c = p.scale_log2;
    float m = -INFINITY;  // running max of raw scores
    float l = 0.f;        // running sum of exp2(c*(s - m))

    for (int j = 0; j < n_tiles; ++j) {
      mbar_wait(BAR_S, j & 1);
      tc_fence_after();
      uint32_t s[128];
#pragma unroll
      for (int q = 0; q < 4; ++q) tmem_ld_32x32b_x32(tS + 32 * q, *reinterpret_cast<uint32_t(*)[32]>(&s[32 * q]));
      tmem_wait_ld();
      reg_fence(s);

      const int rem = lim - j * C::BN;  // visible keys of this row in this tile
      const bool masked = rem < C::BN;  // boundary tile for this row (a5)
      float mt0 = -INFINITY, mt1 = -INFINITY, mt2 = -INFINITY, mt3 = -INFINITY;
      if (masked) {
#pragma unroll
        for (int k = 0; k < 128; k += 4) {
          mt0 = fmaxf(mt0, k + 0 < rem ? __uint_as_float(s[k + 0]) : -INFINITY);
          mt1 = fmaxf(mt1, k + 1 < rem ? __uint_as_float(s[k + 1]) : -INFINITY);
          mt2 = fmaxf(mt2, k + 2 < rem ? __uint_as_float(s[k + 2]) : -INFINITY);
          mt3 = fmaxf(mt3, k + 3 < rem ? __uint_as_float(s[k + 3]) : -INFINITY);
        }
      } else {
#pragma unroll
        for (int k = 0; k < 128; k += 4) {
          mt0 = fmaxf(mt0, __uint_as_float(s[k + 0]));
          mt1 = fmaxf(mt1, __uint_as_float(s[k + 1]));
          mt2 = fmaxf(mt2, __uint_as_float(s[k + 2]));
          mt3 = fmaxf(mt3, __uint_as_float(s[k + 3]));
        }
      }
      const float m_new = fmaxf(m, fmaxf(fmaxf(mt0, mt1), fmaxf(mt2, mt3)));

      if (j > 0) {
        // O correction (a7): O <- alpha * O once PV_{j-1} has landed.
        mbar_wait(BAR_O, (j - 1) & 1);
        tc_fence_after();
        const float alpha = (m_new > m) ? ((m == -INFINITY) ? 0.f : ex2((m - m_new) * c)) : 1.f;
        if (__any_sync(0xffffffffu, alpha != 1.f)) {
#pragma unroll
          for (int q = 0; q < D / 32; ++q) {
            uint32_t o[32];
            tmem_ld_32x32b_x32(tO + 32 * q, o);
            tmem_wait_ld();
            reg_fence(o);
#pragma unroll
            for (int k = 0; k < 32; ++k) o[k] = __float_as_uint(__uint_as_float(o[k]) * alpha);
            tmem_st_32x32b_x32(tO + 32 * q, o);
          }
        }
        l *= alpha;
      }
      m = m_new;
      const float mc = (m == -INFINITY) ? 0.f : m * c;

      // P = exp2(c*s - c*m) (a6), rounded to the I/O type and stored over S in TMEM.
      float l0 = 0.f, l1 = 0.f;
#pragma unroll
      for (int h = 0; h < 2; ++h) {
        uint32_t pk[32];
#pragma unroll
        for (int t = 0; t < 32; ++t) {
          const int k = 64 * h + 2 * t;
          float e0 = ex2(fmaf(__uint_as_float(s[k]), c, -mc));
          float e1 = ex2(fmaf(__uint_as_float(s[k + 1]), c, -mc));
          if (masked) {
            e0 = (k < rem) ? e0 : 0.f;
            e1 = (k + 1 < rem) ? e1 : 0.f;
          }
          l0 += e0;
          l1 += e1;
          pk[t] = pack2<BF16>(e0, e1);
        }
        tmem_st_32x32b_x32(tS + 32 * h, pk);
      }
      l += l0 + l1;
      tmem_wait_st();
      tc_fence_before();
      mbar_arrive(BAR_P);
    }

    // ---------------------------------------------------------------- epilogue (a9)
    if (n_tiles > 0) {
      mbar_wait(BAR_O, (n_tiles - 1) & 1);
      tc_fence_after();
    }
    const float inv_l = (l > 0.f) ? 1.f / l : 0.f;  // fully masked row -> O = 0 (R4)
#pragma unroll
    for (int q = 0; q < D / 32; ++q) {
      uint32_t o[32];
      if (n_tiles > 0) {
        tmem_ld_32x32b_x32(tO + 32 * q, o);
        tmem_wait_ld();
        reg_fence(o);
      } else {
#pragma unroll
        for (int k = 0; k < 32; ++k) o[k] = 0u;
      }
      const int col0 = 32 * q;
      const uint32_t box = sQ + (col0 / 64) * C::CHUNK + row * 128;
#pragma unroll
      for (int u = 0; u < 4; ++u) {
        const int unit = ((col0 % 64) / 8) + u;  // 16-byte unit within the 128-byte row
        const uint32_t addr = box + ((unit ^ (row & 7)) << 4);  // SWIZZLE_128B placement
        st_shared_v4(addr,
                     pack2<BF16>(__uint_as_float(o[8 * u + 0]) * inv_l, __uint_as_float(o[8 * u + 1]) * inv_l),
                     pack2<BF16>(__uint_as_float(o[8 * u + 2]) * inv_l, __uint_as_float(o[8 * u + 3]) * inv_l),
                     pack2<BF16>(__uint_as_float(o[8 * u + 4]) * inv_l, __uint_as_float(o[8 * u + 5]) * inv_l),
                     pack2<BF16>(__uint_as_float(o[8 * u + 6]) * inv_l, __uint_as_float(o[8 * u + 7]) * inv_l));
      }
    }
    fence_proxy_async_smem();
    named_bar_sync(1, 128);
    if (row == 0) {
#pragma unroll
      for (int c2 = 0; c2 < D / 64; ++c2) tma_store_3d(&p.tmO, sQ + c2 * C::CHUNK, c2 * 64, q0, bh);
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

}  // namespace b200
