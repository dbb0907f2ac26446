// fmha_kernel.cuh — FMHA forward for sm_100a (persistent, warp-specialised, two Q tiles ping-pong).
//
// The operation is the paper's fused multi-head attention (§6 "Fused Multi-Head
// Attention"): two back-to-back GEMMs with a softmax between them, per (batch, head).  The paper's
// kernel was written for Ampere (ldmatrix + mma.sync, specialised to BERT shapes, L489); this is
// the B200-native redesign:
//
//   work item     two consecutive 128-row query tiles (t = 0, 1) of one (b, h) sharing every
//                 K/V tile load; persistent CTAs (one per SM) walk a static list of items   [a1]
//   warps 0-3     softmax group for tile 0    (thread = query row; TMEM lane = row)        [a5, a6]
//   warps 4-7     softmax group for tile 1
//   warps 8-11    correction group: rescales O_t in TMEM when a row max moved by more than
//                 2^8 (lazy), then the epilogue O_t / l -> fp16/bf16 -> smem -> TMA store  [a7, a9]
//   warp 12       MMA issuer (one thread): S_t = Q_t K_j^T (SS), O_t += P_t V_j (TS)     [a4, a8]
//   warp 13       TMA producer: Q_t per item, K_j / V_j through an NS-slot smem ring       [a2, a3]
//   warps 14-15   idle (keep warpgroup 3 whole for setmaxnreg)
//
//   TMEM (512 columns x 128 lanes, fp32):  S_0 [0,128)  S_1 [128,256)  O_0 [256,256+D)  O_1 [..+D)
//   P_t (16-bit, two per column) overwrites the first 64 columns of S_t once S_t is in registers.
//
// Ordering facts relied on:
//   * tcgen05.mma ops of one thread execute in issue order: QK_{t,j+1} may overwrite S_t right
//     after PV_{t,j} (which reads P_t from the same columns) has been issued.
//   * tcgen05.commit arrives once all earlier tcgen05 ops of the issuing thread have completed.
//
// Row statistics are thread-local because tcgen05.ld 32x32b gives each thread one whole row
// (SURVEY D6): no warp-shuffle reductions.
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
  int num_items;  // num_units * ceil(num_q_tiles / 2)
  int mask_kind;
  float scale_log2;  // scale * log2(e)
};

template <int D>
struct FmhaCfg {
  static constexpr int BM = 128;                 // query rows per tile (UMMA M)
  static constexpr int BN = 128;                 // keys per KV tile
  static constexpr int CHUNK = 128 * 64 * 2;     // one SW128 TMA box: 128 rows x 64 16-bit elements
  static constexpr int TILE = BM * D * 2;        // bytes of one Q / K / V / O tile
  static constexpr int NS = (D == 64) ? 8 : 3;   // K/V ring slots (K_j, V_j alternate)
  static constexpr int OFF_Q = 0;                // Q_0, Q_1
  static constexpr int OFF_RING = 2 * TILE;
  static constexpr int NSTG = (D == 64) ? 2 : 1;        // O staging buffers (D=128 shares one)
  static constexpr int OFF_STG = OFF_RING + NS * TILE;
  static constexpr int OFF_ALPHA = OFF_STG + NSTG * TILE;  // float alpha[2][128]
  static constexpr int OFF_LSUM = OFF_ALPHA + 2 * 128 * 4;
  static constexpr int OFF_BAR = OFF_LSUM + 2 * 128 * 4;
  // barriers: 2x {q_full, q_empty, s_full, p_full, o_ready, pv_done, st_full, st_empty, l_full}
  //           + NS x {kv_full, kv_empty}
  static constexpr int NUM_BARS = 18 + 2 * NS;
  static constexpr int OFF_TMEMPTR = OFF_BAR + NUM_BARS * 8;
  static constexpr int SMEM_BYTES = OFF_TMEMPTR + 16;
  static constexpr int SMEM_ALLOC = SMEM_BYTES + 1024;  // slack for manual 1024-B alignment
  static constexpr int TMEM_COLS = 512;
  static constexpr int THREADS = 512;
  static_assert(SMEM_ALLOC <= 232448, "shared memory budget");
};

// One work item = q-tiles {2*pair, 2*pair+1} of unit bh.  Every role decodes items identically.
struct WorkItem {
  int bh;
  int q0;         // first query row of tile 0
  int kv_valid;   // keys >= kv_valid are masked for every row (key padding)
  int n[2];       // KV tiles visited by tile t (0 = tile absent or fully masked)
  bool has[2];    // tile t exists (rows < seq_q)
};

__device__ __forceinline__ WorkItem decode_item(const FmhaParams& p, int idx) {
  WorkItem w;
  const int pairs = (p.num_q_tiles + 1) >> 1;
  int pr;
  if (p.mask_kind == MASK_CAUSAL) {  // longest-first: the last query tiles see the most keys
    pr = pairs - 1 - idx / p.num_units;
    w.bh = idx % p.num_units;
  } else {  // both pairs of a (b,h) back to back so K/V are re-read from L2
    w.bh = idx / pairs;
    pr = idx % pairs;
  }
  w.q0 = pr * 256;
  w.kv_valid = p.seq_kv;
  if (p.mask_kind == MASK_KEY_PADDING) w.kv_valid = min(max(__ldg(p.kv_len + w.bh / p.heads), 0), p.seq_kv);
  const int off = p.seq_kv - p.seq_q;
#pragma unroll
  for (int t = 0; t < 2; ++t) {
    const int qt = 2 * pr + t;
    w.has[t] = qt < p.num_q_tiles;
    int kv_end = w.kv_valid;
    if (p.mask_kind == MASK_CAUSAL) kv_end = min(kv_end, max(0, qt * 128 + 128 + off));
    w.n[t] = w.has[t] ? (kv_end + 127) / 128 : 0;
  }
  return w;
}

template <int D, bool BF16>
__global__ void __launch_bounds__(512, 1) fmha_fwd_sm100(const __grid_constant__ FmhaParams p) {
  using C = FmhaCfg<D>;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  const uint32_t sbase = smem_u32(smem);
  const uint32_t bar = sbase + C::OFF_BAR;
  // barrier addresses (t = tile 0/1, s = ring slot)
  auto Q_FULL = [&](int t) { return bar + 8 * (0 + t); };
  auto Q_EMPTY = [&](int t) { return bar + 8 * (2 + t); };
  auto S_FULL = [&](int t) { return bar + 8 * (4 + t); };
  auto P_FULL = [&](int t) { return bar + 8 * (6 + t); };
  auto O_READY = [&](int t) { return bar + 8 * (8 + t); };
  auto PV_DONE = [&](int t) { return bar + 8 * (10 + t); };
  auto ST_FULL = [&](int t) { return bar + 8 * (12 + t); };
  auto ST_EMPTY = [&](int t) { return bar + 8 * (14 + t); };
  auto L_FULL = [&](int t) { return bar + 8 * (16 + t); };
  auto KV_FULL = [&](int s) { return bar + 8 * (18 + s); };
  auto KV_EMPTY = [&](int s) { return bar + 8 * (18 + C::NS + s); };
  float* s_alpha = reinterpret_cast<float*>(smem + C::OFF_ALPHA);
  float* s_lsum = reinterpret_cast<float*>(smem + C::OFF_LSUM);
  uint32_t* tmem_holder = reinterpret_cast<uint32_t*>(smem + C::OFF_TMEMPTR);

  const int warp = warp_id();
  const int lane = lane_id();

  if (threadIdx.x == 0) {
    for (int t = 0; t < 2; ++t) {
      mbar_init(Q_FULL(t), 1);
      mbar_init(Q_EMPTY(t), 1);
      mbar_init(S_FULL(t), 1);
      mbar_init(P_FULL(t), 128);
      mbar_init(O_READY(t), 128);
      mbar_init(PV_DONE(t), 1);
      mbar_init(ST_FULL(t), 128);
      mbar_init(ST_EMPTY(t), 128);
      mbar_init(L_FULL(t), 128);
    }
    for (int s = 0; s < C::NS; ++s) {
      mbar_init(KV_FULL(s), 1);
      mbar_init(KV_EMPTY(s), 1);
    }
    fence_mbar_init();
  }
  if (warp == 13 && lane == 0) {
    tma_prefetch_desc(&p.tmQ);
    tma_prefetch_desc(&p.tmK);
    tma_prefetch_desc(&p.tmV);
    tma_prefetch_desc(&p.tmO);
  }
  if (warp == 12) {
    tmem_alloc(smem_u32(tmem_holder), C::TMEM_COLS);
    tmem_relinquish();
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = *tmem_holder;
  const int first = blockIdx.x, stride = gridDim.x;

  if (warp >= 12) {
    asm volatile("setmaxnreg.dec.sync.aligned.u32 56;");
    if (warp == 13 && lane == 0) {
      // ============================================================ TMA producer (a2, a3)
      const uint64_t keep = policy_evict_last();   // K/V: re-read by the other q-tile pairs
      const uint64_t once = policy_evict_first();  // Q: read once
      uint32_t kv = 0, qc[2] = {0, 0};
      for (int idx = first; idx < p.num_items; idx += stride) {
        const WorkItem w = decode_item(p, idx);
        const int N = max(w.n[0], w.n[1]);
#pragma unroll
        for (int t = 0; t < 2; ++t) {
          if (w.n[t] == 0) continue;
          mbar_wait(Q_EMPTY(t), (qc[t] & 1) ^ 1);
          mbar_arrive_expect_tx(Q_FULL(t), C::TILE);
#pragma unroll
          for (int c = 0; c < D / 64; ++c)
            tma_load_3d_hint(sbase + C::OFF_Q + t * C::TILE + c * C::CHUNK, &p.tmQ, Q_FULL(t), c * 64,
                             w.q0 + 128 * t, w.bh, once);
          ++qc[t];
        }
        for (int j = 0; j < N; ++j) {
#pragma unroll
          for (int m = 0; m < 2; ++m, ++kv) {  // m = 0: K_j, m = 1: V_j
            const int s = kv % C::NS;
            mbar_wait(KV_EMPTY(s), ((kv / C::NS) & 1) ^ 1);
            mbar_arrive_expect_tx(KV_FULL(s), C::TILE);
            const CUtensorMap* map = m ? &p.tmV : &p.tmK;
#pragma unroll
            for (int c = 0; c < D / 64; ++c)
              tma_load_3d_hint(sbase + C::OFF_RING + s * C::TILE + c * C::CHUNK, map, KV_FULL(s), c * 64, j * 128,
                               w.bh, keep);
          }
        }
      }
    } else if (warp == 12 && lane == 0) {
      // ============================================================ MMA issuer (a4, a8)
      constexpr uint32_t IDESC_QK = idesc_f16(BF16, 128, 128, false, false);  // Q, K: K-major
      constexpr uint32_t IDESC_PV = idesc_f16(BF16, 128, D, false, true);     // P: K-major (TMEM), V: MN-major
      uint32_t kv = 0, qc[2] = {0, 0}, pc[2] = {0, 0}, oc[2] = {0, 0};
      auto ring_wait = [&](uint32_t k) {
        const int s = k % C::NS;
        mbar_wait(KV_FULL(s), (k / C::NS) & 1);
        tc_fence_after();
        return sbase + C::OFF_RING + s * C::TILE;
      };
      auto qk = [&](int t, uint32_t sK) {
        const uint32_t sQ = sbase + C::OFF_Q + t * C::TILE;
#pragma unroll
        for (int kk = 0; kk < D / 16; ++kk) {
          const uint32_t off = (kk / 4) * C::CHUNK + (kk % 4) * 32;
          umma_ss(tmem + 128 * t, sdesc_sw128(sQ + off, 16, 1024), sdesc_sw128(sK + off, 16, 1024), IDESC_QK,
                  kk > 0);
        }
        umma_commit(S_FULL(t));
      };
      for (int idx = first; idx < p.num_items; idx += stride) {
        const WorkItem w = decode_item(p, idx);
        const int N = max(w.n[0], w.n[1]);
        if (N == 0) continue;
#pragma unroll
        for (int t = 0; t < 2; ++t)
          if (w.n[t] > 0) {
            mbar_wait(Q_FULL(t), qc[t] & 1);
            ++qc[t];
          }
        tc_fence_after();
        uint32_t kslot = kv++;
        uint32_t sK = ring_wait(kslot);
#pragma unroll
        for (int t = 0; t < 2; ++t)
          if (w.n[t] > 0) {
            qk(t, sK);
            if (w.n[t] == 1) umma_commit(Q_EMPTY(t));
          }
        umma_commit(KV_EMPTY(kslot % C::NS));
        for (int j = 0; j < N; ++j) {
          const uint32_t vslot = kv++;
          const uint32_t sV = ring_wait(vslot);
          bool k_taken = false;
#pragma unroll
          for (int t = 0; t < 2; ++t) {
            if (j >= w.n[t]) continue;
            mbar_wait(P_FULL(t), pc[t] & 1);
            ++pc[t];
            mbar_wait(O_READY(t), oc[t] & 1);
            ++oc[t];
            tc_fence_after();
            const uint32_t tO = tmem + 256 + t * D;
            const uint32_t tP = tmem + 128 * t;
#pragma unroll
            for (int kk = 0; kk < 8; ++kk)
              umma_ts(tO, tP + kk * 8, sdesc_sw128(sV + kk * 2048, C::CHUNK, 1024), IDESC_PV, (j > 0 || kk > 0));
            umma_commit(PV_DONE(t));
            if (j + 1 < w.n[t]) {
              if (!k_taken) {
                kslot = kv++;
                sK = ring_wait(kslot);
                k_taken = true;
              }
              qk(t, sK);
              if (j + 2 == w.n[t]) umma_commit(Q_EMPTY(t));  // last QK of tile t: Q_t slot reusable
            }
          }
          umma_commit(KV_EMPTY(vslot % C::NS));
          if (k_taken) umma_commit(KV_EMPTY(kslot % C::NS));
          if (j + 1 < N && !k_taken) {
            // neither tile needs K_{j+1} (cannot happen: N = max n_t), keep the ring in step anyway
            kslot = kv++;
            ring_wait(kslot);
            umma_commit(KV_EMPTY(kslot % C::NS));
          }
        }
      }
    }
  } else if (warp < 8) {
    asm volatile("setmaxnreg.inc.sync.aligned.u32 176;");
    // ============================================================== softmax group t (a5, a6)
    // The two groups take turns for the exp2 phase (named barriers 2 + t): while one group
    // exponentiates, the other loads/reduces its next S and the tensor core runs the first
    // group's PV and next QK, so MUFU and tensor pipes overlap instead of running in lockstep.
    const int t = warp >> 2;
    const int quad = warp & 3;
    const int row = quad * 32 + lane;
    const uint32_t tS = tmem + (static_cast<uint32_t>(quad * 32) << 16) + 128 * t;
    const float c = p.scale_log2;
    const int off = p.seq_kv - p.seq_q;
    const uint32_t my_turn = 2 + t, other_turn = 3 - t;
    if (t == 1) named_bar_arrive(2, 256);  // tile 0 goes first
    uint32_t sc = 0, stc = 0;
    for (int idx = first; idx < p.num_items; idx += stride) {
      const WorkItem w = decode_item(p, idx);
      const int N = max(w.n[0], w.n[1]);
      const int n = w.n[t];
      const int qi = w.q0 + 128 * t + row;
      int lim = w.kv_valid;  // keys j < lim are visible to this row
      if (p.mask_kind == MASK_CAUSAL) lim = min(lim, qi + off + 1);
      float m_ref = -INFINITY;  // max used as the exp2 reference (lags the true max by < 2^8)
      float l = 0.f;
      for (int j = 0; j < N; ++j) {
        if (j >= n) {  // this tile has no KV tile j: keep the turn order
          named_bar_sync(my_turn, 256);
          named_bar_arrive(other_turn, 256);
          continue;
        }
        mbar_wait(S_FULL(t), sc & 1);
        ++sc;
        tc_fence_after();
        uint32_t s[128];
#pragma unroll
        for (int q = 0; q < 4; ++q) tmem_ld_32x32b_x32(tS + 32 * q, *reinterpret_cast<uint32_t(*)[32]>(&s[32 * q]));
        tmem_wait_ld();
        reg_fence(s);
        const int rem = lim - j * 128;
        if (rem < 128) {  // boundary tile for this row (a5)
#pragma unroll
          for (int k = 0; k < 128; ++k)
            if (k >= rem) s[k] = __float_as_uint(-INFINITY);
        }
        float mx0 = m_ref, mx1 = -INFINITY;
#pragma unroll
        for (int k = 0; k < 128; k += 4) {
          mx0 = fmax3(mx0, __uint_as_float(s[k]), __uint_as_float(s[k + 1]));
          mx1 = fmax3(mx1, __uint_as_float(s[k + 2]), __uint_as_float(s[k + 3]));
        }
        const float m_new = fmaxf(mx0, mx1);
        // Lazy rescale: keep the old reference while the max grows by < 8 in the log2 domain (the
        // p's then stay <= 2^8, exact in fp32 and in fp16/bf16 range); l and O share the reference.
        float alpha = 1.f;
        if (m_new > m_ref && (m_ref == -INFINITY || (m_new - m_ref) * c > 8.f)) {
          alpha = (m_ref == -INFINITY) ? 0.f : ex2((m_ref - m_new) * c);
          m_ref = m_new;
        }
        // hand alpha to the correction group (it rescales O_t before PV_{t,j})
        mbar_wait(ST_EMPTY(t), (stc & 1) ^ 1);
        s_alpha[t * 128 + row] = (j == 0) ? 1.f : alpha;
        mbar_arrive(ST_FULL(t));
        ++stc;

        const float mc = (m_ref == -INFINITY) ? 0.f : m_ref * c;
        float2 acc0 = make_float2(0.f, 0.f), acc1 = make_float2(0.f, 0.f);
        named_bar_sync(my_turn, 256);
#pragma unroll
        for (int h = 0; h < 2; ++h) {
          uint32_t pk[32];
#pragma unroll
          for (int u = 0; u < 32; u += 2) {
            const int k = 64 * h + 2 * u;
            float2 x0 = ffma2(make_float2(__uint_as_float(s[k]), __uint_as_float(s[k + 1])), c, -mc);
            float2 x1 = ffma2(make_float2(__uint_as_float(s[k + 2]), __uint_as_float(s[k + 3])), c, -mc);
            x0.x = ex2(x0.x);
            x0.y = ex2(x0.y);
            x1.x = ex2(x1.x);
            x1.y = ex2(x1.y);
            acc0 = fadd2(acc0, x0);
            acc1 = fadd2(acc1, x1);
            pk[u] = pack2<BF16>(x0.x, x0.y);
            pk[u + 1] = pack2<BF16>(x1.x, x1.y);
          }
          tmem_st_32x32b_x32(tS + 32 * h, pk);
        }
        named_bar_arrive(other_turn, 256);
        tmem_wait_st();
        tc_fence_before();
        mbar_arrive(P_FULL(t));
        l = l * alpha + ((acc0.x + acc0.y) + (acc1.x + acc1.y));
      }
      if (w.has[t]) {
        s_lsum[t * 128 + row] = l;
        mbar_arrive(L_FULL(t));
      }
    }
    if (t == 0) named_bar_sync(2, 256);  // consume tile 1's last hand-over
  } else {
    asm volatile("setmaxnreg.dec.sync.aligned.u32 96;");
    // ================================================================ correction group (a7, a9)
    const int quad = warp & 3;
    const int row = quad * 32 + lane;
    const uint32_t lane_off = static_cast<uint32_t>(quad * 32) << 16;
    uint32_t stc[2] = {0, 0}, pvc[2] = {0, 0}, lc[2] = {0, 0};
    for (int idx = first; idx < p.num_items; idx += stride) {
      const WorkItem w = decode_item(p, idx);
      const int N = max(w.n[0], w.n[1]);
      for (int j = 0; j < N; ++j) {
#pragma unroll
        for (int t = 0; t < 2; ++t) {
          if (j >= w.n[t]) continue;
          mbar_wait(ST_FULL(t), stc[t] & 1);
          const float alpha = s_alpha[t * 128 + row];
          mbar_arrive(ST_EMPTY(t));
          ++stc[t];
          if (j > 0) {
            mbar_wait(PV_DONE(t), pvc[t] & 1);  // PV_{t,j-1} has landed in O_t
            ++pvc[t];
            if (__any_sync(0xffffffffu, alpha != 1.f)) {
              tc_fence_after();
              const uint32_t tO = tmem + lane_off + 256 + t * D;
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
              tmem_wait_st();
            }
          }
          tc_fence_before();
          mbar_arrive(O_READY(t));
        }
      }
      // ------------------------------------------------------------ epilogue per tile (a9)
#pragma unroll 1
      for (int t = 0; t < 2; ++t) {
        if (!w.has[t]) continue;
        mbar_wait(L_FULL(t), lc[t] & 1);
        ++lc[t];
        const float l = s_lsum[t * 128 + row];
        if (w.n[t] > 0) {
          mbar_wait(PV_DONE(t), pvc[t] & 1);  // last PV of this tile
          ++pvc[t];
          tc_fence_after();
        }
        const float inv_l = (l > 0.f) ? 1.f / l : 0.f;  // fully masked row -> 0 (R4)
        const uint32_t stg = sbase + C::OFF_STG + (t % C::NSTG) * C::TILE;
        if (row == 0) tma_store_wait_read0();  // previous store out of this staging buffer done
        named_bar_sync(1, 128);
        const uint32_t tO = tmem + lane_off + 256 + t * D;
#pragma unroll
        for (int q = 0; q < D / 32; ++q) {
          uint32_t o[32];
          if (w.n[t] > 0) {
            tmem_ld_32x32b_x32(tO + 32 * q, o);
            tmem_wait_ld();
            reg_fence(o);
          } else {
#pragma unroll
            for (int k = 0; k < 32; ++k) o[k] = 0u;
          }
          const int col0 = 32 * q;
          const uint32_t box = stg + (col0 / 64) * C::CHUNK + row * 128;
#pragma unroll
          for (int u = 0; u < 4; ++u) {
            const int unit = ((col0 % 64) / 8) + u;
            st_shared_v4(box + ((unit ^ (row & 7)) << 4),
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
          for (int c2 = 0; c2 < D / 64; ++c2)
            tma_store_3d(&p.tmO, stg + c2 * C::CHUNK, c2 * 64, w.q0 + 128 * t, w.bh);
          tma_store_commit();
        }
      }
    }
    if (row == 0) tma_store_wait0();
  }

  tc_fence_before();
  __syncthreads();
  if (warp == 12) {
    tc_fence_after();
    tmem_dealloc(tmem, C::TMEM_COLS);
  }
}

}  // namespace b200
