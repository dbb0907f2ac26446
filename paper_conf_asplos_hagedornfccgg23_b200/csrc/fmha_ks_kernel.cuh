// fmha_ks_kernel.cuh — FMHA forward for sm_100a at head_dim 64: "key-split" streams.
//
// The operation is the paper's fused multi-head attention (§6): per (batch, head)
// O = softmax(scale Q K^T + mask) V, two back-to-back GEMMs with the softmax between them.
//
// Why a second D = 64 kernel (round-1 measurements): with one softmax warp per
// 128-row Q tile per SM sub-partition (SMSP), a KV step of the two-tile kernel (fmha_kernel.cuh) is
// bound by each warp's serial chain -- S_FULL wait, 128-column TMEM load, row max, exponentials,
// P store -- at ~3.4k cycles per step against 1024 tensor-core cycles, with the issue slots 55%
// busy and no pipe saturated.  More independent chains per SMSP is the lever.  TMEM (512 columns)
// does not hold S + O for more than two 128-key tiles, so this kernel splits every 128-key KV tile
// between two independent STREAMS per Q tile instead:
//
//   work item      two 128-row Q tiles (t = 0, 1) sharing every K/V tile load (as the two-tile
//                  kernel: same item decode, schedules and ring protocol)                    [a1]
//   stream (t, h)  query tile t against keys 64h .. 64h+63 of every 128-key KV tile, with its own
//                  running max, row sum and O accumulator: four independent online softmaxes per
//                  item, merged once per item (the split-KV identity, exact up to rounding)   [a6, a7]
//   warps 0-15     softmax: warp w serves stream w >> 2, TMEM lane quarter w & 3 (one thread per
//                  query row, 64 key columns per step, row statistics thread-local); each SMSP
//                  hosts four independent chains.  After an item's last step the two warps of a
//                  (tile, lane quarter) merge their streams (exchanging (max, sum) through shared
//                  memory) and each writes 32 of the 64 output columns                         [a5, a6, a9]
//   warp 16 / 17   MMA issuer of tile 0 / 1: S_th = Q_t K_j[64h..]^T (SS, M128 N64 K64), then
//                  O_th += P_th V_j[64h..] (TS, P from TMEM)                                  [a4, a8]
//   warp 18        TMA producer: Q per item (double-buffered), K_j / V_j ring                 [a2, a3]
//   warp 19        varlen schedule builder (sched mode), otherwise idle
//
//   TMEM (512 columns): stream s = 2t + h owns columns [128 s, 128 s + 128):
//       S_s  [128 s, +64)   fp32 scores of the step; P_s (16-bit pairs) overwrites its first 32
//       O_s  [128 s + 64, +64)
//   QK_{s,j+1} is issued after PV_{s,j} by the same thread (tcgen05.mma ops of one thread execute in
//   issue order), so the P columns are consumed before the next S overwrites them, and S_FULL_{s,j+1}
//   (a commit: all earlier MMAs of the thread complete) also tells the softmax that PV_{s,j} has
//   landed in O_s (the lazy rescale may touch O_s then).
//
// Merge at the end of an item (per query row, mc_h = scale log2(e) m_h of stream h, m_h its
// reference max, l_h its row sum): M = max(mc_0, mc_1), w_h = 2^(mc_h - M),
//     O = (w_0 O_0 + w_1 O_1) / (w_0 l_0 + w_1 l_1),   rows with no visible key -> 0 (R4).
#pragma once
#include "fmha_kernel.cuh"

namespace b200 {

struct FmhaKsCfg {
  static constexpr int D = 64;
  static constexpr int TILE = 128 * 64 * 2;  // one Q / K / V tile: 128 rows x 64 16-bit elements, SW128
#ifndef FMHA_KS_NS
#define FMHA_KS_NS 6
#endif
  static constexpr int NS = FMHA_KS_NS;      // K/V ring slots (K_j and V_j alternate)
  static constexpr int QS = 2;               // Q stages per tile (the next item's Q loads early)
  static constexpr int STG = 32 * 128;       // O staging per (tile, lane quarter): 32 rows x 128 B, SW128
  static constexpr int OFF_Q = 0;            // Q[stage][tile]
  static constexpr int OFF_RING = 2 * QS * TILE;
  static constexpr int OFF_STG = OFF_RING + NS * TILE;     // [tile][quarter]
  static constexpr int OFF_STAT = OFF_STG + 8 * STG;       // float2 (mc, l) [tile][h][row]
  static constexpr int OFF_BAR = OFF_STAT + 2 * 2 * 128 * 8;
  enum : int {
    B_S_FULL = 0,    // [stream]   count 1 (commit)
    B_P_FULL = 4,    // [stream]   count 128 (the stream's softmax threads)
    B_O_FULL = 8,    // [tile]     count 1 (commit after the tile's last PV of an item)
    B_O_EMPTY = 10,  // [tile]     count 256 (both streams' softmax threads read O)
    B_Q_FULL = 12,   // [stage][tile]
    B_Q_EMPTY = 16,  // [stage][tile]
    B_KV = 20        // KV_FULL[NS], KV_EMPTY[NS] (count 2: both MMA warps)
  };
  static constexpr int NUM_BARS = B_KV + 2 * NS;
  static constexpr int OFF_TMEMPTR = OFF_BAR + NUM_BARS * 8;
  static constexpr int OFF_SCHED = (OFF_TMEMPTR + 16 + 15) / 16 * 16;
  static constexpr int SMEM_ALLOC = OFF_SCHED + 4 * (3 * (SCHED_MAX_LEVELS + 2) + SCHED_MAX_SEQS);
  static constexpr int THREADS = 640;
  static constexpr int W_MMA = 16, W_TMA = 18, W_SCHED = 19;
  // registers after setmaxnreg (whole warpgroups): 16 x 32 x 104 + 4 x 32 x 64 = 61440 = 640 x 96,
  // the launch allocation at __launch_bounds__(640, 1)
#ifndef FMHA_KS_REG_SOFTMAX
#define FMHA_KS_REG_SOFTMAX 104
#endif
  static constexpr int REG_SOFTMAX = FMHA_KS_REG_SOFTMAX, REG_MISC = 64;
  static_assert(16 * 32 * REG_SOFTMAX + 4 * 32 * REG_MISC <= THREADS * 96, "register pool");
  static_assert(SMEM_ALLOC <= 232448, "shared memory budget");
  // exp2 of element pairs q (32 per row and step) with (q % 8) < POLY_CNT on the FMA pipe
#ifndef FMHA_KS_POLY_CNT
#define FMHA_KS_POLY_CNT 2
#endif
  static constexpr int POLY_CNT = FMHA_KS_POLY_CNT;
};

template <bool BF16, int MODE>
__global__ void __launch_bounds__(640, 1) fmha_fwd_ks_sm100(const __grid_constant__ FmhaParams p) {
  using C = FmhaKsCfg;
  constexpr int D = 64;
  constexpr bool PAIRX = MODE == MODE_PAIRX, VL = MODE == MODE_VARLEN || MODE == MODE_VARLEN_SCHED,
                 SCHED = MODE == MODE_VARLEN_SCHED;
  static_assert(MODE == MODE_DENSE || MODE == MODE_PAIRX || MODE == MODE_VARLEN || MODE == MODE_VARLEN_SCHED,
                "key-split kernel modes");
  extern __shared__ __align__(1024) uint8_t smem[];
  const uint32_t sbase = smem_u32(smem);
  const uint32_t bar = sbase + C::OFF_BAR;
  auto BAR = [&](int slot) { return bar + 8 * slot; };
  auto Q_FULL = [&](int t, int q) { return BAR(C::B_Q_FULL + 2 * q + t); };
  auto Q_EMPTY = [&](int t, int q) { return BAR(C::B_Q_EMPTY + 2 * q + t); };
  auto KV_FULL = [&](int s) { return BAR(C::B_KV + s); };
  auto KV_EMPTY = [&](int s) { return BAR(C::B_KV + C::NS + s); };
  uint32_t* tmem_holder = reinterpret_cast<uint32_t*>(smem + C::OFF_TMEMPTR);
  const int warp = warp_id();
  const int lane = lane_id();

  if (threadIdx.x == 0) {
    if (sbase & 1023u) __trap();
    for (int s = 0; s < 4; ++s) {
      mbar_init(BAR(C::B_S_FULL + s), 1);
      mbar_init(BAR(C::B_P_FULL + s), 128);
    }
    for (int t = 0; t < 2; ++t) {
      mbar_init(BAR(C::B_O_FULL + t), 1);
      mbar_init(BAR(C::B_O_EMPTY + t), 256);
      for (int q = 0; q < 2; ++q) {
        mbar_init(Q_FULL(t, q), 1);
        mbar_init(Q_EMPTY(t, q), 1);
      }
    }
    for (int s = 0; s < C::NS; ++s) {
      mbar_init(KV_FULL(s), 1);
      mbar_init(KV_EMPTY(s), 2);
    }
    fence_mbar_init();
  }
  if (warp == C::W_TMA && lane == 0) {
    tma_prefetch_desc(&p.tmQ);
    tma_prefetch_desc(&p.tmK);
    tma_prefetch_desc(&p.tmV);
    tma_prefetch_desc(&p.tmO32);
  }
  if (warp == C::W_MMA) {
    tmem_alloc(smem_u32(tmem_holder), 512);
    tmem_relinquish();
  }
  pdl_wait();
  pdl_trigger();
  const SchedTable* sched = reinterpret_cast<const SchedTable*>(smem + C::OFF_SCHED);
  if (SCHED && warp == C::W_SCHED) build_sched(p, reinterpret_cast<SchedTable*>(smem + C::OFF_SCHED), lane);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = *tmem_holder;

  if (warp >= C::W_MMA) {
    asm volatile("setmaxnreg.dec.sync.aligned.u32 %0;" ::"n"(C::REG_MISC));
    if (warp == C::W_TMA) {
      // ============================================================ TMA producer (a2, a3)
      const uint64_t keep = policy_evict_last();
      const uint64_t once = policy_evict_first();
      uint32_t kv = 0, qc0 = 0, qc1 = 0;
      auto load_kv = [&](const WorkItem& w, int t, int j) {
#pragma unroll
        for (int m = 0; m < 2; ++m, ++kv) {  // m = 0: K_j, m = 1: V_j
          const int s = kv % C::NS;
          mbar_wait_at(KV_EMPTY(s), ((kv / C::NS) & 1) ^ 1, 1, kv, j);
          mbar_arrive_expect_tx_elect(KV_FULL(s), C::TILE);
          tma_load_3d_hint_elect(sbase + C::OFF_RING + s * C::TILE, m ? &p.tmV : &p.tmK, KV_FULL(s), 0,
                                 w.c1(VL, t, j * 128), w.c2(VL, t, j * 128), keep);
        }
      };
      for (int kk = 0, idx; (idx = item_at<SCHED>(p, sched, kk)) >= 0; ++kk) {
        const WorkItem w = get_item<PAIRX, VL, false, SCHED>(p, sched, idx);
        const int N = max(w.n0, w.n1);
#pragma unroll
        for (int t = 0; t < 2; ++t) {
          if (w.n(t) == 0) continue;
          uint32_t& qc = t ? qc1 : qc0;
          const int qs = qc % C::QS;
          mbar_wait_at(Q_EMPTY(t, qs), ((qc / C::QS) & 1) ^ 1, 2, qc, t);
          mbar_arrive_expect_tx_elect(Q_FULL(t, qs), C::TILE);
          tma_load_3d_hint_elect(sbase + C::OFF_Q + (2 * qs + t) * C::TILE, &p.tmQ, Q_FULL(t, qs), 0,
                                 w.c1(VL, t, w.row0(t)), w.c2(VL, t, w.row0(t)), once);
          ++qc;
        }
        for (int j = 0; j < N; ++j) {
          if (w.shared) {
            load_kv(w, 0, j);
          } else {
            if (j < w.n0) load_kv(w, 0, j);
            if (j < w.n1) load_kv(w, 1, j);
          }
        }
      }
    } else if (warp == C::W_MMA || warp == C::W_MMA + 1) {
      // ============================================================ MMA issuer of tile t (a4, a8)
      const int t = warp - C::W_MMA;
      constexpr uint32_t IDESC_QK = idesc_f16(BF16, 128, 64, false, false);  // Q, K: K-major
      constexpr uint32_t IDESC_PV = idesc_f16(BF16, 128, 64, false, true);   // P: TMEM, V: MN-major
      const uint64_t desc0 = sdesc_sw128(sbase, 16, 1024);
      const uint64_t vdesc0 = sdesc_sw128(sbase, 128 * 128, 1024);
      const uint32_t tS0 = tmem + 256 * t, tS1 = tS0 + 128;  // streams (t, 0), (t, 1); O at +64
      uint32_t qc = 0, oc = 0, pc0 = 0, pc1 = 0;
      auto ring_wait = [&](uint32_t k) {
        mbar_wait_at(KV_FULL(k % C::NS), (k / C::NS) & 1, 3, k, 0);
        tc_fence_after();
        return sbase + C::OFF_RING + (k % C::NS) * C::TILE;
      };
      auto release = [&](uint32_t k) {
        ring_wait(k);
        umma_commit_elect(KV_EMPTY(k % C::NS));
      };
      // the step whose PVs are still to be issued (PV_{s,j} goes out right before QK_{s,j+1})
      struct Pend {
        uint32_t vidx;
        bool valid, first, last;
      } pend = {0, false, false, false};
      auto pv = [&](int h) {
        const uint32_t sV = ring_wait(pend.vidx);
        if (h == 0 && pend.first) {  // the item's first PV overwrites O_t: the epilogue has read it
          mbar_wait_at(BAR(C::B_O_EMPTY + t), (oc & 1) ^ 1, 7, oc, t);
          ++oc;
        }
        uint32_t& pc = h ? pc1 : pc0;
        mbar_wait_at(BAR(C::B_P_FULL + 2 * t + h), pc & 1, 6, pc, h);
        ++pc;
        tc_fence_after();
        const uint32_t tS = h ? tS1 : tS0;
#pragma unroll
        for (int kk = 0; kk < 4; ++kk)  // keys 64h + 16kk .. of V_j (MN-major rows of 128 B)
          umma_ts_elect(tS + 64, tS + kk * 8, vdesc0 + ((sV - sbase + 8192 * h + 2048 * kk) >> 4), IDESC_PV,
                        (!pend.first || kk > 0));
      };
      auto qk = [&](int h, uint32_t sK, int qs) {
        const uint32_t qoff = C::OFF_Q + (2 * qs + t) * C::TILE;
        const uint32_t koff = sK - sbase + 8192 * h;  // K rows 64h .. 64h+63
#pragma unroll
        for (int kk = 0; kk < 4; ++kk)
          umma_ss_elect(h ? tS1 : tS0, desc0 + ((qoff + 32 * kk) >> 4), desc0 + ((koff + 32 * kk) >> 4), IDESC_QK,
                        kk > 0);
        umma_commit_elect(BAR(C::B_S_FULL + 2 * t + h));
      };
      int qs = 0;
      auto step = [&](uint32_t kidx, int j, int n) {
        const uint32_t sK = ring_wait(kidx);
        if (j == 0) {
          qs = qc % C::QS;
          mbar_wait_at(Q_FULL(t, qs), (qc / C::QS) & 1, 4, qc, t);
          ++qc;
        }
        if (pend.valid) pv(0);
        qk(0, sK, qs);
        if (pend.valid) {
          pv(1);
          if (pend.last) umma_commit_elect(BAR(C::B_O_FULL + t));
          umma_commit_elect(KV_EMPTY(pend.vidx % C::NS));
        }
        qk(1, sK, qs);
        if (j + 1 == n) umma_commit_elect(Q_EMPTY(t, qs));
        umma_commit_elect(KV_EMPTY(kidx % C::NS));
        pend = {kidx + 1, true, j == 0, j + 1 == n};
      };
      uint32_t ring = 0;  // ring index of the current item's first entry
      for (int kk = 0, idx; (idx = item_at<SCHED>(p, sched, kk)) >= 0; ++kk) {
        const WorkItem w = get_item<PAIRX, VL, false, SCHED>(p, sched, idx);
        const int N = max(w.n0, w.n1), n = w.n(t);
        for (int j = 0; j < N; ++j) {  // this step's ring entries in ring order
          if (w.shared) {
            if (j < n) {
              step(ring + 2 * j, j, n);
            } else {
              release(ring + 2 * j);
              release(ring + 2 * j + 1);
            }
          } else {
#pragma unroll
            for (int u = 0; u < 2; ++u) {
              if (j >= w.n(u)) continue;
              const uint32_t k = ring + w.k_index(u, j);
              if (u == t) {
                step(k, j, n);
              } else {
                release(k);
                release(k + 1);
              }
            }
          }
        }
        ring += w.entries();
      }
      if (pend.valid) {
        pv(0);
        pv(1);
        umma_commit_elect(BAR(C::B_O_FULL + t));
        umma_commit_elect(KV_EMPTY(pend.vidx % C::NS));
      }
    }
  } else {
    asm volatile("setmaxnreg.inc.sync.aligned.u32 %0;" ::"n"(C::REG_SOFTMAX));
    // ============================================================== softmax + epilogue (a5-a7, a9)
    const int s = warp >> 2, t = s >> 1, h = s & 1, quad = warp & 3;
    const int row = quad * 32 + lane;
    const uint32_t lane_off = static_cast<uint32_t>(quad * 32) << 16;
    const uint32_t tS = tmem + lane_off + 128 * s;  // S_s / P_s; O_s at +64
    const uint32_t S_FULL = BAR(C::B_S_FULL + s), P_FULL = BAR(C::B_P_FULL + s);
    const uint32_t pair_bar = 1 + 4 * t + quad;  // named barrier of the two warps of (t, quad)
    float2* stat = reinterpret_cast<float2*>(smem + C::OFF_STAT);
    const uint32_t stg = sbase + C::OFF_STG + (4 * t + quad) * C::STG;
    const float c = p.scale_log2;
    const int off = p.seq_kv - p.seq_q;
    uint32_t g = 0, ofc = 0;
    for (int kk = 0, idx; (idx = item_at<SCHED>(p, sched, kk)) >= 0; ++kk) {
      const WorkItem w = get_item<PAIRX, VL, false, SCHED>(p, sched, idx);
      if (!w.has(t)) continue;
      const int n = w.n(t);
      const int qi = w.row0(t) + row;
      int lim = w.kv(t);
      if (p.mask_kind == MASK_CAUSAL) lim = min(lim, qi + off + 1);
      if (qi >= w.len(t)) lim = 0;
      const int lim_w = __reduce_max_sync(0xffffffffu, lim);
      float m_ref = -INFINITY, l = 0.f;
      for (int j = 0; j < n; ++j) {
        const int key0 = j * 128 + 64 * h;
        mbar_wait_at(S_FULL, g & 1, 8, g, j);
        ++g;
        tc_fence_after();
        uint32_t sv[64];
        tmem_ld_32x32b_x32(tS, *reinterpret_cast<uint32_t(*)[32]>(&sv[0]));
        tmem_ld_32x32b_x32(tS + 32, *reinterpret_cast<uint32_t(*)[32]>(&sv[32]));
        tmem_wait_ld();
        reg_fence(sv);
        const int rem = lim - key0, rem_w = lim_w - key0;
        if (rem < 64) {
#pragma unroll
          for (int k = 0; k < 64; ++k)
            if (k >= rem) sv[k] = __float_as_uint(-INFINITY);
        }
        float mx0 = m_ref, mx1 = -INFINITY, mx2 = -INFINITY, mx3 = -INFINITY;
#pragma unroll
        for (int k = 0; k < 64; k += 8) {
          mx0 = fmax3(mx0, __uint_as_float(sv[k]), __uint_as_float(sv[k + 1]));
          mx1 = fmax3(mx1, __uint_as_float(sv[k + 2]), __uint_as_float(sv[k + 3]));
          mx2 = fmax3(mx2, __uint_as_float(sv[k + 4]), __uint_as_float(sv[k + 5]));
          mx3 = fmax3(mx3, __uint_as_float(sv[k + 6]), __uint_as_float(sv[k + 7]));
        }
        const float m_new = fmaxf(fmaxf(mx0, mx1), fmaxf(mx2, mx3));
        // lazy rescale (a7): keep the reference while the max grows by <= 8 in log2 units
        float alpha = 1.f;
        if (m_new > m_ref && (m_ref == -INFINITY || (m_new - m_ref) * c > 8.f)) {
          alpha = (m_ref == -INFINITY) ? 0.f : ex2((m_ref - m_new) * c);
          m_ref = m_new;
        }
        const float mc = (m_ref == -INFINITY) ? 0.f : m_ref * c;
        float2 acc0 = make_float2(0.f, 0.f), acc1 = make_float2(0.f, 0.f);
        auto chunk = [&](int hh) {  // keys 32 hh .. 32 hh + 31 of the stream's 64
          uint32_t pk[16];
#pragma unroll
          for (int u = 0; u < 16; u += 2) {
            const int k = 32 * hh + 2 * u;
            float2 x0 = ffma2(make_float2(__uint_as_float(sv[k]), __uint_as_float(sv[k + 1])), c, -mc);
            float2 x1 = ffma2(make_float2(__uint_as_float(sv[k + 2]), __uint_as_float(sv[k + 3])), c, -mc);
            if (((16 * hh + u) % 8) < C::POLY_CNT) {
              x0 = exp2_poly2(x0);
            } else {
              x0.x = ex2(x0.x);
              x0.y = ex2(x0.y);
            }
            if (((16 * hh + u + 1) % 8) < C::POLY_CNT) {
              x1 = exp2_poly2(x1);
            } else {
              x1.x = ex2(x1.x);
              x1.y = ex2(x1.y);
            }
            acc0 = fadd2(acc0, x0);
            acc1 = fadd2(acc1, x1);
            pk[u] = pack2<BF16>(x0.x, x0.y);
            pk[u + 1] = pack2<BF16>(x1.x, x1.y);
          }
          tmem_st_32x32b_x16(tS + 16 * hh, pk);
        };
        auto zero_chunk = [&](int hh) {
          uint32_t pk[16];
#pragma unroll
          for (int u = 0; u < 16; ++u) pk[u] = 0u;
          tmem_st_32x32b_x16(tS + 16 * hh, pk);
        };
        if (rem_w >= 64) {  // (the common case: no chunk of this warp is fully masked)
          chunk(0);
          chunk(1);
        } else {
          if (rem_w > 0) chunk(0); else zero_chunk(0);
          if (rem_w > 32) chunk(1); else zero_chunk(1);
        }
        // lazy rescale of this row's O_s (PV_{s,j-1} has landed: S_FULL_{s,j} commits after it)
        if (j > 0 && __any_sync(0xffffffffu, alpha != 1.f)) {
#pragma unroll 1
          for (int q = 0; q < 2; ++q) {
            uint32_t o[32];
            tmem_ld_32x32b_x32(tS + 64 + 32 * q, o);
            tmem_wait_ld();
            reg_fence(o);
#pragma unroll
            for (int k = 0; k < 32; ++k) o[k] = __float_as_uint(__uint_as_float(o[k]) * alpha);
            tmem_st_32x32b_x32(tS + 64 + 32 * q, o);
          }
        }
        tmem_wait_st();
        tc_fence_before();
        mbar_arrive(P_FULL);
        l = l * alpha + ((acc0.x + acc0.y) + (acc1.x + acc1.y));
      }
      // ------------------------------------------------------------ merge the two streams (a9)
      stat[(2 * t + h) * 128 + row] = make_float2(m_ref == -INFINITY ? -INFINITY : m_ref * c, l);
      if (h == 0 && lane == 0) tma_store_wait_read0();  // staging buffer free again
      named_bar_sync(pair_bar, 64);
      const float2 st0 = stat[(2 * t) * 128 + row], st1 = stat[(2 * t + 1) * 128 + row];
      const float M = fmaxf(st0.x, st1.x);
      const float w0 = (st0.x == -INFINITY) ? 0.f : ex2(st0.x - M);
      const float w1 = (st1.x == -INFINITY) ? 0.f : ex2(st1.x - M);
      const float L = w0 * st0.y + w1 * st1.y;
      const float inv = L > 0.f ? 1.f / L : 0.f;  // fully masked row -> 0 (R4)
      const float a0 = w0 * inv, a1 = w1 * inv;
      uint32_t o0[32], o1[32];
      if (n > 0) {
        mbar_wait_at(BAR(C::B_O_FULL + t), ofc & 1, 14, ofc, t);
        ++ofc;
        tc_fence_after();
        const uint32_t tOc = tmem + lane_off + 256 * t + 64 + 32 * h;  // columns 32h.. of O_(t,0)
        tmem_ld_32x32b_x32(tOc, o0);
        tmem_ld_32x32b_x32(tOc + 128, o1);                            // ... and of O_(t,1)
        tmem_wait_ld();
        reg_fence(o0);
        reg_fence(o1);
        tc_fence_before();
        mbar_arrive(BAR(C::B_O_EMPTY + t));
      } else {
#pragma unroll
        for (int k = 0; k < 32; ++k) o0[k] = o1[k] = 0u;
      }
      uint32_t pk[16];
#pragma unroll
      for (int u = 0; u < 16; ++u) {
        const float lo = __uint_as_float(o0[2 * u]) * a0 + __uint_as_float(o1[2 * u]) * a1;
        const float hi = __uint_as_float(o0[2 * u + 1]) * a0 + __uint_as_float(o1[2 * u + 1]) * a1;
        pk[u] = pack2<BF16>(lo, hi);
      }
      const bool rowwise = VL && w.row0(t) + 128 > w.len(t);
      if (!rowwise) {
#pragma unroll
        for (int u = 0; u < 4; ++u)
          st_shared_v4(stg + lane * 128 + (((4 * h + u) ^ (lane & 7)) << 4), pk[4 * u], pk[4 * u + 1], pk[4 * u + 2],
                       pk[4 * u + 3]);
        fence_proxy_async_smem();
      } else if (qi < w.len(t)) {  // varlen tile crossing the sequence's end: rows inside only
        const size_t tokn = static_cast<size_t>(w.tok(t) + qi);
        uint8_t* dst = p.o_ptr + 2 * (tokn * p.o_row_elems + (t ? w.head1 : w.head) * D + 32 * h);
#pragma unroll
        for (int u = 0; u < 4; ++u) st_global_v4(dst + 16 * u, pk[4 * u], pk[4 * u + 1], pk[4 * u + 2], pk[4 * u + 3]);
      }
      named_bar_sync(pair_bar, 64);
      if (!rowwise && h == 0 && lane == 0) {
        tma_store_3d(&p.tmO32, stg, 0, w.c1(VL, t, w.row0(t) + 32 * quad), w.c2(VL, t, w.row0(t) + 32 * quad));
        tma_store_commit();
      }
    }
    if (h == 0 && lane == 0) tma_store_wait0();
  }

  tc_fence_before();
  __syncthreads();
  if (warp == C::W_MMA) {
    tc_fence_after();
    tmem_dealloc(tmem, 512);
  }
}

}  // namespace b200
