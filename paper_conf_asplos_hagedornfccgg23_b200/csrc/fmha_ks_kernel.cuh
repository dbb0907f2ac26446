// fmha_ks_kernel.cuh — FMHA forward for sm_100a at head_dim 64: two softmax warps per row quarter.
//
// The operation is the paper's fused multi-head attention (§6): per (batch, head)
// O = softmax(scale Q K^T + mask) V, two back-to-back GEMMs with the softmax between them.
//
// Why a second D = 64 kernel (round-1 measurements): with one softmax warp per
// 128-row Q tile per SM sub-partition (SMSP), a KV step of the two-tile kernel (fmha_kernel.cuh) is
// bound by each warp's serial chain -- S_FULL wait, 128-column TMEM load, row max, 128 exponentials,
// P store -- at ~3.4k cycles per step against 1024 tensor-core cycles, with the issue slots 55%
// busy and no pipe saturated.  Here every 128-key S tile is split between TWO warps per row quarter
// (16 softmax warps, four per SMSP), each loading, masking and exponentiating 64 of the 128 columns:
//
//   work item      two 128-row Q tiles (t = 0, 1) sharing every K/V tile load (the two-tile kernel's
//                  item decode, schedules and K/V ring protocol)                              [a1]
//   warps 0-15     softmax: warp w serves tile t = w >> 3, key half h = (w >> 2) & 1 and TMEM lane
//                  quarter w & 3 (one thread per query row, 64 key columns per step).  The two
//                  tiles' warp pairs of a lane quarter take turns for the exponential phase (named
//                  barriers), so one tile's exponentials overlap the other tile's S load and max.
//                  The row max needs both halves: each warp writes its half-row max to shared memory
//                  before waiting for its turn, and the turn barrier -- which both warps of the pair
//                  pass together -- publishes it to the partner, so the exchange costs no extra
//                  synchronisation.  Both warps take the same lazy-rescale decision; each rescales its
//                  32 of O_t's 64 columns, keeps the row sum of its half and, at the item's end,
//                  stores 32 output columns (after exchanging the half sums)               [a5-a7, a9]
//   warp 16 / 17   MMA issuer of tile t: S_t = Q_t K_j^T (SS, M128 N128 K64) as soon as the softmax
//                  has read S_{t,j-1} (S_FREE), so QK of the next step runs under this step's
//                  softmax; O_t += P_t V_j (TS, M128 N64 K128, P from TMEM) after P_FULL        [a4, a8]
//   warp 18        TMA producer: Q per item (double-buffered), K_j / V_j ring                 [a2, a3]
//   warp 19        varlen schedule builder (sched mode), otherwise idle
//
//   TMEM (512 columns), tile t at [256 t, 256 t + 256): O_t [0, 64), then S and P of step g rotating
//   over three 64-column regions (FmhaKsCfg::col_s / col_p), so neither the next QK nor the P store
//   waits for the previous PV.
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
  static constexpr int STG = 32 * 64;        // O staging per softmax warp: 32 rows x 32 columns (64 B rows)
  static constexpr int OFF_Q = 0;            // Q[stage][tile]
  static constexpr int OFF_RING = 2 * QS * TILE;
  static constexpr int OFF_STG = OFF_RING + NS * TILE;     // [warp]
  static constexpr int OFF_XMAX = OFF_STG + 16 * STG;        // float half-row max [step parity][tile][h][row]
  static constexpr int OFF_LSUM = OFF_XMAX + 2 * 2 * 2 * 128 * 4;  // float half-row sum [item parity][tile][h][row]
  static constexpr int OFF_BAR = OFF_LSUM + 2 * 2 * 2 * 128 * 4;
  // TMEM columns inside tile t's 256: O_t [0, 64), then three 64-column regions A, B, C.  Step g (the
  // tile's step count) puts S_g into AB (g even) / BC (g odd) and P_g into A (g even) / C (g odd):
  // S_{g+1} never covers P_g (still to be read by PV_g), P_g never covers P_{g-1} (PV_{g-1} may still
  // be reading it), and S_{g+1} covering P_{g-1} is safe because PV_{g-1} is issued before QK_{g+1}
  // by the same thread.  So writing P_g waits for nothing but the pair's max exchange (P_g lies on
  // S_g, which both warps of the pair have loaded by then).
  // (ROT = 0: the fixed layout S [0, 128), P [128, 192), O [192, 256); P_g then waits for PV_{g-1})
#ifndef FMHA_KS_ROT
#define FMHA_KS_ROT 1
#endif
  static constexpr bool ROT = FMHA_KS_ROT;
  static constexpr int COL_O = ROT ? 0 : 192;
  __host__ __device__ static constexpr int col_s(uint32_t g) { return ROT ? ((g & 1) ? 128 : 64) : 0; }
  __host__ __device__ static constexpr int col_p(uint32_t g) { return ROT ? ((g & 1) ? 192 : 64) : 128; }
  enum : int {
    B_S_FULL = 0,    // [tile]          count 1 (commit)
    B_P_FULL = 2,    // [tile]          count 8 (one arrival per softmax warp of the tile)
    B_O_FULL = 4,    // [tile]          count 1 (commit after the tile's last PV of an item)
    B_O_EMPTY = 6,   // [tile]          count 8 (the tile's softmax warps read O)
    B_Q_FULL = 8,    // [stage][tile]
    B_Q_EMPTY = 12,  // [stage][tile]
    B_STAT = 16,     // [tile][quarter] count 64 (the two warps' threads of a (tile, lane quarter) wrote their l)
    B_S_FREE = 24,   // [tile]          count 8 (the tile's softmax warps read S)
    B_PV_DONE = 26,  // [tile]          count 1 (commit after each PV)
    B_KV = 28        // KV_FULL[NS], KV_EMPTY[NS] (count 2: both MMA warps)
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
  // TURNS: the two tiles' warp pairs of a lane quarter alternate their exponential phases (128-thread
  // named barriers 1 + 2 quarter + t, which also publish the half-row maxima); otherwise all four
  // softmax warps of an SMSP run freely and each pair exchanges its maxima through its own 64-thread
  // named barrier 1 + 4 t + quarter
#ifndef FMHA_KS_TURNS
#define FMHA_KS_TURNS 0
#endif
  static constexpr bool TURNS = FMHA_KS_TURNS;
  // (no turns) OFFSET: at the start of an item tile 1's pairs wait until tile 0's pairs have done their
  // first exponential phase (named barrier 9 + quarter), so the two tiles' phases start half a step apart
#ifndef FMHA_KS_OFFSET
#define FMHA_KS_OFFSET 0
#endif
  static constexpr bool OFFSET = FMHA_KS_OFFSET && !TURNS;
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
  TRACE_DECL

  if (threadIdx.x == 0) {
    if (sbase & 1023u) __trap();
    for (int t = 0; t < 2; ++t) {
      mbar_init(BAR(C::B_S_FULL + t), 1);
      mbar_init(BAR(C::B_P_FULL + t), 8);   // (one arrival per softmax warp)
      mbar_init(BAR(C::B_O_FULL + t), 1);
      mbar_init(BAR(C::B_O_EMPTY + t), 8);
      for (int q = 0; q < 2; ++q) {
        mbar_init(Q_FULL(t, q), 1);
        mbar_init(Q_EMPTY(t, q), 1);
      }
      for (int q = 0; q < 4; ++q) mbar_init(BAR(C::B_STAT + 4 * t + q), 64);
      mbar_init(BAR(C::B_S_FREE + t), 8);
      mbar_init(BAR(C::B_PV_DONE + t), 1);
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
          TRACE_EV(EV_TMA_KV, m * 64 + j);
          mbar_arrive_expect_tx_elect(KV_FULL(s), C::TILE);
          tma_load_4d_hint_elect(sbase + C::OFF_RING + s * C::TILE, m ? &p.tmV : &p.tmK, KV_FULL(s), 0,
                                 w.c1(VL, t, j * 128), w.c2(VL, t, j * 128), w.c3(VL, t), keep);
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
          tma_load_4d_hint_elect(sbase + C::OFF_Q + (2 * qs + t) * C::TILE, &p.tmQ, Q_FULL(t, qs), 0,
                                 w.c1(VL, t, w.row0(t)), w.c2(VL, t, w.row0(t)), w.c3(VL, t), once);
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
      // QK_{t,j+1} goes out as soon as the softmax has read S_{t,j} (S_FREE), so it runs under the
      // softmax of step j; PV_{t,j} follows once P_{t,j} is written (P_FULL).
      const int t = warp - C::W_MMA;
      constexpr uint32_t IDESC_QK = idesc_f16(BF16, 128, 128, false, false);  // Q, K: K-major
      constexpr uint32_t IDESC_PV = idesc_f16(BF16, 128, 64, false, true);    // P: TMEM, V: MN-major
      const uint64_t desc0 = sdesc_sw128(sbase, 16, 1024);
      const uint64_t vdesc0 = sdesc_sw128(sbase, 128 * 128, 1024);
      const uint32_t tT = tmem + 256 * t, tO = tT + C::COL_O;  // tile t's TMEM columns
      const uint32_t S_FULL = BAR(C::B_S_FULL + t), P_FULL = BAR(C::B_P_FULL + t);
      const uint32_t S_FREE = BAR(C::B_S_FREE + t), PV_DONE = BAR(C::B_PV_DONE + t);
      uint32_t qc = 0, oc = 0, pc = 0, qkc = 0;
      auto ring_wait = [&](uint32_t k) {
        mbar_wait_at(KV_FULL(k % C::NS), (k / C::NS) & 1, 3, k, 0);
        tc_fence_after();
        return sbase + C::OFF_RING + (k % C::NS) * C::TILE;
      };
      struct Pend {  // the step whose PV is still to be issued
        uint32_t vidx;
        bool valid, first, last;
      } pend = {0, false, false, false};
      auto pv = [&]() {
        const uint32_t sV = ring_wait(pend.vidx);
        if (pend.first) {  // the item's first PV overwrites O_t: the previous item's epilogue has read it
          mbar_wait_at(BAR(C::B_O_EMPTY + t), (oc & 1) ^ 1, 7, oc, t);
          ++oc;
        }
        TRACE_EV(EV_COR_ST, 0);
        mbar_wait_at(P_FULL, pc & 1, 6, pc, t);
        TRACE_EV(EV_MMA_P, 0);
        const uint32_t tP = tT + C::col_p(pc);
        ++pc;
        tc_fence_after();
#pragma unroll
        for (int kk = 0; kk < 8; ++kk)  // keys 16kk .. of V_j (MN-major rows of 128 B); P: 8 columns per 16 keys
          umma_ts_elect(tO, tP + kk * 8, vdesc0 + ((sV - sbase + 2048 * kk) >> 4), IDESC_PV, (!pend.first || kk > 0));
        umma_commit_elect(PV_DONE);
        if (pend.last) umma_commit_elect(BAR(C::B_O_FULL + t));
        umma_commit_elect(KV_EMPTY(pend.vidx % C::NS));
        TRACE_EV(EV_MMA_PV, 0);
      };
      // an entry this tile does not use: wait until it is filled, then release it (the pending PV goes
      // first -- its V slot may be the one the TMA needs to fill this entry)
      auto release = [&](uint32_t k) {
        if (pend.valid) {
          pv();
          pend.valid = false;
        }
        ring_wait(k);
        umma_commit_elect(KV_EMPTY(k % C::NS));
      };
      int qs = 0;
      auto step = [&](uint32_t kidx, int j, int n) {
        TRACE_EV(EV_COR_PV, j);
        // QK_{t,j+1} normally goes out before PV_{t,j}.  But when this K entry does not directly
        // follow the pending V entry in the ring (cross-unit pairs: the other tile's entries sit in
        // between), waiting for it first could deadlock: the TMA may need a slot that only this PV
        // frees (through the epilogue -> turn -> other tile chain).  Then the PV goes first.
        if (pend.valid && kidx != pend.vidx + 1) {
          pv();
          pend.valid = false;
        }
        const uint32_t sK = ring_wait(kidx);
        TRACE_EV(EV_COR_ORDY, j);
        if (j == 0) {
          qs = qc % C::QS;
          mbar_wait_at(Q_FULL(t, qs), (qc / C::QS) & 1, 4, qc, t);
          ++qc;
        }
        if (qkc > 0) {  // the softmax has read S_t of the previous step
          mbar_wait_at(S_FREE, (qkc - 1) & 1, 5, qkc, t);
          tc_fence_after();
        }
        const uint32_t tS = tT + C::col_s(qkc);
        ++qkc;
        const uint32_t qoff = C::OFF_Q + (2 * qs + t) * C::TILE;
#pragma unroll
        for (int kk = 0; kk < 4; ++kk)
          umma_ss_elect(tS, desc0 + ((qoff + 32 * kk) >> 4), desc0 + ((sK - sbase + 32 * kk) >> 4), IDESC_QK, kk > 0);
        umma_commit_elect(S_FULL);
        TRACE_EV(EV_MMA_QK, j);
        if (j + 1 == n) umma_commit_elect(Q_EMPTY(t, qs));
        umma_commit_elect(KV_EMPTY(kidx % C::NS));
        if (pend.valid) pv();
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
      if (pend.valid) pv();
    }
  } else {
    asm volatile("setmaxnreg.inc.sync.aligned.u32 %0;" ::"n"(C::REG_SOFTMAX));
    // ============================================================== softmax + epilogue (a5-a7, a9)
    const int t = warp >> 3, h = (warp >> 2) & 1, quad = warp & 3;
    const int row = quad * 32 + lane;
    const uint32_t lane_off = static_cast<uint32_t>(quad * 32) << 16;
    const uint32_t tT = tmem + lane_off + 256 * t;           // tile t's columns, this warp's lanes
    const uint32_t tO = tT + C::COL_O + 32 * h;               // O_t columns 32h .. 32h+31
    const uint32_t S_FULL = BAR(C::B_S_FULL + t), P_FULL = BAR(C::B_P_FULL + t);
    const uint32_t S_FREE = BAR(C::B_S_FREE + t), PV_DONE = BAR(C::B_PV_DONE + t);
    const uint32_t STAT = BAR(C::B_STAT + 4 * t + quad);
    // 128-thread named barriers: the pair (t, quad) waits on my_turn, the other tile's pair arrives
    const uint32_t my_turn = 1 + 2 * quad + t, other_turn = 2 + 2 * quad - t;
    float* xmax = reinterpret_cast<float*>(smem + C::OFF_XMAX);  // [step parity][tile][h][row]
    float* lsum = reinterpret_cast<float*>(smem + C::OFF_LSUM);  // [item parity][tile][h][row]
    const uint32_t stg = sbase + C::OFF_STG + warp * C::STG;
    const float c = p.scale_log2;
    const int off = p.seq_kv - p.seq_q;
    const uint32_t pair_bar = 1 + 4 * t + quad;  // (no turns) the pair's 64-thread exchange barrier
    if (C::TURNS && t == 1) named_bar_arrive(1 + 2 * quad, 128);  // tile 0 goes first
    uint32_t g = 0, ofc = 0, ec = 0;
    for (int kk = 0, idx; (idx = item_at<SCHED>(p, sched, kk)) >= 0; ++kk) {
      const WorkItem w = get_item<PAIRX, VL, false, SCHED>(p, sched, idx);
      const int n = w.n(t);
      const int N = C::TURNS ? max(w.n0, w.n1) : n;
      const int qi = w.row0(t) + row;
      int lim = w.kv(t);
      if (p.mask_kind == MASK_CAUSAL) lim = min(lim, qi + off + 1);
      if (qi >= w.len(t)) lim = 0;
      const int lim_w = __reduce_max_sync(0xffffffffu, lim);
      float m_ref = -INFINITY, l = 0.f;
      for (int j = 0; j < N; ++j) {
        if (j >= n) {  // no KV tile j for this tile: pass the turn on
          named_bar_sync(my_turn, 128);
          named_bar_arrive(other_turn, 128);
          continue;
        }
        if (C::OFFSET && j == 0 && t == 1 && w.n0 > 0) named_bar_sync(9 + quad, 128);
        const int key0 = j * 128 + 64 * h;
        TRACE_EV(EV_S_WAIT, j);
        mbar_wait_at(S_FULL, g & 1, 8, g, j);
        TRACE_EV(EV_S_READY, j);
        tc_fence_after();
        const uint32_t tS = tT + C::col_s(g) + 64 * h;  // this warp's 64 S columns of step g
        const uint32_t tP = tT + C::col_p(g) + 32 * h;  // ... and its 32 P columns
        uint32_t sv[64];
        tmem_ld_32x32b_x32(tS, *reinterpret_cast<uint32_t(*)[32]>(&sv[0]));
        tmem_ld_32x32b_x32(tS + 32, *reinterpret_cast<uint32_t(*)[32]>(&sv[32]));
        tmem_wait_ld();
        reg_fence(sv);
        tc_fence_before();
        mbar_arrive_elect(S_FREE);  // S_t read (wait::ld is warp-wide): QK_{t,j+1} may overwrite it
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
        // this warp's half of the row max goes to shared memory; the turn barrier (which the two
        // warps of the pair pass together) makes the partner's half visible (slots by step parity)
        float* xm = xmax + (g & 1) * 512 + 256 * t;
        xm[128 * h + row] = fmaxf(fmaxf(mx0, mx1), fmaxf(mx2, mx3));
        if (!C::ROT && g > 0) {  // fixed layout: P_g overwrites P_{g-1}
          mbar_wait_at(PV_DONE, (g - 1) & 1, 10, g, j);
          tc_fence_after();
        }
        TRACE_EV(EV_MAX_DONE, j);
        if (C::TURNS)
          named_bar_sync(my_turn, 128);
        else
          named_bar_sync(pair_bar, 64);
        TRACE_EV(EV_XCHG, j);
        const float m_new = fmaxf(xm[row], xm[128 + row]);
        // lazy rescale (a7): keep the reference while the max grows by <= 8 in log2 units (both warps
        // of the pair take the same decision from the same two halves)
        float alpha = 1.f;
        if (m_new > m_ref && (m_ref == -INFINITY || (m_new - m_ref) * c > 8.f)) {
          alpha = (m_ref == -INFINITY) ? 0.f : ex2((m_ref - m_new) * c);
          m_ref = m_new;
        }
        const float mc = (m_ref == -INFINITY) ? 0.f : m_ref * c;
        float2 acc0 = make_float2(0.f, 0.f), acc1 = make_float2(0.f, 0.f);
        auto chunk = [&](int hh) {  // keys 32 hh .. 32 hh + 31 of this warp's 64
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
          tmem_st_32x32b_x16(tP + 16 * hh, pk);
        };
        auto zero_chunk = [&](int hh) {
          uint32_t pk[16];
#pragma unroll
          for (int u = 0; u < 16; ++u) pk[u] = 0u;
          tmem_st_32x32b_x16(tP + 16 * hh, pk);
        };
        if (rem_w >= 64) {  // (the common case: no chunk of this warp is fully masked)
          chunk(0);
          chunk(1);
        } else {
          if (rem_w > 0) chunk(0); else zero_chunk(0);
          if (rem_w > 32) chunk(1); else zero_chunk(1);
        }
        if (C::TURNS) named_bar_arrive(other_turn, 128);
        if (C::OFFSET && j == 0 && t == 0 && w.n1 > 0) named_bar_arrive(9 + quad, 128);
        TRACE_EV(EV_EXP_DONE, j);
        // lazy rescale of O_t columns 32h .. 32h+31 of this row (a7); at j = 0 the PV overwrites O_t.
        // O_t must hold PV_{t,g-1} first (PV_DONE's phases run one behind the softmax's step count,
        // so the parity of completion g-1 is unambiguous even though most steps do not wait)
        if (j > 0 && __any_sync(0xffffffffu, alpha != 1.f)) {
          mbar_wait_at(PV_DONE, (g - 1) & 1, 10, g, j);
          tc_fence_after();
          uint32_t o[32];
          tmem_ld_32x32b_x32(tO, o);
          tmem_wait_ld();
          reg_fence(o);
#pragma unroll
          for (int k = 0; k < 32; ++k) o[k] = __float_as_uint(__uint_as_float(o[k]) * alpha);
          tmem_st_32x32b_x32(tO, o);
        }
        tmem_wait_st();
        // every PV_DONE phase is consumed in order before P_FULL_g lets PV_g start (see fmha_kernel.cuh)
        if (g > 0) mbar_wait_at(PV_DONE, (g - 1) & 1, 10, g, j);
        tc_fence_before();
        mbar_arrive_elect(P_FULL);
        ++g;
        TRACE_EV(EV_EPI, j);
        l = l * alpha + ((acc0.x + acc0.y) + (acc1.x + acc1.y));
      }
      if (!w.has(t)) continue;
      // ------------------------------------------------------------ epilogue (a9)
      TRACE_EV(EV_ITEM, 1);
      // the row sum is split over the pair (same reference max): exchange the halves (slots by item
      // parity, so a warp an item ahead never overwrites what its partner has yet to read)
      float* ls = lsum + (ec & 1) * 512 + 256 * t;
      ls[128 * h + row] = l;
      mbar_arrive(STAT);  // (one arrival per thread: each publishes its own shared-memory write)
      if (lane == 0) tma_store_wait_read0();  // this warp's staging buffer free again
      mbar_wait_at(STAT, ec & 1, 9, ec, t);
      ++ec;
      const float L = ls[row] + ls[128 + row];
      const float inv = L > 0.f ? 1.f / L : 0.f;  // fully masked row -> 0 (R4)
      uint32_t o[32];
      if (n > 0) {
        mbar_wait_at(BAR(C::B_O_FULL + t), ofc & 1, 14, ofc, t);
        TRACE_EV(EV_ITEM, 2);
        ++ofc;
        tc_fence_after();
        tmem_ld_32x32b_x32(tO, o);
        tmem_wait_ld();
        reg_fence(o);
        tc_fence_before();
        mbar_arrive_elect(BAR(C::B_O_EMPTY + t));
      } else {
#pragma unroll
        for (int k = 0; k < 32; ++k) o[k] = 0u;
      }
      uint32_t pk[16];
#pragma unroll
      for (int u = 0; u < 16; ++u)
        pk[u] = pack2<BF16>(__uint_as_float(o[2 * u]) * inv, __uint_as_float(o[2 * u + 1]) * inv);
      const bool rowwise = VL && w.row0(t) + 128 > w.len(t);
      if (!rowwise) {  // 32 rows x 64 B, SWIZZLE_64B: 16-B chunk u of row r at chunk u ^ ((r >> 1) & 3)
#pragma unroll
        for (int u = 0; u < 4; ++u)
          st_shared_v4(stg + lane * 64 + 16 * (u ^ ((lane >> 1) & 3)), pk[4 * u], pk[4 * u + 1], pk[4 * u + 2],
                       pk[4 * u + 3]);
        fence_proxy_async_smem();
        __syncwarp();
        if (lane == 0) {
          tma_store_4d(&p.tmO32, stg, 32 * h, w.c1(VL, t, w.row0(t) + 32 * quad), w.c2(VL, t, w.row0(t) + 32 * quad),
                       w.c3(VL, t));
          tma_store_commit();
        }
      } else if (qi < w.len(t)) {  // varlen tile crossing the sequence's end: rows inside only
        const size_t tokn = static_cast<size_t>(w.tok(t) + qi);
        uint8_t* dst = p.o_ptr + 2 * (tokn * p.o_row_elems + (t ? w.head1 : w.head) * D + 32 * h);
#pragma unroll
        for (int u = 0; u < 4; ++u) st_global_v4(dst + 16 * u, pk[4 * u], pk[4 * u + 1], pk[4 * u + 2], pk[4 * u + 3]);
      }
      TRACE_EV(EV_ITEM, 3);
    }
    if (C::TURNS && t == 0) named_bar_sync(1 + 2 * quad, 128);  // consume tile 1's last hand-over
    if (lane == 0) tma_store_wait0();
  }

  tc_fence_before();
  __syncthreads();
  if (warp == C::W_MMA) {
    tc_fence_after();
    tmem_dealloc(tmem, 512);
  }
}

}  // namespace b200
