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

// Debug timeline (build with -DFMHA_TRACE=1, see Makefile target `trace`): lane 0 of each warp of
// CTA 0 appends (clock64, warp, event, aux) records to a global buffer.  Compiled out otherwise.
#ifndef FMHA_TRACE
#define FMHA_TRACE 0
#endif

namespace b200 {

#if FMHA_TRACE
__device__ unsigned long long* g_fmha_trace = nullptr;
__device__ unsigned int g_fmha_trace_n = 0;
// per-warp slices of 4096 records, plain stores (no atomics on the timed path)
#define TRACE_EV(ev, aux)                                                                                \
  do {                                                                                                   \
    if (blockIdx.x == 0 && (threadIdx.x & 31) == 0 && trace_buf && trace_i < 4096u) {                    \
      trace_buf[(threadIdx.x >> 5) * 4096u + trace_i++] =                                                \
          (static_cast<unsigned long long>(clock64()) << 24) |                                           \
          (static_cast<unsigned long long>(threadIdx.x >> 5) << 18) |                                    \
          (static_cast<unsigned long long>(ev) << 12) | (static_cast<unsigned>(aux) & 0xFFFu);           \
    }                                                                                                    \
  } while (0)
#define TRACE_DECL                                    \
  unsigned long long* trace_buf = g_fmha_trace;      \
  unsigned int trace_i = 0;
#else
#define TRACE_EV(ev, aux) \
  do {                    \
  } while (0)
#define TRACE_DECL
#endif
// event ids
enum : int { EV_S_WAIT = 1, EV_S_READY, EV_MAX_DONE, EV_TURN, EV_EXP_DONE, EV_MMA_P, EV_MMA_O, EV_MMA_PV,
             EV_MMA_QK, EV_COR_ST, EV_COR_PV, EV_COR_ORDY, EV_EPI, EV_TMA_KV, EV_ITEM };

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
  static constexpr int NS = (D == 64) ? 6 : 3;   // K/V ring slots (K_j, V_j alternate)
  static constexpr int QS = (D == 64) ? 2 : 1;   // Q stages per tile: the next item's Q loads early
  static constexpr int OFF_Q = 0;                // Q[stage][tile]
  static constexpr int OFF_RING = 2 * QS * TILE;
  static constexpr int NSTG = (D == 64) ? 2 : 1;        // O staging buffers (D=128 shares one)
  static constexpr int OFF_STG = OFF_RING + NS * TILE;
  static constexpr int OFF_ALPHA = OFF_STG + NSTG * TILE;  // float alpha[2][128]
  static constexpr int OFF_LSUM = OFF_ALPHA + 2 * 128 * 4;
  static constexpr int OFF_BAR = OFF_LSUM + 2 * 128 * 4;
  // barriers: 2x {q_full, q_empty, s_full, p_full, o_ready, pv_done, st_full, st_empty, l_full}
  //           + NS x {kv_full, kv_empty}
  static constexpr int NUM_BARS = 28 + 2 * NS;
  static constexpr int OFF_TMEMPTR = OFF_BAR + NUM_BARS * 8;
  static constexpr int SMEM_BYTES = OFF_TMEMPTR + 16;
  static constexpr int SMEM_ALLOC = SMEM_BYTES;
  static constexpr int TMEM_COLS = 512;
  static constexpr int THREADS = 512;
  // D = 64: S_0, S_1, O_0, O_1 use 384 columns, so P_t gets its own 64 columns at 384 + 64 t and
  // QK_{t,j+1} can be issued as soon as S_{t,j} is in registers (S_FREE), overlapping the softmax.
  // D = 128: TMEM is full; P_t overwrites S_t and QK_{t,j+1} must follow PV_{t,j}.
  static constexpr bool SEP_P = (D == 64);
  static constexpr int TMEM_P = 384;
  // exp-phase turn-taking between the two softmax groups (named barriers 2, 3).  With HALF_TURN
  // the turn passes after half of the exp loop, so the groups overlap by half a phase: one warp's
  // TMEM load + row max runs under the other's exponentials, and MUFU still sees two warps.
  static constexpr bool TURNS = true;
  static constexpr bool HALF_TURN = SEP_P;
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
  // Dynamic shared memory starts at the (1024-byte aligned) base of the CTA's shared window; the
  // SWIZZLE_128B tiles need that alignment.  Using the base directly keeps every smem address a
  // compile-time-uniform value, so UMMA descriptors live in uniform registers.
  extern __shared__ __align__(1024) uint8_t smem[];
  const uint32_t sbase = smem_u32(smem);
  const uint32_t bar = sbase + C::OFF_BAR;
  // barrier addresses (t = tile 0/1, s = ring slot)
  auto Q_FULL = [&](int t, int q) { return bar + 8 * (20 + C::NS * 2 + 2 * q + t); };  // q = Q stage
  auto Q_EMPTY = [&](int t, int q) { return bar + 8 * (24 + C::NS * 2 + 2 * q + t); };
  auto S_FULL = [&](int t) { return bar + 8 * (4 + t); };
  auto P_FULL = [&](int t) { return bar + 8 * (6 + t); };
  auto O_READY = [&](int t) { return bar + 8 * (8 + t); };
  auto PV_DONE = [&](int t) { return bar + 8 * (10 + t); };
  auto ST_FULL = [&](int t) { return bar + 8 * (12 + t); };
  auto ST_EMPTY = [&](int t) { return bar + 8 * (14 + t); };
  auto L_FULL = [&](int t) { return bar + 8 * (16 + t); };
  auto S_FREE = [&](int t) { return bar + 8 * (18 + t); };
  auto KV_FULL = [&](int s) { return bar + 8 * (20 + s); };
  auto KV_EMPTY = [&](int s) { return bar + 8 * (20 + C::NS + s); };
  float* s_alpha = reinterpret_cast<float*>(smem + C::OFF_ALPHA);
  float* s_lsum = reinterpret_cast<float*>(smem + C::OFF_LSUM);
  uint32_t* tmem_holder = reinterpret_cast<uint32_t*>(smem + C::OFF_TMEMPTR);

  const int warp = warp_id();
  const int lane = lane_id();
  TRACE_DECL

  if (threadIdx.x == 0) {
    if (sbase & 1023u) __trap();  // the layout below assumes a 1024-byte aligned window
    for (int t = 0; t < 2; ++t) {
      for (int q = 0; q < 2; ++q) {
        mbar_init(Q_FULL(t, q), 1);
        mbar_init(Q_EMPTY(t, q), 1);
      }
      mbar_init(S_FULL(t), 1);
      mbar_init(P_FULL(t), 128);
      mbar_init(O_READY(t), 128);
      mbar_init(PV_DONE(t), 1);
      mbar_init(ST_FULL(t), 128);
      mbar_init(ST_EMPTY(t), 128);
      mbar_init(L_FULL(t), 128);
      mbar_init(S_FREE(t), 128);
    }
    for (int s = 0; s < C::NS; ++s) {
      mbar_init(KV_FULL(s), 1);
      mbar_init(KV_EMPTY(s), 2);  // released by both MMA warps
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
    if (warp == 13) {
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
          const int qs = qc[t] % C::QS;
          mbar_wait(Q_EMPTY(t, qs), ((qc[t] / C::QS) & 1) ^ 1);
          mbar_arrive_expect_tx_elect(Q_FULL(t, qs), C::TILE);
#pragma unroll
          for (int c = 0; c < D / 64; ++c)
            tma_load_3d_hint_elect(sbase + C::OFF_Q + (2 * qs + t) * C::TILE + c * C::CHUNK, &p.tmQ, Q_FULL(t, qs),
                                   c * 64, w.q0 + 128 * t, w.bh, once);
          ++qc[t];
          TRACE_EV(EV_ITEM, 3 + t);
        }
        for (int j = 0; j < N; ++j) {
#pragma unroll
          for (int m = 0; m < 2; ++m, ++kv) {  // m = 0: K_j, m = 1: V_j
            const int s = kv % C::NS;
            mbar_wait(KV_EMPTY(s), ((kv / C::NS) & 1) ^ 1);
            TRACE_EV(EV_TMA_KV, m * 64 + j);
            mbar_arrive_expect_tx_elect(KV_FULL(s), C::TILE);
            const CUtensorMap* map = m ? &p.tmV : &p.tmK;
#pragma unroll
            for (int c = 0; c < D / 64; ++c)
              tma_load_3d_hint_elect(sbase + C::OFF_RING + s * C::TILE + c * C::CHUNK, map, KV_FULL(s), c * 64, j * 128,
                               w.bh, keep);
          }
        }
      }
    } else if (warp == 12 || warp == 14) {
      // ============================================================ MMA issuers (a4, a8)
      // Warp 12 issues tile 0's MMAs, warp 14 tile 1's: each tile's chain (QK -> softmax -> PV)
      // then depends only on its own softmax group.  Both warps release every K/V slot (count 2).
      const int t = (warp == 12) ? 0 : 1;
      constexpr uint32_t IDESC_QK = idesc_f16(BF16, 128, 128, false, false);  // Q, K: K-major
      constexpr uint32_t IDESC_PV = idesc_f16(BF16, 128, D, false, true);     // P: K-major (TMEM), V: MN-major
      // descriptors differ only in the start-address field: build one base and add (offset >> 4)
      const uint64_t desc0 = sdesc_sw128(sbase, 16, 1024);          // K-major Q / K tiles
      const uint64_t vdesc0 = sdesc_sw128(sbase, C::CHUNK, 1024);   // MN-major V tiles
      const uint32_t tS = tmem + 128 * t;
      const uint32_t tO = tmem + 256 + t * D;
      const uint32_t tP = tmem + (C::SEP_P ? C::TMEM_P + 64 * t : 128 * t);
      uint32_t kv = 0, qc = 0, pc = 0, oc = 0, qkc = 0;
      auto ring_wait = [&](uint32_t k) {
        mbar_wait(KV_FULL(k % C::NS), (k / C::NS) & 1);
        tc_fence_after();
        return sbase + C::OFF_RING + (k % C::NS) * C::TILE;
      };
      for (int idx = first; idx < p.num_items; idx += stride) {
        const WorkItem w = decode_item(p, idx);
        const int N = max(w.n[0], w.n[1]);
        if (N == 0) continue;
        const int n = w.n[t];
        int qs = 0;
        if (n > 0) {
          qs = qc % C::QS;
          mbar_wait(Q_FULL(t, qs), (qc / C::QS) & 1);
          ++qc;
          tc_fence_after();
        }
        const uint32_t qoff = C::OFF_Q + (2 * qs + t) * C::TILE;
        const uint32_t base = kv;  // ring index of K_0 of this item; K_j = base + 2j, V_j = base + 2j + 1
        kv += 2 * N;
        // S_t <- Q_t K_j^T (with separate P buffers: once softmax t has read the previous S_t)
        auto issue_qk = [&](int j) {
          const uint32_t kidx = base + 2 * j;
          const uint32_t sK = ring_wait(kidx);
          if (j < n) {
            if (C::SEP_P && qkc > 0) {
              mbar_wait(S_FREE(t), (qkc - 1) & 1);
              tc_fence_after();
            }
            ++qkc;
            const uint32_t koff = sK - sbase;
#pragma unroll
            for (int kk = 0; kk < D / 16; ++kk) {
              const uint32_t off = (kk / 4) * C::CHUNK + (kk % 4) * 32;
              umma_ss_elect(tS, desc0 + ((qoff + off) >> 4), desc0 + ((koff + off) >> 4), IDESC_QK, kk > 0);
            }
            umma_commit_elect(S_FULL(t));
            TRACE_EV(EV_MMA_QK, t * 64 + j);
            if (j + 1 == n) umma_commit_elect(Q_EMPTY(t, qs));  // last QK of this tile: Q slot reusable
          }
          umma_commit_elect(KV_EMPTY(kidx % C::NS));
        };
        // O_t (+)= P_t V_j once softmax t wrote P_t and the correction group rescaled O_t
        auto issue_pv = [&](int j) {
          const uint32_t vidx = base + 2 * j + 1;
          const uint32_t sV = ring_wait(vidx);
          if (j < n) {
            mbar_wait(P_FULL(t), pc & 1);
            ++pc;
            TRACE_EV(EV_MMA_P, t * 64 + j);
            mbar_wait(O_READY(t), oc & 1);
            ++oc;
            TRACE_EV(EV_MMA_O, t * 64 + j);
            tc_fence_after();
#pragma unroll
            for (int kk = 0; kk < 8; ++kk)
              umma_ts_elect(tO, tP + kk * 8, vdesc0 + ((sV - sbase + kk * 2048) >> 4), IDESC_PV, (j > 0 || kk > 0));
            umma_commit_elect(PV_DONE(t));
            TRACE_EV(EV_MMA_PV, t * 64 + j);
          }
          umma_commit_elect(KV_EMPTY(vidx % C::NS));
        };
        issue_qk(0);
        for (int j = 0; j < N; ++j) {
          if (C::SEP_P) {  // next scores first: they only need S_t free, not P_t
            if (j + 1 < N) issue_qk(j + 1);
            issue_pv(j);
          } else {  // P_t overwrites S_t: QK_{t,j+1} must follow PV_{t,j} (in-order tensor pipe)
            issue_pv(j);
            if (j + 1 < N) issue_qk(j + 1);
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
    if (C::TURNS && t == 1) named_bar_arrive(2, 256);  // tile 0 goes first
    const uint32_t tP = tmem + (static_cast<uint32_t>(quad * 32) << 16) + (C::SEP_P ? C::TMEM_P + 64 * t : 128 * t);
    uint32_t sc = 0, stc = 0, gstep = 0;
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
          if (C::TURNS) {
            named_bar_sync(my_turn, 256);
            named_bar_arrive(other_turn, 256);
          }
          continue;
        }
        TRACE_EV(EV_S_WAIT, j);
        mbar_wait(S_FULL(t), sc & 1);
        ++sc;
        TRACE_EV(EV_S_READY, j);
        tc_fence_after();
        uint32_t s[128];
#pragma unroll
        for (int q = 0; q < 4; ++q) tmem_ld_32x32b_x32(tS + 32 * q, *reinterpret_cast<uint32_t(*)[32]>(&s[32 * q]));
        tmem_wait_ld();
        reg_fence(s);
        if (C::SEP_P) {  // S_t is in registers: the tensor core may overwrite it with S_{t,j+1}
          tc_fence_before();
          mbar_arrive(S_FREE(t));
        }
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
        TRACE_EV(EV_MAX_DONE, j);
        if (C::TURNS) named_bar_sync(my_turn, 256);
        TRACE_EV(EV_TURN, j);
        if (C::SEP_P && gstep > 0) {  // P_t buffer still read by PV_{t,j-1}?
          mbar_wait(PV_DONE(t), (gstep - 1) & 1);
          tc_fence_after();
        }
        ++gstep;
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
          tmem_st_32x32b_x32(tP + 32 * h, pk);
          if (C::TURNS && C::HALF_TURN && h == 0) named_bar_arrive(other_turn, 256);
        }
        if (C::TURNS && !C::HALF_TURN) named_bar_arrive(other_turn, 256);
        TRACE_EV(EV_EXP_DONE, j);
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
    if (C::TURNS && t == 0) named_bar_sync(2, 256);  // consume tile 1's last hand-over
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
          TRACE_EV(EV_COR_ST, t * 64 + j);
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
          TRACE_EV(EV_COR_ORDY, t * 64 + j);
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
