// fmha_kernel.cuh — FMHA forward for sm_100a (persistent, warp-specialised, two Q tiles per CTA).
//
// The operation is the paper's fused multi-head attention (§6 "Fused Multi-Head
// Attention"): two back-to-back GEMMs with a softmax between them, per (batch, head).  The paper's
// kernel was written for Ampere (ldmatrix + mma.sync, specialised to BERT shapes, L489); this is
// the B200-native redesign:
//
//   work item     two consecutive 128-row query tiles (t = 0, 1) of one (b, h) sharing every
//                 K/V tile load; persistent CTAs (one per SM) walk a static item list        [a1]
//   warps 0-7     softmax: warpgroup t (warps 4t..4t+3) owns tile t, one thread per query row
//                 and all 128 key columns of every S tile, so the row max and row sum are
//                 thread-local (192 registers per thread after setmaxnreg)                 [a5, a6]
//                 A softmax warp also rescales its own 32 rows of O_t in TMEM when a row max
//                 grew by more than 2^8 (lazy rescale, rare), so PV_{t,j} waits only for P  [a7]
//   warps 8-11    epilogue: O_t / l -> fp16/bf16 -> smem -> TMA store                      [a9]
//   warps 12, 13  MMA issuers for tile 0 / tile 1 (one elected lane each):
//                 S_t = Q_t K_j^T (SS), O_t += P_t V_j (TS)                                [a4, a8]
//   warp 14       TMA producer: Q_t per item (double-buffered at D=64), K_j / V_j ring     [a2, a3]
//   warp 15       idle (completes warpgroup 3 for setmaxnreg)
//
//   TMEM (512 columns x 128 lanes, fp32):  S_0 [0,128)  S_1 [128,256)  O_0 [256,256+D)  O_1 [..+D)
//   D = 64 : P_t (16-bit, two per column) has its own columns [384 + 64t, 448 + 64t), so
//            QK_{t,j+1} starts as soon as S_{t,j} is in registers (S_FREE).
//   D = 128: TMEM is full; P_t overwrites the first 64 columns of S_t and QK_{t,j+1} follows
//            PV_{t,j} (tcgen05.mma ops of one thread execute in issue order).
//
// Ordering facts relied on:
//   * tcgen05.mma ops of one thread execute in issue order;
//   * tcgen05.commit arrives once all earlier tcgen05 ops of the issuing thread have completed.
//
// Because tcgen05.ld 32x32b gives each thread whole TMEM lanes (= query rows), row statistics are
// thread-local: no warp-shuffle reductions and no cross-warp exchange.
#pragma once
#include <type_traits>

#include "sm100.cuh"

// Debug timeline (build with -DFMHA_TRACE=1, see Makefile target `trace`): lane 0 of each warp of
// CTA 0 appends (clock64, warp, event, aux) records to its slice of a global buffer.
#ifndef FMHA_TRACE
#define FMHA_TRACE 0
#endif

namespace b200 {

#ifndef FMHA_PROF
#define FMHA_PROF 0
#endif
#if FMHA_TRACE || FMHA_PROF
__device__ unsigned long long* g_fmha_trace = nullptr;
__device__ unsigned int g_fmha_trace_n = 0;
#endif
#if FMHA_TRACE
#define TRACE_EV(ev, aux)                                                                                \
  do {                                                                                                   \
    if (blockIdx.x == 0 && (threadIdx.x & 31) == 0 && trace_buf && trace_i < 2048u) {                    \
      trace_buf[(threadIdx.x >> 5) * 2048u + trace_i++] =                                                \
          (static_cast<unsigned long long>(clock64()) << 24) |                                           \
          (static_cast<unsigned long long>(threadIdx.x >> 5) << 18) |                                    \
          (static_cast<unsigned long long>(ev) << 12) | (static_cast<unsigned>(aux) & 0xFFFu);           \
    }                                                                                                    \
  } while (0)
#define TRACE_DECL                               \
  unsigned long long* trace_buf = g_fmha_trace; \
  unsigned int trace_i = 0;
#else
#define TRACE_EV(ev, aux) \
  do {                    \
  } while (0)
#define TRACE_DECL
#endif
// Timing-only ablations (WRONG RESULTS; never in the product build): FMHA_ABL bit 0 skips the S TMEM
// load (registers zeroed), bit 1 the row max (fixed reference), bit 2 the P TMEM stores, bit 3 the
// tensor-core instructions (commits still arrive), bit 4 the exponential phase (its turn kept), bit 5 the
// epilogue's O TMEM loads, bit 6 makes every K/V load read the same (L2-resident) tile.  Used to locate what bounds a step.
#ifndef FMHA_ABL
#define FMHA_ABL 0
#endif
// FMHA_ELECT: the per-row hand-offs (S_FREE, P_FULL, L_FULL, L_EMPTY, O_EMPTY) arrive once per warp
// (elect.sync, barrier count 4) instead of once per thread (count 128): 32x fewer mbarrier updates.
// FMHA_SK_ABL (timing only, wrong results): bit 0 skips the stream-K count + merge, bit 1 the pieces'
// workspace stores
#ifndef FMHA_SK_ABL
#define FMHA_SK_ABL 0
#endif
#ifndef FMHA_SUMCHECK
#define FMHA_SUMCHECK 0
#endif
// FMHA_PREFETCH_FIRST (default on): the first item's Q and FMHA_PREFETCH_STEPS K/V steps into L2 before
// griddepcontrol.wait (below).  Measured in one session (profiles/r02c_ab_prefetch_first.txt): BERT-base
// padded 98.0 -> 105.3 TFLOP/s, BERT-large-384 +2.5%, BERT-large-512 +1.3%, gpt_causal level; the 8-way
// strong-scaling shard of BERT-large-512 11.75 -> 10.96 us per launch.  1, 2 or 4 steps: level.
#ifndef FMHA_PREFETCH_FIRST
#define FMHA_PREFETCH_FIRST 1
#endif
#ifndef FMHA_PREFETCH_STEPS
#define FMHA_PREFETCH_STEPS 2
#endif
#ifndef FMHA_ELECT
#define FMHA_ELECT 0
#endif
#if FMHA_ELECT
#define FMHA_ROW_ARRIVE(bar) mbar_arrive_elect(bar)
#define FMHA_ROW_COUNT 4
#else
#define FMHA_ROW_ARRIVE(bar) mbar_arrive(bar)
#define FMHA_ROW_COUNT 128
#endif
// Phase profile (build with -DFMHA_PROF=1; not the product build): every softmax thread accumulates
// the cycles between consecutive marks into per-phase counters (two clock reads per mark, no memory
// traffic until the end), and lane 0 of each softmax warp writes them to g_fmha_trace[block][warp][16].
#ifndef FMHA_PROF
#define FMHA_PROF 0
#endif
#if FMHA_PROF
#define PROF_DECL                     \
  uint32_t prof_acc[16] = {};         \
  uint32_t prof_t = clock();
#define PROF_MARK(k)                  \
  do {                                \
    const uint32_t prof_now = clock(); \
    prof_acc[k] += prof_now - prof_t; \
    prof_t = prof_now;                \
  } while (0)
#define PROF_COUNT(k) (++prof_acc[k])
#else
#define PROF_DECL
#define PROF_MARK(k) \
  do {               \
  } while (0)
#define PROF_COUNT(k) \
  do {                \
  } while (0)
#endif
enum : int { EV_S_WAIT = 1, EV_S_READY, EV_MAX_DONE, EV_XCHG, EV_EXP_DONE, EV_MMA_P, EV_MMA_O, EV_MMA_PV,
             EV_MMA_QK, EV_COR_ST, EV_COR_PV, EV_COR_ORDY, EV_EPI, EV_TMA_KV, EV_ITEM };

enum : int { MASK_NONE = 0, MASK_KEY_PADDING = 1, MASK_CAUSAL = 2, MASK_KEY_BIAS = 3 };

// Division by a launch constant without the integer-divide sequence (whose MUFU.RCP would queue
// behind the softmax's exponentials): q = (umulhi(n, m) + n) >> s, exact for 0 <= n < 2^31.
struct FastDiv {
  uint32_t d, m, s;
  __host__ void init(uint32_t div) {
    d = div;
    s = 0;
    while ((1ull << s) < div) ++s;
    m = static_cast<uint32_t>(((1ull << 32) * ((1ull << s) - div)) / div + 1);
  }
  __device__ __forceinline__ int div(int n) const {
    return static_cast<int>((__umulhi(static_cast<uint32_t>(n), m) + static_cast<uint32_t>(n)) >> s);
  }
  __device__ __forceinline__ int mod(int n, int q) const { return n - q * static_cast<int>(d); }
};

// Cost-sorted schedule (sched mode 1, varlen non-causal): every (sequence, head, q-tile pair) item
// costs `level` = ceil(len / 128) KV steps.  Items are ordered by decreasing level (sequences of one
// level by index, then head, then pair) and dealt to the CTAs in snake order (CTA c takes positions
// c, 2G-1-c, 2G+c, ...), a near-LPT balance.  Each CTA builds the same table in shared memory.
#ifdef SCHED_SMALL
constexpr int SCHED_MAX_LEVELS = 4, SCHED_MAX_SEQS = 32;
#else
constexpr int SCHED_MAX_LEVELS = 64, SCHED_MAX_SEQS = 1024;
#endif

struct FmhaParams {
  CUtensorMap tmQ;  // 4-D {D, seq_q, H, B} (any row / head / batch strides), box {64, 128, 1, 1}, SWIZZLE_128B
  CUtensorMap tmK;  // 4-D {D, seq_kv, H, B}; varlen maps: {D, H, T, 1}, box {64, 1, 128, 1}
  CUtensorMap tmV;
  CUtensorMap tmO;  // same geometry as Q
  CUtensorMap tmO32;  // O with a 32-row box (key-split kernel: one store per (tile, lane quarter))
  const int32_t* kv_len;
  // Variable-length packed mode (fmha_fwd_varlen): sequence b of the batch is
  // tokens [cu_seqlens[b], cu_seqlens[b+1]) of QKV [T, 3, H, D] / O [T, H, D]; the tensor maps are
  // {D, H, T}, so a tile coordinate is (d, h, token) instead of (d, row, b*H + h).  Rows past the
  // sequence's end are never stored (partial tiles are written row by row, not by TMA).
  const int32_t* cu_seqlens;  // nullptr: dense [B, H, S, D] mode
  uint8_t* o_ptr;             // O base (varlen partial-tile stores)
  int o_row_elems;            // elements between consecutive tokens of O (H * D)
  int sched;                  // 0: item idx = blockIdx.x + k * gridDim.x;  1: cost-sorted (above)
  int snake;                  // sched 0: odd rounds k visit the CTAs in reverse (idx = (k + 1) G - 1 - c), so
                              // longest-first items of decreasing cost (causal) balance like LPT
  int num_seqs;               // varlen
  int max_level;              // ceil(max_seqlen / 128) (sched 1: <= SCHED_MAX_LEVELS)
  int seq_q;
  int seq_kv;
  int heads;
  int num_q_tiles;
  int num_units;  // B*H
  int num_items;  // see pair_mode
  int single_from;  // pair_mode 1: items >= single_from hold one tile (see decode_item)
  int pair_mode;  // 0: items are q-tiles {2i, 2i+1} of one unit (num_units * ceil(num_q_tiles / 2) items)
                  // 1: items are tiles {2i, 2i+1} of the flattened (unit, q-tile) list, so a tile pair
                  //    may straddle two units (odd num_q_tiles, non-causal): no half-empty items
  int mask_kind;
  float scale_log2;  // scale * log2(e)
  FastDiv div_units, div_pairs, div_qtiles, div_heads;  // num_units, ceil(num_q_tiles/2), num_q_tiles, heads
  // Split-KV mode (MODE_SPLIT, fmha_fwd_splitkv): item idx = (unit, q-tile pair) *
  // num_splits + split; split s visits KV tiles [s * split_tiles, (s + 1) * split_tiles) and writes
  // its unnormalised partial O (fp32), its exp2 reference mc = scale*log2e*m and its row sum l to
  // the workspace; fmha_splitkv_combine_kernel merges the splits.
  int num_splits, split_tiles;
  FastDiv div_splits;  // ceil(num_splits / 2) with split_pair, else num_splits
  // split_pair (units with one q-tile; the MODE_SPLIT_PAIR instance): an item's tile 1 is the same q-tile
  // as tile 0 with the NEXT split's key range (its own K/V stream), so both softmax warpgroups work and the
  // items halve
  int split_pair;
  float* ws_o;   // [num_splits][num_units][seq_q][D]
  float* ws_m;   // [num_splits][num_units][seq_q]
  float* ws_l;   // [num_splits][num_units][seq_q]
  // Additive key bias (MODE_BIAS; R20): raw scores get key_bias[b][j] / scale added, so
  // c * s' = c * s + log2(e) * bias and the rest of the softmax is unchanged.
  const float* key_bias;
  int key_bias_stride;
  float inv_scale;
  // General additive (query x key) mask (MODE_BIAS2D; R21): raw scores get
  // attn_bias[b, h, i, j] / scale added (16-bit, the I/O type), element strides below (0 broadcasts);
  // bias_cols8 = min(row stride, seq_kv rounded up to 8) / 8 bounds the 16-byte loads of a row.
  const uint16_t* attn_bias;
  long long ab_sb, ab_sh, ab_sq;
  int bias_cols8;
  // Stream-K tail (MODE_DENSE_TAIL / MODE_PAIRX_TAIL, fmha_fwd_streamk): items
  // idx >= tail_from are pieces of the last, partial round's items: piece idx - tail_from is split
  // s = (idx - tail_from) % tail_splits of tail item r = (idx - tail_from) / tail_splits (= the
  // item tail_from + r of the plain numbering) and visits its KV tiles [s * tail_tiles, (s + 1) *
  // tail_tiles).  Every piece writes its online-softmax state (unnormalised O, mc, l) to ws_tail and
  // counts itself in tail_cnt[r]; the piece that counts last merges the splits and stores O.
  int tail_from, tail_splits, tail_tiles;
  FastDiv div_tail;
  unsigned int* tail_cnt;  // [tail items]; zero before the launch, zero again after it
  float* ws_tail;          // [tail item][split][tile] x {O [D/4][128 rows] float4, mc [128], l [128]} (fp32)
};
constexpr int MAX_TAIL_SPLITS = 4;

template <int D>
struct FmhaCfg {
  static constexpr int BM = 128;                // query rows per tile (UMMA M)
  static constexpr int BN = 128;                // keys per KV tile
  static constexpr int CHUNK = 128 * 64 * 2;    // one SW128 TMA box: 128 rows x 64 16-bit elements
  static constexpr int TILE = BM * D * 2;       // bytes of one Q / K / V / O tile
#ifndef FMHA_NS64
#define FMHA_NS64 6
#endif
  // D128_RING4: at D = 128 a fourth K/V ring slot (the MMA warp waited ~300 cycles per step for K_{j+1}
  // with three), paid for by a half-size O staging buffer (one 64-column chunk, stored before the next)
#ifndef FMHA_D128_RING4
#define FMHA_D128_RING4 0
#endif
  static constexpr bool D128_RING4 = FMHA_D128_RING4 && D == 128;
  static constexpr int NS = (D == 64) ? FMHA_NS64 : (D128_RING4 ? 4 : 3);  // K/V ring slots (K_j, V_j alternate)
  static constexpr int QS = (D == 64) ? 2 : 1;  // Q stages per tile: the next item's Q loads early
  static constexpr int NSTG = (D == 64) ? 2 : 1;  // O staging buffers (D=128: both tiles share one)
  static constexpr int OFF_Q = 0;               // Q[stage][tile]
  static constexpr int OFF_RING = 2 * QS * TILE;
  static constexpr int OFF_STG = OFF_RING + NS * TILE;
  // LSUM_MMA (D = 64): the row sum l comes out of the PV MMA -- V gets 16 extra columns of ones
  // (a constant 16 KB SW128 atom that the V descriptor's leading-byte offset points at), so
  // O_t[:, 64] = sum_k P[:, k]; P then overwrites S_t (as at D = 128) to make room in TMEM for the
  // 80-column O_t.  The softmax threads drop their row-sum adds.
#ifndef FMHA_LSUM_MMA
#define FMHA_LSUM_MMA 0
#endif
  static constexpr bool LSUM_MMA = FMHA_LSUM_MMA && D == 64;
  static constexpr int OW = LSUM_MMA ? D + 16 : D;  // O_t columns in TMEM (and PV MMA N)
  static constexpr int STG_CHUNKS = D128_RING4 ? 1 : D / 64;  // 64-column chunks one staging buffer holds
  static constexpr int OFF_ONES = OFF_STG + NSTG * STG_CHUNKS * CHUNK;  // LSUM_MMA: 128 x 64 ones (16 KB)
  static constexpr int OFF_LSUM = OFF_ONES + (LSUM_MMA ? CHUNK : 0);  // float l[2 tiles][128 rows]
  static constexpr int OFF_MC = OFF_LSUM + 2 * 128 * 4;    // float mc[2 tiles][128 rows] (turn fence)
  static constexpr int OFF_MREF = OFF_MC + 2 * 128 * 4;  // float mc[2 tiles][128 rows] at item end (tail pieces)
  static constexpr int OFF_BAR = OFF_MREF + 2 * 128 * 4;
  // barrier slots
  enum : int {
    B_S_FULL = 0, B_P_FULL = 2, B_O_FULL = 4, B_PV_DONE = 6, B_O_EMPTY = 8, B_L_FULL = 12,
    B_S_FREE = 14, B_Q_FULL = 16, B_Q_EMPTY = 20, B_L_EMPTY = 24, B_KV = 26
  };
  // B_P_FULL2 [tile]: P_FULL of odd steps (ROT).  Without the per-step PV_DONE wait the softmax can
  // be two P hand-offs ahead of the MMA warp (S_FULL_g only implies PV_{g-2} was issued), which one
  // barrier's phase parity cannot tell apart; two barriers by step parity can.
  static constexpr int B_P_FULL2 = B_KV + 2 * NS;
  static constexpr int B_MERGE = B_P_FULL2 + 2;  // stream-K merge: bulk loads of the pieces' states
  static constexpr int NUM_BARS = B_MERGE + 1;
  static constexpr int OFF_TMEMPTR = OFF_BAR + NUM_BARS * 8;
  static constexpr int OFF_SCHED = OFF_TMEMPTR + 16;  // SchedTable (sched mode 1 only)
  static constexpr int SMEM_ALLOC = OFF_SCHED + 4 * (3 * (SCHED_MAX_LEVELS + 2) + SCHED_MAX_SEQS);
  static constexpr int TMEM_COLS = 512;
  static constexpr int THREADS = 512;
  static constexpr int W_CORR = 8, W_MMA = 12, W_TMA = 14;  // first warp of each role
  static constexpr bool SEP_P = (D == 64) && !LSUM_MMA;
  static constexpr int TMEM_P = 384;
  // ROT (D = 64, separate P): tile t owns columns [256 t, 256 t + 256): O_t at +192 and three 64-column
  // regions below it over which S and P rotate with the tile's step count g -- S_g in [0,128) (g even)
  // or [64,192) (g odd), P_g in [0,64) or [128,192).  S_{g+1} never covers P_g (PV_g is issued after
  // QK_{g+1}), P_g never covers P_{g-1} (PV_{g-1} may still be reading it), and S_{g+1} covering
  // P_{g-1} is safe (PV_{g-1} is issued before QK_{g+1} by the same thread, and tcgen05.mma ops of one
  // thread execute in order); P_g lies on S_g, which this warp has loaded.  So the softmax writes P_g
  // without waiting for PV_{g-1} (PV_DONE is waited only before a lazy rescale of O).
// Default off: measured level on BERT-large-512 and +1.7% on BERT-large-384 only while PV_DONE
// phases go unwaited, which compute-sanitizer's synccheck rejects ("Missing wait"); consuming every
// phase (FMHA_ROT_PVWAIT) costs 2% on BERT-large-512 (profiles/r02_fmha_ablation.txt).
#ifndef FMHA_ROT
#define FMHA_ROT 0
#endif
#ifndef FMHA_ROT_PVWAIT
#define FMHA_ROT_PVWAIT 1
#endif
  static constexpr bool ROT = FMHA_ROT && SEP_P;
  static __host__ __device__ constexpr uint32_t col_s(int t, uint32_t g) {
    return ROT ? 256 * t + ((g & 1) ? 64 : 0) : 128 * t;
  }
  static __host__ __device__ constexpr uint32_t col_p(int t, uint32_t g) {
    return ROT ? 256 * t + ((g & 1) ? 128 : 0) : (SEP_P ? TMEM_P + 64 * t : 128 * t);
  }
  static __host__ __device__ constexpr uint32_t col_o(int t) { return ROT ? 256 * t + 192 : 256 + t * OW; }
  // registers after setmaxnreg.  setmaxnreg.inc only draws on the CTA's launch allocation
  // (128 x 512 = 65536), so 8 x 32 x 192 + 4 x 32 x 56 + 4 x 32 x 72 = 65536 must not be exceeded
  // (56 / 72: the MMA and TMA warps spill at 48, and those spills cost 2-12%).
#ifndef FMHA_REG_CORR
#define FMHA_REG_CORR 56
#endif
#ifndef FMHA_REG_MISC
#define FMHA_REG_MISC 72
#endif
  static constexpr int REG_SOFTMAX = 192, REG_CORR = FMHA_REG_CORR, REG_MISC = FMHA_REG_MISC;
  // The two tiles' softmax warps on one SMSP (warps q and 4 + q) take turns for the exp phase, so
  // one tile's exponentials overlap the other's S load and row max (named barriers 2..9).
#ifndef FMHA_TURNS
#define FMHA_TURNS 1
#endif
// (FMHA_TURNS128=0, D = 128 without turns: gpt_causal 871 -> 837 TFLOP/s, 8x32x2048 non-causal 1047 -> 890;
// profiles/r02c_ab_d128_noturns.txt)
#ifndef FMHA_TURNS128
#define FMHA_TURNS128 FMHA_TURNS
#endif
  static constexpr bool TURNS = (D == 128) ? FMHA_TURNS128 : FMHA_TURNS;
  // Split S load: max of the first 64 columns overlaps the TMEM load of the last 64 (A/B knob)
#ifndef FMHA_SPLIT_LD
#define FMHA_SPLIT_LD 0
#endif
  static constexpr bool SPLIT_LD = FMHA_SPLIT_LD;
  // Prefetch S_{t,j+1} into registers at the end of step j, before P_FULL (separate P only)
#ifndef FMHA_PREFETCH_S
#define FMHA_PREFETCH_S 0
#endif
  static constexpr bool PREFETCH_S = FMHA_PREFETCH_S && SEP_P && !SPLIT_LD && !FMHA_ROT;
  // Key bias: prefetch all four 128-B lines of this and the next step's bias into L1 (A/B knob;
  // measured -2% at BERT-large-384, +2% at 512: L1 misses are not the bias cost, left off)
#ifndef FMHA_BIAS_PF4
#define FMHA_BIAS_PF4 0
#endif
  static constexpr bool BIAS_PF4 = FMHA_BIAS_PF4;
  // Key bias: unpredicated loads with the column clamped into the row (stride >= seq_kv, a multiple
  // of 4, so every valid column is unchanged; the clamped ones are past seq_kv and masked) instead
  // of predicated loads with zero fill (A/B knob)
#ifndef FMHA_BIAS_CLAMP
#define FMHA_BIAS_CLAMP 1
#endif
  static constexpr bool BIAS_CLAMP = FMHA_BIAS_CLAMP;
  // The first PRE_CHUNKS of the four 32-column chunks of a row are exponentiated before the turn
  // (overlapping the other tile's turn), the rest inside it.
#ifndef FMHA_PRE_CHUNKS
#define FMHA_PRE_CHUNKS ((D == 128) ? 0 : 1)
#endif
  static constexpr int PRE_CHUNKS = TURNS ? FMHA_PRE_CHUNKS : 4;
#ifndef FMHA_DEFER_ST
#define FMHA_DEFER_ST 0
#endif
  static constexpr int DEFER_ST = FMHA_DEFER_ST;
  static_assert(!TURNS || (PRE_CHUNKS >= 0 && PRE_CHUNKS < 4), "the turn barrier sits before chunk PRE_CHUNKS");
  // exp2 of element pairs q (of 64 per row) with (q % POLY_MOD) < POLY_CNT runs on the FMA pipe
  // (exp2_poly2) instead of MUFU: at D = 64 MUFU (16/clk/SM) is the bound.
#ifndef FMHA_POLY_CNT
#define FMHA_POLY_CNT 2
#endif
#ifndef FMHA_POLY_MOD
#define FMHA_POLY_MOD 8
#endif
#ifndef FMHA_POLY_CNT128
#define FMHA_POLY_CNT128 0
#endif
  static constexpr int POLY_MOD = FMHA_POLY_MOD, POLY_CNT = (D == 64) ? FMHA_POLY_CNT : FMHA_POLY_CNT128;
#ifndef FMHA_POLY_MASK
#define FMHA_POLY_MASK 0
#endif
  // optional explicit 8-bit pattern over (pair index % 8); 0 = use POLY_MOD / POLY_CNT
  static constexpr unsigned POLY_MASK = FMHA_POLY_MASK;
  static __host__ __device__ constexpr bool poly_pair(int q) {
    return POLY_MASK && D == 64 ? ((POLY_MASK >> (q % 8)) & 1u) != 0 : (q % POLY_MOD) < POLY_CNT;
  }
  static_assert(8 * 32 * REG_SOFTMAX + 4 * 32 * REG_CORR + 4 * 32 * REG_MISC <= 128 * THREADS, "register pool");
  static_assert(SMEM_ALLOC <= 232448, "shared memory budget");
};

// Exponential-phase shape per kernel instance.  The cross-unit pair instance (BERT-large-384: each
// tile streams its own K/V) measured best with all exp2 on MUFU (no polynomial pairs), keeping the
// one pre-turn chunk: 525 vs 517 TF/s for (0 pre-turn chunks, 1 of 8) and 509 for the dense
// instance's (1, 2 of 8), which stays best on BERT-large-512 (profiles/r01_ab_pc0.txt,
// r01_ab_pairx_expshape.txt, r01_ab_pairx_sweep.txt).
#ifndef FMHA_PAIRX_PRE_CHUNKS
#define FMHA_PAIRX_PRE_CHUNKS 1
#endif
#ifndef FMHA_PAIRX_POLY_CNT
#define FMHA_PAIRX_POLY_CNT 0
#endif
#ifndef FMHA_VARLEN_ALT
#define FMHA_VARLEN_ALT 0
#endif
// The key-bias instance has its own pair (FMHA_BIAS_PRE_CHUNKS, FMHA_BIAS_POLY_CNT): the bias add
// lengthens the S -> max part of its step, which moves the best split of the exponential phase.
// Sweep of 8 shapes (profiles/r01_ab_bias_shape.txt): (0 pre-turn chunks, all exp2 on MUFU) is
// best, -4.9% at BERT-large-384 and -2.7% at 512 against the dense instance's (1, 2 of 8).
#ifndef FMHA_BIAS_PRE_CHUNKS
#define FMHA_BIAS_PRE_CHUNKS 0
#endif
#ifndef FMHA_BIAS_POLY_CNT
#define FMHA_BIAS_POLY_CNT 0
#endif
// Varlen instances: (FMHA_VARLEN_PRE_CHUNKS, FMHA_VARLEN_POLY_CNT), -1 = the dense instance's shape.
// Sweeps of 13 shapes on bert_large_varlen (profiles/r01_ab_varlen_shape.txt, _shape2.txt): two
// pre-turn chunks with every exp2 on MUFU is best, 173.7 vs 171.1 TF/s for (2, 2 of 8) and 168.6
// for the dense instance's (1, 2 of 8).  (Same exp2 arithmetic as the pair instance.)
#ifndef FMHA_VARLEN_PRE_CHUNKS
#define FMHA_VARLEN_PRE_CHUNKS 2
#endif
#ifndef FMHA_VARLEN_POLY_CNT
#define FMHA_VARLEN_POLY_CNT 0
#endif
template <int D, bool PAIRX, bool VL = false, bool BIAS = false>
struct ExpShape {
  static constexpr bool ALT = (PAIRX || (VL && FMHA_VARLEN_ALT)) && D == 64 && FmhaCfg<D>::TURNS && !FmhaCfg<D>::POLY_MASK;
  static constexpr bool BSH = BIAS && D == 64 && FmhaCfg<D>::TURNS && !FmhaCfg<D>::POLY_MASK;
  static constexpr bool VSH = VL && !ALT && D == 64 && FmhaCfg<D>::TURNS && !FmhaCfg<D>::POLY_MASK;
  static constexpr int PRE_CHUNKS = ALT ? FMHA_PAIRX_PRE_CHUNKS : BSH ? FMHA_BIAS_PRE_CHUNKS
                                  : (VSH && FMHA_VARLEN_PRE_CHUNKS >= 0) ? FMHA_VARLEN_PRE_CHUNKS : FmhaCfg<D>::PRE_CHUNKS;
  static __host__ __device__ constexpr bool poly_pair(int q) {
    return ALT ? (q % 8) < FMHA_PAIRX_POLY_CNT : BSH ? (q % 8) < FMHA_BIAS_POLY_CNT
         : (VSH && FMHA_VARLEN_POLY_CNT >= 0) ? (q % 8) < FMHA_VARLEN_POLY_CNT : FmhaCfg<D>::poly_pair(q);
  }
};

// One work item = two 128-row query tiles t = 0, 1.  Every role decodes items identically.
// shared: both tiles belong to one unit and share every K/V tile; otherwise (pair_mode 1) each tile
// streams its own K/V through the ring (entries of tile 0 then tile 1 for every step j).
struct WorkItem {
  int bh0, bh1;  // units of tile 0 / 1
  int r0, r1;    // first query row of tile 0 / 1
  int kv0, kv1;  // keys >= kv_t are masked for every row of tile t (key padding)
  int n0, n1;    // KV tiles visited by tile t (0 = tile absent or fully masked)
  bool has0;     // tile 0 exists (always, except for varlen tiles past the sequence's end)
  bool has1;     // tile 1 exists
  int tok0, tok1;  // varlen: first token of the sequence of tile 0 / 1; len = its length
  int len0, len1;
  int head, head1;  // h of unit bh0 / bh1
  int bat0, bat1;   // dense: b of unit bh0 / bh1
  int jb;          // split-KV: first KV tile of this item's range (0 otherwise)
  int split;       // split-KV: split index
  int jb1, split1; // the same for tile 1 (differ from tile 0's only with split pairing, FmhaParams::split_pair)
  __device__ __forceinline__ int jbt(int t) const { return t ? jb1 : jb; }
  __device__ __forceinline__ int splt(int t) const { return t ? split1 : split; }
  int tail;        // stream-K tail piece: its tail item r (-1: a whole item)
  // 4-D TMA coordinates (c1, c2, c3) of the block starting at row r of tile t (c0 = d):
  // dense maps are {D, rows, heads, batch}, varlen maps {D, heads, tokens, 1}
  __device__ __forceinline__ int c1(bool varlen, int t, int r) const { return varlen ? (t ? head1 : head) : r; }
  __device__ __forceinline__ int c2(bool varlen, int t, int r) const { return varlen ? tok(t) + r : (t ? head1 : head); }
  __device__ __forceinline__ int c3(bool varlen, int t) const { return varlen ? 0 : (t ? bat1 : bat0); }
  bool shared;
  __device__ __forceinline__ int n(int t) const { return t ? n1 : n0; }
  __device__ __forceinline__ int bh(int t) const { return t ? bh1 : bh0; }
  __device__ __forceinline__ int row0(int t) const { return t ? r1 : r0; }
  __device__ __forceinline__ int kv(int t) const { return t ? kv1 : kv0; }
  __device__ __forceinline__ bool has(int t) const { return t ? has1 : has0; }
  __device__ __forceinline__ int tok(int t) const { return t ? tok1 : tok0; }
  __device__ __forceinline__ int len(int t) const { return t ? len1 : len0; }
  // number of K/V ring entries the item uses, and the ring index of K_{t,j} (V = K + 1)
  __device__ __forceinline__ int entries() const { return shared ? 2 * max(n0, n1) : 2 * (n0 + n1); }
  __device__ __forceinline__ int k_index(int t, int j) const {
    return shared ? 2 * j : 2 * (min(j, n0) + min(j, n1)) + ((t == 1 && j < n0) ? 2 : 0);
  }
};

// SPLIT: 0 none, 1 split-KV, 2 split-KV with split pairing (MODE_SPLIT_PAIR)
template <bool PAIRX, bool VL, int SPLIT = 0, bool TAIL = false, bool NOLOAD = false>
__device__ __forceinline__ WorkItem decode_item(const FmhaParams& p, int idx) {
  WorkItem w;
  int qt0;
  w.jb = w.jb1 = 0;
  w.split = w.split1 = 0;
  w.tail = -1;
  if constexpr (TAIL) {
    if (idx >= p.tail_from) {  // piece (tail item r, split) of item tail_from + r
      const int piece = idx - p.tail_from;
      const int r = p.div_tail.div(piece);
      w.split = piece - r * p.tail_splits;
      w.tail = r;
      idx = p.tail_from + r;
    }
  }
  if constexpr (SPLIT != 0) {
    const int ns = SPLIT == 2 ? (p.num_splits + 1) >> 1 : p.num_splits;  // items per (unit, q-tile pair)
    const int rest = p.div_splits.div(idx);
    const int sp = idx - rest * ns;
    w.split = SPLIT == 2 ? 2 * sp : sp;
    idx = rest;
  }
  if (!PAIRX) {
    const int pairs = (p.num_q_tiles + 1) >> 1;
    int pr;
    if (p.mask_kind == MASK_CAUSAL) {  // longest-first: the last query tiles see the most keys
      const int q = p.div_units.div(idx);
      pr = pairs - 1 - q;
      w.bh0 = p.div_units.mod(idx, q);
    } else {  // both pairs of a (b,h) back to back so K/V are re-read from L2
      w.bh0 = p.div_pairs.div(idx);
      pr = p.div_pairs.mod(idx, w.bh0);
    }
    qt0 = 2 * pr;
    w.bh1 = w.bh0;
    w.has1 = qt0 + 1 < p.num_q_tiles;
    w.shared = true;
    w.r0 = qt0 * 128;
    w.r1 = w.r0 + 128;
  } else {
    // items < single_from pair tiles {2 idx, 2 idx + 1}; later items (the last, partial round of
    // the static schedule) are single tiles, so that round takes about half as long
    const bool single = idx >= p.single_from;
    const int a = single ? 2 * p.single_from + (idx - p.single_from) : 2 * idx;
    const int b = single ? a : a + 1;
    w.bh0 = p.div_qtiles.div(a);
    qt0 = a - w.bh0 * p.num_q_tiles;
    w.bh1 = p.div_qtiles.div(b);
    const int qt1 = b - w.bh1 * p.num_q_tiles;
    w.has1 = !single && b < p.num_units * p.num_q_tiles;
    w.shared = w.has1 && w.bh1 == w.bh0;
    w.r0 = qt0 * 128;
    w.r1 = qt1 * 128;
  }
  if constexpr (SPLIT == 2) {
    {  // tile 1: the same q-tile (one per unit), the next split's key range
      w.has1 = w.split + 1 < p.num_splits;
      w.bh1 = w.bh0;
      w.r1 = w.r0;
      w.shared = false;
    }
  }
  w.has0 = true;
  w.kv0 = w.kv1 = p.seq_kv;
  w.tok0 = w.tok1 = 0;
  w.bat0 = p.div_heads.div(w.bh0);
  w.bat1 = w.shared ? w.bat0 : p.div_heads.div(w.bh1);
  w.head = w.bh0 - w.bat0 * p.heads;
  w.head1 = w.bh1 - w.bat1 * p.heads;
  w.len0 = w.len1 = p.seq_q;
  if constexpr (VL) {  // varlen (pair_mode 0): both tiles belong to unit bh0 = b * H + h
    const int b = p.div_heads.div(w.bh0);
    w.tok0 = w.tok1 = __ldg(p.cu_seqlens + b);
    w.len0 = w.len1 = __ldg(p.cu_seqlens + b + 1) - w.tok0;
    w.kv0 = w.kv1 = w.len0;
    w.head = w.bh0 - b * p.heads;
    w.head1 = w.head;
    w.has0 = w.r0 < w.len0;
    w.has1 = w.has1 && w.r1 < w.len0;
  }
  if (!NOLOAD && p.mask_kind == MASK_KEY_PADDING) {  // (NOLOAD: no global reads -- before pdl_wait)
    w.kv0 = min(max(__ldg(p.kv_len + w.bat0), 0), p.seq_kv);
    w.kv1 = w.shared ? w.kv0
                     : min(max(__ldg(p.kv_len + p.div_heads.div(min(w.bh1, p.num_units - 1))), 0), p.seq_kv);
  }
  const int off = p.seq_kv - p.seq_q;
  int kv_end0 = w.kv0, kv_end1 = w.kv1;
  if (p.mask_kind == MASK_CAUSAL) {
    kv_end0 = min(kv_end0, max(0, w.r0 + 128 + off));
    kv_end1 = min(kv_end1, max(0, w.r1 + 128 + off));
  }
  w.n0 = w.has0 ? (kv_end0 + 127) / 128 : 0;
  w.n1 = w.has1 ? (kv_end1 + 127) / 128 : 0;
  if constexpr (SPLIT != 0) {  // this split's KV tiles [jb, jb + split_tiles) of each tile's range
    w.jb = w.split * p.split_tiles;
    w.split1 = SPLIT == 2 ? w.split + 1 : w.split;
    w.jb1 = SPLIT == 2 ? w.split1 * p.split_tiles : w.jb;
    w.n0 = min(max(w.n0 - w.jb, 0), p.split_tiles);
    w.n1 = min(max(w.n1 - w.jb1, 0), p.split_tiles);
  }
  if constexpr (TAIL) {  // a tail piece: its split's KV tiles [jb, jb + tail_tiles)
    if (w.tail >= 0) {
      w.jb = w.jb1 = w.split * p.tail_tiles;
      w.split1 = w.split;
      w.n0 = min(max(w.n0 - w.jb, 0), p.tail_tiles);
      w.n1 = min(max(w.n1 - w.jb, 0), p.tail_tiles);
    }
  }
  return w;
}

// Shared-memory table of sched mode 1: items_end[l] = number of items of level >= l (levels
// descending), seq_start[l] = first entry of level l in seq_by_level, seq_by_level = sequence indices
// sorted by decreasing level (ascending index within a level).
struct SchedTable {
  int items_end[SCHED_MAX_LEVELS + 2];
  int seq_start[SCHED_MAX_LEVELS + 2];
  int seq_by_level[SCHED_MAX_SEQS];
  int seq_count[SCHED_MAX_LEVELS + 2];  // sequences of level l
};

// Built by one full warp before the CTA's first __syncthreads.  Deterministic (no order-dependent
// atomics), so every CTA derives the same order.
__device__ __forceinline__ void build_sched(const FmhaParams& p, SchedTable* tb, int lane) {
  const int L = p.max_level;
  for (int l = lane; l <= L + 1; l += 32) tb->items_end[l] = tb->seq_start[l] = tb->seq_count[l] = 0;
  __syncwarp();
  auto level_of = [&](int sq) {
    if (sq >= p.num_seqs) return -1;
    const int len = __ldg(p.cu_seqlens + sq + 1) - __ldg(p.cu_seqlens + sq);
    return len <= 0 ? -1 : min((len + 127) >> 7, L);
  };
  for (int base = 0; base < p.num_seqs; base += 32) {  // sequences per level (into seq_start)
    const int lv = level_of(base + lane);
    if (lv > 0) atomicAdd(&tb->seq_start[lv], 1);
  }
  __syncwarp();
  if (lane == 0) {  // prefix over descending levels
    int seqs = 0, items = 0;
    for (int l = L; l >= 1; --l) {
      const int c = tb->seq_start[l];
      tb->seq_count[l] = c;
      tb->seq_start[l] = seqs;
      seqs += c;
      // l >> 1 same-unit tile pairs per (sequence, head); for odd l the units' last tiles are
      // paired across units (two different (sequence, head)), so no item runs half empty
      items += c * p.heads * (l >> 1) + (l & 1) * ((c * p.heads + 1) >> 1);
      tb->items_end[l] = items;
    }
    tb->items_end[L + 1] = 0;
    tb->items_end[0] = items;  // total
  }
  __syncwarp();
  for (int base = 0; base < p.num_seqs; base += 32) {  // stable scatter, 32 sequences at a time
    const int sq = base + lane;
    const int lv = level_of(sq);
    const unsigned same = __match_any_sync(0xffffffffu, lv);
    if (lv > 0) {
      const int rank = __popc(same & ((1u << lane) - 1u));
      tb->seq_by_level[tb->seq_start[lv] + rank] = sq;
    }
    __syncwarp();
    if (lv > 0 && lane == __ffs(same) - 1) tb->seq_start[lv] += __popc(same);
    __syncwarp();
  }
  if (lane == 0) {  // undo the scatter's advance: seq_start[l] = first entry of level l again
    int seqs = 0;
    for (int l = L; l >= 1; --l) {
      const int end = tb->seq_start[l];
      tb->seq_start[l] = seqs;
      seqs = end;
    }
  }
  __syncwarp();
}

// The k-th work item of this CTA: its index in decode_item's numbering, or -1 when exhausted.
template <bool SCHED>
__device__ __forceinline__ int item_at(const FmhaParams& p, const SchedTable* tb, int k) {
  const int G = gridDim.x, c = blockIdx.x;
  if constexpr (!SCHED) {
    const long long idx = ((k & 1) && p.snake ? G - 1 - c : c) + static_cast<long long>(k) * G;
    return idx < p.num_items ? static_cast<int>(idx) : -1;
  } else {
    const long long pos = static_cast<long long>(k) * G + ((k & 1) ? G - 1 - c : c);
    if (pos >= tb->items_end[0]) return -1;
    return static_cast<int>(pos);  // decoded by sched_item
  }
}

// Work item at schedule position pos (sched mode): level l = KV steps; positions of a level list
// its same-unit pairs (sequence, head, pair) first, then the cross-unit pairs of the last tiles of
// odd-level units (units in (sequence, head) order, two per item; the last may be alone).
__device__ __forceinline__ WorkItem sched_item(const FmhaParams& p, const SchedTable* tb, int pos) {
  int l = p.max_level;
  while (pos >= tb->items_end[l]) --l;  // items_end grows as l decreases
  const int r = pos - tb->items_end[l + 1];
  const int H = p.heads, nl = tb->seq_count[l] * H, full = nl * (l >> 1);
  WorkItem w;
  w.jb = w.jb1 = 0;
  w.split = w.split1 = 0;
  w.tail = -1;
  w.has0 = true;
  int si0, h0, si1, h1;
  if (r < full) {  // q-tiles 2 pr, 2 pr + 1 of one unit
    const int pairs_l = l >> 1, per = H * pairs_l;
    si0 = r / per;
    const int rem = r - si0 * per;
    h0 = rem / pairs_l;
    const int pr = rem - h0 * pairs_l;
    si1 = si0;
    h1 = h0;
    w.r0 = 2 * pr * 128;
    w.r1 = w.r0 + 128;
    w.has1 = true;
    w.shared = true;
  } else {  // the last q-tile (l - 1) of units 2 r2 and 2 r2 + 1 of this level
    const int su0 = 2 * (r - full), su1 = su0 + 1;
    si0 = su0 / H;
    h0 = su0 - si0 * H;
    w.has1 = su1 < nl;
    si1 = w.has1 ? su1 / H : si0;
    h1 = w.has1 ? su1 - si1 * H : h0;
    w.r0 = w.r1 = (l - 1) * 128;
    w.shared = false;
  }
  const int sq0 = tb->seq_by_level[tb->seq_start[l] + si0], sq1 = tb->seq_by_level[tb->seq_start[l] + si1];
  w.tok0 = __ldg(p.cu_seqlens + sq0);
  w.len0 = __ldg(p.cu_seqlens + sq0 + 1) - w.tok0;
  w.tok1 = __ldg(p.cu_seqlens + sq1);
  w.len1 = __ldg(p.cu_seqlens + sq1 + 1) - w.tok1;
  w.head = h0;
  w.head1 = h1;
  w.bat0 = w.bat1 = 0;
  w.bh0 = sq0 * H + h0;
  w.bh1 = sq1 * H + h1;
  w.kv0 = w.len0;
  w.kv1 = w.len1;
  w.n0 = (w.len0 + 127) / 128;
  w.n1 = w.has1 ? (w.len1 + 127) / 128 : 0;
  return w;
}

// decode_item, or sched_item in sched mode
template <bool PAIRX, bool VL, int SPLIT, bool SCHED, bool TAIL = false>
__device__ __forceinline__ WorkItem get_item(const FmhaParams& p, const SchedTable* tb, int idx) {
  if constexpr (SCHED) {
    return sched_item(p, tb, idx);
  } else {
    return decode_item<PAIRX, VL, SPLIT, TAIL>(p, idx);
  }
}

// Kernel instances (MODE): dense [B,H,S,D]; dense with cross-unit tile pairing (pair_mode 1, see
// FmhaParams::pair_mode); varlen packed; varlen packed with the cost-sorted schedule.  Separate
// instances keep the varlen and scheduling code out of the dense kernels entirely.
enum : int { MODE_DENSE = 0, MODE_PAIRX = 1, MODE_VARLEN = 2, MODE_VARLEN_SCHED = 3, MODE_SPLIT = 4, MODE_BIAS = 5,
             MODE_BIAS2D = 6, MODE_DENSE_TAIL = 7, MODE_PAIRX_TAIL = 8, MODE_SPLIT_PAIR = 9 };

template <int D, bool BF16, int MODE>
__global__ void __launch_bounds__(512, 1) fmha_fwd_sm100(const __grid_constant__ FmhaParams p) {
  using C = FmhaCfg<D>;
  using XS = ExpShape<D, MODE == MODE_PAIRX || MODE == MODE_PAIRX_TAIL, MODE == MODE_VARLEN || MODE == MODE_VARLEN_SCHED,
                      MODE == MODE_BIAS || MODE == MODE_BIAS2D>;
  constexpr bool TAIL = MODE == MODE_DENSE_TAIL || MODE == MODE_PAIRX_TAIL;
  constexpr int SPLIT_KIND = MODE == MODE_SPLIT_PAIR ? 2 : MODE == MODE_SPLIT ? 1 : 0;
  constexpr bool PAIRX = MODE == MODE_PAIRX || MODE == MODE_PAIRX_TAIL, VL = MODE == MODE_VARLEN || MODE == MODE_VARLEN_SCHED,
                 SCHED = MODE == MODE_VARLEN_SCHED, SPLIT = MODE == MODE_SPLIT || MODE == MODE_SPLIT_PAIR, BIAS = MODE == MODE_BIAS,
                 BIAS2D = MODE == MODE_BIAS2D;
  // FMHA_SUMCHECK: the row max is taken over the polynomial columns only once a row has a reference,
  // and the step's sum of p guards the rest (softmax loop, redo_step)
  // (bit 0: the D = 64 instances, bit 1: D = 128, where P overwrites S in TMEM -- s[] stays in registers)
  constexpr bool SUMCHK = ((D == 64 && (FMHA_SUMCHECK & 1)) || (D == 128 && (FMHA_SUMCHECK & 2))) && !C::ROT &&
                          !C::PREFETCH_S && !C::SPLIT_LD && !C::LSUM_MMA && !BIAS && !BIAS2D && !SPLIT && FMHA_ABL == 0 &&
                          C::DEFER_ST == 0;
  // Dynamic shared memory starts at the (1024-byte aligned) base of the CTA's shared window; the
  // SWIZZLE_128B tiles need that alignment.  Using the base directly keeps smem addresses uniform.
  extern __shared__ __align__(1024) uint8_t smem[];
  const uint32_t sbase = smem_u32(smem);
  const uint32_t bar = sbase + C::OFF_BAR;
  auto BAR = [&](int slot) { return bar + 8 * slot; };
  auto Q_FULL = [&](int t, int q) { return BAR(C::B_Q_FULL + 2 * q + t); };
  auto Q_EMPTY = [&](int t, int q) { return BAR(C::B_Q_EMPTY + 2 * q + t); };
  auto KV_FULL = [&](int s) { return BAR(C::B_KV + s); };
  auto KV_EMPTY = [&](int s) { return BAR(C::B_KV + C::NS + s); };
  float* s_lsum = reinterpret_cast<float*>(smem + C::OFF_LSUM);
  uint32_t* tmem_holder = reinterpret_cast<uint32_t*>(smem + C::OFF_TMEMPTR);

  const int warp = warp_id();
  const int lane = lane_id();
  TRACE_DECL

  if (threadIdx.x == 0) {
    if (sbase & 1023u) __trap();  // the layout below assumes a 1024-byte aligned window
    for (int t = 0; t < 2; ++t) {
      mbar_init(BAR(C::B_S_FULL + t), 1);
      mbar_init(BAR(C::B_P_FULL + t), FMHA_ROW_COUNT);   // softmax warps (threads) of tile t
      mbar_init(BAR(C::B_P_FULL2 + t), FMHA_ROW_COUNT);
      mbar_init(BAR(C::B_O_FULL + t), 1);     // last PV of the tile committed
      mbar_init(BAR(C::B_O_EMPTY + t), FMHA_ROW_COUNT);  // epilogue warps (threads) have read O_t
      mbar_init(BAR(C::B_PV_DONE + t), 1);
      mbar_init(BAR(C::B_L_FULL + t), FMHA_ROW_COUNT);
      mbar_init(BAR(C::B_L_EMPTY + t), FMHA_ROW_COUNT);  // epilogue, after reading the row sums
      mbar_init(BAR(C::B_S_FREE + t), FMHA_ROW_COUNT);
      for (int q = 0; q < 2; ++q) {
        mbar_init(Q_FULL(t, q), 1);
        mbar_init(Q_EMPTY(t, q), 1);
      }
    }
    mbar_init(BAR(C::B_MERGE), 1);
    for (int s = 0; s < C::NS; ++s) {
      mbar_init(KV_FULL(s), 1);
      mbar_init(KV_EMPTY(s), 2);  // released by both MMA warps
    }
    fence_mbar_init();
  }
  if (warp == C::W_TMA && lane == 0) {
    tma_prefetch_desc(&p.tmQ);
    tma_prefetch_desc(&p.tmK);
    tma_prefetch_desc(&p.tmV);
    tma_prefetch_desc(&p.tmO);
  }
  if constexpr (C::LSUM_MMA) {  // the ones atom for the row-sum columns of the PV MMA (1.0 in fp16 / bf16)
    const uint32_t one2 = BF16 ? 0x3F803F80u : 0x3C003C00u;
    const uint32_t a = sbase + C::OFF_ONES + threadIdx.x * 32;
    st_shared_v4(a, one2, one2, one2, one2);
    st_shared_v4(a + 16, one2, one2, one2, one2);
    fence_proxy_async_smem();  // visible to the tensor core's operand reads
  }
  if (warp == C::W_MMA) {
    tmem_alloc(smem_u32(tmem_holder), C::TMEM_COLS);
    tmem_relinquish();
  }
  // PDL: the setup above overlaps the previous kernel's tail; global memory only from here on
  // FMHA_PREFETCH_FIRST: while the previous kernel on the stream drains (PDL), the TMA warp prefetches its
  // CTA's first item's Q and first two K/V steps into L2.  A prefetch reads no data into the CTA and
  // writes nothing, so it is safe before griddepcontrol.wait; the item is decoded without the kv_len
  // read (which may be the previous kernel's output).
  if constexpr (FMHA_PREFETCH_FIRST && !VL) {
    if (warp == C::W_TMA) {
      const int idx0 = blockIdx.x;
      if (idx0 < p.num_items) {
        const WorkItem w = decode_item<PAIRX, false, SPLIT_KIND, TAIL, true>(p, idx0);
#pragma unroll
        for (int t = 0; t < 2; ++t) {
          if (w.n(t) == 0) continue;
#pragma unroll
          for (int c = 0; c < D / 64; ++c)
            tma_prefetch_l2_4d_elect(&p.tmQ, c * 64, w.c1(false, t, w.row0(t)), w.c2(false, t, w.row0(t)), w.c3(false, t));
          if (t == 1 && w.shared) continue;
          for (int j = 0; j < min(w.n(t), FMHA_PREFETCH_STEPS); ++j)
#pragma unroll
            for (int c = 0; c < D / 64; ++c) {
              const int r = (w.jbt(t) + j) * 128;
              tma_prefetch_l2_4d_elect(&p.tmK, c * 64, w.c1(false, t, r), w.c2(false, t, r), w.c3(false, t));
              tma_prefetch_l2_4d_elect(&p.tmV, c * 64, w.c1(false, t, r), w.c2(false, t, r), w.c3(false, t));
            }
        }
      }
    }
  }
  pdl_wait();
  pdl_trigger();
  const SchedTable* sched = reinterpret_cast<const SchedTable*>(smem + C::OFF_SCHED);
  if (SCHED && warp == C::W_TMA + 1) build_sched(p, reinterpret_cast<SchedTable*>(smem + C::OFF_SCHED), lane);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = *tmem_holder;
  // this CTA's k-th item: item_at<SCHED>(p, sched, k) (-1 when exhausted)

  if (warp >= C::W_MMA) {
    asm volatile("setmaxnreg.dec.sync.aligned.u32 %0;" ::"n"(C::REG_MISC));
    if (warp == C::W_TMA) {
      // ============================================================ TMA producer (a2, a3)
      const uint64_t keep = policy_evict_last();   // K/V: re-read by the other q-tile pairs
      const uint64_t once = policy_evict_first();  // Q: read once
      uint32_t kv = 0, qc0 = 0, qc1 = 0;
      constexpr bool vl = VL;
      auto load_kv = [&](const WorkItem& w, int t, int j) {
#pragma unroll
        for (int m = 0; m < 2; ++m, ++kv) {  // m = 0: K_j, m = 1: V_j
          const int s = kv % C::NS;
          mbar_wait_at(KV_EMPTY(s), ((kv / C::NS) & 1) ^ 1, 1, kv, j);
          TRACE_EV(EV_TMA_KV, m * 64 + j);
          mbar_arrive_expect_tx_elect(KV_FULL(s), C::TILE);
          const CUtensorMap* map = m ? &p.tmV : &p.tmK;
#pragma unroll
          for (int c = 0; c < D / 64; ++c)
            if (FMHA_ABL & 64)  // (timing ablation: every K/V load hits the same L2-resident tile)
              tma_load_4d_hint_elect(sbase + C::OFF_RING + s * C::TILE + c * C::CHUNK, map, KV_FULL(s), c * 64, 0, 0, 0,
                                     keep);
            else
              tma_load_4d_hint_elect(sbase + C::OFF_RING + s * C::TILE + c * C::CHUNK, map, KV_FULL(s), c * 64,
                                     w.c1(vl, t, (w.jbt(t) + j) * 128), w.c2(vl, t, (w.jbt(t) + j) * 128), w.c3(vl, t), keep);
        }
      };
      for (int kk = 0, idx; (idx = item_at<SCHED>(p, sched, kk)) >= 0; ++kk) {
        const WorkItem w = get_item<PAIRX, VL, SPLIT_KIND, SCHED, TAIL>(p, sched, idx);
        const int N = max(w.n0, w.n1);
#pragma unroll
        for (int t = 0; t < 2; ++t) {
          if (w.n(t) == 0) continue;
          uint32_t& qc = t ? qc1 : qc0;
          const int qs = qc % C::QS;
          mbar_wait_at(Q_EMPTY(t, qs), ((qc / C::QS) & 1) ^ 1, 2, qc, t);
          mbar_arrive_expect_tx_elect(Q_FULL(t, qs), C::TILE);
#pragma unroll
          for (int c = 0; c < D / 64; ++c)
            tma_load_4d_hint_elect(sbase + C::OFF_Q + (2 * qs + t) * C::TILE + c * C::CHUNK, &p.tmQ, Q_FULL(t, qs),
                                   c * 64, w.c1(vl, t, w.row0(t)), w.c2(vl, t, w.row0(t)), w.c3(vl, t), once);
          ++qc;
          TRACE_EV(EV_ITEM, 4 + t);
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
      // ============================================================ MMA issuers (a4, a8)
      // Warp W_MMA issues tile 0's MMAs, warp W_MMA + 1 tile 1's, so each tile's chain (QK -> softmax ->
      // PV) depends only on its own softmax warps.  Both warps release every K/V entry (count 2).
      const int t = warp - C::W_MMA;
      constexpr uint32_t IDESC_QK = idesc_f16(BF16, 128, 128, false, false);  // Q, K: K-major
      constexpr uint32_t IDESC_PV = idesc_f16(BF16, 128, C::OW, false, true);  // P: K-major (TMEM), V: MN-major
      // descriptors differ only in the start-address field: one base, plus (offset >> 4)
      const uint64_t desc0 = sdesc_sw128(sbase, 16, 1024);         // K-major Q / K tiles
      const uint64_t vdesc0 = sdesc_sw128(sbase, C::CHUNK, 1024);  // MN-major V tiles
      const uint32_t tO = tmem + C::col_o(t);
      const uint32_t S_FULL = BAR(C::B_S_FULL + t), P_FULL = BAR(C::B_P_FULL + t), P_FULL2 = BAR(C::B_P_FULL2 + t);
      const uint32_t O_FULL = BAR(C::B_O_FULL + t), O_EMPTY = BAR(C::B_O_EMPTY + t);
      const uint32_t PV_DONE = BAR(C::B_PV_DONE + t), S_FREE = BAR(C::B_S_FREE + t);
      uint32_t qc = 0, pc = 0, oc = 0, qkc = 0;
      PROF_DECL
      auto ring_wait = [&](uint32_t k) {
        mbar_wait_at(KV_FULL(k % C::NS), (k / C::NS) & 1, 3, k, 0);
        tc_fence_after();
        return sbase + C::OFF_RING + (k % C::NS) * C::TILE;
      };
      // Two cursors walk the same sequence of (item, KV step j): the QK cursor runs one step ahead
      // of the PV cursor (behind it when P aliases S), across item boundaries, so the next item's
      // first S is computed while the current item's last P is still being produced.
      struct Ring {  // the part of a WorkItem the ring arithmetic needs
        int n0, n1;
        bool shared;
        __device__ __forceinline__ int n(int t) const { return t ? n1 : n0; }
        __device__ __forceinline__ int entries() const { return shared ? 2 * max(n0, n1) : 2 * (n0 + n1); }
        __device__ __forceinline__ int k_index(int t, int j) const {
          return shared ? 2 * j : 2 * (min(j, n0) + min(j, n1)) + ((t == 1 && j < n0) ? 2 : 0);
        }
      };
      struct Cursor {
        Ring w;
        int idx, k, j, N, qs;
        uint32_t base;  // ring index of the item's first K/V entry (WorkItem::k_index)
        bool valid;
      };
      auto seek = [&](Cursor& cu, int k, uint32_t base) {
        cu.valid = false;
        for (int idx; (idx = item_at<SCHED>(p, sched, k)) >= 0; ++k) {
          const WorkItem w = get_item<PAIRX, VL, SPLIT_KIND, SCHED, TAIL>(p, sched, idx);
          const int N = max(w.n0, w.n1);
          if (N == 0) continue;
          cu.w.n0 = w.n0;
          cu.w.n1 = w.n1;
          cu.w.shared = w.shared;
          cu.idx = idx;
          cu.k = k;
          cu.j = 0;
          cu.N = N;
          cu.base = base;
          cu.valid = true;
          return;
        }
      };
      auto advance = [&](Cursor& cu) {
        if (++cu.j == cu.N) seek(cu, cu.k + 1, cu.base + cu.w.entries());
      };
      Cursor cq, cp;
      seek(cq, 0, 0);
      cp = cq;
      // S_t <- Q_t K_j^T (separate P: once the softmax warps have read the previous S_t)
      // Every K/V ring entry is released exactly once by each MMA warp (KV_EMPTY count 2): a warp
      // that does not use an entry waits for it to be filled, then commits.  (Two back-to-back
      // commits from one thread to one barrier are not a reliable way to arrive twice.)
      auto release = [&](uint32_t kidx) {
        ring_wait(kidx);
        umma_commit_elect(KV_EMPTY(kidx % C::NS));
      };
      // S_t <- Q_t K_{t,j}^T (separate P: once the softmax warps have read the previous S_t)
      auto qk_entry = [&](Cursor& cu, uint32_t kidx) {
        const int n = cu.w.n(t);
        PROF_MARK(8);  // (between MMA phases)
        const uint32_t sK = ring_wait(kidx);
        PROF_MARK(0);  // K ring wait
        if (cu.j == 0) {  // first QK of this item's tile t: its Q tile must have landed
          cu.qs = qc % C::QS;
          mbar_wait_at(Q_FULL(t, cu.qs), (qc / C::QS) & 1, 4, qc, cu.idx);
          ++qc;
        }
        PROF_MARK(1);  // Q wait
        if (C::SEP_P && qkc > 0) {
          mbar_wait_at(S_FREE, (qkc - 1) & 1, 5, qkc, cu.idx);
          tc_fence_after();
        }
        PROF_MARK(2);  // S_FREE wait
        const uint32_t tS = tmem + C::col_s(t, qkc);
        ++qkc;
        const uint32_t qoff = C::OFF_Q + (2 * cu.qs + t) * C::TILE;
        const uint32_t koff = sK - sbase;
#pragma unroll
        for (int kk = 0; kk < D / 16; ++kk) {
          const uint32_t off = (kk / 4) * C::CHUNK + (kk % 4) * 32;
          if (!(FMHA_ABL & 8)) umma_ss_elect(tS, desc0 + ((qoff + off) >> 4), desc0 + ((koff + off) >> 4), IDESC_QK, kk > 0);
        }
        umma_commit_elect(S_FULL);
        TRACE_EV(EV_MMA_QK, t * 64 + cu.j);
        if (cu.j + 1 == n) umma_commit_elect(Q_EMPTY(t, cu.qs));  // last QK of the tile: Q slot reusable
        umma_commit_elect(KV_EMPTY(kidx % C::NS));
        PROF_MARK(3);  // QK issue
      };
      // O_t (+)= P_t V_{t,j} once the softmax wrote P_t (and rescaled its rows of O_t if needed);
      // the first PV of an item overwrites O_t, so it also waits until the epilogue has read O_t
      auto pv_entry = [&](Cursor& cu, uint32_t vidx) {
        PROF_MARK(8);
        const uint32_t sV = ring_wait(vidx);
        PROF_MARK(4);  // V ring wait
        if (cu.j == 0) {
          mbar_wait_at(O_EMPTY, (oc & 1) ^ 1, 7, oc, cu.idx);
          ++oc;
        }
        PROF_MARK(5);  // O_EMPTY wait
        if (C::ROT)
          mbar_wait_at((pc & 1) ? P_FULL2 : P_FULL, (pc >> 1) & 1, 6, pc, cu.idx);
        else
          mbar_wait_at(P_FULL, pc & 1, 6, pc, cu.idx);
        const uint32_t tP = tmem + C::col_p(t, pc);
        ++pc;
        PROF_MARK(6);  // P_FULL wait
        TRACE_EV(EV_MMA_P, t * 64 + cu.j);
        tc_fence_after();
        // LSUM_MMA: the second 64-column N chunk of B (columns 64..79 used) is the ones atom, one
        // leading-byte offset above this ring slot
        const uint64_t vdesc = C::LSUM_MMA ? sdesc_sw128(sbase, C::OFF_ONES - (sV - sbase), 1024) : vdesc0;
#pragma unroll
        for (int kk = 0; kk < 8; ++kk)
          if (!(FMHA_ABL & 8)) umma_ts_elect(tO, tP + kk * 8, vdesc + ((sV - sbase + kk * 2048) >> 4), IDESC_PV, (cu.j > 0 || kk > 0));
        if (C::SEP_P) umma_commit_elect(PV_DONE);   // P_t may be overwritten
        if (cu.j + 1 == cu.w.n(t)) umma_commit_elect(O_FULL);  // O_t final: epilogue
        TRACE_EV(EV_MMA_PV, t * 64 + cu.j);
        umma_commit_elect(KV_EMPTY(vidx % C::NS));
        PROF_MARK(7);  // PV issue
      };
      // walk the ring entries of step j in ring order: use this tile's, release the rest
      auto issue_qk = [&](Cursor& cu) {
        for (int u = 0; u < (cu.w.shared ? 1 : 2); ++u) {
          const int uu = cu.w.shared ? t : u;  // tile whose entry this is
          if (cu.j >= cu.w.n(uu)) {
            if (cu.w.shared) release(cu.base + cu.w.k_index(t, cu.j));
            continue;
          }
          const uint32_t kidx = cu.base + cu.w.k_index(uu, cu.j);
          if (uu == t) qk_entry(cu, kidx);
          else release(kidx);
        }
      };
      auto issue_pv = [&](Cursor& cu) {
        for (int u = 0; u < (cu.w.shared ? 1 : 2); ++u) {
          const int uu = cu.w.shared ? t : u;
          if (cu.j >= cu.w.n(uu)) {
            if (cu.w.shared) release(cu.base + cu.w.k_index(t, cu.j) + 1);
            continue;
          }
          const uint32_t vidx = cu.base + cu.w.k_index(uu, cu.j) + 1;
          if (uu == t) pv_entry(cu, vidx);
          else release(vidx);
        }
      };
      // One loop, one call site each (keeps the issuing code small).  With separate P the QK
      // cursor leads (QK of step s+1 before PV of step s); with P over S it follows.
      bool started = false;
      while (cp.valid) {
        if (!C::SEP_P && started) {
          issue_pv(cp);
          advance(cp);
          if (!cp.valid) break;
        }
        if (cq.valid) {
          issue_qk(cq);
          advance(cq);
        }
        if (C::SEP_P && started) {
          issue_pv(cp);
          advance(cp);
        }
        started = true;
      }
#if FMHA_PROF
      PROF_MARK(9);
      if (lane == 0 && g_fmha_trace) {
        unsigned long long* dst = g_fmha_trace + (static_cast<size_t>(blockIdx.x) * 16 + warp) * 16;
        for (int k = 0; k < 16; ++k) dst[k] = prof_acc[k];
        dst[15] = qkc;
      }
#endif
    }
  } else if (warp < C::W_CORR) {
    asm volatile("setmaxnreg.inc.sync.aligned.u32 %0;" ::"n"(C::REG_SOFTMAX));
    // ============================================================== softmax (a5, a6)
    const int t = warp >> 2, quad = warp & 3;
    const int row = quad * 32 + lane;
    const uint32_t lane_off = static_cast<uint32_t>(quad * 32) << 16;
    // this row's S (128 columns) and P (64) of step g: tmem + lane_off + col_s / col_p(t, g)
    const uint32_t S_FULL = BAR(C::B_S_FULL + t), P_FULL = BAR(C::B_P_FULL + t), P_FULL2 = BAR(C::B_P_FULL2 + t);
    const uint32_t PV_DONE = BAR(C::B_PV_DONE + t), S_FREE = BAR(C::B_S_FREE + t);
    const uint32_t L_FULL = BAR(C::B_L_FULL + t), L_EMPTY = BAR(C::B_L_EMPTY + t);
    const uint32_t tO = tmem + lane_off + C::col_o(t);  // this row of O_t
    const uint32_t my_turn = 2 + 2 * quad + t, other_turn = 3 + 2 * quad - t;  // 64-thread barriers
    if (C::TURNS && t == 1) named_bar_arrive(2 + 2 * quad, 64);  // tile 0 goes first
    const float c = p.scale_log2;
    const int off = p.seq_kv - p.seq_q;
    // g = real steps this thread has done so far: the phase count of S_FULL and PV_DONE
    uint32_t g = 0, lc = 0;
    PROF_DECL
    for (int kk = 0, idx; (idx = item_at<SCHED>(p, sched, kk)) >= 0; ++kk) {
      const WorkItem w = get_item<PAIRX, VL, SPLIT_KIND, SCHED, TAIL>(p, sched, idx);
      const int n = w.n(t);
      const int N = C::TURNS ? max(w.n0, w.n1) : n;
      TRACE_EV(EV_ITEM, 1);
      const int qi = w.row0(t) + row;
      int lim = w.kv(t);  // keys j < lim are visible to this row
      if (p.mask_kind == MASK_CAUSAL) lim = min(lim, qi + off + 1);
      if (qi >= w.len(t)) lim = 0;  // row past the sequence's end: never stored, so no work
      const int lim_w = __reduce_max_sync(0xffffffffu, lim);  // keys >= lim_w: masked for the warp
      float m_ref = -INFINITY;  // max used as the exp2 reference (lags the true max by < 2^8)
      float l = 0.f;            // row sum relative to m_ref
      uint32_t s[128];  // this row's scores S_{t,j}
      bool pre = false;  // PREFETCH_S: S_{t,j} already requested into s
      for (int j = 0; j < N; ++j) {
        if (j >= n) {  // no KV tile j for this tile: pass the turn on
          named_bar_sync(my_turn, 64);
          TRACE_EV(EV_XCHG, 100 + j);
          named_bar_arrive(other_turn, 64);
          continue;
        }
        const uint32_t tS = tmem + lane_off + C::col_s(t, g);  // this row's 128 S columns of step g
        if constexpr (BIAS && C::BIAS_PF4) {  // lanes 0-3: this step's four bias lines, 4-7: the next step's
          if (lane < 8) {
            const float* brow = p.key_bias + static_cast<size_t>(p.div_heads.div(w.bh(t))) * p.key_bias_stride;
            const int pf = (w.jbt(t) + j) * 128 + 32 * lane;
            if (pf < p.seq_kv) asm volatile("prefetch.global.L1 [%0];" ::"l"(brow + pf));
          }
        }
        PROF_COUNT(15);
        PROF_MARK(0);  // loop turnaround since the last P_FULL (or the item start)
        if (!pre) {
          TRACE_EV(EV_S_WAIT, j);
          mbar_wait_at(S_FULL, g & 1, 8, g, idx);
          PROF_MARK(1);  // S_FULL wait
          TRACE_EV(EV_S_READY, j);
          tc_fence_after();
          if constexpr (C::PREFETCH_S) {
#pragma unroll
            for (int q = 0; q < 4; ++q)
              tmem_ld_32x32b_x32(tS + 32 * q, *reinterpret_cast<uint32_t(*)[32]>(&s[32 * q]));
          }
        }
        if constexpr (C::PREFETCH_S) {
          tmem_wait_ld();
          reg_fence(s);
        }
        // SPLIT_LD: load the first 64 columns, wait, start the second 64 and take the first half's
        // max while they land (the max of the second half follows the second wait)
        float mxh = -INFINITY;
        if constexpr (C::PREFETCH_S) {
          // (loaded above)
        } else if constexpr (C::SPLIT_LD) {
          tmem_ld_32x32b_x32(tS, *reinterpret_cast<uint32_t(*)[32]>(&s[0]));
          tmem_ld_32x32b_x32(tS + 32, *reinterpret_cast<uint32_t(*)[32]>(&s[32]));
          tmem_wait_ld();
          reg_fence(*reinterpret_cast<uint32_t(*)[64]>(&s[0]));
          tmem_ld_32x32b_x32(tS + 64, *reinterpret_cast<uint32_t(*)[32]>(&s[64]));
          tmem_ld_32x32b_x32(tS + 96, *reinterpret_cast<uint32_t(*)[32]>(&s[96]));
          const int rem0 = lim - (w.jbt(t) + j) * 128;
          if (!BIAS && rem0 >= 64) {
            float a0 = -INFINITY, a1 = -INFINITY, a2 = -INFINITY, a3 = -INFINITY;
#pragma unroll
            for (int k = 0; k < 64; k += 8) {
              a0 = fmax3(a0, __uint_as_float(s[k]), __uint_as_float(s[k + 1]));
              a1 = fmax3(a1, __uint_as_float(s[k + 2]), __uint_as_float(s[k + 3]));
              a2 = fmax3(a2, __uint_as_float(s[k + 4]), __uint_as_float(s[k + 5]));
              a3 = fmax3(a3, __uint_as_float(s[k + 6]), __uint_as_float(s[k + 7]));
            }
            mxh = fmaxf(fmaxf(a0, a1), fmaxf(a2, a3));
          }
          tmem_wait_ld();
          reg_fence(*reinterpret_cast<uint32_t(*)[64]>(&s[64]));
        } else if (FMHA_ABL & 1) {
#pragma unroll
          for (int k = 0; k < 128; ++k) s[k] = __float_as_uint(0.01f * (k & 7));
          reg_fence(s);
        } else {
#pragma unroll
          for (int q = 0; q < 4; ++q)
            tmem_ld_32x32b_x32(tS + 32 * q, *reinterpret_cast<uint32_t(*)[32]>(&s[32 * q]));
          tmem_wait_ld();
          reg_fence(s);
        }
        PROF_MARK(2);  // S TMEM load
        if (C::SEP_P) {  // S_t read: the tensor core may overwrite it with S_{t,j+1}
          tc_fence_before();
          FMHA_ROW_ARRIVE(S_FREE);
        }
        const int rem = lim - (w.jbt(t) + j) * 128;
        // 32-key chunks no row of this warp can see are skipped: their P is stored as zeros
        const int rem_w = lim_w - (w.jbt(t) + j) * 128;
        if constexpr (BIAS) {  // s' = s + bias / scale (R20), 32 keys at a time; L1-resident, the
                               // next step's keys prefetched (every softmax warp reads the same row)
          const int b = p.div_heads.div(w.bh(t));
          const float* brow = p.key_bias + static_cast<size_t>(b) * p.key_bias_stride;
          const int key0 = (w.jbt(t) + j) * 128;
          // a step's 128 keys are 512 B = four 128-B lines (BIAS_PF4 prefetches all of this and the
          // next step's; otherwise only the next step's first line, and the other three miss L1)
          if constexpr (C::BIAS_PF4) {
            // (issued at the top of the step, before the S wait)
          } else if (key0 + 128 < p.seq_kv) {
            asm volatile("prefetch.global.L1 [%0];" ::"l"(brow + key0 + 128));
          }
          // (clamp: last float4 of the row, >= 0 since key0 < seq_kv <= stride, all multiples of 4)
          const unsigned cap4 = static_cast<unsigned>(p.key_bias_stride - 4 - key0) >> 2;
          const float4* bk0 = reinterpret_cast<const float4*>(brow + key0);
#pragma unroll
          for (int q = 0; q < 4; ++q) {
            float4 bq[8];
#pragma unroll
            for (int u = 0; u < 8; ++u) {
              const int col = key0 + 32 * q + 4 * u;
              if constexpr (C::BIAS_CLAMP)  // keys >= seq_kv are set to -inf below, whatever they load
                bq[u] = __ldg(bk0 + min(static_cast<unsigned>(8 * q + u), cap4));
              else
                bq[u] = col < p.seq_kv ? __ldg(reinterpret_cast<const float4*>(brow + col)) : make_float4(0.f, 0.f, 0.f, 0.f);
            }
#pragma unroll
            for (int u = 0; u < 8; ++u) {
              const int k = 32 * q + 4 * u;
              const float2 is2 = make_float2(p.inv_scale, p.inv_scale);
              const float2 a = ffma2(make_float2(bq[u].x, bq[u].y), is2,
                                     make_float2(__uint_as_float(s[k]), __uint_as_float(s[k + 1])));
              const float2 bb2 = ffma2(make_float2(bq[u].z, bq[u].w), is2,
                                       make_float2(__uint_as_float(s[k + 2]), __uint_as_float(s[k + 3])));
              s[k] = __float_as_uint(a.x);
              s[k + 1] = __float_as_uint(a.y);
              s[k + 2] = __float_as_uint(bb2.x);
              s[k + 3] = __float_as_uint(bb2.y);
            }
          }
        }
        if constexpr (BIAS2D) {  // s' = s + attn_bias[b, h, qi, key] / scale (R21): this row's 128 keys as
                                 // 16 x 16-byte loads (clamped to the row; keys >= seq_kv are masked below)
          const int bb = t ? w.bat1 : w.bat0, hh = t ? w.head1 : w.head;
          const uint4* brow = reinterpret_cast<const uint4*>(
              p.attn_bias + bb * p.ab_sb + hh * p.ab_sh + static_cast<long long>(min(qi, p.seq_q - 1)) * p.ab_sq);
          const int c80 = (w.jbt(t) + j) * 16;  // first 8-key group of this step
          const float2 is2 = make_float2(p.inv_scale, p.inv_scale);
#pragma unroll
          for (int q = 0; q < 4; ++q) {
            uint4 bq[4];
#pragma unroll
            for (int u = 0; u < 4; ++u) bq[u] = __ldg(brow + min(c80 + 4 * q + u, p.bias_cols8 - 1));
#pragma unroll
            for (int u = 0; u < 4; ++u) {
              const uint32_t hw[4] = {bq[u].x, bq[u].y, bq[u].z, bq[u].w};
#pragma unroll
              for (int e = 0; e < 4; ++e) {
                const int k = 32 * q + 8 * u + 2 * e;
                float2 bf;
                if constexpr (BF16) {
                  bf = __bfloat1622float2(*reinterpret_cast<const __nv_bfloat162*>(&hw[e]));
                } else {
                  bf = __half22float2(*reinterpret_cast<const __half2*>(&hw[e]));
                }
                const float2 r = ffma2(bf, is2, make_float2(__uint_as_float(s[k]), __uint_as_float(s[k + 1])));
                s[k] = __float_as_uint(r.x);
                s[k + 1] = __float_as_uint(r.y);
              }
            }
          }
        }
        if (rem < 128) {  // boundary tile for this row (a5)
#pragma unroll
          for (int k = 0; k < 128; ++k)
            if (k >= rem) s[k] = __float_as_uint(-INFINITY);
        }
        // SUMCHK: once the row has a reference, only the scores of the polynomial-exp2 columns are
        // max-reduced (the polynomial needs x <= 8); the MUFU columns are checked after the fact by
        // the step's sum of p (a p > 2^15 makes the sum exceed 2^15, an overflow makes it inf), and a
        // step that fails the check is redone from the full max (redo_step below).
        bool full_max = true;
        if constexpr (SUMCHK) {
          if (m_ref != -INFINITY) {
            float pa = -INFINITY, pb = -INFINITY;
#pragma unroll
            for (int q = 0; q < 64; q += 2) {
              if (XS::poly_pair(q)) pa = fmax3(pa, __uint_as_float(s[2 * q]), __uint_as_float(s[2 * q + 1]));
              if (XS::poly_pair(q + 1)) pb = fmax3(pb, __uint_as_float(s[2 * q + 2]), __uint_as_float(s[2 * q + 3]));
            }
            full_max = (fmaxf(pa, pb) - m_ref) * c > 8.f;
          }
        }
        float m_new = m_ref;
        if (full_max) {
        // (SPLIT_LD: the first 64 columns' max is mxh when none of them is masked, else recomputed)
        const int k_max0 = (C::SPLIT_LD && mxh != -INFINITY) ? 64 : 0;
        float mx0 = fmaxf(m_ref, mxh), mx1 = -INFINITY, mx2 = -INFINITY, mx3 = -INFINITY;
#pragma unroll
        for (int k = 0; k < 128; k += 8) {
          if (C::SPLIT_LD && k < k_max0) continue;
          mx0 = fmax3(mx0, __uint_as_float(s[k]), __uint_as_float(s[k + 1]));
          mx1 = fmax3(mx1, __uint_as_float(s[k + 2]), __uint_as_float(s[k + 3]));
          mx2 = fmax3(mx2, __uint_as_float(s[k + 4]), __uint_as_float(s[k + 5]));
          mx3 = fmax3(mx3, __uint_as_float(s[k + 6]), __uint_as_float(s[k + 7]));
        }
        m_new = (FMHA_ABL & 2) ? 1.f : fmaxf(fmaxf(mx0, mx1), fmaxf(mx2, mx3));
        }
        PROF_MARK(3);  // masks, bias, row max
        TRACE_EV(EV_MAX_DONE, j);
        // Lazy rescale: keep the old reference while the max grows by < 8 in the log2 domain (the
        // p's then stay <= 2^8, exact in fp32 and in fp16/bf16 range); l and O share the reference.
        float alpha = 1.f;
        if (m_new > m_ref && (m_ref == -INFINITY || (m_new - m_ref) * c > 8.f)) {
          alpha = (m_ref == -INFINITY) ? 0.f : ex2((m_ref - m_new) * c);
          m_ref = m_new;
        }
        float mc = (m_ref == -INFINITY) ? 0.f : m_ref * c;
        TRACE_EV(EV_COR_ST, j);
        // PV_{t,j-1} must be done before P_t is overwritten (separate P) and before O_t is rescaled.
        // (With P over S, S_{t,j} was computed after PV_{t,j-1}: S_FULL already implies it.)
        // (ROT: P_g has its own region; PV_DONE is then waited only before a rescale, below)
        if (C::SEP_P && !C::ROT && g > 0) {
          mbar_wait_at(PV_DONE, (g - 1) & 1, 10, g, idx);
          tc_fence_after();
        }
        PROF_MARK(4);  // rescale decision + PV_DONE wait
        TRACE_EV(EV_COR_PV, j);  // after the PV_DONE wait
        const uint32_t gs = g;  // this step's index (the rotation of S / P)
        const uint32_t tP = tmem + lane_off + C::col_p(t, gs);
        ++g;
        // P = exp2(c*s - c*m_ref) (a6), rounded to the I/O type, stored to TMEM for the PV MMA
        float2 acc0 = make_float2(0.f, 0.f), acc1 = make_float2(0.f, 0.f);
        float mcv = mc;
        // two instances: no chunk test at all on unmasked steps (the common case), so ptxas can
        // interleave the chunks freely; per-chunk skipping on steps with masked columns
        auto exp_phase = [&](auto skip_tag, auto turn_tag) {
          constexpr bool SKIP = decltype(skip_tag)::value;
          constexpr bool TURN = decltype(turn_tag)::value;  // false: a SUMCHK redo, already inside the turn
          // DEFER_ST: the tcgen05.st of a post-turn chunk's P is issued after the next chunk's math
          // (1: all at the end of the phase; 2: one chunk later) -- ptxas does not move MUFU work of
          // a later chunk above a tcgen05.st, so storing each chunk right away left a burst of
          // back-to-back MUFUs with nothing else to issue at the end of every chunk.
          uint32_t pk_all[4][16];
#pragma unroll
        for (int hh = 0; hh < 4; ++hh) {
          if (TURN && hh == XS::PRE_CHUNKS) {
            // The exponentials are register-only work that ptxas would hoist above the barrier:
            // round-trip their input through shared memory, which bar.sync does order.
            const uint32_t slot = sbase + C::OFF_MC + (t * 128 + row) * 4;
            asm volatile("st.shared.f32 [%0], %1;" ::"r"(slot), "f"(mc) : "memory");
            PROF_MARK(5);  // pre-turn chunks
            named_bar_sync(my_turn, 64);
            PROF_MARK(6);  // turn wait
            TRACE_EV(EV_XCHG, j);  // turn granted
            asm volatile("ld.volatile.shared.f32 %0, [%1];" : "=f"(mcv) : "r"(slot) : "memory");
          }
          uint32_t (&pk)[16] = pk_all[hh];
          const bool defer = C::DEFER_ST != 0 && hh >= XS::PRE_CHUNKS;
          if (C::DEFER_ST == 2 && hh > XS::PRE_CHUNKS) tmem_st_32x32b_x16(tP + 16 * (hh - 1), pk_all[hh - 1]);
          if (SKIP && 32 * hh >= rem_w) {
#pragma unroll
            for (int u = 0; u < 16; ++u) pk[u] = 0u;
            if (!defer) tmem_st_32x32b_x16(tP + 16 * hh, pk);
            continue;
          }
#pragma unroll
          for (int u = 0; u < 16; u += 2) {
            const int k = 32 * hh + 2 * u;
            float2 x0 = ffma2(make_float2(__uint_as_float(s[k]), __uint_as_float(s[k + 1])), c, -mcv);
            float2 x1 = ffma2(make_float2(__uint_as_float(s[k + 2]), __uint_as_float(s[k + 3])), c, -mcv);
#ifdef FMHA_FAKE_EXP  // timing experiment only: exponentials replaced by a trivial op (wrong results)
            if (true) {
              x0 = fadd2(x0, make_float2(1.f, 1.f));
            } else
#endif
            if (XS::poly_pair(16 * hh + u)) {
              x0 = exp2_poly2(x0);
            } else {
              x0.x = ex2(x0.x);
              x0.y = ex2(x0.y);
            }
#ifdef FMHA_FAKE_EXP
            if (true) {
              x1 = fadd2(x1, make_float2(1.f, 1.f));
            } else
#endif
            if (XS::poly_pair(16 * hh + u + 1)) {
              x1 = exp2_poly2(x1);
            } else {
              x1.x = ex2(x1.x);
              x1.y = ex2(x1.y);
            }
            if constexpr (!C::LSUM_MMA) {  // (LSUM_MMA: the PV MMA sums P)
              acc0 = fadd2(acc0, x0);
              acc1 = fadd2(acc1, x1);
            }
            pk[u] = pack2<BF16>(x0.x, x0.y);
            pk[u + 1] = pack2<BF16>(x1.x, x1.y);
          }
          if (!defer && !(FMHA_ABL & 4)) tmem_st_32x32b_x16(tP + 16 * hh, pk);
          if (FMHA_ABL & 4) reg_fence(pk);
        }
        if constexpr (C::DEFER_ST == 1) {
#pragma unroll
          for (int hh = XS::PRE_CHUNKS; hh < 4; ++hh) tmem_st_32x32b_x16(tP + 16 * hh, pk_all[hh]);
        } else if constexpr (C::DEFER_ST == 2) {
          tmem_st_32x32b_x16(tP + 16 * 3, pk_all[3]);
        }
        };
        if (FMHA_ABL & 16) {  // (timing ablation: no exponential phase, only its turn)
          if (C::TURNS) named_bar_sync(my_turn, 64);
        } else if (rem_w >= 128)
          exp_phase(std::false_type{}, std::true_type{});
        else
          exp_phase(std::true_type{}, std::true_type{});
        if constexpr (SUMCHK) {  // redo_step: some p of this row exceeded 2^15 (rare; inside the turn)
          const bool bad = !(((acc0.x + acc0.y) + (acc1.x + acc1.y)) <= 32768.f);
          if (__any_sync(0xffffffffu, bad)) {
            if (bad) {  // full max, lazy-rescale factor, new reference (alpha was 1: no full max ran)
              float mx0 = m_ref, mx1 = -INFINITY;
#pragma unroll
              for (int k = 0; k < 128; k += 4) {
                mx0 = fmax3(mx0, __uint_as_float(s[k]), __uint_as_float(s[k + 1]));
                mx1 = fmax3(mx1, __uint_as_float(s[k + 2]), __uint_as_float(s[k + 3]));
              }
              const float mn = fmaxf(mx0, mx1);
              alpha = ex2((m_ref - mn) * c);
              m_ref = mn;
              mc = m_ref * c;
            }
            mcv = mc;  // (rows that passed recompute bit-identical p)
            acc0 = make_float2(0.f, 0.f);
            acc1 = make_float2(0.f, 0.f);
            tmem_wait_st();  // the first pass's P stores have landed before they are overwritten
            if (rem_w >= 128)
              exp_phase(std::false_type{}, std::false_type{});
            else
              exp_phase(std::true_type{}, std::false_type{});
          }
        }
        if (C::TURNS) named_bar_arrive(other_turn, 64);
        PROF_MARK(7);  // exponentials inside the turn
        TRACE_EV(EV_EXP_DONE, j);
        // lazy rescale of this warp's rows of O_t (a7), after the exponentials so that S is no
        // longer live; at j = 0 PV overwrites O_t instead
        if (j > 0 && __any_sync(0xffffffffu, alpha != 1.f)) {
          if (C::ROT) {  // O_t must hold PV_{t,gs-1}: PV_DONE's completions run one behind the step count,
                         // so the parity of completion gs-1 is unambiguous although most steps skip it
            mbar_wait_at(PV_DONE, (gs - 1) & 1, 10, gs, idx);
            tc_fence_after();
          }
#pragma unroll 1
          for (int q = 0; q < D / 32; ++q) {
            uint32_t o[32];
            tmem_ld_32x32b_x32(tO + 32 * q, o);
            tmem_wait_ld();
            reg_fence(o);
#pragma unroll
            for (int k = 0; k < 32; ++k) o[k] = __float_as_uint(__uint_as_float(o[k]) * alpha);
            tmem_st_32x32b_x32(tO + 32 * q, o);
          }
          if constexpr (C::LSUM_MMA) {  // the row-sum columns share O_t's reference
            uint32_t o[16];
            tmem_ld_32x32b_x16(tO + D, o);
            tmem_wait_ld();
            reg_fence(o);
#pragma unroll
            for (int k = 0; k < 16; ++k) o[k] = __float_as_uint(__uint_as_float(o[k]) * alpha);
            tmem_st_32x32b_x16(tO + D, o);
          }
        }
        // PREFETCH_S: request S_{t,j+1} before releasing P_{t,j}, so its TMEM load overlaps the P
        // stores draining and the loop turnaround.  Safe only with a separate P buffer: QK_{t,j+1} is
        // then issued before PV_{t,j} (it waits for S_FREE_{t,j}, not for P_FULL_{t,j}), and its K
        // tile never waits for a V slot released by PV_{t,j} (ring order, NS = 6).
        // Only when S_{t,j+1} is already there (a blocking wait here would hold back P_FULL_{t,j}).
        pre = C::PREFETCH_S && j + 1 < n && __all_sync(0xffffffffu, mbar_try_wait(S_FULL, g & 1));
        if (pre) {
          TRACE_EV(EV_S_READY, j + 1);
          tc_fence_after();
#pragma unroll
          for (int q = 0; q < 4; ++q)
            tmem_ld_32x32b_x32(tS + 32 * q, *reinterpret_cast<uint32_t(*)[32]>(&s[32 * q]));
        }
        PROF_MARK(8);  // rescale of O
        tmem_wait_st();
        PROF_MARK(9);  // P store drain
        TRACE_EV(EV_EPI, j);  // P stores landed
        // ROT: every PV_DONE phase is still consumed in order, here, before P_FULL_g lets PV_g start
        // (PV_{g-1} has had a whole exponential phase to finish, so this rarely blocks; waiting any
        // later could alias two phases, and compute-sanitizer's synccheck requires each phase waited)
        if (C::ROT && FMHA_ROT_PVWAIT && gs > 0) mbar_wait_at(PV_DONE, (gs - 1) & 1, 10, gs, idx);
        tc_fence_before();
        FMHA_ROW_ARRIVE((C::ROT && (gs & 1)) ? P_FULL2 : P_FULL);
        l = l * alpha + ((acc0.x + acc0.y) + (acc1.x + acc1.y));
      }
      if (!w.has(t)) continue;
      // the epilogue has read the previous item's sums (without this wait the softmax can run two
      // items ahead and L_FULL's phase parity would alias)
      TRACE_EV(EV_ITEM, 2);
      mbar_wait_at(L_EMPTY, (lc & 1) ^ 1, 15, lc, idx);
      TRACE_EV(EV_ITEM, 3);
      ++lc;
      s_lsum[t * 128 + row] = l;
      if constexpr (TAIL) reinterpret_cast<float*>(smem + C::OFF_MREF)[t * 128 + row] = (m_ref == -INFINITY) ? -INFINITY : m_ref * c;
      if constexpr (SPLIT) {  // this split's row statistics (rows inside the sequence only)
        if (qi < p.seq_q) {
          const size_t o = (static_cast<size_t>(w.splt(t)) * p.num_units + w.bh(t)) * p.seq_q + qi;
          p.ws_m[o] = (m_ref == -INFINITY) ? -INFINITY : m_ref * c;
          if constexpr (!C::LSUM_MMA) p.ws_l[o] = l;  // (LSUM_MMA: the epilogue reads l from TMEM)
        }
      }
      __syncwarp();
      FMHA_ROW_ARRIVE(L_FULL);
      PROF_MARK(10);  // item end: L_EMPTY wait, row sums
    }
    if (C::TURNS && t == 0) named_bar_sync(2 + 2 * quad, 64);  // consume tile 1's last hand-over
#if FMHA_PROF
    PROF_MARK(11);
    if (lane == 0 && g_fmha_trace) {
      unsigned long long* dst = g_fmha_trace + (static_cast<size_t>(blockIdx.x) * 16 + warp) * 16;
      for (int k = 0; k < 16; ++k) dst[k] = prof_acc[k];
    }
#endif
  } else {
    asm volatile("setmaxnreg.dec.sync.aligned.u32 %0;" ::"n"(C::REG_CORR));
    // ================================================================ epilogue (a9)
    const int quad = warp & 3;
    const int row = quad * 32 + lane;
    const uint32_t lane_off = static_cast<uint32_t>(quad * 32) << 16;
    // phase parities of L_FULL / O_FULL per tile (bit t): registers, not a runtime-indexed array
    // (which lived in local memory)
    uint32_t ofbits = 0, lbits = 0;
    for (int kk = 0, idx; (idx = item_at<SCHED>(p, sched, kk)) >= 0; ++kk) {
      const WorkItem w = get_item<PAIRX, VL, SPLIT_KIND, SCHED, TAIL>(p, sched, idx);
      // ------------------------------------------------------------ epilogue per tile (a9)
#pragma unroll 1
      for (int t = 0; t < 2; ++t) {
        if (!w.has(t)) continue;
        mbar_wait_at(BAR(C::B_L_FULL + t), (lbits >> t) & 1, 13, t, idx);
        TRACE_EV(EV_EPI, 100 + t);
        lbits ^= 1u << t;
        float l = s_lsum[t * 128 + row];
        const float mref = TAIL ? reinterpret_cast<const float*>(smem + C::OFF_MREF)[t * 128 + row] : 0.f;
        __syncwarp();
        FMHA_ROW_ARRIVE(BAR(C::B_L_EMPTY + t));
        const int n = w.n(t);
        if (n > 0) {
          mbar_wait_at(BAR(C::B_O_FULL + t), (ofbits >> t) & 1, 14, t, idx);  // last PV of this tile
          TRACE_EV(EV_EPI, 110 + t);
          ofbits ^= 1u << t;
          tc_fence_after();
        }
        if constexpr (TAIL) {
          if (w.tail >= 0 && !(FMHA_SK_ABL & 2)) {  // stream-K piece: this split's state to the workspace, O
                              // as float4 columns [D/4][128 rows] (a warp's store instruction writes 512
                              // contiguous bytes; the merge reads it back the same way, conflict-free)
            float* dst = p.ws_tail + static_cast<size_t>((w.tail * p.tail_splits + w.split) * 2 + t) * (128 * (D + 2));
            const uint32_t tO = tmem + lane_off + C::col_o(t);
#pragma unroll 1
            for (int q = 0; q < D / 32; ++q) {
              uint32_t o[32];
              if (n > 0) {
                tmem_ld_32x32b_x32(tO + 32 * q, o);
                tmem_wait_ld();
                reg_fence(o);
              } else {
#pragma unroll
                for (int k = 0; k < 32; ++k) o[k] = 0u;
              }
#pragma unroll
              for (int c4 = 0; c4 < 8; ++c4)
                st_global_v4(dst + ((8 * q + c4) * 128 + row) * 4, o[4 * c4], o[4 * c4 + 1], o[4 * c4 + 2], o[4 * c4 + 3]);
            }
            dst[D * 128 + row] = mref;
            dst[(D + 1) * 128 + row] = l;
            if (n > 0) {
              tc_fence_before();
              FMHA_ROW_ARRIVE(BAR(C::B_O_EMPTY + t));
            }
            continue;
          }
        }
        if constexpr (C::LSUM_MMA) {  // l = O_t[row, D] (the ones column of the PV MMA)
          l = 0.f;
          if (n > 0) {
            uint32_t lv[1];
            tmem_ld_32x32b_x1(tmem + lane_off + C::col_o(t) + D, lv);
            tmem_wait_ld();
            l = __uint_as_float(lv[0]);
          }
          if constexpr (SPLIT) {
            const int qi = w.row0(t) + row;
            if (qi < p.seq_q) p.ws_l[(static_cast<size_t>(w.splt(t)) * p.num_units + w.bh(t)) * p.seq_q + qi] = l;
          }
        }
        const float inv_l = (l > 0.f) ? 1.f / l : 0.f;  // fully masked row -> 0 (R4)
        // varlen tile that crosses its sequence's end: a TMA store would overwrite the next
        // sequence's rows, so each thread stores its own row (if inside the sequence) instead
        const bool rowwise = VL && w.row0(t) + 128 > w.len(t);
        const uint32_t stg = sbase + C::OFF_STG + (t % C::NSTG) * C::STG_CHUNKS * C::CHUNK;
        if (row == 0) tma_store_wait_read0();  // previous store out of this staging buffer done
        named_bar_sync(1, 128);
        const uint32_t tO = tmem + lane_off + C::col_o(t);
#pragma unroll 1
        for (int q = 0; q < D / 32; ++q) {
          uint32_t o[32];
          if (n > 0 && !(FMHA_ABL & 32)) {
            tmem_ld_32x32b_x32(tO + 32 * q, o);
            tmem_wait_ld();
            reg_fence(o);
          } else {
#pragma unroll
            for (int k = 0; k < 32; ++k) o[k] = 0u;
          }
          const int col0 = 32 * q;
          if constexpr (SPLIT) {  // unnormalised fp32 partial O of this split, rows inside the sequence
            const int qi = w.row0(t) + row;
            if (qi < p.seq_q) {
              float* dst = p.ws_o + ((static_cast<size_t>(w.splt(t)) * p.num_units + w.bh(t)) * p.seq_q + qi) * D + col0;
#pragma unroll
              for (int u = 0; u < 8; ++u)
                st_global_v4(dst + 4 * u, o[4 * u], o[4 * u + 1], o[4 * u + 2], o[4 * u + 3]);
            }
            continue;
          }
          const uint32_t box = stg + ((col0 / 64) % C::STG_CHUNKS) * C::CHUNK + row * 128;
#pragma unroll
          for (int u = 0; u < 4; ++u) {
            const int unit = ((col0 % 64) / 8) + u;
            const uint32_t v0 = pack2<BF16>(__uint_as_float(o[8 * u + 0]) * inv_l, __uint_as_float(o[8 * u + 1]) * inv_l);
            const uint32_t v1 = pack2<BF16>(__uint_as_float(o[8 * u + 2]) * inv_l, __uint_as_float(o[8 * u + 3]) * inv_l);
            const uint32_t v2 = pack2<BF16>(__uint_as_float(o[8 * u + 4]) * inv_l, __uint_as_float(o[8 * u + 5]) * inv_l);
            const uint32_t v3 = pack2<BF16>(__uint_as_float(o[8 * u + 6]) * inv_l, __uint_as_float(o[8 * u + 7]) * inv_l);
            if (!rowwise) {
              st_shared_v4(box + ((unit ^ (row & 7)) << 4), v0, v1, v2, v3);
            } else if (row < w.len(t) - w.row0(t)) {  // varlen partial tile: rows inside the sequence
              const size_t tokn = static_cast<size_t>(w.tok(t) + w.row0(t) + row);
              st_global_v4(p.o_ptr + 2 * (tokn * p.o_row_elems + (t ? w.head1 : w.head) * D + col0 + 8 * u), v0, v1, v2, v3);
            }
          }
          if constexpr (C::STG_CHUNKS < D / 64) {  // half staging: store this 64-column chunk before the next
            if (!rowwise && (q & 1) && q + 1 < D / 32) {
              fence_proxy_async_smem();
              named_bar_sync(1, 128);
              if (row == 0) {
                constexpr bool vl = VL;
                tma_store_4d(&p.tmO, stg, (q / 2) * 64, w.c1(vl, t, w.row0(t)), w.c2(vl, t, w.row0(t)), w.c3(vl, t));
                tma_store_commit();
                tma_store_wait_read0();
              }
              named_bar_sync(1, 128);
            }
          }
        }
        if (n > 0) {  // O_t read: the next item's first PV may overwrite it
          tc_fence_before();
          FMHA_ROW_ARRIVE(BAR(C::B_O_EMPTY + t));
        }
        if (!rowwise && !SPLIT) {
          fence_proxy_async_smem();
          named_bar_sync(1, 128);
          if (row == 0) {
            constexpr bool vl = VL;
#pragma unroll
            for (int c2 = D / 64 - C::STG_CHUNKS; c2 < D / 64; ++c2)  // (half staging: the last chunk)
              tma_store_4d(&p.tmO, stg + (c2 % C::STG_CHUNKS) * C::CHUNK, c2 * 64, w.c1(vl, t, w.row0(t)),
                           w.c2(vl, t, w.row0(t)), w.c3(vl, t));
            tma_store_commit();
          }
        }
        TRACE_EV(EV_EPI, 120 + t);
      }
      if constexpr (TAIL && !(FMHA_SK_ABL & 1)) {
        if (w.tail >= 0) {
          // count this piece (after its stores are visible GPU-wide); the piece that counts last merges
          //   M = max_s mc_s,  O = sum_s 2^(mc_s - M) O_s / sum_s 2^(mc_s - M) l_s
          // (as fmha_splitkv_combine_kernel) and stores O through the usual staging buffer + TMA
          __threadfence();
          named_bar_sync(1, 128);
          volatile uint32_t* last_flag = reinterpret_cast<volatile uint32_t*>(smem + C::OFF_TMEMPTR + 4);
          if (row == 0) {
            const unsigned prev = atomicAdd(p.tail_cnt + w.tail, 1u);
            const bool last = prev == static_cast<unsigned>(p.tail_splits - 1);
            if (last) atomicExch(p.tail_cnt + w.tail, 0u);  // every piece has counted: reset for the next launch
            *last_flag = last ? 1u : 0u;
          }
          named_bar_sync(1, 128);
          if (*last_flag) {
            // The merging piece is its CTA's last item (the pieces fill the final round), so the Q + K/V
            // ring region [0, OFF_STG) is idle: the splits' states land there by bulk copies, 64 columns
            // of every split at a time (S x 32 KB) plus their row statistics (S x 1 KB), then each
            // thread merges its own row out of shared memory.
            const int S = p.tail_splits;
            constexpr int TS = 128 * (D + 2);       // floats per (piece, tile)
            constexpr uint32_t HALF = 128 * 64 * 4; // bytes of 64 columns of one split
            constexpr uint32_t STAT = MAX_TAIL_SPLITS * HALF;  // landing offset of the statistics
            static_assert(STAT + MAX_TAIL_SPLITS * 1024 <= C::OFF_STG, "merge landing zone");
            const uint32_t mbar = BAR(C::B_MERGE);
            uint32_t mph = 0;
            if (row == 0) {
              __threadfence();
              fence_proxy_async_all();  // the other pieces' generic stores, then async-proxy reads
            }
#pragma unroll 1
            for (int t = 0; t < 2; ++t) {
              if (!w.has(t)) continue;
              const float* src = p.ws_tail + static_cast<size_t>(w.tail * S * 2 + t) * TS;  // split s at + 2 s TS
              float wt[MAX_TAIL_SPLITS];
              float inv = 0.f;
              const uint32_t stg = sbase + C::OFF_STG + (t % C::NSTG) * C::STG_CHUNKS * C::CHUNK;
              if (row == 0) tma_store_wait_read0();
#pragma unroll 1
              for (int hf = 0; hf < D / 64; ++hf) {
                if (row == 0) {
                  fence_proxy_async_smem();  // earlier generic reads of the landing zone, then async writes
                  mbar_arrive_expect_tx(mbar, S * HALF + (hf == 0 ? S * 1024u : 0u));
                  for (int sp = 0; sp < S; ++sp) {
                    bulk_load(sbase + sp * HALF, src + sp * 2 * TS + hf * (HALF / 4), HALF, mbar);
                    if (hf == 0) bulk_load(sbase + STAT + sp * 1024, src + sp * 2 * TS + D * 128, 1024, mbar);
                  }
                }
                mbar_wait(mbar, mph);
                mph ^= 1;
                if (hf == 0) {  // M = max_s mc_s, weights 2^(mc_s - M), L = sum_s w_s l_s
                  const float* st = reinterpret_cast<const float*>(smem + STAT);
                  float M = -INFINITY, L = 0.f;
#pragma unroll
                  for (int sp = 0; sp < MAX_TAIL_SPLITS; ++sp)
                    if (sp < S) M = fmaxf(M, st[sp * 256 + row]);
#pragma unroll
                  for (int sp = 0; sp < MAX_TAIL_SPLITS; ++sp) {
                    wt[sp] = 0.f;
                    if (sp < S) {
                      const float m = st[sp * 256 + row];
                      if (m != -INFINITY) {  // (a split with no visible key for this row has l = 0, O = 0)
                        wt[sp] = ex2(m - M);
                        L += wt[sp] * st[sp * 256 + 128 + row];
                      }
                    }
                  }
                  inv = (L > 0.f) ? 1.f / L : 0.f;  // fully masked row -> 0 (R4)
#pragma unroll
                  for (int sp = 0; sp < MAX_TAIL_SPLITS; ++sp) wt[sp] *= inv;
                  named_bar_sync(1, 128);  // (the staging buffer's previous store has been read)
                }
#pragma unroll 1
                for (int q = 0; q < 2; ++q) {  // 32-column chunks of this half
                  float v[32];
#pragma unroll
                  for (int k = 0; k < 32; ++k) v[k] = 0.f;
#pragma unroll
                  for (int sp = 0; sp < MAX_TAIL_SPLITS; ++sp) {
                    if (sp < S) {
#pragma unroll
                      for (int c4 = 0; c4 < 8; ++c4) {
                        const float4 x = ld_shared_f4(sbase + sp * HALF + ((8 * q + c4) * 128 + row) * 16);
                        v[4 * c4] += wt[sp] * x.x;
                        v[4 * c4 + 1] += wt[sp] * x.y;
                        v[4 * c4 + 2] += wt[sp] * x.z;
                        v[4 * c4 + 3] += wt[sp] * x.w;
                      }
                    }
                  }
                  const int col0 = 64 * hf + 32 * q;
                  const uint32_t box = stg + ((col0 / 64) % C::STG_CHUNKS) * C::CHUNK + row * 128;
#pragma unroll
                  for (int u = 0; u < 4; ++u) {
                    const int unit = ((col0 % 64) / 8) + u;
                    st_shared_v4(box + ((unit ^ (row & 7)) << 4), pack2<BF16>(v[8 * u], v[8 * u + 1]),
                                 pack2<BF16>(v[8 * u + 2], v[8 * u + 3]), pack2<BF16>(v[8 * u + 4], v[8 * u + 5]),
                                 pack2<BF16>(v[8 * u + 6], v[8 * u + 7]));
                  }
                }
                if constexpr (C::STG_CHUNKS < D / 64) {  // half staging: store this chunk now
                  fence_proxy_async_smem();
                  named_bar_sync(1, 128);  // (also: every thread has read this half's landing zone)
                  if (row == 0) {
                    tma_store_4d(&p.tmO, stg, hf * 64, w.c1(false, t, w.row0(t)), w.c2(false, t, w.row0(t)), w.c3(false, t));
                    tma_store_commit();
                    tma_store_wait_read0();
                  }
                }
                named_bar_sync(1, 128);  // every thread has read this half's landing zone
              }
              if constexpr (C::STG_CHUNKS == D / 64) {
                fence_proxy_async_smem();
                named_bar_sync(1, 128);
                if (row == 0) {
#pragma unroll
                  for (int c2 = 0; c2 < D / 64; ++c2)
                    tma_store_4d(&p.tmO, stg + c2 * C::CHUNK, c2 * 64, w.c1(false, t, w.row0(t)), w.c2(false, t, w.row0(t)),
                                 w.c3(false, t));
                  tma_store_commit();
                }
              }
            }
          }
        }
      }
    }
    if (row == 0) tma_store_wait0();
  }

  tc_fence_before();
  __syncthreads();
  if (warp == C::W_MMA) {
    tc_fence_after();
    tmem_dealloc(tmem, C::TMEM_COLS);
  }
}

}  // namespace b200
