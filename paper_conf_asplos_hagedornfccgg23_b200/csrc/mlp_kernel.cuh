// mlp_kernel.cuh — the paper's fused multi-layer MLP on sm_100a (Fig. 11):
// L layers h_l = act(h_{l-1} W_l^T + b_l) of width N = K <= 128 in ONE kernel, every intermediate
// h_l kept on chip ("all intermediate tensors fit into the GPU's shared memory allowing to avoid
// communication via the slower global memory", L453).  SURVEY §8(f) f4.
//
// Persistent, one CTA per SM.  A CTA owns S <= R row tiles of 128 rows at a time (a "group"; S is
// a launch parameter, R the template's maximum: 2 at N = 128, 4 at N = 64) and walks them through
// all L layers in lockstep, so every W_l tile loaded into shared memory feeds S MMAs, and while one
// tile's epilogue runs the tensor core works on the others (a layer of one tile is a serial chain
// MMA -> epilogue -> next MMA; S tiles in flight hide it):
//   warp 0        TMA producer: the group's X tiles into ACT[r], then W_1 .. W_L (WS-stage ring)
//   warp 1 + r    MMA issuer of slot r: for each layer l, ACC_r = h_{l-1} W_l^T (tcgen05.mma M=128
//                 N=NW K=16, fp32 in TMEM columns [r NW, (r + 1) NW); layer 1 reads X from ACT[r] in
//                 shared memory (SS form), later layers h_{l-1} from TMEM (TS form)); commit to ACC_FULL[r]
//   last 16 warps four epilogue warpgroups.  Warpgroup w owns 64-column chunks h, h + H, ... of
//                 slots r = w / H, w / H + 4 / H, ... (thread = accumulator row): TMEM -> + b_l ->
//                 act -> one RNE rounding -> h_l, stored as the next layer's A operand:
//                 TA (default): fp16 pairs into TMEM columns A_r (K-major, the TS-form MMA's A, as the
//                   FMHA's P), so the MMA reads only W from shared memory;
//                 else: swizzled st.shared back into ACT[r] (K-major SW128, the layout TMA produces).
//                 After layer L, h_L goes to ACT[r] in shared memory and is TMA-stored to Y
//
//   smem  ACT[R] (X in, Y out) | W ring[WS] | fp32 bias ring
//   TMEM  ACC_r = columns [r NW, (r + 1) NW); TA: A_r = [R NW + r NW / 2, ...) (R = 2 at N = 128:
//         384 of 512 columns; the shared-memory variant uses R = 512 / N accumulators)
//
// Barriers (every producer -> consumer edge has its consumer -> producer partner):
//   X_FULL[r] / ACT_EMPTY[r]   TMA (X into ACT[r]) -> MMA;  the Y store out of ACT[r] has been read
//                              (bulk read-completion, signalled by the storing thread) -> TMA
//   W_FULL[s] / W_EMPTY[s]     TMA -> MMA warps -> TMA (count R: every slot warp commits once per layer)
//   ACC_FULL[r]                MMA commit -> epilogue of slot r
//   ACT_FULL[r] (count 128 H)  epilogue -> MMA: ACC_r drained AND ACT[r] holds h_l (the generic-proxy
//                              stores are fenced into the async proxy first)
// ACT[r] is overwritten by layer l's epilogue only after ACC_FULL: layer l's MMA, the last reader
// of ACT[r] = h_{l-1}, has completed.
#pragma once
#include "gemm_kernel.cuh"  // apply_act, make_map_2d_rows
#include "sm100.cuh"

namespace b200 {

struct MlpParams {
  CUtensorMap tmX;  // {NW, M, 1} box {64, 128, 1}, SWIZZLE_128B
  CUtensorMap tmW;  // {NW, NW, L} box {64, NW, 1}
  CUtensorMap tmY;  // as tmX
  const __half* bias;  // [L, NW] or nullptr
  int M, layers;
  int slots;       // S: row tiles per group (1 .. R)
  int num_groups;  // ceil(num_tiles / S)
  int num_tiles;   // ceil(M / 128)
};

template <int NW, bool TA>
struct MlpCfg {
  // TA: the intermediates h_1..h_{L-1} live in TMEM as the A operand of a TS-form MMA (fp16 pairs,
  // NW / 2 columns per slot) instead of shared memory; slots then need 1.5 NW columns each.
  static constexpr int R = TA ? (NW == 128 ? 2 : 4) : 512 / NW;  // slots in flight per CTA
  static constexpr int TMEM_A = R * NW;               // TA: A_r = columns [TMEM_A + r NW / 2, ...)
  // epilogue warpgroups per slot (H = 1: one warpgroup drains all NW columns of a slot, 64 at a time;
  // H = 2: two warpgroups, 64 columns each) -- one warpgroup per slot when there are 4 slots, so
  // the four slots' epilogues run side by side
  static constexpr int H = (TA && NW == 128) ? 2 : 1;
  static constexpr int EPI_WG = 4;                    // epilogue warpgroups
  static constexpr int SG = EPI_WG / H;               // slot groups: slot r -> warpgroups (r % SG) H + h
  static constexpr int SPW = (R + SG - 1) / SG;       // slots per epilogue warpgroup
  static constexpr int CHUNK = 128 * 128;             // one SW128 box of 128 rows x 64 16-bit elements
  static constexpr int ATILE = 128 * NW * 2;          // 128 rows x NW
  static constexpr int WCHUNK = NW * 128;             // NW rows x 64 elements
  static constexpr int WTILE = NW * NW * 2;
  static constexpr int WS = (NW == 128) ? (TA ? 3 : 2) : 4;  // W ring stages (smem budget at N = 128)
  static constexpr int OFF_ACT = 0;
  static constexpr int OFF_W = OFF_ACT + R * ATILE;
  static constexpr int OFF_BIAS = OFF_W + WS * WTILE;  // fp32 b_l ring: [slot group][2][NW]
  static constexpr int OFF_BAR = OFF_BIAS + SG * 2 * NW * 4;
  // barriers: X_FULL[R], ACT_EMPTY[R], ACC_FULL[R], ACT_FULL[R], W_FULL[WS], W_EMPTY[WS]
  static constexpr int NUM_BARS = 4 * R + 2 * WS;
  static constexpr int OFF_TMEMPTR = OFF_BAR + NUM_BARS * 8;
  static constexpr int SMEM_ALLOC = OFF_TMEMPTR + 16;
  // control warpgroups: warp 0 the TMA producer, warps 1..R one MMA issuer per slot (an mbarrier
  // wait of an issuing warp queues behind that warp's in-flight MMAs, so one warp walking all slots
  // left the tensor core idle between slots: measured ~420 cycles per slot)
  static constexpr int CW = (1 + R + 3) / 4;
  static constexpr int W_EPI = 4 * CW;                // first epilogue warp
  static constexpr int THREADS = 128 * CW + 128 * EPI_WG;
  static constexpr int REG_LAUNCH = (65536 / THREADS) / 8 * 8;
  static constexpr int REG_CTRL = 48;
  static constexpr int REG_EPI = (REG_LAUNCH + (REG_LAUNCH - REG_CTRL) * CW / EPI_WG) / 8 * 8;
  static_assert(128 * CW * REG_CTRL + 128 * EPI_WG * REG_EPI <= THREADS * REG_LAUNCH, "register pool");
  static_assert(NW == 64 || NW == 128, "width");
  static_assert(SMEM_ALLOC <= 232448, "shared memory budget");
};

template <int NW, int ACT, bool TA>
__global__ void __launch_bounds__(MlpCfg<NW, TA>::THREADS, 1) mlp_fused_kernel(const __grid_constant__ MlpParams p) {
  using C = MlpCfg<NW, TA>;
  constexpr int R = C::R;
  extern __shared__ __align__(1024) uint8_t smem[];
  const uint32_t sbase = smem_u32(smem);
  const uint32_t bar = sbase + C::OFF_BAR;
  auto X_FULL = [&](int r) { return bar + 8 * r; };
  auto ACT_EMPTY = [&](int r) { return bar + 8 * (R + r); };
  auto ACC_FULL = [&](int r) { return bar + 8 * (2 * R + r); };
  auto ACT_FULL = [&](int r) { return bar + 8 * (3 * R + r); };
  auto W_FULL = [&](int s) { return bar + 8 * (4 * R + s); };
  auto W_EMPTY = [&](int s) { return bar + 8 * (4 * R + C::WS + s); };
  uint32_t* tmem_holder = reinterpret_cast<uint32_t*>(smem + C::OFF_TMEMPTR);
  const int warp = warp_id(), lane = lane_id();
  const int S = p.slots, L = p.layers;
  TRACE_DECL  // debug timeline build only (FMHA_TRACE, tools/trace_mlp.py)

  if (threadIdx.x == 0) {
    if (sbase & 1023u) __trap();
    for (int r = 0; r < R; ++r) {
      mbar_init(X_FULL(r), 1);
      mbar_init(ACT_EMPTY(r), 1);
      mbar_init(ACC_FULL(r), 1);
      mbar_init(ACT_FULL(r), 128 * C::H);
    }
    for (int s = 0; s < C::WS; ++s) {
      mbar_init(W_FULL(s), 1);
      mbar_init(W_EMPTY(s), R);  // one commit per slot MMA warp (idle slots commit at once)
    }
    fence_mbar_init();
  }
  if (warp == 0 && lane == 0) {
    tma_prefetch_desc(&p.tmX);
    tma_prefetch_desc(&p.tmW);
    tma_prefetch_desc(&p.tmY);
  }
  if (warp == 1) {
    tmem_alloc(smem_u32(tmem_holder), 512);
    tmem_relinquish();
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  pdl_wait();  // global memory only from here on (PDL)
  pdl_trigger();
  const uint32_t tmem = *tmem_holder;
  // tiles of group g: g * S + r for r < ntiles(g)
  auto ntiles = [&](int g) { return min(S, p.num_tiles - g * S); };

  // registers: the launch gives every thread 65536 / THREADS; the control warpgroups (TMA, MMA,
  // idle warps) give some back to the epilogue warps (setmaxnreg inside each role's branch, so
  // ptxas allocates each region with its own budget)
  if (warp < C::W_EPI) {
    asm volatile("setmaxnreg.dec.sync.aligned.u32 %0;" ::"n"(C::REG_CTRL));
    if (warp == 0) {
      // -------------------------------------------------------------- TMA producer
      const uint64_t keep = policy_evict_last();   // W: re-read by every group of every CTA
      const uint64_t once = policy_evict_first();  // X rows: read once
      uint32_t wl = 0, xbits = 0;  // bit r: parity of the X loads into ACT[r] so far
      for (int g = blockIdx.x; g < p.num_groups; g += gridDim.x) {
        const int nt = ntiles(g);
#pragma unroll 1
        for (int r = 0; r < nt; ++r) {
          mbar_wait(ACT_EMPTY(r), ((xbits >> r) & 1) ^ 1);  // the previous group's Y store has read ACT[r]
          xbits ^= 1u << r;
          mbar_arrive_expect_tx_elect(X_FULL(r), C::ATILE);
#pragma unroll
          for (int c = 0; c < NW / 64; ++c)
            tma_load_3d_hint_elect(sbase + C::OFF_ACT + r * C::ATILE + c * C::CHUNK, &p.tmX, X_FULL(r), 64 * c,
                                   (g * S + r) * 128, 0, once);
        }
        for (int l = 0; l < L; ++l, ++wl) {
          const int s = wl % C::WS;
          mbar_wait(W_EMPTY(s), ((wl / C::WS) & 1) ^ 1);
          mbar_arrive_expect_tx_elect(W_FULL(s), C::WTILE);
#pragma unroll
          for (int c = 0; c < NW / 64; ++c)
            tma_load_3d_hint_elect(sbase + C::OFF_W + s * C::WTILE + c * C::WCHUNK, &p.tmW, W_FULL(s), 64 * c, 0,
                                   l, keep);
        }
      }
    } else if (warp <= R) {
      // -------------------------------------------------------------- MMA issuer of slot r
      const int r = warp - 1;
      constexpr uint32_t IDESC = idesc_f16(false, 128, NW, false, false);  // A, W: K-major
      const uint64_t desc0 = sdesc_sw128(sbase, 16, 1024);
      const uint32_t aoff = C::OFF_ACT + r * C::ATILE;
      uint32_t wl = 0, use = 0, xc = 0;
      for (int g = blockIdx.x; g < p.num_groups; g += gridDim.x) {
        const bool active = r < ntiles(g);
        for (int l = 0; l < L; ++l, ++wl) {
          const int s = wl % C::WS;
          mbar_wait(W_FULL(s), (wl / C::WS) & 1);  // (also keeps an idle slot's W_EMPTY arrival in phase)
          if (active) {
            if (l == 0) {
              mbar_wait(X_FULL(r), xc & 1);  // (the previous group's last epilogue of slot r drained ACC_r
              ++xc;                          //  before its Y store: implied)
            } else {
              mbar_wait(ACT_FULL(r), (use - 1) & 1);  // ACC_r drained, ACT[r] = h_{l-1}
            }
            tc_fence_after();
            TRACE_EV(5, r * 64 + l);
            const uint32_t woff = C::OFF_W + s * C::WTILE;
            if (TA && l > 0) {  // A = h_{l-1} in TMEM (K-major, fp16 pairs), W_l from shared memory
#pragma unroll
              for (int kk = 0; kk < NW / 16; ++kk)
                umma_ts_elect(tmem + r * NW, tmem + C::TMEM_A + r * (NW / 2) + kk * 8,
                              desc0 + ((woff + (kk / 4) * C::WCHUNK + (kk % 4) * 32) >> 4), IDESC, kk > 0);
            } else {
#pragma unroll
              for (int kk = 0; kk < NW / 16; ++kk)
                umma_ss_elect(tmem + r * NW, desc0 + ((aoff + (kk / 4) * C::CHUNK + (kk % 4) * 32) >> 4),
                              desc0 + ((woff + (kk / 4) * C::WCHUNK + (kk % 4) * 32) >> 4), IDESC, kk > 0);
            }
            umma_commit_elect(ACC_FULL(r));
            TRACE_EV(6, r * 64 + l);
            ++use;
          }
          umma_commit_elect(W_EMPTY(s));  // this slot's reads of W_l are done
        }
      }
    }
  } else {
    asm volatile("setmaxnreg.inc.sync.aligned.u32 %0;" ::"n"(C::REG_EPI));
    // ---------------------------------------------------------------- epilogue
    // warp W_EPI + 4 w + quad: accumulator rows 32 quad.., columns 64 h .. 64 h + 63 (= SW128 chunk h of
    // the next layer's A operand) of slots sg, sg + SG, ...
    const int w = (warp - C::W_EPI) >> 2, h = w % C::H, sg = w / C::H, quad = warp & 3;
    const int row = quad * 32 + lane;
    const uint32_t lane_off = static_cast<uint32_t>(quad * 32) << 16;
    constexpr uint32_t EPI_THREADS = 128 * C::H;  // threads writing one slot's ACT tile
    constexpr int CPG = NW / C::H;                 // columns per warpgroup: chunks c = h, h + H, ...
    uint32_t use[C::SPW];
#pragma unroll
    for (int j = 0; j < C::SPW; ++j) use[j] = 0;
    const int bcol = CPG * h + row;  // the bias column this thread converts (row < CPG)
    auto bias_at = [&](int l) { return p.bias ? __half2float(p.bias[static_cast<size_t>(l) * NW + bcol]) : 0.f; };
    float bnext = 0.f;
    bool first = true;
    for (int g = blockIdx.x; g < p.num_groups; g += gridDim.x) {
      const int nt = ntiles(g);
      for (int l = 0; l < L; ++l) {
        // b_l in fp32 for this slot group: thread (row < CPG, h) converts column CPG h + row into the
        // ring entry l % 2 (its previous readers, layer l - 2, are past the last layer's barrier)
        const uint32_t bring = sbase + C::OFF_BIAS + (sg * 2 + (l & 1)) * NW * 4;
        // (its global load was issued one layer ahead, so the L2 latency is off the chain)
        if (row < CPG) {
          const float bv = first ? bias_at(l) : bnext;
          bnext = bias_at(l + 1 < L ? l + 1 : 0);
          first = false;
          asm volatile("st.shared.f32 [%0], %1;" ::"r"(bring + bcol * 4), "f"(bv) : "memory");
        }
        named_bar_sync(1 + sg, EPI_THREADS);
#pragma unroll
        for (int j = 0; j < C::SPW; ++j) {  // this warpgroup's slots, in the MMA warp's issue order
          const int r = sg + j * C::SG;
          if (r >= nt) continue;
          mbar_wait(ACC_FULL(r), use[j] & 1);
          TRACE_EV(1, r * 64 + l);
          ++use[j];
          tc_fence_after();
          const bool to_tmem = TA && l + 1 < L;  // h_l -> TMEM A_r (next layer's TS operand)
#pragma unroll
          for (int ci = 0; ci < NW / 64 / C::H; ++ci) {  // 64-column chunk c = SW128 chunk c of h_l
            const int c = h + ci * C::H;
            uint32_t v[64];
            const uint32_t tacc = tmem + lane_off + r * NW + 64 * c;
            tmem_ld_32x32b_x32(tacc, *reinterpret_cast<uint32_t(*)[32]>(&v[0]));
            tmem_ld_32x32b_x32(tacc + 32, *reinterpret_cast<uint32_t(*)[32]>(&v[32]));
            tmem_wait_ld();
            reg_fence(v);
            TRACE_EV(2, r * 64 + l);
            const uint32_t act_box = sbase + C::OFF_ACT + r * C::ATILE + c * C::CHUNK + row * 128;
            const float4* bias4 = reinterpret_cast<const float4*>(smem + (bring - sbase)) + 16 * c;
            uint32_t pk[32];  // this chunk of h_l as fp16 pairs
            // bias: broadcast reads (every thread the same address), software-pipelined one 8-column
            // unit ahead so the shared-memory latency is off each unit's add -> convert -> store chain
            float4 nb0 = bias4[0], nb1 = bias4[1];
#pragma unroll
            for (int u = 0; u < 8; ++u) {  // 8 columns -> one 16-byte unit of the 128-byte row
              const float4 b0 = nb0, b1 = nb1;
              if (u + 1 < 8) {
                nb0 = bias4[2 * u + 2];
                nb1 = bias4[2 * u + 3];
              }
              const float bb[8] = {b0.x, b0.y, b0.z, b0.w, b1.x, b1.y, b1.z, b1.w};
#pragma unroll
              for (int e = 0; e < 4; ++e) {
                const float2 x = fadd2(make_float2(__uint_as_float(v[8 * u + 2 * e]), __uint_as_float(v[8 * u + 2 * e + 1])),
                                       make_float2(bb[2 * e], bb[2 * e + 1]));
                uint32_t& d = pk[4 * u + e];
                if constexpr (ACT == 1) {
                  // ReLU inside the conversion: cvt.rn.relu clamps the rounded pair at 0 (rounding is
                  // monotonic and keeps 0, so this equals rounding max(x, 0))
                  asm("cvt.rn.relu.f16x2.f32 %0, %1, %2;" : "=r"(d) : "f"(x.y), "f"(x.x));
                } else if constexpr (ACT == 0) {
                  d = pack2<false>(x.x, x.y);
                } else {
                  d = pack2<false>(apply_act<ACT>(x.x), apply_act<ACT>(x.y));
                }
              }
              if (!to_tmem)
                asm volatile("st.shared.v4.b32 [%0], {%1, %2, %3, %4};" ::"r"(act_box + ((u ^ (row & 7)) << 4)),
                             "r"(pk[4 * u]), "r"(pk[4 * u + 1]), "r"(pk[4 * u + 2]), "r"(pk[4 * u + 3]));
            }
            TRACE_EV(7, r * 64 + l);
            if (to_tmem) {  // row `row`, K columns 64 c .. 64 c + 63 = TMEM columns A_r + 32 c ..
              tmem_st_32x32b_x32(tmem + lane_off + C::TMEM_A + r * (NW / 2) + 32 * c, pk);
              tmem_wait_st();
            }
          }
          TRACE_EV(3, r * 64 + l);
          if (!TA || l + 1 == L) fence_proxy_async_smem();  // smem h_l visible to the async proxy
          tc_fence_before();
          mbar_arrive(ACT_FULL(r));
          TRACE_EV(4, r * 64 + l);
          if (l == L - 1) {  // Y rows of tile r (rows >= M clipped by the tensor map)
            named_bar_sync(1 + sg, EPI_THREADS);
            if (row == 0 && h == 0) {
#pragma unroll
              for (int c = 0; c < NW / 64; ++c)
                tma_store_3d(&p.tmY, sbase + C::OFF_ACT + r * C::ATILE + c * C::CHUNK, 64 * c, (g * S + r) * 128, 0);
              tma_store_commit();
              tma_store_wait_read0();  // ACT[r] read out: the next group's X may land in it
              mbar_arrive(ACT_EMPTY(r));
            }
          }
        }
      }
    }
    if (row == 0 && h == 0) tma_store_wait0();
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 1) {
    tc_fence_after();
    tmem_dealloc(tmem, 512);
  }
}

int make_map_3d_rows(CUtensorMap* m, const void* base, uint64_t cols, uint64_t rows, uint64_t units,
                     uint32_t box_rows, char* err, size_t errlen);

template <int NW, bool TA>
inline int launch_mlp_fused_w(MlpParams& prm, int act, int sms, cudaStream_t stream, char* err, size_t errlen) {
  using C = MlpCfg<NW, TA>;
  constexpr int R = C::R;
  void (*kern)(MlpParams) = act == 1 ? mlp_fused_kernel<NW, 1, TA>
                            : act == 2 ? mlp_fused_kernel<NW, 2, TA>
                            : act == 3 ? mlp_fused_kernel<NW, 3, TA>
                            : act == 4 ? mlp_fused_kernel<NW, 4, TA>
                                       : mlp_fused_kernel<NW, 0, TA>;
  if (cudaError_t e = ensure_smem_attr(reinterpret_cast<const void*>(kern), C::SMEM_ALLOC); e != cudaSuccess) {
    snprintf(err, errlen, "cudaFuncSetAttribute(mlp_fused): %s", cudaGetErrorString(e));
    return 4;
  }
  // Slots per group S.  One tile's layer is a serial chain: MMA (t) -> epilogue (E ~ e t, e ~ 3) ->
  // next MMA.  With S tiles in flight a group's layer takes about max(S t, t + E ceil(S / SG)) (an
  // epilogue warpgroup serves ceil(S / SG) slots in turn), and a CTA runs ceil(groups / SMs) rounds;
  // pick the S with the least rounds x that, the larger S on ties (more reuse of each W_l tile).
  {
    const double e = 3.0;
    double best = 1e300;
    for (int s = 1; s <= R; ++s) {
      const long long groups = (prm.num_tiles + s - 1) / s;
      const long long rounds = (groups + sms - 1) / std::max(sms, 1);
      const double per = std::max(static_cast<double>(s), 1.0 + e * ((s + C::SG - 1) / C::SG));
      const double cost = static_cast<double>(rounds) * per;
      if (cost <= best) {
        best = cost;
        prm.slots = s;
      }
    }
  }
  if (const char* ov = getenv("B200_MLP_SLOTS")) {  // tuning experiments only (tools/mlp_sweep.py)
    const int v = atoi(ov);
    if (v >= 1 && v <= R) prm.slots = v;
  }
  prm.num_groups = (prm.num_tiles + prm.slots - 1) / prm.slots;
  const int grid = std::min(prm.num_groups, sms);
  cudaError_t e = launch_pdl(true, kern, dim3(grid), dim3(C::THREADS), C::SMEM_ALLOC, stream, prm);
  if (e != cudaSuccess) {
    snprintf(err, errlen, "mlp_fused_kernel launch: %s", cudaGetErrorString(e));
    return 4;
  }
  return 0;
}

// Y = h_L of the chain (see the file comment); W [L, NW, NW], bias [L, NW] or nullptr.
inline int launch_mlp_fused(const void* X, const void* W, const void* bias, void* Y, int M, int NW, int L, int act,
                            int sms, cudaStream_t stream, char* err, size_t errlen) {
  MlpParams prm;
  memset(&prm, 0, sizeof(prm));
  int st;
  if ((st = make_map_2d_rows(&prm.tmX, X, NW, M, 128, err, errlen)) != 0) return st;
  if ((st = make_map_2d_rows(&prm.tmY, Y, NW, M, 128, err, errlen)) != 0) return st;
  if ((st = make_map_3d_rows(&prm.tmW, W, NW, NW, L, NW, err, errlen)) != 0) return st;
  prm.bias = static_cast<const __half*>(bias);
  prm.M = M;
  prm.layers = L;
  prm.num_tiles = (M + 127) / 128;
  // h_l in TMEM (TS-form MMAs; 2 slots at N = 128, 4 at N = 64).  The shared-memory variant (4 / 8
  // slots) measured 824 vs 887 TF/s at N = 128 (its SS MMAs and the epilogue's h_l stores compete
  // for the SM's 128 B/clk of shared-memory bandwidth) and 406 vs 439 at N = 64;
  // B200_MLP_VARIANT=1 selects it (A/B experiments only).
  static const bool smem_a = getenv("B200_MLP_VARIANT") != nullptr;
  if (NW == 128)
    return smem_a ? launch_mlp_fused_w<128, false>(prm, act, sms, stream, err, errlen)
                  : launch_mlp_fused_w<128, true>(prm, act, sms, stream, err, errlen);
  return smem_a ? launch_mlp_fused_w<64, false>(prm, act, sms, stream, err, errlen)
                : launch_mlp_fused_w<64, true>(prm, act, sms, stream, err, errlen);
}

}  // namespace b200
