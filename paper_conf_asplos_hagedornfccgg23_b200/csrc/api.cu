// api.cu — the C ABI declared in include/fmha.h: argument validation, TMA tensor-map encoding,
// kernel selection and launch.  No allocation, no synchronisation, no CPU fallback.
#include <cuda.h>
#include <cuda_runtime.h>

#include <cmath>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <algorithm>
#include <mutex>

#include "../../include/fmha.h"
#include "fmha_kernel.cuh"
#include "fmha_ks_kernel.cuh"
#include "gemm_kernel.cuh"
#include "mlp_kernel.cuh"
#include "splitkv_kernel.cuh"

namespace {

thread_local char g_last_cuda_error[256] = "";

int cuda_fail(cudaError_t e, const char* where) {
  snprintf(g_last_cuda_error, sizeof(g_last_cuda_error), "%s: %s", where, cudaGetErrorString(e));
  return FMHA_ERR_CUDA;
}


using EncodeTiledFn = CUresult (*)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                                   const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                                   CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

EncodeTiledFn get_encode_fn() {
  static EncodeTiledFn fn = nullptr;
  static std::once_flag once;
  std::call_once(once, [] {
    void* ptr = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPointByVersion("cuTensorMapEncodeTiled", &ptr, 12000, cudaEnableDefault, &q) ==
            cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = reinterpret_cast<EncodeTiledFn>(ptr);
  });
  return fn;
}

// Checks that the current device is an sm_100 part.  Cached per device ordinal.
int check_device(int* sm_count) {
  int dev = 0;
  cudaError_t e = cudaGetDevice(&dev);
  if (e != cudaSuccess) {
    cudaGetLastError();
    return FMHA_ERR_NO_DEVICE;
  }
  static int cached_major[64], cached_sms[64];
  static bool cached[64];
  static std::mutex mu;
  std::lock_guard<std::mutex> lk(mu);
  if (dev < 64 && cached[dev]) {
    if (sm_count) *sm_count = cached_sms[dev];
    return cached_major[dev] == 10 ? FMHA_OK : FMHA_ERR_NO_DEVICE;
  }
  int major = 0, minor = 0, sms = 0;
  if (cudaDeviceGetAttribute(&major, cudaDevAttrComputeCapabilityMajor, dev) != cudaSuccess ||
      cudaDeviceGetAttribute(&minor, cudaDevAttrComputeCapabilityMinor, dev) != cudaSuccess ||
      cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess) {
    cudaGetLastError();
    return FMHA_ERR_NO_DEVICE;
  }
  if (dev < 64) {
    cached_major[dev] = (major == 10 && minor == 0) ? 10 : -1;
    cached_sms[dev] = sms;
    cached[dev] = true;
  }
  if (sm_count) *sm_count = sms;
  return (major == 10 && minor == 0) ? FMHA_OK : FMHA_ERR_NO_DEVICE;
}

// 3-D tile map over a [units, rows, cols] row-major tensor of 16-bit elements.
// Box = {64 cols (128 B, the SWIZZLE_128B span), box_rows, 1}.  OOB elements read as zero.
int make_map_3d(CUtensorMap* m, const void* base, bool bf16, uint64_t cols, uint64_t rows, uint64_t units,
                uint32_t box_rows, uint32_t box_cols = 64) {
  EncodeTiledFn enc = get_encode_fn();
  if (!enc) {
    snprintf(g_last_cuda_error, sizeof(g_last_cuda_error), "cuTensorMapEncodeTiled entry point unavailable");
    return FMHA_ERR_CUDA;
  }
  cuuint64_t dims[3] = {cols, rows, units};
  cuuint64_t strides[2] = {cols * 2, cols * rows * 2};
  cuuint32_t box[3] = {box_cols, box_rows, 1};
  cuuint32_t estr[3] = {1, 1, 1};
  CUresult r = enc(m, bf16 ? CU_TENSOR_MAP_DATA_TYPE_BFLOAT16 : CU_TENSOR_MAP_DATA_TYPE_FLOAT16, 3,
                   const_cast<void*>(base), dims, strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
                   box_cols == 64 ? CU_TENSOR_MAP_SWIZZLE_128B : CU_TENSOR_MAP_SWIZZLE_64B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                   CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) {
    snprintf(g_last_cuda_error, sizeof(g_last_cuda_error), "cuTensorMapEncodeTiled failed (%d)", int(r));
    return FMHA_ERR_CUDA;
  }
  return FMHA_OK;
}

// 4-D tile map over a 16-bit tensor with head_dim contiguous and arbitrary row / head / batch strides
// (elements; multiples of 8, i.e. 16 bytes, as TMA requires): dims {D, rows, heads, batch}, box
// {box_cols, box_rows, 1, 1}.  SWIZZLE_128B for 64-column boxes, SWIZZLE_64B for 32-column ones.
// Rows >= `rows` read as zero and are clipped on stores.
int make_map_4d(CUtensorMap* m, const void* base, bool bf16, uint64_t d, uint64_t rows, uint64_t heads,
                uint64_t batch, uint64_t s_row, uint64_t s_head, uint64_t s_batch, uint32_t box_rows,
                uint32_t box_cols = 64) {
  EncodeTiledFn enc = get_encode_fn();
  if (!enc) {
    snprintf(g_last_cuda_error, sizeof(g_last_cuda_error), "cuTensorMapEncodeTiled entry point unavailable");
    return FMHA_ERR_CUDA;
  }
  cuuint64_t dims[4] = {d, rows, heads, batch};
  cuuint64_t strides[3] = {s_row * 2, s_head * 2, s_batch * 2};
  cuuint32_t box[4] = {box_cols, box_rows, 1, 1};
  cuuint32_t estr[4] = {1, 1, 1, 1};
  CUresult r = enc(m, bf16 ? CU_TENSOR_MAP_DATA_TYPE_BFLOAT16 : CU_TENSOR_MAP_DATA_TYPE_FLOAT16, 4,
                   const_cast<void*>(base), dims, strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
                   box_cols == 64 ? CU_TENSOR_MAP_SWIZZLE_128B : CU_TENSOR_MAP_SWIZZLE_64B,
                   CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) {
    snprintf(g_last_cuda_error, sizeof(g_last_cuda_error), "cuTensorMapEncodeTiled (4-D) failed (%d)", int(r));
    return FMHA_ERR_INVALID_ARG;  // e.g. a stride that is not a multiple of 16 bytes
  }
  return FMHA_OK;
}

bool aligned16(const void* p) { return (reinterpret_cast<uintptr_t>(p) & 15u) == 0; }

// Key-split kernel (fmha_ks_kernel.cuh: two softmax warps per row quarter and tile) for D = 64 in the
// dense, cross-unit pair and varlen modes, selected with B200_FMHA_KS=1.  Off by default: measured
// against the two-tile kernel on the same boxes it is level on BERT-large-512 (640 vs 657 TFLOP/s),
// slower on BERT-large-384 and BERT-base and +3% on the packed varlen batch.
bool split_pair_enabled() {  // B200_SPLIT_PAIR=0 turns split pairing off (A/B only)
  static const bool on = [] {
    const char* v = std::getenv("B200_SPLIT_PAIR");
    return !(v && v[0] == '0');
  }();
  return on;
}

bool snake_enabled() {  // B200_FMHA_SNAKE=0 turns the causal snake order off (A/B only)
  static const bool on = [] {
    const char* v = std::getenv("B200_FMHA_SNAKE");
    return !(v && v[0] == '0');
  }();
  return on;
}

bool ks_enabled() {
  static const bool on = [] {
    const char* v = std::getenv("B200_FMHA_KS");
    return v && v[0] == '1';
  }();
  return on;
}

template <bool BF16>
int launch_fmha_ks(const b200::FmhaParams& prm, int mode, int sm_count, cudaStream_t stream) {
  using C = b200::FmhaKsCfg;
  void (*kern)(b200::FmhaParams) = mode == b200::MODE_DENSE    ? b200::fmha_fwd_ks_sm100<BF16, b200::MODE_DENSE>
                                   : mode == b200::MODE_PAIRX  ? b200::fmha_fwd_ks_sm100<BF16, b200::MODE_PAIRX>
                                   : mode == b200::MODE_VARLEN ? b200::fmha_fwd_ks_sm100<BF16, b200::MODE_VARLEN>
                                                               : b200::fmha_fwd_ks_sm100<BF16, b200::MODE_VARLEN_SCHED>;
  if (cudaError_t e = b200::ensure_smem_attr(reinterpret_cast<const void*>(kern), C::SMEM_ALLOC); e != cudaSuccess)
    return cuda_fail(e, "cudaFuncSetAttribute(fmha_ks)");
  dim3 grid(static_cast<unsigned>(std::min(prm.num_items, sm_count)), 1, 1);
  const bool pdl = mode != b200::MODE_VARLEN && mode != b200::MODE_VARLEN_SCHED;
  cudaError_t e = b200::launch_pdl(pdl, kern, grid, dim3(C::THREADS), C::SMEM_ALLOC, stream, prm);
  if (e != cudaSuccess) return cuda_fail(e, "fmha_fwd_ks_kernel launch");
  return FMHA_OK;
}

template <int D, bool BF16>
int launch_fmha(const b200::FmhaParams& prm, int sm_count, cudaStream_t stream) {
  using C = b200::FmhaCfg<D>;
  const int mode = prm.num_splits > 1 ? (prm.split_pair ? b200::MODE_SPLIT_PAIR : b200::MODE_SPLIT)
                   : prm.tail_splits > 1 ? (prm.pair_mode ? b200::MODE_PAIRX_TAIL : b200::MODE_DENSE_TAIL)
                   : prm.attn_bias  ? b200::MODE_BIAS2D
                   : prm.key_bias   ? b200::MODE_BIAS
                   : prm.cu_seqlens ? (prm.sched ? b200::MODE_VARLEN_SCHED : b200::MODE_VARLEN)
                                    : (prm.pair_mode ? b200::MODE_PAIRX : b200::MODE_DENSE);
  void (*kern)(b200::FmhaParams) = mode == b200::MODE_DENSE    ? b200::fmha_fwd_sm100<D, BF16, b200::MODE_DENSE>
                                   : mode == b200::MODE_PAIRX  ? b200::fmha_fwd_sm100<D, BF16, b200::MODE_PAIRX>
                                   : mode == b200::MODE_VARLEN ? b200::fmha_fwd_sm100<D, BF16, b200::MODE_VARLEN>
                                   : mode == b200::MODE_SPLIT  ? b200::fmha_fwd_sm100<D, BF16, b200::MODE_SPLIT>
                                   : mode == b200::MODE_SPLIT_PAIR ? b200::fmha_fwd_sm100<D, BF16, b200::MODE_SPLIT_PAIR>
                                   : mode == b200::MODE_BIAS   ? b200::fmha_fwd_sm100<D, BF16, b200::MODE_BIAS>
                                   : mode == b200::MODE_BIAS2D ? b200::fmha_fwd_sm100<D, BF16, b200::MODE_BIAS2D>
                                   : mode == b200::MODE_DENSE_TAIL ? b200::fmha_fwd_sm100<D, BF16, b200::MODE_DENSE_TAIL>
                                   : mode == b200::MODE_PAIRX_TAIL ? b200::fmha_fwd_sm100<D, BF16, b200::MODE_PAIRX_TAIL>
                                                               : b200::fmha_fwd_sm100<D, BF16, b200::MODE_VARLEN_SCHED>;
  if (D == 64 && mode <= b200::MODE_VARLEN_SCHED && ks_enabled()) return launch_fmha_ks<BF16>(prm, mode, sm_count, stream);
  if (cudaError_t e = b200::ensure_smem_attr(reinterpret_cast<const void*>(kern), C::SMEM_ALLOC); e != cudaSuccess)
    return cuda_fail(e, "cudaFuncSetAttribute(fmha)");
  // persistent: one CTA per SM (or fewer when there is less work)
  dim3 grid(static_cast<unsigned>(std::min(prm.num_items, sm_count)), 1, 1);
  // PDL measured: +0.5% (BERT-large-512) to +4.5% (BERT-base, padded); -5% on the varlen schedule
  // (B200_VARLEN_PDL=1 turns it on for varlen too, A/B only)
  static const bool varlen_pdl = [] {
    const char* v = std::getenv("B200_VARLEN_PDL");
    return v && v[0] == '1';
  }();
  const bool pdl = varlen_pdl || (mode != b200::MODE_VARLEN && mode != b200::MODE_VARLEN_SCHED);
  cudaError_t e = b200::launch_pdl(pdl, kern, grid, dim3(C::THREADS), C::SMEM_ALLOC, stream, prm);
  if (e != cudaSuccess) return cuda_fail(e, "fmha_fwd_kernel launch");
  if (mode == b200::MODE_SPLIT || mode == b200::MODE_SPLIT_PAIR) {  // merge the splits into O (same stream, after the kernel)
    const long long rows = static_cast<long long>(prm.num_units) * prm.seq_q;
    const long long blocks = (rows * 32 + 255) / 256;
    b200::fmha_splitkv_combine_kernel<D, BF16><<<static_cast<unsigned>(blocks), 256, 0, stream>>>(
        prm.ws_o, prm.ws_m, prm.ws_l, prm.o_ptr, prm.num_splits, rows);
    e = cudaGetLastError();
    if (e != cudaSuccess) return cuda_fail(e, "fmha_splitkv_combine_kernel launch");
  }
  return FMHA_OK;
}

// Split-KV (fmha_fwd_splitkv): workspace floats for `splits` splits.
size_t splitkv_ws_bytes(long long units, int seq_q, int head_dim, int splits) {
  return static_cast<size_t>(splits) * units * seq_q * (head_dim + 2) * sizeof(float);
}

// Default split count.  A CTA runs ceil(items * s / SMs) rounds of items of ceil(nkv / s) KV tiles
// plus a fixed per-item cost (Q load, pipeline fill, the fp32 partial-O store; ~2 tiles); pick the
// s with the least rounds x (tiles + 2), at least one KV tile per split.  1 when the dense schedule
// already fills the SMs.
int splitkv_default(long long units, int seq_q, int seq_kv, int sms) {
  const long long items = units * (((seq_q + 127) / 128 + 1) / 2);  // (unit, q-tile pair) items
  const bool pair = (seq_q + 127) / 128 == 1 && split_pair_enabled();  // two splits per item (split_pair)
  const int nkv = (seq_kv + 127) / 128;
  if (items <= 0 || items >= sms || nkv <= 1) return 1;
  int best_s = 1;
  long long best = -1;
  for (int s = 1; s <= std::min(nkv, 64); ++s) {
    const int per = (nkv + s - 1) / s;
    if ((nkv + per - 1) / per != s) continue;  // s not reachable with whole tiles per split
    const long long rounds = ((pair ? items * ((s + 1) / 2) : items * s) + sms - 1) / sms;
    const long long cost = rounds * (per + 2);
    if (best < 0 || cost < best) {
      best = cost;
      best_s = s;
    }
  }
  return best_s;
}

// Work items of the dense schedule and its pairing mode: (unit, q-tile pair) items, or (pair_mode 1)
// pairs of the flattened (unit, q-tile) list when a unit has an odd number of q-tiles (>= 3, or 1 with
// more units than SMs) and the mask is not causal / a bias (BERT-large-384: no half-empty items, +8%).
long long dense_items(long long units, int num_q_tiles, int kind, int sms, int* pair_mode, long long decide_units = -1) {
  // Single-q-tile units (seq_q <= 128) are paired too once they fill more than one round unpaired (one
  // round of pair steps is shorter than two of single-tile steps); with fewer units than SMs pairing
  // would halve the busy SMs.  Measured on BERT-base padded (384 units): 105 -> 117 TFLOP/s
  // (profiles/r02c_ab_pair1.txt).  B200_FMHA_PAIR1=0 restores round 1's rule (A/B only).
  static const bool pair1 = [] {
    const char* v = std::getenv("B200_FMHA_PAIR1");
    return !(v && v[0] == '0');
  }();
  // (decide_units: the whole problem's units when this launch is one batch chunk of it, so every chunk of
  // fmha_fwd_from_host takes the same decision and the results stay bitwise those of fmha_fwd)
  const long long du = decide_units >= 0 ? decide_units : units;
  const bool odd = (num_q_tiles & 1) && (num_q_tiles >= 3 || (pair1 && num_q_tiles == 1 && du > sms));
  *pair_mode = (kind != FMHA_MASK_CAUSAL && kind != FMHA_MASK_KEY_BIAS && kind != FMHA_MASK_ATTN_BIAS && odd) ? 1 : 0;
  return *pair_mode ? (units * num_q_tiles + 1) / 2 : units * ((num_q_tiles + 1) / 2);
}

// Stream-K tail plan (fmha_fwd_streamk): the persistent grid runs `items` two-tile items in rounds of
// `sms`; the last, partial round's `rest` items are cut into s key ranges of whole 128-key tiles
// (s <= nkv, rest * s <= sms: the pieces still fit one round, s <= MAX_TAIL_SPLITS), so that round
// takes ceil(nkv / s) instead of nkv KV steps.  The merge (the last piece's stores, release / acquire
// through L2, bulk loads of the other pieces' states, the combine) costs ~5 us on B200, about 2.5 KV
// steps of a BERT-large item, and fmha_fwd already runs a cross-unit-paired last round as single
// tiles (`singles`, ~0.65 of a pair step), so a split is planned only when the modelled
// round time drops by >= 1.5 steps (profiles/r02_streamk_probe.txt: BERT-large-384 and
// 8 x 14 x 384 x 1024 measured slower split, long key ranges 13-39% faster).  Returns s (1: no
// split), *tail_items = rest.
int streamk_plan(long long items, int nkv, int sms, bool singles, long long* tail_items) {
  *tail_items = 0;
  if (items <= 0 || sms <= 0 || nkv < 2) return 1;
  const long long rest = items % sms;
  if (rest == 0) return 1;
  long long s = std::min<long long>(std::min<long long>(nkv, sms / rest), b200::MAX_TAIL_SPLITS);
  if (s < 2) return 1;
  const int per = static_cast<int>((nkv + s - 1) / s);
  s = (nkv + per - 1) / per;  // every piece gets at least one key tile
  const long long cost_fwd = (singles ? 65LL : 100LL) * nkv, cost_sk = 100LL * per + 250;
  if (s < 2 || cost_fwd - cost_sk < 150) return 1;
  *tail_items = rest;
  return static_cast<int>(s);
}

// fmha_fwd's last round runs as single tiles (pair_mode 1 with at least one full round, and the
// last round's tiles fit one round)
bool singles_tail(long long items, long long tiles, int pair_mode, int sms) {
  const long long full = items / sms * sms;
  return pair_mode && full > 0 && tiles - 2 * full > 0 && tiles - 2 * full <= sms;
}

// Stream-K workspace: tail counters (one per tail item, < sms) then the pieces' states (< sms pieces
// of two tiles x 128 rows x (D + 2) floats).
size_t streamk_cnt_bytes(int sms) { return (static_cast<size_t>(sms) * 4 + 255) / 256 * 256; }
size_t streamk_ws_bytes(int head_dim, int sms) {
  return streamk_cnt_bytes(sms) + static_cast<size_t>(sms) * 2 * 128 * (head_dim + 2) * sizeof(float);
}

// The argument checks of fmha_common that need no pointers to be valid device memory: shapes, scale,
// head_dim, mask kind.  FMHA_OK with *empty = true means there is nothing to launch.
int validate_shape(int batch, int heads, int seq_q, int seq_kv, int head_dim, float scale, const fmha_mask_t* mask,
                   int splits, bool* empty) {
  *empty = false;
  if (batch < 0 || heads < 0 || seq_q < 0 || seq_kv < 0) return FMHA_ERR_INVALID_ARG;
  if (!std::isfinite(scale)) return FMHA_ERR_INVALID_ARG;
  if (head_dim != 64 && head_dim != 128) return FMHA_ERR_UNSUPPORTED;
  if (scale < 0.f) return FMHA_ERR_UNSUPPORTED;
  const int kind = mask ? mask->kind : FMHA_MASK_NONE;
  if (kind != FMHA_MASK_NONE && kind != FMHA_MASK_KEY_PADDING && kind != FMHA_MASK_CAUSAL &&
      kind != FMHA_MASK_KEY_BIAS && kind != FMHA_MASK_ATTN_BIAS)
    return FMHA_ERR_UNSUPPORTED;
  if (kind == FMHA_MASK_ATTN_BIAS) {  // (R21) fmha_fwd / fmha_fwd_bf16 / fmha_fwd_strided; added as bias / scale
    if (splits != 1 || !(scale > 0.f)) return FMHA_ERR_UNSUPPORTED;
    if ((mask->attn_bias_stride_q != 0 && mask->attn_bias_stride_q < seq_kv) || mask->attn_bias_stride_q < 0 ||
        (mask->attn_bias_stride_q % 8) != 0 || mask->attn_bias_stride_b < 0 ||
        mask->attn_bias_stride_h < 0 || (mask->attn_bias_stride_b % 8) != 0 || (mask->attn_bias_stride_h % 8) != 0)
      return FMHA_ERR_INVALID_ARG;
  }
  if (kind == FMHA_MASK_KEY_BIAS) {  // (R20) fmha_fwd / fmha_fwd_bf16 only; the bias is added as bias / scale
    if (splits != 1 || !(scale > 0.f)) return FMHA_ERR_UNSUPPORTED;
    if (mask->key_bias_stride < seq_kv || (mask->key_bias_stride % 4) != 0) return FMHA_ERR_INVALID_ARG;
  }
  const long long units = static_cast<long long>(batch) * heads;
  if (units == 0 || seq_q == 0) {
    *empty = true;
    return FMHA_OK;
  }
  if (seq_kv == 0) return FMHA_ERR_INVALID_ARG;
  if (kind == FMHA_MASK_KEY_PADDING && !mask->kv_len) return FMHA_ERR_INVALID_ARG;
  if (units > 2147483647LL || static_cast<long long>(seq_q) * head_dim * units * 2 > (1LL << 40))
    return FMHA_ERR_INVALID_ARG;
  return FMHA_OK;
}

int fmha_common(bool bf16, const void* Q, const void* K, const void* V, void* O, const fmha_mask_t* mask,
                int batch, int heads, int seq_q, int seq_kv, int head_dim, float scale, cudaStream_t stream,
                int splits = 1, void* workspace = nullptr, size_t workspace_bytes = 0,
                const fmha_strides_t* strides = nullptr, bool streamk = false, long long decide_units = -1) {
  g_last_cuda_error[0] = 0;
  bool empty = false;
  if (int vs = validate_shape(batch, heads, seq_q, seq_kv, head_dim, scale, mask, splits, &empty); vs != FMHA_OK || empty)
    return vs;
  const int kind = mask ? mask->kind : FMHA_MASK_NONE;
  const long long units = static_cast<long long>(batch) * heads;
  if (!Q || !K || !V || !O) return FMHA_ERR_INVALID_ARG;
  if (kind == FMHA_MASK_KEY_BIAS && !mask->key_bias) return FMHA_ERR_INVALID_ARG;
  if (kind == FMHA_MASK_KEY_BIAS && !aligned16(mask->key_bias)) return FMHA_ERR_MISALIGNED;
  if (kind == FMHA_MASK_ATTN_BIAS && !mask->attn_bias) return FMHA_ERR_INVALID_ARG;
  if (kind == FMHA_MASK_ATTN_BIAS && !aligned16(mask->attn_bias)) return FMHA_ERR_MISALIGNED;
  if (!aligned16(Q) || !aligned16(K) || !aligned16(V) || !aligned16(O)) return FMHA_ERR_MISALIGNED;
  int sm_count = 0;
  int st = check_device(&sm_count);
  if (st != FMHA_OK) return st;

  b200::FmhaParams prm;
  memset(&prm, 0, sizeof(prm));
  // element strides {row, head, batch} of Q, K, V, O (contiguous [B, H, S, D] unless given)
  const uint64_t D_ = head_dim;
  fmha_strides_t cs;
  const uint64_t qsz = D_ * seq_q, ksz = D_ * seq_kv;
  const int64_t cq[3] = {static_cast<int64_t>(qsz * heads), static_cast<int64_t>(qsz), static_cast<int64_t>(D_)};
  const int64_t ck[3] = {static_cast<int64_t>(ksz * heads), static_cast<int64_t>(ksz), static_cast<int64_t>(D_)};
  for (int i = 0; i < 3; ++i) {
    cs.q[i] = strides ? strides->q[i] : cq[i];
    cs.k[i] = strides ? strides->k[i] : ck[i];
    cs.v[i] = strides ? strides->v[i] : ck[i];
    cs.o[i] = strides ? strides->o[i] : cq[i];
  }
  auto map4 = [&](CUtensorMap* m, const void* base, const int64_t* st3, uint64_t rows, uint32_t box_rows,
                  uint32_t box_cols) {
    return make_map_4d(m, base, bf16, D_, rows, heads, batch, st3[2], st3[1], st3[0], box_rows, box_cols);
  };
  if ((st = map4(&prm.tmQ, Q, cs.q, seq_q, 128, 64)) != FMHA_OK) return st;
  if ((st = map4(&prm.tmK, K, cs.k, seq_kv, 128, 64)) != FMHA_OK) return st;
  if ((st = map4(&prm.tmV, V, cs.v, seq_kv, 128, 64)) != FMHA_OK) return st;
  if ((st = map4(&prm.tmO, O, cs.o, seq_q, 128, 64)) != FMHA_OK) return st;
  if ((st = map4(&prm.tmO32, O, cs.o, seq_q, 32, 32)) != FMHA_OK) return st;
  prm.kv_len = (kind == FMHA_MASK_KEY_PADDING) ? mask->kv_len : nullptr;
  prm.cu_seqlens = nullptr;
  prm.seq_q = seq_q;
  prm.seq_kv = seq_kv;
  prm.heads = heads;
  prm.num_q_tiles = (seq_q + 127) / 128;
  prm.num_units = static_cast<int>(units);
  prm.mask_kind = kind;
  // scale = 0 is legal (every visible key gets weight 1); keep c strictly positive so masked
  // scores (-inf) still map to exp2(-inf) = 0 instead of -inf * 0 = NaN.  1e-30 perturbs visible
  // scores by < 1e-25 in the exponent.
  prm.scale_log2 = std::max(scale * 1.4426950408889634f, 1e-30f);
  long long items = dense_items(units, prm.num_q_tiles, kind, sm_count, &prm.pair_mode, decide_units);
  if (kind == FMHA_MASK_KEY_BIAS) {
    prm.key_bias = mask->key_bias;
    prm.key_bias_stride = mask->key_bias_stride;
    prm.inv_scale = 1.4426950408889634f / prm.scale_log2;  // c * inv_scale = log2(e) exactly as used
    prm.mask_kind = FMHA_MASK_NONE;  // no key bound beyond seq_kv; the bias does the masking
  }
  if (kind == FMHA_MASK_ATTN_BIAS) {
    prm.attn_bias = static_cast<const uint16_t*>(mask->attn_bias);
    prm.ab_sb = mask->attn_bias_stride_b;
    prm.ab_sh = mask->attn_bias_stride_h;
    prm.ab_sq = mask->attn_bias_stride_q;
    const long long row8 = (seq_kv + 7) / 8 * 8;  // a broadcast row (stride 0) must hold row8 elements
    prm.bias_cols8 = static_cast<int>((mask->attn_bias_stride_q == 0 ? row8 : std::min<long long>(mask->attn_bias_stride_q, row8)) / 8);
    prm.inv_scale = 1.4426950408889634f / prm.scale_log2;  // c * inv_scale = log2(e) exactly as used
    prm.mask_kind = FMHA_MASK_NONE;
  }
  prm.single_from = 0x7fffffff;
  prm.tail_from = 0x7fffffff;
  long long tail_items = 0;
  const int tail_s = (streamk && splits == 1 && kind != FMHA_MASK_KEY_BIAS && kind != FMHA_MASK_ATTN_BIAS)
                         ? streamk_plan(items, (seq_kv + 127) / 128, sm_count,
                                        singles_tail(items, units * prm.num_q_tiles, prm.pair_mode, sm_count), &tail_items)
                         : 1;
  if (tail_s > 1) {  // stream-K tail: the last round's items as key-range pieces, merged in the kernel
    if (!workspace || workspace_bytes < streamk_ws_bytes(head_dim, sm_count)) return FMHA_ERR_INVALID_ARG;
    if (reinterpret_cast<uintptr_t>(workspace) % 256 != 0) return FMHA_ERR_MISALIGNED;
    const int nkv = (seq_kv + 127) / 128;
    prm.tail_from = static_cast<int>(items - tail_items);
    prm.tail_splits = tail_s;
    prm.tail_tiles = (nkv + tail_s - 1) / tail_s;
    prm.div_tail.init(static_cast<uint32_t>(tail_s));
    prm.tail_cnt = static_cast<unsigned int*>(workspace);
    prm.ws_tail = reinterpret_cast<float*>(static_cast<uint8_t*>(workspace) + streamk_cnt_bytes(sm_count));
    items = prm.tail_from + tail_items * tail_s;
  } else if (prm.pair_mode) {  // a last, partial round of tile pairs runs as single tiles (half as long)
    const long long tiles = units * prm.num_q_tiles;
    const long long full = items / sm_count * sm_count;  // pair items in full rounds
    const long long rest = tiles - 2 * full;              // tiles left for the last round
    if (full > 0 && rest > 0 && rest <= sm_count) {
      prm.single_from = static_cast<int>(full);
      items = full + rest;
    }
  }
  if (items > 2147483647LL || units * prm.num_q_tiles > 2147483647LL) return FMHA_ERR_UNSUPPORTED;
  prm.num_items = static_cast<int>(items);
  // causal items come longest first with decreasing cost: deal them in snake order (gpt_causal: the
  // busiest SM 132 -> 126 KV steps for a 124.5 mean); equal-cost items need no snake
  prm.snake = (kind == FMHA_MASK_CAUSAL && snake_enabled()) ? 1 : 0;
  prm.div_units.init(static_cast<uint32_t>(std::max(prm.num_units, 1)));
  prm.div_pairs.init(static_cast<uint32_t>(std::max((prm.num_q_tiles + 1) / 2, 1)));
  prm.div_qtiles.init(static_cast<uint32_t>(std::max(prm.num_q_tiles, 1)));
  prm.div_heads.init(static_cast<uint32_t>(std::max(heads, 1)));
  if (splits == 0) splits = splitkv_default(units, seq_q, seq_kv, sm_count);
  if (splits > 1) {
    const int nkv = (seq_kv + 127) / 128;
    const int per = (nkv + splits - 1) / splits;
    splits = (nkv + per - 1) / per;  // every split gets at least one KV tile
  }
  if (splits > 1) {
    if (!workspace || workspace_bytes < splitkv_ws_bytes(units, seq_q, head_dim, splits)) return FMHA_ERR_INVALID_ARG;
    if (reinterpret_cast<uintptr_t>(workspace) % 16 != 0) return FMHA_ERR_MISALIGNED;
    const int nkv = (seq_kv + 127) / 128;
    prm.num_splits = splits;
    prm.split_tiles = (nkv + splits - 1) / splits;
    prm.pair_mode = 0;  // (pairs of one unit's q-tiles; the split index is the fastest item digit)
    // one q-tile per unit: pair consecutive splits of the unit in one item (tile 1 = the same rows, the
    // next key range), so the second softmax warpgroup is not idle (decode_splitkv: 4 -> 8 splits)
    prm.split_pair = (prm.num_q_tiles == 1 && split_pair_enabled()) ? 1 : 0;
    const int per_item = prm.split_pair ? (splits + 1) / 2 : splits;
    const long long items = units * ((prm.num_q_tiles + 1) / 2) * per_item;
    if (items > 2147483647LL) return FMHA_ERR_UNSUPPORTED;
    prm.num_items = static_cast<int>(items);
    prm.div_splits.init(static_cast<uint32_t>(per_item));
    float* ws = static_cast<float*>(workspace);
    const size_t rows = static_cast<size_t>(units) * seq_q;
    prm.ws_o = ws;
    prm.ws_m = ws + static_cast<size_t>(splits) * rows * head_dim;
    prm.ws_l = prm.ws_m + static_cast<size_t>(splits) * rows;
    prm.o_ptr = static_cast<uint8_t*>(O);
  }

  if (head_dim == 64)
    return bf16 ? launch_fmha<64, true>(prm, sm_count, stream) : launch_fmha<64, false>(prm, sm_count, stream);
  return bf16 ? launch_fmha<128, true>(prm, sm_count, stream) : launch_fmha<128, false>(prm, sm_count, stream);
}

size_t round_up(size_t x, size_t a) { return (x + a - 1) / a * a; }

int fmha_varlen_common(bool bf16, const void* QKV, void* O, const int32_t* cu_seqlens, int num_seqs, int max_seqlen,
                       int total_tokens, int heads, int head_dim, float scale, int causal, cudaStream_t stream) {
  g_last_cuda_error[0] = 0;
  if (num_seqs < 0 || max_seqlen < 0 || total_tokens < 0 || heads < 0) return FMHA_ERR_INVALID_ARG;
  if (!std::isfinite(scale)) return FMHA_ERR_INVALID_ARG;
  if (head_dim != 64 && head_dim != 128) return FMHA_ERR_UNSUPPORTED;
  if (scale < 0.f || (causal != 0 && causal != 1)) return FMHA_ERR_UNSUPPORTED;
  const long long units = static_cast<long long>(num_seqs) * heads;
  if (units == 0 || max_seqlen == 0 || total_tokens == 0) return FMHA_OK;
  if (!QKV || !O || !cu_seqlens) return FMHA_ERR_INVALID_ARG;
  if (!aligned16(QKV) || !aligned16(O) || (reinterpret_cast<uintptr_t>(cu_seqlens) & 3u)) return FMHA_ERR_MISALIGNED;
  if (units > 2147483647LL || static_cast<long long>(total_tokens) * 3 * heads * head_dim > (1LL << 40))
    return FMHA_ERR_INVALID_ARG;
  int sm_count = 0;
  int st = check_device(&sm_count);
  if (st != FMHA_OK) return st;

  b200::FmhaParams prm;
  memset(&prm, 0, sizeof(prm));
  const uint64_t hd = static_cast<uint64_t>(heads) * head_dim;
  const uint8_t* base = static_cast<const uint8_t*>(QKV);
  // {D, H, T, 1}: a tile coordinate is (d, h, token, 0); box {64, 1, 128, 1} = one head's 128 tokens
  auto mapv = [&](CUtensorMap* m, const void* b, uint64_t tok_stride, uint32_t box_tokens, uint32_t box_d) {
    EncodeTiledFn enc = get_encode_fn();
    if (!enc) return static_cast<int>(FMHA_ERR_CUDA);
    cuuint64_t dims[4] = {static_cast<cuuint64_t>(head_dim), static_cast<cuuint64_t>(heads),
                          static_cast<cuuint64_t>(total_tokens), 1};
    cuuint64_t strd[3] = {static_cast<cuuint64_t>(head_dim) * 2, tok_stride * 2, tok_stride * 2 * total_tokens};
    cuuint32_t box[4] = {box_d, 1, box_tokens, 1};
    cuuint32_t estr[4] = {1, 1, 1, 1};
    CUresult r = enc(m, bf16 ? CU_TENSOR_MAP_DATA_TYPE_BFLOAT16 : CU_TENSOR_MAP_DATA_TYPE_FLOAT16, 4, const_cast<void*>(b),
                     dims, strd, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
                     box_d == 64 ? CU_TENSOR_MAP_SWIZZLE_128B : CU_TENSOR_MAP_SWIZZLE_64B,
                     CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    if (r != CUDA_SUCCESS) {
      snprintf(g_last_cuda_error, sizeof(g_last_cuda_error), "cuTensorMapEncodeTiled (varlen) failed (%d)", int(r));
      return static_cast<int>(FMHA_ERR_CUDA);
    }
    return static_cast<int>(FMHA_OK);
  };
  if ((st = mapv(&prm.tmQ, base, 3 * hd, 128, 64)) != FMHA_OK) return st;
  if ((st = mapv(&prm.tmK, base + 2 * hd, 3 * hd, 128, 64)) != FMHA_OK) return st;
  if ((st = mapv(&prm.tmV, base + 4 * hd, 3 * hd, 128, 64)) != FMHA_OK) return st;
  if ((st = mapv(&prm.tmO, O, hd, 128, 64)) != FMHA_OK) return st;
  if ((st = mapv(&prm.tmO32, O, hd, 32, 32)) != FMHA_OK) return st;
  prm.kv_len = nullptr;
  prm.cu_seqlens = cu_seqlens;
  prm.o_ptr = static_cast<uint8_t*>(O);
  prm.o_row_elems = static_cast<int>(hd);
  prm.seq_q = prm.seq_kv = max_seqlen;  // self-attention within each sequence: causal offset 0
  prm.heads = heads;
  prm.num_q_tiles = (max_seqlen + 127) / 128;
  prm.num_units = static_cast<int>(units);
  prm.mask_kind = causal ? FMHA_MASK_CAUSAL : FMHA_MASK_NONE;
  prm.scale_log2 = std::max(scale * 1.4426950408889634f, 1e-30f);
  prm.pair_mode = 0;  // both tiles of an item belong to one (sequence, head)
  prm.num_seqs = num_seqs;
  prm.max_level = prm.num_q_tiles;
  // non-causal items cost ceil(len/128) KV steps: visit them in decreasing-cost order, dealt in snake
  // order over the CTAs (see fmha_kernel.cuh).  Causal keeps the static longest-pair-first order.
  prm.sched = (!causal && num_seqs <= b200::SCHED_MAX_SEQS && prm.max_level <= b200::SCHED_MAX_LEVELS) ? 1 : 0;
  const long long items = units * ((prm.num_q_tiles + 1) / 2);
  if (items > 2147483647LL) return FMHA_ERR_UNSUPPORTED;
  prm.num_items = static_cast<int>(items);
  prm.div_units.init(static_cast<uint32_t>(std::max(prm.num_units, 1)));
  prm.div_pairs.init(static_cast<uint32_t>(std::max((prm.num_q_tiles + 1) / 2, 1)));
  prm.div_qtiles.init(static_cast<uint32_t>(std::max(prm.num_q_tiles, 1)));
  prm.div_heads.init(static_cast<uint32_t>(std::max(heads, 1)));
  if (head_dim == 64)
    return bf16 ? launch_fmha<64, true>(prm, sm_count, stream) : launch_fmha<64, false>(prm, sm_count, stream);
  return bf16 ? launch_fmha<128, true>(prm, sm_count, stream) : launch_fmha<128, false>(prm, sm_count, stream);
}

}  // namespace

namespace b200 {
int make_map_2d_rows(CUtensorMap* m, const void* base, uint64_t cols, uint64_t rows, uint32_t box_rows, char* err,
                     size_t errlen) {
  int st = make_map_3d(m, base, false, cols, rows, 1, box_rows);
  if (st != FMHA_OK && err && errlen) snprintf(err, errlen, "%s", g_last_cuda_error);
  return st;
}
int make_map_3d_rows(CUtensorMap* m, const void* base, uint64_t cols, uint64_t rows, uint64_t units,
                     uint32_t box_rows, char* err, size_t errlen) {
  int st = make_map_3d(m, base, false, cols, rows, units, box_rows);
  if (st != FMHA_OK && err && errlen) snprintf(err, errlen, "%s", g_last_cuda_error);
  return st;
}
}  // namespace b200

extern "C" {

int fmha_fwd(const void* Q, const void* K, const void* V, void* O, const fmha_mask_t* mask, int batch, int heads,
             int seq_q, int seq_kv, int head_dim, float scale, fmha_stream_t stream) {
  return fmha_common(false, Q, K, V, O, mask, batch, heads, seq_q, seq_kv, head_dim, scale,
                     reinterpret_cast<cudaStream_t>(stream));
}

int fmha_fwd_bf16(const void* Q, const void* K, const void* V, void* O, const fmha_mask_t* mask, int batch,
                  int heads, int seq_q, int seq_kv, int head_dim, float scale, fmha_stream_t stream) {
  return fmha_common(true, Q, K, V, O, mask, batch, heads, seq_q, seq_kv, head_dim, scale,
                     reinterpret_cast<cudaStream_t>(stream));
}

int fmha_fwd_strided(int dtype, const void* Q, const void* K, const void* V, void* O, const fmha_strides_t* strides,
                     const fmha_mask_t* mask, int batch, int heads, int seq_q, int seq_kv, int head_dim, float scale,
                     fmha_stream_t stream) {
  g_last_cuda_error[0] = 0;
  if (dtype != 0 && dtype != 1) return FMHA_ERR_UNSUPPORTED;
  if (strides) {
    const int64_t* all[4] = {strides->q, strides->k, strides->v, strides->o};
    for (const int64_t* st3 : all) {
      for (int i = 0; i < 3; ++i)
        if (st3[i] <= 0 || (st3[i] % 8) != 0 || st3[i] > (int64_t(1) << 36)) return FMHA_ERR_INVALID_ARG;
      if (st3[2] < head_dim) return FMHA_ERR_INVALID_ARG;
    }
  }
  return fmha_common(dtype == 1, Q, K, V, O, mask, batch, heads, seq_q, seq_kv, head_dim, scale,
                     reinterpret_cast<cudaStream_t>(stream), 1, nullptr, 0, strides);
}

int fmha_fwd_varlen(const void* QKV, void* O, const int32_t* cu_seqlens, int num_seqs, int max_seqlen,
                    int total_tokens, int heads, int head_dim, float scale, int causal, int dtype,
                    fmha_stream_t stream) {
  if (dtype != 0 && dtype != 1) return FMHA_ERR_UNSUPPORTED;
  return fmha_varlen_common(dtype == 1, QKV, O, cu_seqlens, num_seqs, max_seqlen, total_tokens, heads, head_dim,
                            scale, causal, reinterpret_cast<cudaStream_t>(stream));
}

size_t transformer_layer_workspace_bytes(int tokens, int d_model, int d_ff) {
  if (tokens < 0 || d_model < 0 || d_ff < 0) return 0;
  const size_t t = static_cast<size_t>(tokens);
  return round_up(t * 3 * d_model * 2, 256) + 2 * round_up(t * d_model * 2, 256) + round_up(t * d_ff * 2, 256);
}

int transformer_layer_fwd(const void* X, const void* Wqkv, const void* bqkv, const void* Wo, const void* bo,
                          const void* W1, const void* b1, const void* W2, const void* b2, void* Y,
                          const int32_t* cu_seqlens, int num_seqs, int max_seqlen, int tokens, int d_model,
                          int heads, int d_ff, float scale, int causal, void* workspace, size_t workspace_bytes,
                          fmha_stream_t stream) {
  g_last_cuda_error[0] = 0;
  if (tokens < 0 || d_model <= 0 || heads <= 0 || d_ff <= 0 || num_seqs < 0 || max_seqlen < 0)
    return FMHA_ERR_INVALID_ARG;
  if (d_model % heads != 0) return FMHA_ERR_INVALID_ARG;
  const int head_dim = d_model / heads;
  if (head_dim != 64 && head_dim != 128) return FMHA_ERR_UNSUPPORTED;
  if (tokens == 0) return FMHA_OK;
  if (!X || !Wqkv || !Wo || !W1 || !W2 || !Y || !cu_seqlens || !workspace) return FMHA_ERR_INVALID_ARG;
  if (workspace_bytes < transformer_layer_workspace_bytes(tokens, d_model, d_ff)) return FMHA_ERR_INVALID_ARG;
  if ((reinterpret_cast<uintptr_t>(workspace) & 255u) != 0) return FMHA_ERR_MISALIGNED;
  const size_t t = static_cast<size_t>(tokens);
  uint8_t* w = static_cast<uint8_t*>(workspace);
  uint8_t* qkv = w;                                       // [T, 3, H, D]
  uint8_t* attn = qkv + round_up(t * 3 * d_model * 2, 256);  // [T, H, D] = [T, d_model]
  uint8_t* z = attn + round_up(t * d_model * 2, 256);     // [T, d_model]
  uint8_t* h = z + round_up(t * d_model * 2, 256);        // [T, d_ff]
  int st;
  if ((st = gemm_bias_act(X, Wqkv, bqkv, qkv, tokens, 3 * d_model, d_model, ACT_NONE, stream)) != FMHA_OK) return st;
  if ((st = fmha_varlen_common(false, qkv, attn, cu_seqlens, num_seqs, max_seqlen, tokens, heads, head_dim, scale,
                               causal, reinterpret_cast<cudaStream_t>(stream))) != FMHA_OK)
    return st;
  if ((st = gemm_bias_act(attn, Wo, bo, z, tokens, d_model, d_model, ACT_NONE, stream)) != FMHA_OK) return st;
  if ((st = gemm_bias_act(z, W1, b1, h, tokens, d_ff, d_model, ACT_GELU_ERF, stream)) != FMHA_OK) return st;
  return gemm_bias_act(h, W2, b2, Y, tokens, d_model, d_ff, ACT_NONE, stream);
}

size_t fmha_workspace_bytes(int batch, int heads, int seq_q, int seq_kv, int head_dim) {
  if (batch < 0 || heads < 0 || seq_q < 0 || seq_kv < 0 || head_dim < 0) return 0;
  const size_t u = static_cast<size_t>(batch) * heads;
  const size_t q = round_up(u * seq_q * head_dim * 2, 256);
  const size_t kv = round_up(u * seq_kv * head_dim * 2, 256);
  return 2 * q + 2 * kv + round_up(static_cast<size_t>(batch) * 4, 256);
}

int fmha_fwd_from_host(int dtype, const void* hQ, const void* hK, const void* hV, void* hO, const fmha_mask_t* mask,
                       void* workspace, size_t workspace_bytes, int batch, int heads, int seq_q, int seq_kv,
                       int head_dim, float scale, fmha_stream_t stream_) {
  g_last_cuda_error[0] = 0;
  cudaStream_t stream = reinterpret_cast<cudaStream_t>(stream_);
  if (dtype != 0 && dtype != 1) return FMHA_ERR_UNSUPPORTED;
  // every argument check happens before anything is enqueued (include/fmha.h)
  if (mask && (mask->kind == FMHA_MASK_KEY_BIAS || mask->kind == FMHA_MASK_ATTN_BIAS))
    return FMHA_ERR_UNSUPPORTED;  // (device-pointer masks: fmha_fwd / fmha_fwd_strided only)
  bool empty = false;
  if (int vs = validate_shape(batch, heads, seq_q, seq_kv, head_dim, scale, mask, 1, &empty); vs != FMHA_OK || empty)
    return vs;
  const size_t u = static_cast<size_t>(batch) * heads;
  if (!hQ || !hK || !hV || !hO || !workspace) return FMHA_ERR_INVALID_ARG;
  if (workspace_bytes < fmha_workspace_bytes(batch, heads, seq_q, seq_kv, head_dim)) return FMHA_ERR_INVALID_ARG;
  if ((reinterpret_cast<uintptr_t>(workspace) & 255u) != 0) return FMHA_ERR_MISALIGNED;
  const size_t qb = u * seq_q * head_dim * 2, kvb = u * seq_kv * head_dim * 2;
  uint8_t* w = static_cast<uint8_t*>(workspace);
  uint8_t* dQ = w;
  uint8_t* dO = dQ + round_up(qb, 256);
  uint8_t* dK = dO + round_up(qb, 256);
  uint8_t* dV = dK + round_up(kvb, 256);
  int32_t* dL = reinterpret_cast<int32_t*>(dV + round_up(kvb, 256));
  fmha_mask_t dmask = {FMHA_MASK_NONE, nullptr, nullptr, 0};
  if (mask) {
    dmask.kind = mask->kind;
    if (mask->kind == FMHA_MASK_KEY_PADDING) {
      if (!mask->kv_len) return FMHA_ERR_INVALID_ARG;
      cudaError_t e = cudaMemcpyAsync(dL, mask->kv_len, sizeof(int32_t) * batch, cudaMemcpyHostToDevice, stream);
      if (e != cudaSuccess) return cuda_fail(e, "H2D kv_len");
      dmask.kv_len = dL;
    }
  }
  // Pipelined over batch chunks on three streams: the host->device copy of chunk c+1 and the
  // device->host copy of chunk c-1 overlap the kernel on chunk c (PCIe is full duplex), ordered by
  // events; `stream` waits for the last copy-out, so a caller that syncs `stream` sees O complete.
  // Each (b, h) is independent, so a chunk is just a smaller batch.  The streams and events are
  // created once per thread and device and reused (thread-local, so concurrent callers on other
  // threads never share them).
  cudaError_t e;
  // B200_E2E_CHUNKS: A/B of the pipelining depth (BERT-large-512 e2e: 4 chunks 15.5 TFLOP/s, 8 15.0-15.1,
  // 16 13.3-13.6 -- smaller copies lose more PCIe efficiency than the shorter tail gains)
  static const int max_chunks = [] {
    const char* v = std::getenv("B200_E2E_CHUNKS");
    const int c = v ? std::atoi(v) : 4;
    return (c >= 1 && c <= 16) ? c : 4;
  }();
  const int chunks = std::min(batch, max_chunks);
  const size_t qb1 = qb / batch, kvb1 = kvb / batch;  // bytes per batch element
  struct HostPipe {
    cudaStream_t sh = nullptr, sc = nullptr, sd = nullptr;
    cudaEvent_t start = nullptr, d = nullptr, h[16] = {}, c[16] = {};
    bool ok = false;
  };
  thread_local HostPipe pipes[64];
  int dev = 0;
  if ((e = cudaGetDevice(&dev)) != cudaSuccess || dev >= 64) return cuda_fail(e, "fmha_fwd_from_host device");
  HostPipe& hp = pipes[dev];
  if (!hp.ok) {
    bool ok = cudaStreamCreateWithFlags(&hp.sh, cudaStreamNonBlocking) == cudaSuccess &&
              cudaStreamCreateWithFlags(&hp.sc, cudaStreamNonBlocking) == cudaSuccess &&
              cudaStreamCreateWithFlags(&hp.sd, cudaStreamNonBlocking) == cudaSuccess &&
              cudaEventCreateWithFlags(&hp.start, cudaEventDisableTiming) == cudaSuccess &&
              cudaEventCreateWithFlags(&hp.d, cudaEventDisableTiming) == cudaSuccess;
    for (int c = 0; ok && c < 16; ++c)
      ok = cudaEventCreateWithFlags(&hp.h[c], cudaEventDisableTiming) == cudaSuccess &&
           cudaEventCreateWithFlags(&hp.c[c], cudaEventDisableTiming) == cudaSuccess;
    if (!ok) return cuda_fail(cudaGetLastError(), "fmha_fwd_from_host streams/events");
    hp.ok = true;
  }
  cudaStream_t sh = hp.sh, sc = hp.sc, sd = hp.sd;
  cudaEvent_t ev_start = hp.start, ev_d = hp.d, *ev_h = hp.h, *ev_c = hp.c;
  // everything already queued on `stream` (incl. the kv_len copy) happens first
  if ((e = cudaEventRecord(ev_start, stream)) != cudaSuccess ||
      (e = cudaStreamWaitEvent(sh, ev_start, 0)) != cudaSuccess) {
    return cuda_fail(e, "fmha_fwd_from_host ordering");
  }
  int st = FMHA_OK;
  for (int c = 0; c < chunks && st == FMHA_OK; ++c) {
    const int b0 = static_cast<int>(static_cast<long long>(batch) * c / chunks);
    const int b1 = static_cast<int>(static_cast<long long>(batch) * (c + 1) / chunks);
    const int nb = b1 - b0;
    const size_t oq = b0 * qb1, okv = b0 * kvb1;
    const uint8_t* hq = static_cast<const uint8_t*>(hQ) + oq;
    const uint8_t* hk = static_cast<const uint8_t*>(hK) + okv;
    const uint8_t* hv = static_cast<const uint8_t*>(hV) + okv;
    if ((e = cudaMemcpyAsync(dQ + oq, hq, nb * qb1, cudaMemcpyHostToDevice, sh)) != cudaSuccess ||
        (e = cudaMemcpyAsync(dK + okv, hk, nb * kvb1, cudaMemcpyHostToDevice, sh)) != cudaSuccess ||
        (e = cudaMemcpyAsync(dV + okv, hv, nb * kvb1, cudaMemcpyHostToDevice, sh)) != cudaSuccess ||
        (e = cudaEventRecord(ev_h[c], sh)) != cudaSuccess || (e = cudaStreamWaitEvent(sc, ev_h[c], 0)) != cudaSuccess) {
      st = cuda_fail(e, "H2D chunk");
      break;
    }
    fmha_mask_t cm = dmask;
    if (cm.kv_len) cm.kv_len = dL + b0;
    st = fmha_common(dtype == 1, dQ + oq, dK + okv, dV + okv, dO + oq, &cm, nb, heads, seq_q, seq_kv, head_dim, scale,
                     sc, 1, nullptr, 0, nullptr, false, static_cast<long long>(batch) * heads);
    if (st != FMHA_OK) break;
    if ((e = cudaEventRecord(ev_c[c], sc)) != cudaSuccess || (e = cudaStreamWaitEvent(sd, ev_c[c], 0)) != cudaSuccess ||
        (e = cudaMemcpyAsync(static_cast<uint8_t*>(hO) + oq, dO + oq, nb * qb1, cudaMemcpyDeviceToHost, sd)) !=
            cudaSuccess) {
      st = cuda_fail(e, "D2H chunk");
      break;
    }
  }
  // `stream` continues after the last copy-out (sd is in order, so it covers every chunk)
  if ((e = cudaEventRecord(ev_d, sd)) != cudaSuccess || (e = cudaStreamWaitEvent(stream, ev_d, 0)) != cudaSuccess)
    if (st == FMHA_OK) st = cuda_fail(e, "fmha_fwd_from_host join");
  return st;
}

int gemm_bias_act(const void* A, const void* W, const void* bias, void* Cm, int M, int N, int K, int act,
                  fmha_stream_t stream) {
  g_last_cuda_error[0] = 0;
  if (M < 0 || N < 0 || K < 0) return FMHA_ERR_INVALID_ARG;
  if (act < ACT_NONE || act > ACT_TANH) return FMHA_ERR_UNSUPPORTED;
  if (M == 0 || N == 0) return FMHA_OK;
  if (!A || !W || !Cm || K == 0) return FMHA_ERR_INVALID_ARG;
  if ((K % 8) != 0 || (N % 8) != 0) return FMHA_ERR_UNSUPPORTED;
  if (!aligned16(A) || !aligned16(W) || !aligned16(Cm) || (bias && !aligned16(bias))) return FMHA_ERR_MISALIGNED;
  int sms = 0;
  int st = check_device(&sms);
  if (st != FMHA_OK) return st;
  return b200::launch_gemm_bias_act(A, W, nullptr, nullptr, bias, Cm, M, N, K, 0, act, sms,
                                    reinterpret_cast<cudaStream_t>(stream), g_last_cuda_error,
                                    sizeof(g_last_cuda_error));
}

int dual_gemm_bias_act(const void* A1, const void* W1, const void* A2, const void* W2, const void* bias, void* Cm,
                       int M, int N, int K1, int K2, int act, fmha_stream_t stream) {
  g_last_cuda_error[0] = 0;
  if (M < 0 || N < 0 || K1 < 0 || K2 < 0) return FMHA_ERR_INVALID_ARG;
  if (act < ACT_NONE || act > ACT_TANH) return FMHA_ERR_UNSUPPORTED;
  if (M == 0 || N == 0) return FMHA_OK;
  if (!A1 || !W1 || !A2 || !W2 || !Cm || K1 == 0 || K2 == 0) return FMHA_ERR_INVALID_ARG;
  if ((K1 % 8) != 0 || (K2 % 8) != 0 || (N % 8) != 0) return FMHA_ERR_UNSUPPORTED;
  if (!aligned16(A1) || !aligned16(W1) || !aligned16(A2) || !aligned16(W2) || !aligned16(Cm) ||
      (bias && !aligned16(bias)))
    return FMHA_ERR_MISALIGNED;
  int sms = 0;
  int st = check_device(&sms);
  if (st != FMHA_OK) return st;
  return b200::launch_gemm_bias_act(A1, W1, A2, W2, bias, Cm, M, N, K1, K2, act, sms,
                                    reinterpret_cast<cudaStream_t>(stream), g_last_cuda_error,
                                    sizeof(g_last_cuda_error));
}

size_t fmha_splitkv_workspace_bytes(int batch, int heads, int seq_q, int head_dim, int num_splits) {
  if (batch <= 0 || heads <= 0 || seq_q <= 0 || head_dim <= 0 || num_splits <= 1) return 0;
  return splitkv_ws_bytes(static_cast<long long>(batch) * heads, seq_q, head_dim, num_splits);
}

int fmha_splitkv_default_splits(int batch, int heads, int seq_q, int seq_kv) {
  int sms = 0;
  if (batch <= 0 || heads <= 0 || seq_q <= 0 || seq_kv <= 0 || check_device(&sms) != FMHA_OK) return 1;
  return splitkv_default(static_cast<long long>(batch) * heads, seq_q, seq_kv, sms);
}

int fmha_fwd_splitkv(int dtype, const void* Q, const void* K, const void* V, void* O, const fmha_mask_t* mask,
                     int batch, int heads, int seq_q, int seq_kv, int head_dim, float scale, int num_splits,
                     void* workspace, size_t workspace_bytes, fmha_stream_t stream) {
  if (dtype != 0 && dtype != 1) return FMHA_ERR_UNSUPPORTED;
  if (num_splits < 0 || num_splits > 1024) return FMHA_ERR_UNSUPPORTED;
  return fmha_common(dtype == 1, Q, K, V, O, mask, batch, heads, seq_q, seq_kv, head_dim, scale,
                     reinterpret_cast<cudaStream_t>(stream), num_splits, workspace, workspace_bytes);
}

int fmha_streamk_plan(int batch, int heads, int seq_q, int seq_kv, int mask_kind, int sm_count, int* tail_items) {
  if (tail_items) *tail_items = 0;
  if (batch <= 0 || heads <= 0 || seq_q <= 0 || seq_kv <= 0 || sm_count <= 0) return 1;
  if (mask_kind == FMHA_MASK_KEY_BIAS || mask_kind == FMHA_MASK_ATTN_BIAS) return 1;
  int pair_mode = 0;
  const long long units = static_cast<long long>(batch) * heads;
  const int nq = (seq_q + 127) / 128;
  const long long items = dense_items(units, nq, mask_kind, sm_count, &pair_mode);
  long long rest = 0;
  const int s = streamk_plan(items, (seq_kv + 127) / 128, sm_count, singles_tail(items, units * nq, pair_mode, sm_count),
                             &rest);
  if (tail_items) *tail_items = static_cast<int>(rest);
  return s;
}

size_t fmha_streamk_workspace_bytes(int head_dim, int sm_count) {
  if (head_dim != 64 && head_dim != 128) return 0;
  if (sm_count <= 0 && check_device(&sm_count) != FMHA_OK) return 0;
  return streamk_ws_bytes(head_dim, sm_count);
}

int fmha_fwd_streamk(int dtype, const void* Q, const void* K, const void* V, void* O, const fmha_mask_t* mask,
                     int batch, int heads, int seq_q, int seq_kv, int head_dim, float scale, void* workspace,
                     size_t workspace_bytes, fmha_stream_t stream) {
  if (dtype != 0 && dtype != 1) return FMHA_ERR_UNSUPPORTED;
  return fmha_common(dtype == 1, Q, K, V, O, mask, batch, heads, seq_q, seq_kv, head_dim, scale,
                     reinterpret_cast<cudaStream_t>(stream), 1, workspace, workspace_bytes, nullptr, true);
}

int mlp_fused_fwd(const void* X, const void* W, const void* bias, void* Y, int M, int width, int layers, int act,
                  fmha_stream_t stream) {
  g_last_cuda_error[0] = 0;
  if (M < 0 || width < 0 || layers < 0) return FMHA_ERR_INVALID_ARG;
  if (act < ACT_NONE || act > ACT_TANH) return FMHA_ERR_UNSUPPORTED;
  if (width != 64 && width != 128) return FMHA_ERR_UNSUPPORTED;
  if (layers < 1 || layers > 65535) return FMHA_ERR_UNSUPPORTED;
  if (M == 0) return FMHA_OK;
  if (!X || !W || !Y) return FMHA_ERR_INVALID_ARG;
  if (!aligned16(X) || !aligned16(W) || !aligned16(Y) || (bias && !aligned16(bias))) return FMHA_ERR_MISALIGNED;
  int sms = 0;
  int st = check_device(&sms);
  if (st != FMHA_OK) return st;
  return b200::launch_mlp_fused(X, W, bias, Y, M, width, layers, act, sms, reinterpret_cast<cudaStream_t>(stream),
                                g_last_cuda_error, sizeof(g_last_cuda_error));
}

const char* fmha_status_string(int status) {
  switch (status) {
    case FMHA_OK: return "FMHA_OK";
    case FMHA_ERR_INVALID_ARG: return "FMHA_ERR_INVALID_ARG: invalid argument";
    case FMHA_ERR_UNSUPPORTED: return "FMHA_ERR_UNSUPPORTED: unsupported configuration";
    case FMHA_ERR_MISALIGNED: return "FMHA_ERR_MISALIGNED: pointer not 16-byte aligned";
    case FMHA_ERR_CUDA: return "FMHA_ERR_CUDA: CUDA error (see fmha_last_cuda_error)";
    case FMHA_ERR_NO_DEVICE: return "FMHA_ERR_NO_DEVICE: no sm_100 device is current";
    default: return "unknown status";
  }
}

const char* fmha_last_cuda_error(void) { return g_last_cuda_error; }

#if FMHA_TRACE || FMHA_PROF
// Debug-build only (not part of include/fmha.h): point the timeline recorder at a device buffer
// of 65536 uint64 records and reset its counter; fmha_trace_count() returns the record count.
FMHA_API int fmha_trace_set(void* dev_buf) {
  unsigned int zero = 0;
  if (cudaMemcpyToSymbol(b200::g_fmha_trace, &dev_buf, sizeof(void*)) != cudaSuccess) return FMHA_ERR_CUDA;
  if (cudaMemcpyToSymbol(b200::g_fmha_trace_n, &zero, sizeof(zero)) != cudaSuccess) return FMHA_ERR_CUDA;
  return FMHA_OK;
}
FMHA_API unsigned int fmha_trace_count(void) {
  unsigned int n = 0;
  cudaMemcpyFromSymbol(&n, b200::g_fmha_trace_n, sizeof(n));
  return n;
}
#endif

const char* fmha_version(void) { return "b200fmha 0.1 (sm_100a)"; }

}  // extern "C"
