/* fmha.h — C ABI of libb200fmha: B200-native (sm_100a) fused multi-head attention forward and
 * GEMM + bias + activation.
 *
 * Operation (paper §6 "Fused Multi-Head Attention": "two back-to-back GEMMs with a
 * softmax computation in between"; shapes of MLPerf BERT inference, L489):
 *
 *     O[b,h,i,:] = sum_j softmax_j( scale * <Q[b,h,i,:], K[b,h,j,:]> + mask[b,i,j] ) * V[b,h,j,:]
 *
 * for every batch b < batch, head h < heads, query row i < seq_q, key j < seq_kv.
 * Precision ("FP16 tensors using FP32 Tensor Core accumulation"): inputs and output
 * fp16 (fmha_fwd) or bf16 (fmha_fwd_bf16); both GEMMs accumulate in fp32 on the tensor cores;
 * the softmax runs in fp32; P is rounded to the I/O type before the second GEMM; O is rounded
 * once, round-to-nearest-even.
 *
 * Layout: Q, O are [batch, heads, seq_q, head_dim] and K, V are [batch, heads, seq_kv, head_dim],
 * dense row-major (head_dim contiguous), no padding between rows.
 *
 * Masks (the paper's FMHA has none; BASELINE.json configs add them; R3-R6):
 *   FMHA_MASK_NONE         every key visible.
 *   FMHA_MASK_KEY_PADDING  key j visible iff j < kv_len[b] (right padding, shared by all heads).
 *                          kv_len is a DEVICE int32 array [batch]; values are clamped to [0, seq_kv].
 *   FMHA_MASK_CAUSAL       key j visible iff j <= i + (seq_kv - seq_q)  (bottom-right aligned).
 *   FMHA_MASK_KEY_BIAS     additive per-key bias (the HF BERT "extended attention mask"; DESIGN.md
 *                          R20): S[i,j] = scale * <q_i, k_j> + key_bias[b * key_bias_stride + j],
 *                          natural-log units, shared by all heads and queries of batch b; -inf
 *                          excludes the key.  key_bias: DEVICE fp32, 16-byte aligned;
 *                          key_bias_stride >= seq_kv and a multiple of 4; scale must be > 0.
 *                          fmha_fwd / fmha_fwd_bf16 only (other entry points: FMHA_ERR_UNSUPPORTED).
 *   FMHA_MASK_ATTN_BIAS    general additive (query x key) mask (R21; the HF extended
 *                          attention mask in its [B, 1 or H, Sq, Skv] form): S[i,j] = scale * <q_i,
 *                          k_j> + attn_bias[b, h, i, j] (layout and strides in fmha_mask_t), natural-
 *                          log units, -inf excludes the pair; scale must be > 0.  fmha_fwd,
 *                          fmha_fwd_bf16 and fmha_fwd_strided only.
 * The kinds are exclusive.  A query row with no visible key produces O = 0 (never NaN).
 *
 * Ownership and errors: every tensor pointer is caller-owned; the library never allocates device
 * memory, never synchronises the stream and retains no pointer past the call (kv_len must stay
 * valid until the kernel completes, stream-ordered).  `mask` is read on the host during the call.
 * Validation failures return a non-zero fmha_status_t before anything is launched; launch failures
 * return FMHA_ERR_CUDA.  Device faults surface at the caller's next synchronisation.  The library
 * is thread-safe; its host state is a cache (the driver entry point for tensor-map encoding, per-device
 * kernel attributes and device properties, all mutex-protected) plus fmha_fwd_from_host's per-thread
 * copy streams.  There is no CPU fallback: without an sm_100 device every entry point that
 * launches returns FMHA_ERR_NO_DEVICE.
 */
#ifndef B200FMHA_FMHA_H
#define B200FMHA_FMHA_H

#include <stddef.h>
#include <stdint.h>

#if defined(__GNUC__)
#define FMHA_API __attribute__((visibility("default")))
#else
#define FMHA_API
#endif

#ifdef __cplusplus
extern "C" {
#endif

typedef struct CUstream_st* fmha_stream_t; /* == cudaStream_t; NULL = legacy default stream */

typedef enum {
  FMHA_OK = 0,
  FMHA_ERR_INVALID_ARG = 1, /* null pointer, negative size, non-finite scale, ...            */
  FMHA_ERR_UNSUPPORTED = 2, /* head_dim not in {64,128}, negative scale, unknown mask / act   */
  FMHA_ERR_MISALIGNED = 3,  /* a tensor pointer is not 16-byte aligned (TMA requirement)       */
  FMHA_ERR_CUDA = 4,        /* a CUDA runtime/driver call failed; see fmha_last_cuda_error()   */
  FMHA_ERR_NO_DEVICE = 5    /* no sm_100 device is current                                    */
} fmha_status_t;

typedef enum {
  FMHA_MASK_NONE = 0,
  FMHA_MASK_KEY_PADDING = 1,
  FMHA_MASK_CAUSAL = 2,
  FMHA_MASK_KEY_BIAS = 3,
  FMHA_MASK_ATTN_BIAS = 4
} fmha_mask_kind_t;

typedef struct {
  int32_t kind;            /* fmha_mask_kind_t                                                 */
  const int32_t* kv_len;   /* DEVICE pointer, [batch]; required for KEY_PADDING, else ignored  */
  const float* key_bias;   /* DEVICE pointer, [batch, key_bias_stride]; KEY_BIAS only          */
  int32_t key_bias_stride; /* elements between batches of key_bias; KEY_BIAS only              */
  /* ATTN_BIAS only: DEVICE pointer to the additive bias in the I/O type (fp16 for fmha_fwd, bf16
   * for fmha_fwd_bf16 / dtype 1), element (b, h, i, j) at attn_bias[b * attn_bias_stride_b +
   * h * attn_bias_stride_h + i * attn_bias_stride_q + j]; strides in elements, 0 broadcasts (e.g.
   * attn_bias_stride_h = 0 for the HF [B, 1, Sq, Skv] mask); attn_bias_stride_q 0 (one row for every
   * query; it must then hold seq_kv rounded up to 8 elements) or >= seq_kv and a multiple of 8; the
   * pointer 16-byte aligned; columns j >= seq_kv of a row may be read, never used. */
  const void* attn_bias;
  int64_t attn_bias_stride_b;
  int64_t attn_bias_stride_h;
  int64_t attn_bias_stride_q;
} fmha_mask_t;

/* Element strides {batch, head, row} of Q, K, V and O for fmha_fwd_strided (head_dim is always
 * contiguous).  Contiguous [B, H, S, D] is {H*S*D, S*D, D}; the HF / packed-projection layout
 * [B, S, H, D] is {S*H*D, D, H*D}.  Every stride must be a multiple of 8 elements (16 bytes, the
 * TMA requirement) and the row stride >= head_dim; overlapping outputs are not detected. */
typedef struct {
  int64_t q[3];
  int64_t k[3];
  int64_t v[3];
  int64_t o[3];
} fmha_strides_t;

/* FMHA forward, fp16 in / fp16 out.
 *   Q, K, V, O : DEVICE pointers, 16-byte aligned, layouts above.
 *   mask       : HOST pointer or NULL (= FMHA_MASK_NONE).
 *   batch, heads, seq_q, seq_kv >= 0 (seq_kv >= 1 unless batch*heads*seq_q == 0);
 *   head_dim   : 64 or 128.
 *   scale      : finite, >= 0; usually 1/sqrt(head_dim).
 *   stream     : CUDA stream the kernel is enqueued on.
 * batch*heads*seq_q == 0 returns FMHA_OK without launching. */
FMHA_API int fmha_fwd(const void* Q, const void* K, const void* V, void* O, const fmha_mask_t* mask, int batch,
             int heads, int seq_q, int seq_kv, int head_dim, float scale, fmha_stream_t stream);

/* Identical contract with bf16 tensors. */
FMHA_API int fmha_fwd_bf16(const void* Q, const void* K, const void* V, void* O, const fmha_mask_t* mask, int batch,
                  int heads, int seq_q, int seq_kv, int head_dim, float scale, fmha_stream_t stream);

/* Strided layouts: the same operation as fmha_fwd with Q, K, V, O addressed
 * through per-tensor {batch, head, row} element strides (fmha_strides_t, HOST pointer, read during the
 * call), e.g. [B, S, H, D] tensors straight out of a QKV projection without a transpose.  dtype: 0 =
 * fp16, 1 = bf16.  Masks, precision, ownership and errors as fmha_fwd; a stride TMA cannot address
 * returns FMHA_ERR_INVALID_ARG before anything is launched.  strides == NULL means contiguous. */
FMHA_API int fmha_fwd_strided(int dtype, const void* Q, const void* K, const void* V, void* O,
                              const fmha_strides_t* strides, const fmha_mask_t* mask, int batch, int heads,
                              int seq_q, int seq_kv, int head_dim, float scale, fmha_stream_t stream);

/* Variable-length packed input: the MLPerf BERT inference format the paper's FMHA serves
 * (SURVEY.md §8(f) f2).  A batch of num_seqs sequences is stored back to back:
 *   QKV        DEVICE [total_tokens, 3, heads, head_dim]  (Q, K, V of token t, e.g. the output of one
 *              fused QKV projection GEMM: row t = [q_h0 .. q_hH-1 | k_h0 .. | v_h0 ..])
 *   O          DEVICE [total_tokens, heads, head_dim]
 *   cu_seqlens DEVICE int32 [num_seqs + 1]: sequence s is tokens [cu_seqlens[s], cu_seqlens[s+1]);
 *              cu_seqlens[0] = 0, nondecreasing, cu_seqlens[num_seqs] = total_tokens (not checked:
 *              out-of-range values make the kernel read or write outside the buffers).
 *   max_seqlen HOST int >= every sequence length (sizes the work decomposition; larger is legal).
 * For every sequence s, head h and token i of s:
 *     O[i,h,:] = sum_{j in s} softmax_j( scale * <Q[i,h,:], K[j,h,:]> + mask ) * V[j,h,:]
 * with mask = none (causal = 0) or j <= i (causal = 1, positions within the sequence).  Tokens of
 * different sequences never attend to each other; zero-length sequences are allowed.
 * dtype: 0 = fp16, 1 = bf16.  Precision, ownership, errors: as fmha_fwd.  QKV and O 16-byte
 * aligned, cu_seqlens 4-byte aligned. */
FMHA_API int fmha_fwd_varlen(const void* QKV, void* O, const int32_t* cu_seqlens, int num_seqs, int max_seqlen,
                             int total_tokens, int heads, int head_dim, float scale, int causal, int dtype,
                             fmha_stream_t stream);

/* End-to-end variant: Q/K/V/O and kv_len are HOST buffers (pinned memory for asynchronous copies).
 * Copies Q, K, V (and kv_len) host->device into `workspace`, runs the same kernel, copies O
 * device->host.  The work is ordered after everything already queued on `stream` and pipelined over
 * up to 4 batch chunks on three internal streams (created on a thread's first call for a device and
 * reused by that thread; the copy-in of chunk c+1 and the copy-out of chunk c-1 overlap the kernel on
 * chunk c); `stream` is made to wait for the
 * last copy-out, so syncing `stream` (no synchronisation happens inside) makes O complete on the host.
 * Results are bitwise those of fmha_fwd (every (b, h) is independent of the batch it runs in).
 * dtype: 0 = fp16, 1 = bf16.  `workspace` is a DEVICE buffer of at least
 * fmha_workspace_bytes(batch, heads, seq_q, seq_kv, head_dim) bytes, 256-byte aligned.
 * For this entry point mask->kv_len is a HOST pointer. */
FMHA_API size_t fmha_workspace_bytes(int batch, int heads, int seq_q, int seq_kv, int head_dim);
FMHA_API int fmha_fwd_from_host(int dtype, const void* hQ, const void* hK, const void* hV, void* hO,
                       const fmha_mask_t* mask, void* workspace, size_t workspace_bytes, int batch, int heads,
                       int seq_q, int seq_kv, int head_dim, float scale, fmha_stream_t stream);

/* Split-KV FMHA: the same operation as fmha_fwd / fmha_fwd_bf16 (dtype 0 = fp16,
 * 1 = bf16; same layouts, mask and scale rules), for shapes where (batch x heads x query-tile pairs)
 * would leave SMs idle -- few heads, short query blocks (seq_q <= 128: decode-like) and long keys.
 * Each row's keys are cut into `num_splits` contiguous ranges of whole 128-key tiles; one kernel
 * computes every (b, h, q-tile pair, split) as its own work item and writes the split's online-softmax
 * state (unnormalised O in fp32, the exp2 reference scale*log2(e)*m and the row sum l, PAPER.md L487's
 * softmax restricted to the range) into `workspace`; a second kernel merges the splits
 * (O = sum_s 2^(m_s - M) O_s / sum_s 2^(m_s - M) l_s) and rounds O once.  num_splits = 0 picks
 * fmha_splitkv_default_splits(); the count is clamped so every split holds at least one key tile, and
 * a count of 1 runs the fmha_fwd kernel (no workspace needed).  `workspace`: DEVICE, 16-byte aligned,
 * >= fmha_splitkv_workspace_bytes(batch, heads, seq_q, head_dim, splits) bytes (else
 * FMHA_ERR_INVALID_ARG), owned by the caller, used until both kernels complete (stream order).
 * Two launches on `stream`; errors as fmha_fwd. */
FMHA_API int fmha_splitkv_default_splits(int batch, int heads, int seq_q, int seq_kv);
FMHA_API size_t fmha_splitkv_workspace_bytes(int batch, int heads, int seq_q, int head_dim, int num_splits);
FMHA_API int fmha_fwd_splitkv(int dtype, const void* Q, const void* K, const void* V, void* O,
                              const fmha_mask_t* mask, int batch, int heads, int seq_q, int seq_kv, int head_dim,
                              float scale, int num_splits, void* workspace, size_t workspace_bytes,
                              fmha_stream_t stream);

/* Stream-K tail FMHA: the same operation, layouts, masks and scale rules as
 * fmha_fwd / fmha_fwd_bf16 (dtype 0 = fp16, 1 = bf16), in ONE launch of the persistent
 * kernel whose last, partial round is split along the keys.  The full rounds run the fmha_fwd schedule;
 * each of the last round's `tail_items` items is cut into s ranges of whole 128-key tiles
 * (fmha_streamk_plan), every piece writes its online-softmax state (unnormalised fp32 O, the exp2
 * reference scale*log2(e)*m and the row sum l) to `workspace` and counts itself in a per-item counter,
 * and the piece that counts last merges O = sum_s 2^(m_s - M) O_s / sum_s 2^(m_s - M) l_s and stores
 * it (one RNE rounding).  The last round then takes ~1/s of the time (BERT-large-384: 28 of 768
 * items in the last round of 148 SMs, s = 3).  When the plan gives s = 1 (or the mask is a bias) this
 * runs exactly fmha_fwd's kernel and schedule and does not touch `workspace`.
 * `workspace`: DEVICE, 256-byte aligned, >= fmha_streamk_workspace_bytes(head_dim, 0) bytes, owned by
 * the caller; it MUST be zero-filled before its first use, and every launch leaves it zero-filled
 * again (the merging piece resets its counter), so one buffer serves any number of launches on one
 * stream (not concurrent launches).  Results agree with fmha_fwd within the oracle tolerance, not
 * bitwise (the tail rows are summed in another order).  Errors as fmha_fwd; too small a workspace ->
 * FMHA_ERR_INVALID_ARG, misaligned -> FMHA_ERR_MISALIGNED. */
FMHA_API int fmha_fwd_streamk(int dtype, const void* Q, const void* K, const void* V, void* O,
                              const fmha_mask_t* mask, int batch, int heads, int seq_q, int seq_kv, int head_dim,
                              float scale, void* workspace, size_t workspace_bytes, fmha_stream_t stream);
/* Bytes of fmha_fwd_streamk's workspace for head_dim on a GPU with sm_count SMs (sm_count <= 0: the
 * current device; 0 if there is none or head_dim is unsupported).  Host-only. */
FMHA_API size_t fmha_streamk_workspace_bytes(int head_dim, int sm_count);
/* The key-split count s of fmha_fwd_streamk's tail for this shape and mask kind on sm_count SMs
 * (1 = no split), and *tail_items (may be NULL) = the items of the last, partial round.  Host-only,
 * needs no device. */
FMHA_API int fmha_streamk_plan(int batch, int heads, int seq_q, int seq_kv, int mask_kind, int sm_count,
                               int* tail_items);

/* GEMM + bias + activation, the MLP building block:
 *     C[m,n] = act( sum_k A[m,k] * W[n,k] + bias[n] )
 * A [M,K], W [N,K] (nn.Linear layout), bias [N] (or NULL), C [M,N]: fp16, row-major, DEVICE,
 * 16-byte aligned; fp32 accumulation, bias and activation in fp32, one RNE rounding to fp16.
 * Requires K % 8 == 0 and N % 8 == 0 (16-byte row pitch for TMA).
 * act: 0 none, 1 ReLU, 2 GELU (erf), 3 GELU (tanh), 4 tanh. */
typedef enum { ACT_NONE = 0, ACT_RELU = 1, ACT_GELU_ERF = 2, ACT_GELU_TANH = 3, ACT_TANH = 4 } fmha_act_t;
FMHA_API int gemm_bias_act(const void* A, const void* W, const void* bias, void* C, int M, int N, int K, int act,
                  fmha_stream_t stream);

/* Dual GEMM + bias + activation in one kernel: the paper's simplified LSTM cell (PAPER.md L471-L475,
 * Fig. 12: "two independent GEMMs followed by an addition and two more pointwise operations"):
 *     C[m,n] = act( sum_k A1[m,k] W1[n,k] + sum_k A2[m,k] W2[n,k] + bias[n] )
 * A1 [M,K1], W1 [N,K1], A2 [M,K2], W2 [N,K2], bias [N] or NULL, C [M,N]; fp16, row-major, DEVICE,
 * 16-byte aligned; both products accumulate into ONE fp32 accumulator (no intermediate tensor),
 * then bias, activation (act as gemm_bias_act, plus 4 = tanh, the LSTM cell's usual activation)
 * and one RNE rounding.  Requires K1, K2, N multiples of 8.  Errors as gemm_bias_act. */
FMHA_API int dual_gemm_bias_act(const void* A1, const void* W1, const void* A2, const void* W2, const void* bias,
                                void* C, int M, int N, int K1, int K2, int act, fmha_stream_t stream);

/* Fused multi-layer MLP in ONE kernel: the paper's Fig. 11 ("Fusing
 * multiple MLP-Layers (GEMM + bias-add + ReLU activation) into a single kernel", possible "for
 * N=K<=128 with arbitrary M", up to 20 layers), SURVEY.md §8(f) f4:
 *     h_0 = X;   h_l[m,n] = act( sum_k h_{l-1}[m,k] * W[l-1][n][k] + bias[l-1][n] ),  l = 1..layers;
 *     Y = h_layers
 * X, Y [M, width]; W [layers, width, width] (each layer nn.Linear [out, in]); bias [layers, width] or
 * NULL: fp16, row-major, DEVICE, 16-byte aligned.  Every layer accumulates in fp32 and rounds once
 * (RNE) to fp16; the intermediates h_1..h_{layers-1} are fp16 tiles that never leave shared memory
 * (R19).  width must be 64 or 128 (FMHA_ERR_UNSUPPORTED otherwise), 1 <= layers <= 65535,
 * any M >= 0 (M = 0: no launch).  act as gemm_bias_act (the paper's is 1 = ReLU).  Y must not
 * overlap W or bias; Y == X (in place) is allowed (each 128-row tile is read before it is written,
 * by the same CTA).  Errors: as gemm_bias_act. */
FMHA_API int mlp_fused_fwd(const void* X, const void* W, const void* bias, void* Y, int M, int width, int layers,
                           int act, fmha_stream_t stream);

/* End-to-end synthetic Transformer layer (the paper's end-to-end use of its
 * fused kernels), fp16, tokens packed as in fmha_fwd_varlen:
 *     QKV = X Wqkv^T + bqkv        X [T, d_model], Wqkv [3 d_model, d_model] (rows: Q heads, K heads,
 *                                  V heads, so QKV is the [T, 3, heads, head_dim] layout)
 *     A   = fmha_varlen(QKV)       per-sequence attention, [T, heads, head_dim] = [T, d_model]
 *     Z   = A Wo^T + bo            Wo [d_model, d_model]
 *     H   = GELU_erf(Z W1^T + b1)  W1 [d_ff, d_model]
 *     Y   = H W2^T + b2            W2 [d_model, d_ff], Y [T, d_model]
 * (no residual adds or LayerNorm: DESIGN.md R18).  Five launches on `stream` (three of them the
 * gemm_bias_act kernel, one fmha).  head_dim = d_model / heads must be 64 or 128; d_model and d_ff
 * multiples of 8; biases may be NULL.  Intermediates live in `workspace` (DEVICE, 256-byte aligned,
 * >= transformer_layer_workspace_bytes(T, d_model, d_ff) bytes).  Errors: as the component calls;
 * the first failing launch's status is returned and later stages are not launched. */
FMHA_API size_t transformer_layer_workspace_bytes(int tokens, int d_model, int d_ff);
FMHA_API int transformer_layer_fwd(const void* X, const void* Wqkv, const void* bqkv, const void* Wo,
                                   const void* bo, const void* W1, const void* b1, const void* W2, const void* b2,
                                   void* Y, const int32_t* cu_seqlens, int num_seqs, int max_seqlen, int tokens,
                                   int d_model, int heads, int d_ff, float scale, int causal, void* workspace,
                                   size_t workspace_bytes, fmha_stream_t stream);

/* Human-readable text for a status code (static storage). */
FMHA_API const char* fmha_status_string(int status);
/* Text of the last CUDA error seen by this thread inside the library ("" if none). */
FMHA_API const char* fmha_last_cuda_error(void);
/* Library version string. */
FMHA_API const char* fmha_version(void);

#ifdef __cplusplus
}
#endif
#endif /* B200FMHA_FMHA_H */
