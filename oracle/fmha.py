"""Unfused fp64 FMHA forward — the plain definition the fused kernel must reach.

TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).  Pinned by tests/test_oracle.py.

What it computes (paper §6 "Fused Multi-Head Attention"):
  "two back-to-back GEMMs with a softmax computation in between.  The softmax
   computation itself consists of two reductions and several pointwise
   operations."
For every (batch b, head h), with Q:[Sq,D], K:[Skv,D], V:[Skv,D]:

  1. S   = (Q @ K^T) * scale            GEMM #1, then a pointwise scale
  2. S[i,j] = -inf where masked         pointwise (R3, R5, R6)
  3. m_i = max_j S[i,j]                 reduction #1
  4. E   = exp(S - m_i)                 pointwise
  5. l_i = sum_j E[i,j]                 reduction #2
  6. P   = E / l_i                      pointwise
  7. O   = P @ V                        GEMM #2

Precision: all arithmetic in float64 on the widened (exactly representable)
fp16/bf16 inputs; ``scale`` is taken as the float32 value the kernel receives
(R1).  O is returned in float64, unrounded (R9 says the GPU rounds O
to the I/O dtype; the tolerance absorbs that rounding).

Masking readings (the paper's FMHA has no mask; BASELINE.json configs add them):
  R3  masked keys are excluded (-inf), so they contribute exactly zero.
  R4  a row with no unmasked key yields O_i = 0 (never NaN).
  R5  key padding: per-batch kv_len[b] valid keys (right padding), shared by all
      heads; query rows are computed regardless of kv_len.
  R6  causal is bottom-right aligned: key j is visible to query i iff
      j <= i + (Skv - Sq); with Sq == Skv this is j <= i.
  R20 additive key bias (the HF BERT "extended attention mask"; SURVEY §8(f) f2
      "arbitrary boolean/additive masks"): step 1 becomes
      S = (Q @ K^T) * scale + bias[b, None, :], bias in natural-log units, shared by
      all heads and queries of batch b; bias = -inf excludes the key (R3), and a row
      whose every score is -inf yields O_i = 0 (R4).
  R21 general additive (query x key) mask (SURVEY §8(f) f2 "arbitrary boolean/additive masks"; the
      HF "extended attention mask" in its general [B, 1 or H, Sq, Skv] form): step 1 becomes
      S = (Q @ K^T) * scale + attn_bias[b, h, i, j], attn_bias broadcastable to [B, H, Sq, Skv],
      natural-log units; -inf excludes the pair (query i, key j) (R3); a row whose every score is
      -inf yields O_i = 0 (R4).  A boolean mask M is the bias 0 where M, -inf elsewhere.
"""

from __future__ import annotations

import numpy as np


def _as_f64(x) -> np.ndarray:
    """Widen fp16/bf16/fp32 input (numpy array or torch CPU tensor) to fp64 exactly."""
    if hasattr(x, "detach"):  # torch tensor: widen on the torch side (bf16 has no numpy dtype)
        return x.detach().to("cpu").double().numpy()
    return np.asarray(x, dtype=np.float64)


def _scale_f64(scale: float) -> float:
    """R1: the kernel receives ``scale`` as a float32; the oracle uses that exact value."""
    return float(np.float32(scale))


def visible_mask(sq: int, skv: int, kv_len: int | None, causal: bool) -> np.ndarray:
    """Boolean [sq, skv]: True where key j is visible to query i (R3, R5, R6)."""
    vis = np.ones((sq, skv), dtype=bool)
    if kv_len is not None:
        vis[:, max(0, int(kv_len)):] = False
    if causal:
        i = np.arange(sq)[:, None]
        j = np.arange(skv)[None, :]
        vis &= j <= i + (skv - sq)
    return vis


def softmax_probs_fp64(q_bh, k_bh, scale: float, kv_len: int | None = None,
                       causal: bool = False, key_bias=None, attn_bias=None) -> np.ndarray:
    """Steps 1-6 for one (b,h): the row-stochastic matrix P [Sq, Skv] (rows of zeros
    where every key is masked, R4).  Exposed so tests can pin sum_j P[i,j] = 1.
    attn_bias: None or this (b, h)'s [Sq, Skv] additive bias (R21)."""
    q = _as_f64(q_bh)
    k = _as_f64(k_bh)
    sq, skv = q.shape[0], k.shape[0]
    s = (q @ k.T) * _scale_f64(scale)                       # step 1 (GEMM #1, scale)
    vis = visible_mask(sq, skv, kv_len, causal)
    if key_bias is not None:                                 # R20: additive key bias
        kb = np.asarray(key_bias, dtype=np.float64)[:skv]
        s = s + kb[None, :]
        vis = vis & (kb > -np.inf)[None, :]
    if attn_bias is not None:                                # R21: general additive mask
        ab = np.broadcast_to(np.asarray(attn_bias, dtype=np.float64), (sq, skv))
        s = s + ab
        vis = vis & (ab > -np.inf)
    s = np.where(vis, s, -np.inf)                            # step 2 (mask)
    any_vis = vis.any(axis=1)
    m = np.where(any_vis, s.max(axis=1, initial=-np.inf), 0.0)  # step 3 (max reduction)
    e = np.where(vis, np.exp(s - m[:, None]), 0.0)           # step 4 (exp)
    l = e.sum(axis=1)                                        # step 5 (sum reduction)
    p = np.where(any_vis[:, None], e / np.where(l > 0, l, 1.0)[:, None], 0.0)  # step 6
    return p


def attention_fp64(q, k, v, scale: float, kv_len=None, causal: bool = False, key_bias=None,
                   attn_bias=None) -> np.ndarray:
    """O = softmax(scale * Q K^T + mask) V for Q:[B,H,Sq,D], K,V:[B,H,Skv,D].

    ``kv_len`` is None or a length-B integer sequence (R5); ``key_bias`` None or
    [B, >= Skv] additive bias (R20); ``attn_bias`` None or an additive bias broadcastable
    to [B, H, Sq, Skv] (R21).  Returns float64 [B,H,Sq,D].  One (b,h) at a time, exactly
    steps 1-7 above.
    """
    q = _as_f64(q)
    k = _as_f64(k)
    v = _as_f64(v)
    b_, h_, sq, d = q.shape
    skv = k.shape[2]
    assert k.shape == (b_, h_, skv, d) and v.shape == (b_, h_, skv, d)
    out = np.zeros((b_, h_, sq, d), dtype=np.float64)
    ab = None if attn_bias is None else np.broadcast_to(_as_f64(attn_bias), (b_, h_, sq, skv))
    for b in range(b_):
        kl = None if kv_len is None else int(kv_len[b])
        for h in range(h_):
            kb = None if key_bias is None else np.asarray(key_bias, dtype=np.float64)[b]
            p = softmax_probs_fp64(q[b, h], k[b, h], scale, kl, causal, kb, None if ab is None else ab[b, h])
            out[b, h] = p @ v[b, h]                          # step 7 (GEMM #2)
    return out


def attention_rows_fp64(q, k, v, scale: float, units, kv_len=None,
                        causal: bool = False, key_bias=None, attn_bias=None) -> np.ndarray:
    """Steps 1-7 for a sample of output rows only: ``units`` is a list of
    (b, h, i) triples; returns float64 [len(units), D].  Used for parity at full
    BASELINE sizes, where the whole oracle would take too long on the sampled
    launch configuration (every row still sees all its keys)."""
    res = []
    for (b, h, i) in units:
        qi = _as_f64(q[b, h, i:i + 1])
        kb = _as_f64(k[b, h])
        vb = _as_f64(v[b, h])
        sq = q.shape[2]
        skv = kb.shape[0]
        kl = None if kv_len is None else int(kv_len[b])
        s = (qi @ kb.T)[0] * _scale_f64(scale)
        vis = visible_mask(sq, skv, kl, causal)[i]
        if key_bias is not None:                             # R20
            bb = np.asarray(key_bias, dtype=np.float64)[b][:skv]
            s = s + bb
            vis = vis & (bb > -np.inf)
        if attn_bias is not None:                            # R21
            ab = np.broadcast_to(_as_f64(attn_bias), (q.shape[0], q.shape[1], sq, skv))[b, h, i]
            s = s + ab
            vis = vis & (ab > -np.inf)
        if not vis.any():
            res.append(np.zeros(vb.shape[1]))
            continue
        s = np.where(vis, s, -np.inf)
        m = s.max()
        e = np.where(vis, np.exp(s - m), 0.0)
        p = e / e.sum()
        res.append(p @ vb)
    return np.stack(res) if res else np.zeros((0, v.shape[-1]))


def attention_varlen_fp64(qkv, cu_seqlens, scale: float, causal: bool = False) -> np.ndarray:
    """Variable-length packed attention (MLPerf BERT inference layout; R17).

    ``qkv`` [T, 3, H, D] holds Q, K, V of every token; sequence s is tokens
    cu_seqlens[s] .. cu_seqlens[s+1]-1.  Each sequence is an independent problem:
    for every head h, steps 1-7 above on Q = qkv[a:b, 0, h], K = qkv[a:b, 1, h],
    V = qkv[a:b, 2, h] (causal: key j visible to query i iff j <= i, positions
    within the sequence).  Returns float64 O [T, H, D]."""
    x = _as_f64(qkv)
    t_, three, h_, d = x.shape
    assert three == 3
    cu = [int(c) for c in cu_seqlens]
    out = np.zeros((t_, h_, d), dtype=np.float64)
    for s in range(len(cu) - 1):
        a, b = cu[s], cu[s + 1]
        if b <= a:
            continue
        for h in range(h_):
            p = softmax_probs_fp64(x[a:b, 0, h], x[a:b, 1, h], scale, None, causal)
            out[a:b, h] = p @ x[a:b, 2, h]                   # step 7 (GEMM #2)
    return out


def fmha_flops(batch: int, heads: int, sq: int, skv: int, d: int, kv_len=None,
               causal: bool = False) -> float:
    """Algorithmic flops: 4*D per visible (i,j) pair (2*D for Q.K, 2*D for P.V).
    Masked pairs are not counted; neither is softmax arithmetic."""
    total = 0
    for b in range(batch):
        kl = skv if kv_len is None else max(0, min(int(kv_len[b]), skv))
        if causal:
            off = skv - sq
            # visible pairs per row i: clamp(min(kl, i + off + 1), 0)
            i = np.arange(sq)
            total += int(np.clip(np.minimum(kl, i + off + 1), 0, None).sum()) * heads
        else:
            total += sq * kl * heads
    return 4.0 * d * total
