"""fp64 synthetic Transformer layer: QKV projection -> FMHA -> out-projection -> MLP.

TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).

The paper's end-to-end result is its fused kernels -- the FMHA of
P:L487 and the GEMM+bias+activation MLP blocks of P:L439-L445 / L453 -- running
inside a BERT model.  SURVEY.md §8(f) f1 fixes the synthetic layer built from
exactly those kernels (R18; no residual adds, no LayerNorm):

    QKV = X Wqkv^T + bqkv          (gemm_bias_act_fp64, act none)
    A   = attention per sequence   (attention_varlen_fp64 on QKV viewed [T,3,H,D])
    Z   = A Wo^T + bo
    H   = GELU_erf(Z W1^T + b1)
    Y   = H W2^T + b2

Storage between the stages is the layer's I/O type: every stage reads fp16
operands and its result is stored as fp16 (round-to-nearest-even), so each stage
here is computed in fp64 from fp16-rounded inputs and rounded to fp16 before the
next stage reads it -- the same rounding points as the GPU layer.  The final Y is
returned unrounded (float64).
"""

from __future__ import annotations

import numpy as np

from .fmha import _as_f64, attention_varlen_fp64
from .gemm import ACT_GELU_ERF, ACT_NONE, gemm_bias_act_fp64


def round_fp16(x: np.ndarray) -> np.ndarray:
    """RNE rounding of float64 values to fp16, returned as float64 (numpy's cast is RNE)."""
    return np.asarray(x, dtype=np.float64).astype(np.float16).astype(np.float64)


def transformer_layer_fp64(x, wqkv, bqkv, wo, bo, w1, b1, w2, b2, cu_seqlens, heads: int, scale: float,
                           causal: bool = False) -> np.ndarray:
    """Returns Y [T, d_model] (float64) for packed tokens x [T, d_model]."""
    x = _as_f64(x)
    t, d = x.shape
    qkv = round_fp16(gemm_bias_act_fp64(x, wqkv, bqkv, ACT_NONE))            # [T, 3d]
    a = attention_varlen_fp64(qkv.reshape(t, 3, heads, d // heads), cu_seqlens, scale, causal)
    a = round_fp16(a.reshape(t, d))                                          # [T, d]
    z = round_fp16(gemm_bias_act_fp64(a, wo, bo, ACT_NONE))                  # [T, d]
    h = round_fp16(gemm_bias_act_fp64(z, w1, b1, ACT_GELU_ERF))              # [T, d_ff]
    return gemm_bias_act_fp64(h, w2, b2, ACT_NONE)                           # [T, d]
