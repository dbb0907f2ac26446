"""fp64 fused multi-layer MLP — the paper's Fig. 11 computation.

TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).

P:L443 (Fig. 11 caption): "Fusing multiple MLP-Layers (GEMM + bias-add + ReLU activation) into a
single kernel"; "it is possible to fuse multiple MLP layers into a single kernel. In these
cases, all intermediate tensors fit into the GPU's shared memory"; footnote 2: "For example
N=K<=128 with arbitrary M"; up to 20 layers.

    h_0 = X                                   [M, N]
    h_l = act(h_{l-1} W_l^T + b_l)            W_l [N, N] (nn.Linear layout), b_l [N], l = 1..L
    Y   = h_L

The intermediates h_1 .. h_{L-1} are tensors of the layer's I/O type (fp16) held in shared memory
(P:L453), so each is rounded to fp16 (RNE) before the next layer reads it (R19); the final
h_L is returned unrounded (float64).  Every layer is computed in fp64 on its fp16 operands, in the
order the caption lists the nodes: GEMM, bias-add, activation.
"""

from __future__ import annotations

import numpy as np

from .fmha import _as_f64
from .gemm import ACT_RELU, gemm_bias_act_fp64


def _round_fp16(x: np.ndarray) -> np.ndarray:
    return np.asarray(x, dtype=np.float64).astype(np.float16).astype(np.float64)


def mlp_fused_fp64(x, w, b=None, act: int = ACT_RELU) -> np.ndarray:
    """x [M, N], w [L, N, N], b [L, N] or None  ->  Y [M, N] float64 (h_L unrounded)."""
    h = _as_f64(x)
    w = _as_f64(w)
    bb = None if b is None else _as_f64(b)
    layers = w.shape[0]
    for l in range(layers):
        h = gemm_bias_act_fp64(h, w[l], None if bb is None else bb[l], act)   # GEMM + bias-add + act
        if l + 1 < layers:
            h = _round_fp16(h)                                                 # stored as fp16 (R19)
    return h


def mlp_fused_rows_fp64(x, w, b, rows, act: int = ACT_RELU) -> np.ndarray:
    """The same for the selected rows of x only (rows are independent): [len(rows), N]."""
    x = np.asarray(x)
    return mlp_fused_fp64(x[np.asarray(rows)], w, b, act)


def mlp_fused_flops(m: int, n: int, layers: int) -> int:
    """Algorithmic flops: 2 M N N per layer (the bias and activation are not counted)."""
    return 2 * m * n * n * layers
