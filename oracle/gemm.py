"""fp64 GEMM + bias + activation — the MLP building block (paper §6, Fig 10/11).

TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).

P:L439-L445: "GEMM kernels with fused pointwise operations, like addition of a
bias tensor or applying the Rectified Linear Unit (ReLU) activation function";
P:L443/L453: an MLP layer is "GEMM + bias-add + ReLU activation".
BASELINE.json config 5 uses GELU (R14): GELU_ERF is
0.5*x*(1+erf(x/sqrt 2)); GELU_TANH is 0.5*x*(1+tanh(sqrt(2/pi)*(x+0.044715 x^3))).

C[M,N] = act(A[M,K] @ W[N,K]^T + b[N])   (W in nn.Linear layout, R15)
"""

from __future__ import annotations

import math

import numpy as np

from .fmha import _as_f64

ACT_NONE, ACT_RELU, ACT_GELU_ERF, ACT_GELU_TANH, ACT_TANH = 0, 1, 2, 3, 4


def relu(x: np.ndarray) -> np.ndarray:
    return np.maximum(x, 0.0)


_erf = np.vectorize(math.erf, otypes=[np.float64])


def gelu_erf(x: np.ndarray) -> np.ndarray:
    x = np.asarray(x, dtype=np.float64)
    return 0.5 * x * (1.0 + _erf(x / math.sqrt(2.0)))


def gelu_tanh(x: np.ndarray) -> np.ndarray:
    x = np.asarray(x, dtype=np.float64)
    return 0.5 * x * (1.0 + np.tanh(math.sqrt(2.0 / math.pi) * (x + 0.044715 * x ** 3)))


def gemm_bias_act_fp64(a, w, bias=None, act: int = ACT_NONE) -> np.ndarray:
    """act(A @ W^T + b) in float64 on the widened inputs."""
    a = _as_f64(a)
    w = _as_f64(w)
    c = a @ w.T                                  # GEMM (fp64)
    if bias is not None:
        c = c + _as_f64(bias)[None, :]           # pointwise bias
    if act == ACT_NONE:
        return c
    if act == ACT_RELU:
        return relu(c)
    if act == ACT_GELU_ERF:
        return gelu_erf(c)
    if act == ACT_GELU_TANH:
        return gelu_tanh(c)
    if act == ACT_TANH:
        return np.tanh(c)
    raise ValueError(f"unknown act {act}")


def dual_gemm_bias_act_fp64(a1, w1, a2, w2, bias=None, act: int = ACT_RELU) -> np.ndarray:
    """The paper's simplified LSTM cell (Fig. 12): two independent GEMMs, their
    addition, the bias addition and the activation -- act(A1 @ W1^T + A2 @ W2^T + b) -- in float64,
    in the order the paper lists the nodes."""
    g1 = _as_f64(a1) @ _as_f64(w1).T             # GEMM 1
    g2 = _as_f64(a2) @ _as_f64(w2).T             # GEMM 2 (independent)
    c = g1 + g2                                  # addition
    if bias is not None:
        c = c + _as_f64(bias)[None, :]           # pointwise bias
    return _act(c, act)                          # activation


def _act(c: np.ndarray, act: int) -> np.ndarray:
    if act == ACT_NONE:
        return c
    if act == ACT_RELU:
        return relu(c)
    if act == ACT_GELU_ERF:
        return gelu_erf(c)
    if act == ACT_GELU_TANH:
        return gelu_tanh(c)
    if act == ACT_TANH:
        return np.tanh(c)
    raise ValueError(f"unknown act {act}")
