"""CPU oracle for the FMHA forward pass and the GEMM+bias+activation block.

TEST INFRASTRUCTURE ONLY.  Nothing in the product path (the CUDA library under
``paper_conf_asplos_hagedornfccgg23_b200/csrc`` and its Python binding) may
import, call, link or execute anything in this package.  The only permitted
callers are ``tests/``, ``__graft_entry__.smoke()`` and the ``cpu_baseline`` /
``--impl reference`` legs of ``bench.py``.

The oracle shares no code with the CUDA path: no kernels, headers, helpers,
constants or pre/post-processing.  Inputs come from ``workloads`` (seeded
generators that hold none of the method's arithmetic).

Citation key: ``P:Lnnn`` = line nnn of the paper text (Hagedorn et al.,
"Graphene: An IR for Optimized Tensor Computations on GPUs", ASPLOS '23),
section/figure named beside it.  ``DESIGN.md R<n>`` = a reading of the paper
recorded in DESIGN.md §3 where the paper is silent.

Modules
-------
fmha   numpy fp64, unfused GEMM -> softmax -> GEMM per (batch, head);
       the same per (sequence, head) of a packed variable-length batch   [pinned]
brute  pure-Python scalar loops with math.fsum, tiny shapes only        [pinned]
gemm   numpy fp64 act(A @ W^T + b); act(A1 W1^T + A2 W2^T + b) (LSTM cell) [pinned]
layer  QKV GEMM -> varlen FMHA -> out GEMM -> MLP, fp16 storage between  [pinned]
mlp    L chained (GEMM + bias + act) layers, N = K, fp16 between layers  [pinned]

Every function is pinned by ``tests/test_oracle.py`` against closed forms,
invariants, a hand-derived golden fixture (``tests/golden/``), brute force and
torch's fp64 CPU ``scaled_dot_product_attention``.  There is no "parity
unpinned" function in this package.
"""

from .fmha import attention_fp64, attention_rows_fp64, attention_varlen_fp64, softmax_probs_fp64, fmha_flops
from .brute import attention_brute
from .gemm import dual_gemm_bias_act_fp64, gemm_bias_act_fp64, gelu_erf, gelu_tanh, relu
from .layer import round_fp16, transformer_layer_fp64
from .mlp import mlp_fused_flops, mlp_fused_fp64, mlp_fused_rows_fp64

__all__ = [
    "attention_fp64",
    "attention_rows_fp64",
    "attention_varlen_fp64",
    "softmax_probs_fp64",
    "fmha_flops",
    "attention_brute",
    "gemm_bias_act_fp64",
    "dual_gemm_bias_act_fp64",
    "gelu_erf",
    "gelu_tanh",
    "relu",
    "round_fp16",
    "transformer_layer_fp64",
    "mlp_fused_fp64",
    "mlp_fused_rows_fp64",
    "mlp_fused_flops",
]
