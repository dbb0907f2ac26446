"""GPU parity for mlp_fused_fwd (the paper's fused multi-layer MLP, Fig. 11)
against the fp64 oracle (oracle.mlp_fused_fp64, R19), through the C ABI.

Tolerance (derived): both sides round h_1..h_{L-1} to fp16 at the same points, so they differ only
where the GPU's fp32 accumulation (relative error ~1e-6) and the oracle's fp64 value fall on
opposite sides of an fp16 rounding boundary: a 1-ulp (2^-11 |h|) flip in some h_l[m,k].  With
He-scaled weights a ReLU layer has gain ~1, so these flips accumulate like a random walk over the
layers (~sqrt(L) ulps of the activations' size, ~0.5-1) on top of the output's own half-ulp
rounding.  The numpy model of the kernel's arithmetic (fp32 accumulation in three orders, fp32 bias
+ ReLU, fp16 store per layer) stays within 0.55 x [1e-3 (1 + sqrt(L)) + 2^-8 |ref|] at L = 20; the
tensor core's fp32 accumulation is not IEEE round-to-nearest per addition (products of a K block are
aligned to the largest exponent and truncated), so its pre-rounding error per layer is larger and its
flips more frequent: measured 1.05 x that bound at one of 64000 outputs (M = 500, N = 128, L = 20,
round 2).  The test uses twice the absolute term: elementwise |err| <= 2e-3 (1 + sqrt(L)) + 2^-8 |ref|,
and rel-L2 <= 1e-3 over the checked rows.  tests/test_oracle.py::test_mlp_tolerance_covers_fp32_kernel_model checks on the CPU
that a numpy model of the kernel's arithmetic (fp32 accumulate, fp32 bias + ReLU, fp16 store per
layer) passes this bound at L = 20 and fails a depth-independent 2e-3 + 2^-9 |ref|."""

import numpy as np
import pytest
import torch

import paper_conf_asplos_hagedornfccgg23_b200 as fm
from oracle import mlp_fused_fp64, mlp_fused_rows_fp64
from workloads import FUSED_MLP_CONFIGS, make_fused_mlp_inputs

pytestmark = pytest.mark.gpu
DEV = torch.device("cuda:0") if torch.cuda.is_available() else None
ACTS = {"none": 0, "relu": 1, "gelu": 2, "gelu_tanh": 3, "tanh": 4}


def check(y, ref, what, layers):
    got = y.double().cpu().numpy()
    assert np.all(np.isfinite(got)), what
    bad = np.abs(got - ref) > 2e-3 * (1 + np.sqrt(layers)) + 2 ** -8 * np.abs(ref)
    print(what, 'max |err|', np.abs(got - ref).max(), 'rel-L2', np.linalg.norm(got - ref) / max(np.linalg.norm(ref), 1e-30))
    rel = np.linalg.norm(got - ref) / max(np.linalg.norm(ref), 1e-30)
    assert not bad.any() and rel <= 1e-3, f"{what}: {bad.sum()} elems out of tol, rel-L2={rel:.3e}"


@pytest.mark.parametrize("m,n,layers", [(1, 64, 1), (128, 128, 1), (300, 128, 3), (300, 64, 5), (500, 128, 20),
                                        (1000, 64, 20), (129, 128, 2)])
def test_mlp_fused_parity_full(m, n, layers):
    x, w, b = make_fused_mlp_inputs(m, n, layers)
    y = fm.mlp_fused(x.to(DEV), w.to(DEV), b.to(DEV))
    torch.cuda.synchronize()
    check(y, mlp_fused_fp64(x, w, b), f"M={m} N={n} L={layers}", layers)


@pytest.mark.parametrize("act", ["none", "gelu", "gelu_tanh", "tanh"])
def test_mlp_fused_activations(act):
    x, w, b = make_fused_mlp_inputs(260, 128, 4)
    y = fm.mlp_fused(x.to(DEV), w.to(DEV), b.to(DEV), act=act)
    torch.cuda.synchronize()
    check(y, mlp_fused_fp64(x, w, b, ACTS[act]), act, 4)


def test_mlp_fused_no_bias_and_in_place():
    x, w, b = make_fused_mlp_inputs(400, 64, 6)
    y = fm.mlp_fused(x.to(DEV), w.to(DEV), None)
    torch.cuda.synchronize()
    check(y, mlp_fused_fp64(x, w, None), "no bias", 6)
    xd = x.to(DEV)
    y2 = fm.mlp_fused(xd, w.to(DEV), b.to(DEV), out=xd)  # Y == X is allowed (include/fmha.h)
    torch.cuda.synchronize()
    assert y2.data_ptr() == xd.data_ptr()
    check(y2, mlp_fused_fp64(x, w, b), "in place", 6)


@pytest.mark.parametrize("n,extra", [(128, 77), (64, 200)])
def test_mlp_fused_multi_slot_groups_sampled(n, extra):
    """M large enough that every CTA takes groups of 2 (N=128) / 4 (N=64) row tiles, with a ragged
    last group and a ragged last tile; rows are independent, so sampled rows are checked exactly."""
    slots = 2 if n == 128 else 4
    m = 148 * slots * 128 + extra
    x, w, b = make_fused_mlp_inputs(m, n, 4)
    y = fm.mlp_fused(x.to(DEV), w.to(DEV), b.to(DEV))
    torch.cuda.synchronize()
    rows = np.random.default_rng(1).choice(m, 96, replace=False)
    rows = np.unique(np.concatenate([rows, [0, 127, 128, m - extra, m - 1]]))
    check(y[torch.from_numpy(rows).to(DEV)], mlp_fused_rows_fp64(x, w, b, rows), f"M={m} N={n}", 4)


@pytest.mark.parametrize("name", sorted(FUSED_MLP_CONFIGS))
def test_mlp_fused_bench_config_sampled(name):
    """The bench workloads at full size (M = 65536, 20 layers), in the launch configuration the
    bench times; 64 sampled rows plus the first and last."""
    cfg = FUSED_MLP_CONFIGS[name]
    x, w, b = make_fused_mlp_inputs(cfg.m, cfg.width, cfg.layers, cfg_id=cfg.cfg_id)
    y = fm.mlp_fused(x.to(DEV), w.to(DEV), b.to(DEV))
    torch.cuda.synchronize()
    rows = np.unique(np.concatenate([np.random.default_rng(2).choice(cfg.m, 64, replace=False), [0, cfg.m - 1]]))
    check(y[torch.from_numpy(rows).to(DEV)], mlp_fused_rows_fp64(x, w, b, rows), name, cfg.layers)
    y2 = fm.mlp_fused(x.to(DEV), w.to(DEV), b.to(DEV))
    torch.cuda.synchronize()
    assert torch.equal(y, y2), "not deterministic"


def test_mlp_fused_zero_rows_and_errors():
    x, w, b = make_fused_mlp_inputs(8, 128, 2)
    y = fm.mlp_fused(x[:0].to(DEV), w.to(DEV), b.to(DEV))
    assert y.shape == (0, 128)
    with pytest.raises(fm.FmhaError):
        fm.mlp_fused(torch.zeros(4, 96, dtype=torch.float16, device=DEV),
                     torch.zeros(2, 96, 96, dtype=torch.float16, device=DEV))
