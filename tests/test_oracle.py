"""Pins for the CPU oracle (runs without a GPU).

The oracle is pinned to things other than itself (SURVEY.md §8(c) pins P1-P13):
closed forms, invariants, a hand-derived golden fixture, pure-Python brute force,
and torch's float64 CPU scaled_dot_product_attention.  Each pin is chosen so a
plausible slip in oracle/fmha.py (dropped scale, wrong sign in the max shift,
transposed K, off-by-one causal diagonal, mask on the wrong axis) fails.
"""

import json
import math
import os

import numpy as np
import pytest
import torch

from oracle import (attention_brute, attention_fp64, attention_rows_fp64, attention_varlen_fp64, fmha_flops,
                    gemm_bias_act_fp64, gelu_erf, gelu_tanh, softmax_probs_fp64)
from oracle.gemm import ACT_GELU_ERF, ACT_GELU_TANH, ACT_NONE, ACT_RELU
from workloads import CONFIGS, make_fmha_inputs

GOLDEN = os.path.join(os.path.dirname(__file__), "golden", "fmha_hand.json")


def rnd(shape, seed, sigma=1.0):
    return np.random.default_rng(seed).standard_normal(shape) * sigma


# ---------------------------------------------------------------- golden (hand-derived)
@pytest.mark.parametrize("case", json.load(open(GOLDEN))["cases"], ids=lambda c: c["name"])
def test_golden_hand_cases(case):
    o = attention_fp64(np.array(case["q"]), np.array(case["k"]), np.array(case["v"]),
                       case["scale"], case["kv_len"], case["causal"])
    np.testing.assert_allclose(o, np.array(case["expected"]), atol=1e-12, rtol=0)
    ob = attention_brute(case["q"], case["k"], case["v"], case["scale"], case["kv_len"], case["causal"])
    np.testing.assert_allclose(np.array(ob), np.array(case["expected"]), atol=1e-12, rtol=0)


# ---------------------------------------------------------------- P11 closed form S=2, D=1
@pytest.mark.parametrize("a,b,v0,v1", [(0.3, -1.2, 2.0, -5.0), (10.0, 9.0, 1.0, 0.0), (-3, 4, 0.5, 0.25)])
def test_p11_two_keys_closed_form(a, b, v0, v1):
    q = np.array([[[[1.0]]]])
    k = np.array([[[[a], [b]]]])
    v = np.array([[[[v0], [v1]]]])
    want = (v0 * math.exp(a) + v1 * math.exp(b)) / (math.exp(a) + math.exp(b))
    assert attention_fp64(q, k, v, 1.0)[0, 0, 0, 0] == pytest.approx(want, abs=1e-14)


# ---------------------------------------------------------------- P11 brute force vs numpy
@pytest.mark.parametrize("seed", range(6))
def test_p11_brute_force_small(seed):
    r = np.random.default_rng(100 + seed)
    b, h = 2, 2
    sq, skv, d = int(r.integers(1, 9)), int(r.integers(1, 9)), int(r.integers(1, 9))
    causal = bool(seed % 2)
    kv_len = None if seed % 3 else [int(r.integers(0, skv + 1)) for _ in range(b)]
    q, k, v = rnd((b, h, sq, d), seed), rnd((b, h, skv, d), seed + 50), rnd((b, h, skv, d), seed + 99)
    scale = 1 / math.sqrt(d)
    o = attention_fp64(q, k, v, scale, kv_len, causal)
    ob = np.array(attention_brute(q.tolist(), k.tolist(), v.tolist(), scale, kv_len, causal))
    np.testing.assert_allclose(o, ob, atol=1e-12, rtol=1e-12)


# ---------------------------------------------------------------- P12 library special case
@pytest.mark.parametrize("causal,pad", [(False, False), (True, False), (False, True), (True, True)])
def test_p12_torch_sdpa_fp64(causal, pad):
    b, h, sq, skv, d = 3, 2, 37, 53, 16
    q, k, v = rnd((b, h, sq, d), 1), rnd((b, h, skv, d), 2), rnd((b, h, skv, d), 3)
    kv_len = [53, 20, 41] if pad else None
    scale = 0.3
    o = attention_fp64(q, k, v, scale, kv_len, causal)
    i = np.arange(sq)[:, None]
    j = np.arange(skv)[None, :]
    vis = np.ones((b, 1, sq, skv), dtype=bool)
    if causal:
        vis &= (j <= i + (skv - sq))[None, None]
    if pad:
        for bb in range(b):
            vis[bb, :, :, kv_len[bb]:] = False
    ref = torch.nn.functional.scaled_dot_product_attention(
        torch.from_numpy(q), torch.from_numpy(k), torch.from_numpy(v),
        attn_mask=torch.from_numpy(vis), scale=float(np.float32(scale))).numpy()
    rows = np.broadcast_to(vis.any(-1), (b, h, sq))  # SDPA gives NaN on fully masked rows
    np.testing.assert_allclose(o[rows], ref[rows], atol=1e-12, rtol=1e-10)
    assert np.all(o[~rows] == 0.0)


# ---------------------------------------------------------------- P1 single key
def test_p1_single_key_returns_v0():
    q, k, v = rnd((2, 3, 5, 8), 4, 5.0), rnd((2, 3, 1, 8), 5, 5.0), rnd((2, 3, 1, 8), 6)
    o = attention_fp64(q, k, v, 0.7)
    np.testing.assert_array_equal(o, np.broadcast_to(v, o.shape))
    # kv_len = 1 reduces to the same thing
    k2, v2 = rnd((2, 3, 9, 8), 7), rnd((2, 3, 9, 8), 8)
    o2 = attention_fp64(q, k2, v2, 0.7, kv_len=[1, 1])
    np.testing.assert_allclose(o2, np.broadcast_to(v2[:, :, :1], o2.shape), atol=0, rtol=0)


# ---------------------------------------------------------------- P2 constant Q,K with huge scores
@pytest.mark.parametrize("mag", [1.0, 100.0, 1e4])
def test_p2_constant_qk_gives_mean_of_visible_v(mag):
    sq, skv, d = 6, 11, 4
    q = np.full((1, 1, sq, d), mag)
    k = np.full((1, 1, skv, d), mag)
    v = rnd((1, 1, skv, d), 9)
    o = attention_fp64(q, k, v, 1.0)          # scores = 4*mag^2, up to 4e8: needs max-shift
    assert np.all(np.isfinite(o))
    np.testing.assert_allclose(o[0, 0], np.broadcast_to(v[0, 0].mean(0), (sq, d)), atol=1e-12)
    o = attention_fp64(q, k, v, 1.0, kv_len=[5])
    np.testing.assert_allclose(o[0, 0], np.broadcast_to(v[0, 0, :5].mean(0), (sq, d)), atol=1e-12)
    o = attention_fp64(q, k[:, :, :sq], v[:, :, :sq], 1.0, causal=True)
    for i in range(sq):
        np.testing.assert_allclose(o[0, 0, i], v[0, 0, :i + 1].mean(0), atol=1e-12)


# ---------------------------------------------------------------- P3 uniform V
def test_p3_uniform_v_identity():
    q, k = rnd((2, 2, 7, 5), 10, 3.0), rnd((2, 2, 13, 5), 11, 3.0)
    vrow = rnd((5,), 12)
    v = np.broadcast_to(vrow, (2, 2, 13, 5)).copy()
    for kw in ({}, {"causal": True}, {"kv_len": [3, 13]}):
        o = attention_fp64(q, k, v, 0.4, **kw)
        np.testing.assert_allclose(o, np.broadcast_to(vrow, o.shape), atol=1e-13)


# ---------------------------------------------------------------- P4 scale = 0
def test_p4_scale_zero_gives_mean():
    q, k, v = rnd((1, 2, 4, 6), 13, 9.0), rnd((1, 2, 10, 6), 14, 9.0), rnd((1, 2, 10, 6), 15)
    o = attention_fp64(q, k, v, 0.0)
    np.testing.assert_allclose(o, np.broadcast_to(v.mean(2, keepdims=True), o.shape), atol=1e-13)


# ---------------------------------------------------------------- P5 / P6 permutations
def test_p5_joint_kv_permutation_invariance():
    q, k, v = rnd((2, 2, 9, 8), 16), rnd((2, 2, 17, 8), 17), rnd((2, 2, 17, 8), 18)
    perm = np.random.default_rng(0).permutation(17)
    o = attention_fp64(q, k, v, 0.35)
    op = attention_fp64(q, k[:, :, perm], v[:, :, perm], 0.35)
    np.testing.assert_allclose(o, op, atol=1e-13)
    # within the valid prefix under key padding
    perm2 = np.concatenate([np.random.default_rng(1).permutation(10), np.arange(10, 17)])
    o = attention_fp64(q, k, v, 0.35, kv_len=[10, 10])
    op = attention_fp64(q, k[:, :, perm2], v[:, :, perm2], 0.35, kv_len=[10, 10])
    np.testing.assert_allclose(o, op, atol=1e-13)
    # a K-only permutation must change the result (catches a kernel/oracle ignoring K order)
    assert not np.allclose(attention_fp64(q, k[:, :, perm], v, 0.35), o)


def test_p6_query_permutation_equivariance():
    q, k, v = rnd((1, 3, 12, 8), 19), rnd((1, 3, 12, 8), 20), rnd((1, 3, 12, 8), 21)
    perm = np.random.default_rng(2).permutation(12)
    o = attention_fp64(q, k, v, 0.5)
    np.testing.assert_allclose(attention_fp64(q[:, :, perm], k, v, 0.5), o[:, :, perm], atol=1e-13)


# ---------------------------------------------------------------- P7 masked rows are inert
def test_p7_garbage_in_masked_kv_rows():
    q, k, v = rnd((2, 2, 8, 8), 22), rnd((2, 2, 16, 8), 23), rnd((2, 2, 16, 8), 24)
    kv_len = [5, 16]
    o = attention_fp64(q, k, v, 0.35, kv_len=kv_len)
    k2, v2 = k.copy(), v.copy()
    k2[0, :, 5:] = 6e4
    v2[0, :, 5:] = -6e4
    np.testing.assert_array_equal(attention_fp64(q, k2, v2, 0.35, kv_len=kv_len), o)
    # causal: keys after the diagonal are inert
    qc, kc, vc = q[:, :, :8], k[:, :, :8].copy(), v[:, :, :8].copy()
    oc = attention_fp64(qc, kc, vc, 0.35, causal=True)
    kc[:, :, 7] = 6e4
    vc[:, :, 7] = 6e4
    np.testing.assert_array_equal(attention_fp64(qc, kc, vc, 0.35, causal=True)[:, :, :7], oc[:, :, :7])


# ---------------------------------------------------------------- P8 convex hull, P9 rows sum to 1
def test_p8_p9_convexity():
    q, k, v = rnd((1, 1, 20, 8), 25, 3.0), rnd((1, 1, 30, 8), 26, 3.0), rnd((1, 1, 30, 8), 27)
    for kw in ({}, {"causal": True}, {"kv_len": [17]}):
        p = softmax_probs_fp64(q[0, 0], k[0, 0], 0.2, kw.get("kv_len", [None])[0], kw.get("causal", False))
        assert np.all(p >= 0)
        np.testing.assert_allclose(p.sum(1), 1.0, atol=1e-12)
        o = attention_fp64(q, k, v, 0.2, **kw)[0, 0]
        assert np.all(o <= v[0, 0].max(0) + 1e-12) and np.all(o >= v[0, 0].min(0) - 1e-12)


# ---------------------------------------------------------------- P10 row score shift
def test_p10_row_shift_invariance():
    q, k, v = rnd((1, 2, 6, 8), 28), rnd((1, 2, 9, 8), 29), rnd((1, 2, 9, 8), 30)
    outs = []
    for c in (0.0, 37.0):
        q2, k2 = q.copy(), k.copy()
        q2[..., 7] = c
        k2[..., 7] = 1.0
        outs.append(attention_fp64(q2, k2, v, 0.5))
    np.testing.assert_allclose(outs[0], outs[1], atol=1e-12)


# ---------------------------------------------------------------- sampled rows == full oracle
def test_rows_sampler_matches_full():
    cfg = CONFIGS["bert_base_pad"].with_(batch=3, heads=2, seq_q=40, seq_kv=40)
    q, k, v, kl = make_fmha_inputs(cfg)
    full = attention_fp64(q, k, v, cfg.scale, kl)
    units = [(0, 1, 3), (2, 0, 39), (1, 1, 0)]
    rows = attention_rows_fp64(q, k, v, cfg.scale, units, kl)
    for n, (b, h, i) in enumerate(units):
        np.testing.assert_allclose(rows[n], full[b, h, i], atol=1e-14)
    fullc = attention_fp64(q, k, v, cfg.scale, causal=True)
    rowsc = attention_rows_fp64(q, k, v, cfg.scale, units, causal=True)
    for n, (b, h, i) in enumerate(units):
        np.testing.assert_allclose(rowsc[n], fullc[b, h, i], atol=1e-14)


def test_flop_count():
    assert fmha_flops(1, 1, 4, 4, 8) == 4 * 8 * 16
    assert fmha_flops(1, 1, 4, 4, 8, causal=True) == 4 * 8 * 10            # 1+2+3+4
    assert fmha_flops(2, 3, 4, 6, 8, kv_len=[2, 6]) == 4 * 8 * 3 * (4 * 2 + 4 * 6)
    assert fmha_flops(1, 1, 3, 2, 1, causal=True) == 4 * (0 + 1 + 2)        # bottom-right


# ---------------------------------------------------------------- P13 gemm pins
def test_p13_gemm_pins():
    r = np.random.default_rng(31)
    a = r.uniform(-1, 1, (7, 5))
    b = r.uniform(-1, 1, 5)
    eye = np.eye(5)
    np.testing.assert_allclose(gemm_bias_act_fp64(a, eye, b, ACT_NONE), a + b, atol=1e-15)
    np.testing.assert_allclose(gemm_bias_act_fp64(a, eye, b, ACT_RELU), np.maximum(a + b, 0), atol=1e-15)
    np.testing.assert_allclose(gemm_bias_act_fp64(np.zeros((3, 5)), r.normal(size=(5, 5)), b, ACT_GELU_ERF),
                               np.broadcast_to(gelu_erf(b), (3, 5)), atol=1e-15)
    x = np.linspace(-6, 6, 101)
    np.testing.assert_allclose(gelu_erf(x) - gelu_erf(-x), x, atol=1e-14)
    np.testing.assert_allclose(gelu_tanh(x) - gelu_tanh(-x), x, atol=1e-14)
    # GELU known values: gelu(1) = Phi(1) = 0.8413447460685429; tanh form within 1e-3 of erf form
    assert gelu_erf(np.array([1.0]))[0] == pytest.approx(0.8413447460685429, abs=1e-15)
    assert np.max(np.abs(gelu_tanh(x) - gelu_erf(x))) < 1e-3
    w = r.normal(size=(6, 5))
    bias6 = r.normal(size=6)
    ref = torch.nn.functional.linear(torch.from_numpy(a), torch.from_numpy(w), torch.from_numpy(bias6)).numpy()
    np.testing.assert_allclose(gemm_bias_act_fp64(a, w, bias6, ACT_NONE), ref, atol=1e-13)
    np.testing.assert_allclose(gemm_bias_act_fp64(a, w, None, ACT_GELU_TANH),
                               torch.nn.functional.gelu(torch.from_numpy(a @ w.T), approximate="tanh").numpy(),
                               atol=1e-14)
    np.testing.assert_allclose(gemm_bias_act_fp64(a, w, None, ACT_GELU_ERF),
                               torch.nn.functional.gelu(torch.from_numpy(a @ w.T)).numpy(), atol=1e-14)


# ---------------------------------------------------------------- workload generator sanity
def test_workloads_shard_reproducible():
    cfg = CONFIGS["bert_base_pad"].with_(batch=4, heads=2, seq_q=16, seq_kv=16)
    q, k, v, kl = make_fmha_inputs(cfg)
    q2, k2, v2, kl2 = make_fmha_inputs(cfg.with_(batch=2), batch_offset=2)
    assert torch.equal(q[2:], q2) and torch.equal(v[2:], v2)
    assert list(kl[2:]) == list(kl2)
    assert kl[0] == 16 and all(16 >= x >= 16 for x in kl[:1])
    assert q.dtype == torch.float16


# ---------------------------------------------------------------- varlen packed layout (f2)
def _brute_varlen(x, cu, scale, causal):
    """Pin for attention_varlen_fp64 via the pure-Python brute force, one sequence at a time."""
    t, _, h_, d = x.shape
    out = np.zeros((t, h_, d))
    for s in range(len(cu) - 1):
        a, b = int(cu[s]), int(cu[s + 1])
        if b <= a:
            continue
        q = [[[list(map(float, x[i, 0, h])) for i in range(a, b)] for h in range(h_)]]
        k = [[[list(map(float, x[i, 1, h])) for i in range(a, b)] for h in range(h_)]]
        v = [[[list(map(float, x[i, 2, h])) for i in range(a, b)] for h in range(h_)]]
        o = attention_brute(q, k, v, scale, None, causal)[0]
        for h in range(h_):
            out[a:b, h] = np.array(o[h])
    return out


@pytest.mark.parametrize("causal", [False, True])
def test_varlen_brute_force(causal):
    lens = [3, 0, 5, 1, 4]
    cu = np.concatenate([[0], np.cumsum(lens)]).astype(np.int32)
    x = rnd((int(cu[-1]), 3, 2, 4), 7)
    o = attention_varlen_fp64(x, cu, 0.5, causal)
    np.testing.assert_allclose(o, _brute_varlen(x, cu, 0.5, causal), atol=1e-13, rtol=0)


def test_varlen_equal_lengths_is_dense_layout():
    """Equal lengths: the packed problem is the dense [B,H,S,D] one with Q/K/V transposed."""
    b, s, h, d = 3, 7, 2, 8
    x = rnd((b * s, 3, h, d), 11)
    cu = np.arange(0, b * s + 1, s, dtype=np.int32)
    o = attention_varlen_fp64(x, cu, 1 / math.sqrt(d))
    xs = x.reshape(b, s, 3, h, d).transpose(2, 0, 3, 1, 4)  # [3, B, H, S, D]
    od = attention_fp64(xs[0], xs[1], xs[2], 1 / math.sqrt(d))  # [B, H, S, D]
    np.testing.assert_allclose(o, od.transpose(0, 2, 1, 3).reshape(b * s, h, d), atol=1e-14, rtol=0)


def test_varlen_sequences_do_not_interact():
    """Garbage in one sequence's tokens leaves every other sequence's output unchanged, and the
    first token of a causal sequence returns its own V (closed form)."""
    lens = [6, 9, 4]
    cu = np.concatenate([[0], np.cumsum(lens)]).astype(np.int32)
    x = rnd((int(cu[-1]), 3, 2, 8), 5)
    o = attention_varlen_fp64(x, cu, 0.3)
    y = x.copy()
    y[cu[1]:cu[2]] = rnd((lens[1], 3, 2, 8), 6, sigma=50.0)
    o2 = attention_varlen_fp64(y, cu, 0.3)
    keep = np.r_[cu[0]:cu[1], cu[2]:cu[3]]
    np.testing.assert_array_equal(o[keep], o2[keep])
    assert not np.allclose(o[cu[1]:cu[2]], o2[cu[1]:cu[2]])
    oc = attention_varlen_fp64(x, cu, 0.3, causal=True)
    for s in range(3):
        np.testing.assert_array_equal(oc[cu[s]], x[cu[s], 2])


# ---------------------------------------------------------------- synthetic Transformer layer (f1)
def test_layer_matches_torch_fp64_composition():
    """Library special case: the same five stages written with torch's float64 CPU linear, SDPA and
    erf-GELU, rounding every stored intermediate to fp16 (R18)."""
    from oracle import transformer_layer_fp64
    from workloads import LayerConfig, make_layer_inputs
    import torch.nn.functional as F
    cfg = LayerConfig("tiny_layer", 31, 3, 0, 16, 2, 32)
    (x, wqkv, bqkv, wo, bo, w1, b1, w2, b2), cu = make_layer_inputs(cfg, lengths=[5, 9, 3])
    y = transformer_layer_fp64(x, wqkv, bqkv, wo, bo, w1, b1, w2, b2, cu, cfg.heads, cfg.scale)
    d64 = lambda t: t.double()
    r16 = lambda t: t.half().double()
    qkv = r16(F.linear(d64(x), d64(wqkv), d64(bqkv))).view(-1, 3, 2, 8)
    a = torch.zeros(qkv.shape[0], 2, 8, dtype=torch.float64)
    for s in range(3):
        lo, hi = int(cu[s]), int(cu[s + 1])
        q, k, v = (qkv[lo:hi, i].transpose(0, 1) for i in range(3))
        a[lo:hi] = F.scaled_dot_product_attention(q, k, v, scale=float(np.float32(cfg.scale))).transpose(0, 1)
    z = r16(F.linear(r16(a.reshape(-1, 16)), d64(wo), d64(bo)))
    h = r16(F.gelu(F.linear(z, d64(w1), d64(b1))))
    yt = F.linear(h, d64(w2), d64(b2))
    # fp16 rounding can flip on ~1e-16 differences between the two fp64 evaluations: allow one fp16
    # ulp of an intermediate, propagated (tiny next to the GPU tolerance)
    np.testing.assert_allclose(y, yt.numpy(), atol=2e-3, rtol=0)
    assert np.abs(y - yt.numpy()).mean() < 1e-6


# ---------------------------------------------------------------- simplified LSTM cell (f4)
def test_dual_gemm_pins():
    """act(A1 W1^T + A2 W2^T + b): equals one GEMM over the K-concatenated operands (a block-matrix
    identity), torch fp64 linear + linear, and ReLU / tanh closed forms on hand values."""
    from oracle import dual_gemm_bias_act_fp64
    from oracle.gemm import ACT_NONE, ACT_RELU, ACT_TANH
    r = np.random.default_rng(5)
    a1, w1 = r.standard_normal((7, 5)), r.standard_normal((4, 5))
    a2, w2 = r.standard_normal((7, 3)), r.standard_normal((4, 3))
    b = r.standard_normal(4)
    cat = gemm_bias_act_fp64(np.hstack([a1, a2]), np.hstack([w1, w2]), b, ACT_NONE)
    np.testing.assert_allclose(dual_gemm_bias_act_fp64(a1, w1, a2, w2, b, ACT_NONE), cat, atol=1e-13, rtol=0)
    lin = (torch.nn.functional.linear(torch.from_numpy(a1), torch.from_numpy(w1))
           + torch.nn.functional.linear(torch.from_numpy(a2), torch.from_numpy(w2), torch.from_numpy(b)))
    np.testing.assert_allclose(dual_gemm_bias_act_fp64(a1, w1, a2, w2, b, ACT_RELU), lin.clamp_min(0).numpy(),
                               atol=1e-13, rtol=0)
    np.testing.assert_allclose(dual_gemm_bias_act_fp64(a1, w1, a2, w2, b, ACT_TANH), torch.tanh(lin).numpy(),
                               atol=1e-13, rtol=0)
    # by hand: 1x1 operands
    one = np.ones((1, 1))
    assert dual_gemm_bias_act_fp64(2 * one, 3 * one, -4 * one, 2 * one, np.array([1.0]), ACT_RELU)[0, 0] == 0.0
    assert dual_gemm_bias_act_fp64(2 * one, 3 * one, 1 * one, 2 * one, np.array([-1.0]), ACT_RELU)[0, 0] == 7.0
    assert dual_gemm_bias_act_fp64(one, one, one, -one, None, ACT_TANH)[0, 0] == 0.0


# ---------------------------------------------------------------------------------------------
# Fused multi-layer MLP (Fig. 11): pins for oracle.mlp_fused_fp64


def _fp16_round_scalar(x: float) -> float:
    import struct
    return struct.unpack("<e", struct.pack("<e", x))[0]  # IEEE half, round-to-nearest-even


def _mlp_brute(x, w, b, act_relu=True):
    """Pure-Python scalar loops (math.fsum), fp16 rounding between layers: an implementation that
    shares nothing with numpy's GEMM."""
    h = [list(map(float, r)) for r in x]
    L = len(w)
    for l in range(L):
        out = []
        for r in h:
            row = []
            for n in range(len(w[l])):
                z = math.fsum([r[k] * float(w[l][n][k]) for k in range(len(r))] + [float(b[l][n])])
                z = max(z, 0.0) if act_relu else z
                row.append(z if l + 1 == L else _fp16_round_scalar(z))
            out.append(row)
        h = out
    return np.array(h)


@pytest.mark.parametrize("seed", [0, 1, 2])
def test_mlp_brute_force_tiny(seed):
    from oracle import mlp_fused_fp64
    rng = np.random.default_rng(seed)
    m, n, L = 3, 5, 4
    x = rng.uniform(-1, 1, (m, n)).astype(np.float16)
    w = (rng.standard_normal((L, n, n)) * 0.6).astype(np.float16)
    b = rng.uniform(-0.3, 0.3, (L, n)).astype(np.float16)
    got = mlp_fused_fp64(x, w, b, ACT_RELU)
    want = _mlp_brute(x.tolist(), w.tolist(), b.tolist())
    np.testing.assert_allclose(got, want, rtol=0, atol=1e-12)
    got_lin = mlp_fused_fp64(x, w, b, ACT_NONE)
    np.testing.assert_allclose(got_lin, _mlp_brute(x.tolist(), w.tolist(), b.tolist(), act_relu=False),
                               rtol=0, atol=1e-12)


@pytest.mark.parametrize("seed", [3, 4])
def test_mlp_rows_sampler_brute_force(seed):
    """mlp_fused_rows_fp64 (the row-sampled checker of the GPU tests) against the pure-Python loops
    on the selected rows only: rows in any order, duplicated, first and last."""
    from oracle import mlp_fused_rows_fp64
    rng = np.random.default_rng(seed)
    m, n, L = 7, 6, 3
    x = rng.uniform(-1, 1, (m, n)).astype(np.float16)
    w = (rng.standard_normal((L, n, n)) * 0.6).astype(np.float16)
    b = rng.uniform(-0.3, 0.3, (L, n)).astype(np.float16)
    rows = [6, 0, 3, 3, 5]
    got = mlp_fused_rows_fp64(x, w, b, rows, ACT_RELU)
    want = _mlp_brute([x[r].tolist() for r in rows], w.tolist(), b.tolist())
    assert got.shape == (len(rows), n)
    np.testing.assert_allclose(got, want, rtol=0, atol=1e-12)


def test_mlp_identity_weights_closed_form():
    """W_l = I, b_l = c >= 0, X >= 0 (ReLU): every layer adds c exactly, so Y = X + L c."""
    from oracle import mlp_fused_fp64
    n, L = 16, 20
    x = (np.arange(4 * n).reshape(4, n) % 7).astype(np.float16)
    w = np.stack([np.eye(n)] * L).astype(np.float16)
    c = np.float16(0.5)
    b = np.full((L, n), c, dtype=np.float16)
    np.testing.assert_array_equal(mlp_fused_fp64(x, w, b), x.astype(np.float64) + L * 0.5)


def test_mlp_zero_weights_leave_last_bias():
    from oracle import mlp_fused_fp64
    rng = np.random.default_rng(5)
    n, L = 8, 3
    x = rng.uniform(-1, 1, (6, n)).astype(np.float16)
    b = rng.uniform(-1, 1, (L, n)).astype(np.float16)
    y = mlp_fused_fp64(x, np.zeros((L, n, n), np.float16), b)
    np.testing.assert_array_equal(y, np.broadcast_to(np.maximum(b[-1].astype(np.float64), 0), y.shape))


def test_mlp_hidden_permutation_invariance():
    """Relabelling the hidden units between two layers (W_l -> P W_l, b_l -> P b_l,
    W_{l+1} -> W_{l+1} P^T) leaves Y unchanged bit for bit: ReLU and the fp16 rounding are
    elementwise.  A transposed operand or a mixed-up row/column index breaks it."""
    from oracle import mlp_fused_fp64
    rng = np.random.default_rng(11)
    n, L = 12, 3
    x = rng.uniform(-1, 1, (7, n)).astype(np.float16)
    w = (rng.standard_normal((L, n, n)) / np.sqrt(n) * np.sqrt(2)).astype(np.float16)
    b = rng.uniform(-0.2, 0.2, (L, n)).astype(np.float16)
    perm = rng.permutation(n)
    w2, b2 = w.copy(), b.copy()
    w2[0] = w[0][perm]
    b2[0] = b[0][perm]
    w2[1] = w[1][:, perm]
    np.testing.assert_array_equal(mlp_fused_fp64(x, w, b), mlp_fused_fp64(x, w2, b2))
    w3 = w.copy()
    w3[0] = w[0].T.copy()  # the transposed-operand mistake is visible
    assert not np.array_equal(mlp_fused_fp64(x, w, b), mlp_fused_fp64(x, w3, b))


def test_mlp_matches_torch_fp64_sequential():
    """Library special case: torch.nn.functional.linear + relu in float64, rounded to fp16 between
    layers by numpy's direct float64 -> float16 cast (torch's double -> half goes through float32,
    a double rounding that flips rare near-tie elements)."""
    from oracle import mlp_fused_fp64
    rng = np.random.default_rng(3)
    m, n, L = 33, 64, 6
    x = rng.uniform(-1, 1, (m, n)).astype(np.float16)
    w = (rng.standard_normal((L, n, n)) * np.sqrt(2.0 / n)).astype(np.float16)
    b = rng.uniform(-0.1, 0.1, (L, n)).astype(np.float16)
    h = torch.from_numpy(x).double()
    for l in range(L):
        h = torch.relu(torch.nn.functional.linear(h, torch.from_numpy(w[l]).double(), torch.from_numpy(b[l]).double()))
        if l + 1 < L:
            h = torch.from_numpy(h.numpy().astype(np.float16).astype(np.float64))
    np.testing.assert_allclose(mlp_fused_fp64(x, w, b), h.numpy(), rtol=0, atol=1e-12)


def test_mlp_positive_homogeneity():
    """b = 0 and ReLU: Y(2 X) = 2 Y(X) exactly (scaling by 2 commutes with fp16 rounding)."""
    from oracle import mlp_fused_fp64
    rng = np.random.default_rng(8)
    n, L = 16, 5
    x = rng.uniform(-1, 1, (9, n)).astype(np.float16)
    w = (rng.standard_normal((L, n, n)) * np.sqrt(2.0 / n)).astype(np.float16)
    b = np.zeros((L, n), np.float16)
    np.testing.assert_array_equal(mlp_fused_fp64(2 * x, w, b), 2 * mlp_fused_fp64(x, w, b))


def test_mlp_tolerance_covers_fp32_kernel_model():
    """The fused-MLP GPU tolerance (tests/test_mlp_fused_gpu.py) against a numpy model of the
    kernel's arithmetic: fp32 accumulation, fp32 bias add and ReLU, fp16 (RNE) store per layer.
    At 20 layers the model must pass the depth-scaled bound and fail the depth-independent one
    (so the scaling is needed, not slack)."""
    from oracle import mlp_fused_fp64
    from workloads import make_fused_mlp_inputs
    x, w, b = (t.numpy() for t in make_fused_mlp_inputs(500, 128, 20))
    ref = mlp_fused_fp64(x, w, b)
    h = x.astype(np.float32)
    for l in range(20):
        h = np.maximum(h @ w[l].astype(np.float32).T + b[l].astype(np.float32), 0).astype(np.float16).astype(np.float32)
    d = np.abs(h.astype(np.float64) - ref)
    assert not (d > 1e-3 * (1 + np.sqrt(20)) + 2 ** -8 * np.abs(ref)).any()
    assert np.linalg.norm(d) / np.linalg.norm(ref) <= 1e-3
    assert (d > 2e-3 + 2 ** -9 * np.abs(ref)).any()


# ---------------------------------------------------------------------------------------------
# Additive key bias (R20): pins for attention_fp64(..., key_bias=)


def _bias_case(seed=0, b=2, h=2, sq=5, skv=7, d=4):
    rng = np.random.default_rng(seed)
    q = rng.standard_normal((b, h, sq, d)).astype(np.float16)
    k = rng.standard_normal((b, h, skv, d)).astype(np.float16)
    v = rng.uniform(-1, 1, (b, h, skv, d)).astype(np.float16)
    return q, k, v


@pytest.mark.parametrize("seed", [0, 1])
def test_key_bias_brute_force(seed):
    q, k, v = _bias_case(seed)
    rng = np.random.default_rng(100 + seed)
    kb = rng.uniform(-3, 3, (2, 7))
    kb[1, 2] = -np.inf
    got = attention_fp64(q, k, v, 0.5, key_bias=kb)
    want = np.array(attention_brute(q.astype(np.float64).tolist(), k.astype(np.float64).tolist(),
                                    v.astype(np.float64).tolist(), 0.5, key_bias=kb.tolist()))
    np.testing.assert_allclose(got, want, rtol=0, atol=1e-12)


def test_key_bias_special_cases():
    q, k, v = _bias_case(3)
    base = attention_fp64(q, k, v, 0.5)
    # zero bias = no mask; a constant bias cancels in the softmax (shift invariance)
    np.testing.assert_allclose(attention_fp64(q, k, v, 0.5, key_bias=np.zeros((2, 7))), base, rtol=0, atol=1e-14)
    np.testing.assert_allclose(attention_fp64(q, k, v, 0.5, key_bias=np.full((2, 7), 123.25)), base, rtol=0, atol=1e-12)
    # -inf past kv_len is exactly key padding (R5)
    kl = np.array([7, 3])
    kb = np.where(np.arange(7)[None, :] < kl[:, None], 0.0, -np.inf)
    np.testing.assert_array_equal(attention_fp64(q, k, v, 0.5, key_bias=kb), attention_fp64(q, k, v, 0.5, kv_len=kl))
    # all keys excluded -> zero rows (R4)
    assert not attention_fp64(q, k, v, 0.5, key_bias=np.full((2, 7), -np.inf)).any()


def test_key_bias_reweighting_closed_form():
    """scale = 0: the weights are softmax(bias), so bias = log w gives O_i = sum_j w_j v_j / sum_j w_j."""
    q, k, v = _bias_case(4)
    w = np.array([[1.0, 2.0, 0.5, 4.0, 1.0, 3.0, 0.25], [2.0, 2.0, 2.0, 1.0, 1.0, 1.0, 8.0]])
    got = attention_fp64(q, k, v, 0.0, key_bias=np.log(w))
    vv = v.astype(np.float64)
    want = np.einsum("bj,bhjd->bhd", w / w.sum(1, keepdims=True), vv)[:, :, None, :].repeat(5, axis=2)
    np.testing.assert_allclose(got, want, rtol=0, atol=1e-12)


def test_key_bias_rows_sampler_matches_full():
    q, k, v = _bias_case(5)
    kb = np.random.default_rng(6).uniform(-2, 2, (2, 7))
    full = attention_fp64(q, k, v, 0.25, key_bias=kb)
    units = [(0, 0, 0), (1, 1, 4), (0, 1, 2)]
    np.testing.assert_allclose(attention_rows_fp64(q, k, v, 0.25, units, key_bias=kb),
                               np.stack([full[b, h, i] for b, h, i in units]), rtol=0, atol=1e-13)


# ---------------------------------------------------------------------------------------------
# General additive (query x key) mask (R21): pins for attention_fp64(..., attn_bias=)


@pytest.mark.parametrize("seed", [0, 1])
def test_attn_bias_brute_force(seed):
    q, k, v = _bias_case(seed, b=2, h=2, sq=5, skv=6)
    rng = np.random.default_rng(200 + seed)
    ab = rng.uniform(-3, 3, (2, 2, 5, 6))
    ab[0, 1, 2, :4] = -np.inf
    ab[1, 0, 4, :] = -np.inf  # a fully excluded row -> 0
    got = attention_fp64(q, k, v, 0.5, attn_bias=ab)
    want = np.array(attention_brute(q.astype(np.float64).tolist(), k.astype(np.float64).tolist(),
                                    v.astype(np.float64).tolist(), 0.5, attn_bias=ab.tolist()))
    np.testing.assert_allclose(got, want, rtol=0, atol=1e-12)
    assert not got[1, 0, 4].any()


def test_attn_bias_torch_sdpa_fp64():
    """Library special case: torch SDPA with a float additive attn_mask [B, 1, Sq, Skv] (broadcast over
    heads), in float64 on the CPU."""
    b, h, sq, skv, d = 2, 3, 19, 23, 8
    q, k, v = rnd((b, h, sq, d), 21), rnd((b, h, skv, d), 22), rnd((b, h, skv, d), 23)
    ab = np.random.default_rng(24).uniform(-4, 2, (b, 1, sq, skv))
    got = attention_fp64(q, k, v, 0.25, attn_bias=ab)
    ref = torch.nn.functional.scaled_dot_product_attention(
        torch.from_numpy(q), torch.from_numpy(k), torch.from_numpy(v), attn_mask=torch.from_numpy(ab),
        scale=float(np.float32(0.25))).numpy()
    np.testing.assert_allclose(got, ref, atol=1e-12, rtol=1e-10)


def test_attn_bias_reduces_to_key_bias_causal_and_padding():
    q, k, v = _bias_case(5, b=2, h=2, sq=6, skv=6)
    kb = np.random.default_rng(25).uniform(-2, 2, (2, 6))
    # a bias that does not depend on the query row is the key bias (R20)
    np.testing.assert_array_equal(attention_fp64(q, k, v, 0.5, attn_bias=kb[:, None, None, :]),
                                  attention_fp64(q, k, v, 0.5, key_bias=kb))
    # -inf above the diagonal is the causal mask (R6, Sq = Skv); -inf past kv_len is key padding (R5)
    tri = np.where(np.arange(6)[None, :] <= np.arange(6)[:, None], 0.0, -np.inf)
    np.testing.assert_array_equal(attention_fp64(q, k, v, 0.5, attn_bias=tri), attention_fp64(q, k, v, 0.5, causal=True))
    kl = np.array([6, 2])
    pad = np.where(np.arange(6)[None, :] < kl[:, None], 0.0, -np.inf)[:, None, None, :]
    np.testing.assert_array_equal(attention_fp64(q, k, v, 0.5, attn_bias=pad), attention_fp64(q, k, v, 0.5, kv_len=kl))
    # sampled rows agree with the full oracle
    ab = np.random.default_rng(26).uniform(-2, 2, (2, 2, 6, 6))
    full = attention_fp64(q, k, v, 0.5, attn_bias=ab)
    units = [(0, 1, 3), (1, 0, 5)]
    rows = attention_rows_fp64(q, k, v, 0.5, units, attn_bias=ab)
    for n, (bb, hh, ii) in enumerate(units):
        np.testing.assert_allclose(rows[n], full[bb, hh, ii], rtol=0, atol=1e-14)
