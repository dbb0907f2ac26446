"""GPU parity of SURVEY.md §8(f) f2's remaining pieces through the C ABI, against the fp64 oracle:

* strided layouts (fmha_fwd_strided): Q, K, V, O addressed through {batch, head, row} strides, e.g. the
  [B, S, H, D] layout of a QKV projection's output viewed as [B, H, S, D] with .transpose(1, 2), and the
  packed [B, S, 3, H, D] QKV tensor; outputs written through a strided O view;
* the general additive (query x key) mask (FMHA_MASK_ATTN_BIAS, R21): attn_bias broadcastable
  to [B, H, Sq, Skv] in the I/O type, -inf excluding pairs, pinned in the oracle by tests/test_oracle.py.

Tolerances as tests/test_fmha_gpu.py (R10).  The inputs are the seeded workloads; the bias
values are drawn here (uniform log-weights, with -inf patterns) from fixed seeds.
"""

import numpy as np
import pytest
import torch

import paper_conf_asplos_hagedornfccgg23_b200 as fm
from oracle import attention_fp64
from workloads import FmhaConfig, make_fmha_inputs

pytestmark = pytest.mark.gpu
DEV = torch.device("cuda:0") if torch.cuda.is_available() else None
TOL = {"fp16": (2e-3, 1e-3), "bf16": (8e-3, 3e-3)}


def check(got, ref, dtype, what):
    got = got.double().cpu().numpy()
    assert np.all(np.isfinite(got)), what
    err = np.abs(got - ref).max() if got.size else 0.0
    nrm = np.linalg.norm(ref)
    rel = np.linalg.norm(got - ref) / nrm if nrm > 0 else np.linalg.norm(got)
    amax, rmax = TOL[dtype]
    assert err <= amax and rel <= rmax, f"{what}: max|err|={err:.3e} rel-L2={rel:.3e}"


# ------------------------------------------------------------------ strided layouts
@pytest.mark.parametrize("dtype", ["fp16", "bf16"])
@pytest.mark.parametrize("d", [64, 128])
@pytest.mark.parametrize("sq,skv,mask", [(512, 512, 0), (200, 520, 1), (384, 384, 0), (300, 300, 2), (77, 129, 0)])
def test_bshd_layout(dtype, d, sq, skv, mask):
    """Q, K, V, O all [B, S, H, D] (the HF layout), passed as [B, H, S, D] views."""
    cfg = FmhaConfig("strided", 40, 2, 3, sq, skv, d, dtype, mask)
    q, k, v, _ = make_fmha_inputs(cfg)
    kl = np.array([skv, skv // 2 + 3], dtype=np.int32) if mask == 1 else None
    qs, ks, vs = (t.transpose(1, 2).contiguous().to(DEV).transpose(1, 2) for t in (q, k, v))
    assert not qs.is_contiguous()
    out = torch.empty((2, sq, 3, d), dtype=q.dtype, device=DEV).transpose(1, 2)
    o = fm.fmha_fwd(qs, ks, vs, kv_len=None if kl is None else torch.from_numpy(kl).to(DEV), causal=mask == 2,
                    scale=cfg.scale, out=out)
    torch.cuda.synchronize()
    assert o.data_ptr() == out.data_ptr()
    check(o, attention_fp64(q, k, v, cfg.scale, kl, causal=mask == 2), dtype, f"bshd {dtype} d={d} {sq}x{skv} m{mask}")
    # bitwise the same as the contiguous path (only the addressing differs)
    oc = fm.fmha_fwd(q.to(DEV), k.to(DEV), v.to(DEV), kv_len=None if kl is None else torch.from_numpy(kl).to(DEV),
                     causal=mask == 2, scale=cfg.scale)
    torch.cuda.synchronize()
    assert torch.equal(o, oc)


@pytest.mark.parametrize("d", [64, 128])
def test_packed_qkv_bs3hd_and_mixed_strides(d):
    """A packed QKV projection output [B, S, 3, H, D] (Q, K, V interleaved per token) consumed in place,
    and a batch padded with extra rows (row stride > the next dimension) for K only."""
    cfg = FmhaConfig("packed", 41, 3, 4, 256, 256, d, "fp16")
    q, k, v, _ = make_fmha_inputs(cfg)
    qkv = torch.stack([q, k, v], dim=2).permute(0, 3, 2, 1, 4).contiguous().to(DEV)  # [B, S, 3, H, D]
    qv, kv_, vv = (qkv[:, :, i].transpose(1, 2) for i in range(3))
    o = fm.fmha_fwd(qv, kv_, vv, scale=cfg.scale)
    torch.cuda.synchronize()
    ref = attention_fp64(q, k, v, cfg.scale)
    check(o, ref, "fp16", "packed qkv")
    kpad = torch.zeros((3, 4, 300, d), dtype=q.dtype, device=DEV)
    kpad[:, :, :256] = k.to(DEV)
    o2 = fm.fmha_fwd(q.to(DEV), kpad[:, :, :256], v.to(DEV), scale=cfg.scale)
    torch.cuda.synchronize()
    assert torch.equal(o2, o)


def test_strided_rejects_unaligned_strides():
    x = torch.zeros((1, 2, 10, 64), dtype=torch.float16, device=DEV)
    bad = torch.zeros((1, 10, 2, 68), dtype=torch.float16, device=DEV)[..., :64].transpose(1, 2)  # row stride 136 ok, head 68 -> not /8
    with pytest.raises((fm.FmhaError, ValueError)):
        fm.fmha_fwd(bad, x, x)


# ------------------------------------------------------------------ general additive mask (R21)
def make_attn_bias(shape, seed, kind):
    rng = np.random.default_rng(seed)
    ab = np.zeros(shape, dtype=np.float32)
    if kind == "random":  # log-weights in [-3, 3], ~15% of pairs excluded, one fully excluded row
        ab[:] = rng.uniform(-3, 3, shape)
        ab[rng.random(shape) < 0.15] = -np.inf
        ab[(0,) * (len(shape) - 2) + (min(1, shape[-2] - 1), slice(None))] = -np.inf
    elif kind == "block":  # block-diagonal packing mask: query i sees keys of its own 100-token segment
        sq, skv = shape[-2:]
        i, j = np.arange(sq)[:, None], np.arange(skv)[None, :]
        ab[:] = np.where(i // 100 == j // 100, 0.0, -np.inf)
    elif kind == "hf":  # HF extended mask values: 0 or -10000
        ab[:] = np.where(rng.random(shape) < 0.3, -10000.0, 0.0)
    return ab


@pytest.mark.parametrize("dtype", ["fp16", "bf16"])
@pytest.mark.parametrize("d", [64, 128])
@pytest.mark.parametrize("kind", ["random", "block", "hf"])
@pytest.mark.parametrize("sq,skv,heads_dim", [(128, 128, 1), (200, 520, 3), (384, 384, 1), (77, 300, 3), (1, 9, 1)])
def test_attn_bias_parity(dtype, d, kind, sq, skv, heads_dim):
    cfg = FmhaConfig("attnbias", 42, 2, 3, sq, skv, d, dtype)
    q, k, v, _ = make_fmha_inputs(cfg)
    skv8 = (skv + 7) // 8 * 8
    ab = make_attn_bias((2, heads_dim, sq, skv), seed=sq * 7 + skv, kind=kind)
    # the kernel reads 16-bit biases in q's dtype: the oracle gets the same rounded values
    abt = torch.from_numpy(ab).to(q.dtype)
    buf = torch.full((2, heads_dim, sq, skv8), float("nan"), dtype=q.dtype)  # row stride padded to 8, NaN padding
    buf[..., :skv] = abt
    o = fm.fmha_fwd(q.to(DEV), k.to(DEV), v.to(DEV), scale=cfg.scale, attn_bias=buf.to(DEV)[..., :skv])
    torch.cuda.synchronize()
    ref = attention_fp64(q, k, v, cfg.scale, attn_bias=abt.double().numpy())
    check(o, ref, dtype, f"attn_bias {kind} {dtype} d={d} {sq}x{skv} hb={heads_dim}")


def test_attn_bias_equals_causal_and_key_padding_paths():
    """-inf above the diagonal is the causal mask; -inf past kv_len (broadcast over queries and heads,
    batch stride from the tensor) is key padding -- the same operation through different kernel paths."""
    cfg = FmhaConfig("attnbias_eq", 43, 3, 2, 256, 256, 64, "fp16")
    q, k, v, _ = make_fmha_inputs(cfg)
    qd, kd, vd = q.to(DEV), k.to(DEV), v.to(DEV)
    tri = torch.where(torch.arange(256)[None, :] <= torch.arange(256)[:, None], 0.0, float("-inf")).half().to(DEV)
    oa = fm.fmha_fwd(qd, kd, vd, scale=cfg.scale, attn_bias=tri)
    oc = fm.fmha_fwd(qd, kd, vd, scale=cfg.scale, causal=True)
    kl = torch.tensor([256, 100, 1], dtype=torch.int32, device=DEV)
    pad = torch.where(torch.arange(256, device=DEV)[None, :] < kl[:, None], 0.0, float("-inf")).half()
    ob = fm.fmha_fwd(qd, kd, vd, scale=cfg.scale, attn_bias=pad[:, None, None, :].expand(3, 1, 256, 256))
    op = fm.fmha_fwd(qd, kd, vd, scale=cfg.scale, kv_len=kl)
    torch.cuda.synchronize()
    assert (oa.float() - oc.float()).abs().max().item() <= 1e-3
    assert (ob.float() - op.float()).abs().max().item() <= 1e-3


def test_attn_bias_bert_large_full_size():
    """BERT-large seq 384 with a per-batch HF mask [B, 1, S, S] (broadcast over 16 heads), full oracle."""
    cfg = FmhaConfig("attnbias_bl3", 44, 32, 16, 384, 384, 64, "fp16")
    q, k, v, _ = make_fmha_inputs(cfg)
    ab = torch.from_numpy(make_attn_bias((32, 1, 384, 384), 45, "hf")).half()
    o = fm.fmha_fwd(q.to(DEV), k.to(DEV), v.to(DEV), scale=cfg.scale, attn_bias=ab.to(DEV))
    torch.cuda.synchronize()
    check(o, attention_fp64(q, k, v, cfg.scale, attn_bias=ab.double().numpy()), "fp16", "bert_large_384 attn_bias")


def test_attn_bias_errors():
    x = torch.zeros((1, 1, 8, 64), dtype=torch.float16, device=DEV)
    with pytest.raises((fm.FmhaError, ValueError)):  # row stride not a multiple of 8
        fm.fmha_fwd(x, x, x, attn_bias=torch.zeros((1, 1, 8, 12), dtype=torch.float16, device=DEV)[..., :8])
    with pytest.raises(ValueError):  # dtype must be q's
        fm.fmha_fwd(x, x, x, attn_bias=torch.zeros((1, 1, 8, 8), dtype=torch.float32, device=DEV))
    with pytest.raises(fm.FmhaError):  # scale 0 (the bias is added as bias / scale)
        fm.fmha_fwd(x, x, x, scale=0.0, attn_bias=torch.zeros((1, 1, 8, 8), dtype=torch.float16, device=DEV))
