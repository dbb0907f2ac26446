"""GPU parity for the additive key bias mask (FMHA_MASK_KEY_BIAS, R20: the HF BERT
"extended attention mask"; SURVEY §8(f) f2 "arbitrary boolean/additive masks") through the C ABI,
against the fp64 oracle (attention_fp64(..., key_bias=)).  Tolerances as the dense path (R10)."""

import numpy as np
import pytest
import torch

import paper_conf_asplos_hagedornfccgg23_b200 as fm
from oracle import attention_fp64, attention_rows_fp64
from workloads import CONFIGS, FmhaConfig, make_fmha_inputs

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


def make_bias(batch, skv, kind, seed, stride=None):
    stride = stride or (skv + 3) // 4 * 4
    rng = np.random.default_rng(seed)
    kb = np.zeros((batch, stride), dtype=np.float32)
    if kind == "random":  # log-weights in [-3, 3], ~20% of keys excluded
        kb[:, :skv] = rng.uniform(-3, 3, (batch, skv))
        kb[:, :skv][rng.random((batch, skv)) < 0.2] = -np.inf
    elif kind == "hf":  # HF BERT extended mask: 0 for real tokens, -10000 for padding
        for b in range(batch):
            n = skv if b == 0 else int(rng.integers(1, skv + 1))
            kb[b, n:skv] = -10000.0
    elif kind == "excluded":  # batch 1 sees no key at all -> zero rows
        kb[1, :] = -np.inf
    kb[:, skv:] = np.nan  # padding columns past seq_kv must never be read into a result
    return kb


@pytest.mark.parametrize("dtype", ["fp16", "bf16"])
@pytest.mark.parametrize("d", [64, 128])
@pytest.mark.parametrize("kind", ["random", "hf", "excluded"])
@pytest.mark.parametrize("sq,skv", [(1, 1), (64, 64), (127, 129), (200, 520), (384, 384), (77, 300)])
def test_key_bias_parity(dtype, d, kind, sq, skv):
    cfg = FmhaConfig("keybias", 18, 2, 3, sq, skv, d, dtype)
    q, k, v, _ = make_fmha_inputs(cfg)
    kb = make_bias(2, skv, kind, seed=sq * 1000 + skv)
    o = fm.fmha_fwd(q.to(DEV), k.to(DEV), v.to(DEV), scale=cfg.scale, key_bias=torch.from_numpy(kb).to(DEV))
    torch.cuda.synchronize()
    ref = attention_fp64(q, k, v, cfg.scale, key_bias=kb[:, :skv])
    check(o, ref, dtype, f"{dtype} d={d} {kind} sq={sq} skv={skv}")
    if kind == "excluded":
        assert torch.count_nonzero(o[1]).item() == 0


def test_key_bias_minus_inf_equals_key_padding():
    """bias = -inf past kv_len and the KEY_PADDING mask are the same operation (R5, R20)."""
    cfg = CONFIGS["bert_base_pad"].with_(batch=4)
    q, k, v, kl = make_fmha_inputs(cfg)
    kb = np.where(np.arange(cfg.seq_kv)[None, :] < kl[:, None], 0.0, -np.inf).astype(np.float32)
    qd, kd, vd = q.to(DEV), k.to(DEV), v.to(DEV)
    ob = fm.fmha_fwd(qd, kd, vd, scale=cfg.scale, key_bias=torch.from_numpy(kb).to(DEV))
    op = fm.fmha_fwd(qd, kd, vd, scale=cfg.scale, kv_len=torch.from_numpy(kl).to(DEV))
    torch.cuda.synchronize()
    assert (ob.float() - op.float()).abs().max().item() <= 1e-3


def test_key_bias_full_size_sampled():
    """BERT-large seq 384 (the paper's MLPerf shape) with HF-style padding bias, full batch."""
    cfg = CONFIGS["bert_large_384"]
    q, k, v, _ = make_fmha_inputs(cfg)
    kb = make_bias(cfg.batch, cfg.seq_kv, "hf", seed=7)
    o = fm.fmha_fwd(q.to(DEV), k.to(DEV), v.to(DEV), scale=cfg.scale, key_bias=torch.from_numpy(kb).to(DEV))
    torch.cuda.synchronize()
    rng = np.random.default_rng(8)
    units = [(int(b), int(h), int(i)) for b, h, i in zip(rng.integers(0, cfg.batch, 24), rng.integers(0, cfg.heads, 24),
                                                         rng.integers(0, cfg.seq_q, 24))] + [(31, 15, 383)]
    ref = attention_rows_fp64(q, k, v, cfg.scale, units, key_bias=kb[:, :cfg.seq_kv])
    check(torch.stack([o[b, h, i] for b, h, i in units]), ref, "fp16", "bert_large_384 hf bias")


def test_key_bias_errors():
    cfg = FmhaConfig("keybias_err", 19, 1, 1, 8, 30, 64, "fp16")
    q, k, v, _ = make_fmha_inputs(cfg)
    qd, kd, vd = q.to(DEV), k.to(DEV), v.to(DEV)
    with pytest.raises(fm.FmhaError):  # stride not a multiple of 4
        fm.fmha_fwd(qd, kd, vd, key_bias=torch.zeros(1, 30, device=DEV))
    with pytest.raises(fm.FmhaError):  # stride < seq_kv
        fm.fmha_fwd(qd, kd, vd, key_bias=torch.zeros(1, 28, device=DEV))
    with pytest.raises(fm.FmhaError):  # scale 0 (the bias is added as bias / scale)
        fm.fmha_fwd(qd, kd, vd, scale=0.0, key_bias=torch.zeros(1, 32, device=DEV))


@pytest.mark.parametrize("skv,extra", [(260, 0), (200, 60), (129, 380), (512, 4)])
def test_key_bias_row_stride_and_clamped_tail(skv, extra):
    """Bias rows longer than seq_kv (stride = seq_kv rounded to 4 + extra, NaN past seq_kv): the
    kernel's bias loads are clamped to the row's last float4 (FMHA_BIAS_CLAMP) and every column past
    seq_kv is masked before the row max, so neither the stride nor the padding reaches a result."""
    cfg = FmhaConfig("keybias_stride", 20, 3, 2, 150, skv, 64, "fp16")
    q, k, v, _ = make_fmha_inputs(cfg)
    kb = make_bias(3, skv, "random", seed=skv + extra, stride=(skv + 3) // 4 * 4 + extra)
    o = fm.fmha_fwd(q.to(DEV), k.to(DEV), v.to(DEV), scale=cfg.scale, key_bias=torch.from_numpy(kb).to(DEV))
    torch.cuda.synchronize()
    check(o, attention_fp64(q, k, v, cfg.scale, key_bias=kb[:, :skv]), "fp16", f"skv={skv} extra={extra}")
