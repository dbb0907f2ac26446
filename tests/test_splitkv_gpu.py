"""GPU parity for the split-KV FMHA path (fmha_fwd_splitkv) against the fp64 oracle
(the same plain definition as fmha_fwd: splitting the keys is an implementation choice, not part of
the method, so the tolerances are the dense path's, R10)."""

import numpy as np
import pytest
import torch

import paper_conf_asplos_hagedornfccgg23_b200 as fm
from oracle import attention_fp64, attention_rows_fp64
from workloads import MASK_CAUSAL, MASK_KEY_PADDING, MASK_NONE, SPLITKV_CONFIGS, FmhaConfig, make_fmha_inputs

pytestmark = pytest.mark.gpu
DEV = torch.device("cuda:0") if torch.cuda.is_available() else None
TOL = {"fp16": (2e-3, 1e-3), "bf16": (8e-3, 3e-3)}


def check(got, ref, dtype, what):
    got = got.double().cpu().numpy()
    assert np.all(np.isfinite(got)), what
    err = np.abs(got - ref).max()
    nrm = np.linalg.norm(ref)
    rel = np.linalg.norm(got - ref) / nrm if nrm > 0 else np.linalg.norm(got)
    amax, rmax = TOL[dtype]
    assert err <= amax and rel <= rmax, f"{what}: max|err|={err:.3e} rel-L2={rel:.3e}"


def run(cfg, q, k, v, kl, splits):
    kld = None if kl is None else torch.from_numpy(np.asarray(kl, dtype=np.int32)).to(DEV)
    o = fm.fmha_fwd_splitkv(q.to(DEV), k.to(DEV), v.to(DEV), kv_len=kld, causal=cfg.mask == MASK_CAUSAL,
                            scale=cfg.scale, num_splits=splits)
    torch.cuda.synchronize()
    return o


@pytest.mark.parametrize("dtype", ["fp16", "bf16"])
@pytest.mark.parametrize("d", [64, 128])
@pytest.mark.parametrize("mask", [MASK_NONE, MASK_CAUSAL, MASK_KEY_PADDING])
@pytest.mark.parametrize("sq,skv", [(1, 1000), (16, 2049), (100, 700), (128, 1280), (200, 900), (1, 129)])
@pytest.mark.parametrize("splits", [0, 2, 3, 7])
def test_splitkv_parity(dtype, d, mask, sq, skv, splits):
    cfg = FmhaConfig("splitkv", 15, 2, 2, sq, skv, d, dtype, mask)
    q, k, v, kl = make_fmha_inputs(cfg)
    if mask == MASK_KEY_PADDING:
        kl = np.array([skv, max(0, skv // 3 - 1)], dtype=np.int32)
    o = run(cfg, q, k, v, kl, splits)
    ref = attention_fp64(q, k, v, cfg.scale, kl, causal=mask == MASK_CAUSAL)
    check(o, ref, dtype, f"{dtype} d={d} mask={mask} sq={sq} skv={skv} splits={splits}")


def test_splitkv_fully_masked_rows_and_empty_splits():
    """kv_len = 0 (every split empty -> O = 0) and kv_len shorter than one split (later splits empty)."""
    cfg = FmhaConfig("splitkv_pad", 16, 3, 2, 8, 4096, 64, "fp16", MASK_KEY_PADDING)
    q, k, v, _ = make_fmha_inputs(cfg)
    kl = np.array([0, 100, 4096], dtype=np.int32)
    o = run(cfg, q, k, v, kl, 8)
    assert torch.count_nonzero(o[0]).item() == 0
    check(o, attention_fp64(q, k, v, cfg.scale, kl), "fp16", "padding")


def test_splitkv_matches_dense_within_rounding():
    """One split = the dense kernel; many splits differ from it only by fp32 rounding order."""
    cfg = FmhaConfig("splitkv_eq", 17, 1, 4, 64, 3000, 128, "bf16")
    q, k, v, _ = make_fmha_inputs(cfg)
    o1 = run(cfg, q, k, v, None, 1)
    od = fm.fmha_fwd(q.to(DEV), k.to(DEV), v.to(DEV), scale=cfg.scale)
    torch.cuda.synchronize()
    assert torch.equal(o1, od)
    o8 = run(cfg, q, k, v, None, 8)
    assert (o8.float() - od.float()).abs().max().item() <= 8e-3


@pytest.mark.parametrize("name", sorted(SPLITKV_CONFIGS))
def test_splitkv_bench_config_sampled(name):
    """The bench workload at full size, default splits (the launch the bench times); sampled rows."""
    cfg = SPLITKV_CONFIGS[name]
    q, k, v, _ = make_fmha_inputs(cfg)
    o = run(cfg, q, k, v, None, 0)
    rng = np.random.default_rng(4)
    units = [(b, h, int(i)) for b, h in [(0, 0), (cfg.batch - 1, cfg.heads - 1), (1, 3)]
             for i in np.unique(np.concatenate([rng.choice(cfg.seq_q, min(8, cfg.seq_q), replace=False),
                                                [cfg.seq_q - 1]]))]
    ref = attention_rows_fp64(q, k, v, cfg.scale, units)
    got = torch.stack([o[b, h, i] for b, h, i in units])
    check(got, ref, cfg.dtype, name)
