"""GPU parity: the CUDA FMHA path (through the C ABI) against the fp64 CPU oracle.

Tolerances (BASELINE.json north_star; R10): fp16 output max|err| <= 2e-3 and
rel-L2 <= 1e-3; bf16 output max|err| <= 8e-3 and rel-L2 <= 3e-3 (bf16 output rounding alone
gives rel-L2 ~1.6e-3, so the north star's 1e-3 cannot bind bf16).
"""

import math

import numpy as np
import pytest
import torch

import paper_conf_asplos_hagedornfccgg23_b200 as fm
from oracle import attention_fp64
from workloads import (CONFIGS, MASK_CAUSAL, MASK_KEY_PADDING, MASK_NONE, FmhaConfig, make_fmha_inputs)

pytestmark = pytest.mark.gpu
DEV = torch.device("cuda:0") if torch.cuda.is_available() else None
TOL = {"fp16": (2e-3, 1e-3), "bf16": (8e-3, 3e-3)}


def run(cfg: FmhaConfig, q, k, v, kv_len, scale=None):
    scale = cfg.scale if scale is None else scale
    kl = None if kv_len is None else torch.from_numpy(np.asarray(kv_len, dtype=np.int32)).to(DEV)
    o = fm.fmha_fwd(q.to(DEV), k.to(DEV), v.to(DEV), kv_len=kl, causal=cfg.mask == MASK_CAUSAL, scale=scale)
    torch.cuda.synchronize()
    return o


def check(got, ref, dtype, what=""):
    got = got.double().cpu().numpy() if torch.is_tensor(got) else got
    assert np.all(np.isfinite(got)), f"{what}: non-finite output"
    err = np.abs(got - ref).max() if got.size else 0.0
    nrm = np.linalg.norm(ref)
    rel = np.linalg.norm(got - ref) / nrm if nrm > 0 else np.linalg.norm(got)
    amax, rmax = TOL[dtype]
    assert err <= amax and rel <= rmax, f"{what}: max|err|={err:.3e} rel-L2={rel:.3e}"
    return err, rel


SHAPES = [(1, 1), (17, 17), (64, 64), (127, 129), (128, 128), (129, 200), (200, 520), (384, 384), (77, 300),
          (300, 77)]


@pytest.mark.parametrize("dtype", ["fp16", "bf16"])
@pytest.mark.parametrize("d", [64, 128])
@pytest.mark.parametrize("mask", [MASK_NONE, MASK_CAUSAL, MASK_KEY_PADDING])
@pytest.mark.parametrize("sq,skv", SHAPES)
def test_parity_sweep(dtype, d, mask, sq, skv):
    cfg = FmhaConfig("sweep", 11, 2, 3, sq, skv, d, dtype, mask)
    q, k, v, kl = make_fmha_inputs(cfg)
    if mask == MASK_KEY_PADDING:
        kl = np.array([skv, max(0, skv // 3 - 1)], dtype=np.int32)  # incl. possibly 0 -> zero rows
    o = run(cfg, q, k, v, kl)
    ref = attention_fp64(q, k, v, cfg.scale, kl, causal=mask == MASK_CAUSAL)
    check(o, ref, dtype, f"{dtype} d={d} mask={mask} sq={sq} skv={skv}")
    if mask == MASK_KEY_PADDING and kl[1] == 0:
        assert torch.count_nonzero(o[1]).item() == 0


@pytest.mark.parametrize("dtype,d", [("fp16", 64), ("bf16", 128)])
def test_kv_len_edge_values(dtype, d):
    cfg = FmhaConfig("kvedge", 12, 6, 2, 150, 260, d, dtype, MASK_KEY_PADDING)
    q, k, v, _ = make_fmha_inputs(cfg)
    kl = np.array([0, 1, 127, 128, 129, 260], dtype=np.int32)
    o = run(cfg, q, k, v, kl)
    check(o, attention_fp64(q, k, v, cfg.scale, kl), dtype, "kv_len edges")
    # out-of-range lengths are clamped to [0, seq_kv]
    kl2 = np.array([-5, 1, 127, 128, 129, 10**6], dtype=np.int32)
    o2 = run(cfg, q, k, v, kl2)
    assert torch.equal(o, o2)


def test_garbage_in_masked_kv_rows_is_inert():
    cfg = FmhaConfig("garbage", 13, 2, 2, 130, 300, 64, "fp16", MASK_KEY_PADDING)
    q, k, v, _ = make_fmha_inputs(cfg)
    kl = np.array([140, 300], dtype=np.int32)
    o = run(cfg, q, k, v, kl)
    k2, v2 = k.clone(), v.clone()
    k2[0, :, 140:] = 6e4
    v2[0, :, 140:] = -6e4
    o2 = run(cfg, q, k2, v2, kl)
    assert torch.equal(o, o2)


@pytest.mark.parametrize("mag", [1.0, 30.0])
def test_large_equal_scores_need_max_shift(mag):
    # constant Q and K rows: every score equal and large -> O = mean of V (pin P2)
    cfg = FmhaConfig("const", 14, 1, 2, 200, 333, 64, "fp16")
    _, _, v, _ = make_fmha_inputs(cfg)
    q = torch.full((1, 2, 200, 64), mag, dtype=torch.float16)
    k = torch.full((1, 2, 333, 64), mag, dtype=torch.float16)
    o = run(cfg, q, k, v, None)
    ref = np.broadcast_to(v.double().numpy().mean(2, keepdims=True), o.shape)
    check(o, ref, "fp16", "equal scores")


def test_scale_zero_and_uniform_v():
    cfg = FmhaConfig("s0", 15, 2, 2, 140, 270, 128, "bf16", MASK_CAUSAL)
    q, k, v, _ = make_fmha_inputs(cfg)
    o = run(cfg, q, k, v, None, scale=0.0)
    check(o, attention_fp64(q, k, v, 0.0, causal=True), "bf16", "scale=0 causal")
    vu = torch.empty_like(v)
    vu[:] = v[:, :, :1, :]
    o = run(cfg, q, k, vu, None)
    ref = np.broadcast_to(vu[:, :, :1].double().numpy(), o.shape)
    check(o, ref, "bf16", "uniform V")


def test_stress_distribution():
    cfg = CONFIGS["bert_large_512"].with_(batch=2, qk_sigma=3.0)
    q, k, v, _ = make_fmha_inputs(cfg)
    check(run(cfg, q, k, v, None), attention_fp64(q, k, v, cfg.scale), "fp16", "sigma=3")


def test_determinism_and_shard_consistency():
    cfg = CONFIGS["bert_large_384"].with_(batch=4)
    q, k, v, _ = make_fmha_inputs(cfg)
    o1 = run(cfg, q, k, v, None)
    o2 = run(cfg, q, k, v, None)
    assert torch.equal(o1, o2)
    # O of a (b,h) does not depend on the batch it is computed with (the multi-GPU sharding rule)
    o3 = run(cfg.with_(batch=2), q[2:].contiguous(), k[2:].contiguous(), v[2:].contiguous(), None)
    assert torch.equal(o1[2:], o3)


# ------------------------------------------------------------------ BASELINE sizes, full tensors
FULL = ["bert_base_pad", "bert_large_384", "bert_large_512", "gpt_causal"]


@pytest.mark.timeout(600)
@pytest.mark.parametrize("name", FULL)
def test_full_size_full_oracle(name):
    """Every BASELINE config at full size, in the launch configuration bench.py times (the same
    fmha_fwd call: persistent grid, its item schedule incl. BERT-large-384's single-tile tail items),
    compared with the full fp64 oracle on every element (BL5: 16.8M outputs, ~3 s of oracle; GPT
    causal: 67M outputs, ~40 s)."""
    cfg = CONFIGS[name]
    q, k, v, kl = make_fmha_inputs(cfg)
    o = run(cfg, q, k, v, kl)
    assert torch.isfinite(o).all()
    ref = attention_fp64(q, k, v, cfg.scale, kl, causal=cfg.mask == MASK_CAUSAL)
    check(o, ref, cfg.dtype, name)


def test_tiny_config_full_oracle():
    cfg = CONFIGS["tiny"]
    q, k, v, _ = make_fmha_inputs(cfg)
    check(run(cfg, q, k, v, None), attention_fp64(q, k, v, cfg.scale), "fp16", "tiny")


@pytest.mark.parametrize("name,batch", [("bert_base_pad", 2), ("gpt_causal", 2), ("bert_base_pad", 5),
                                        ("bert_large_384", 7), ("bert_base_pad", 19), ("tiny", 1)])
def test_from_host_entry_point_matches(name, batch):
    """fmha_fwd_from_host pipelines over up to 4 batch chunks on its own streams and joins `stream`:
    bitwise equal to fmha_fwd, and complete after synchronising only the stream passed in."""
    cfg = CONFIGS[name].with_(batch=batch)
    q, k, v, kl = make_fmha_inputs(cfg)
    o = run(cfg, q, k, v, kl)
    pq, pk, pv = q.pin_memory(), k.pin_memory(), v.pin_memory()
    out = torch.empty_like(pq).pin_memory()
    ws = torch.empty(fm.workspace_bytes(cfg.batch, cfg.heads, cfg.seq_q, cfg.seq_kv, cfg.head_dim),
                     dtype=torch.uint8, device=DEV)
    klh = None if kl is None else torch.from_numpy(kl).pin_memory()
    torch.cuda.synchronize()
    s = torch.cuda.Stream(DEV)
    fm.fmha_fwd_from_host(pq, pk, pv, out, ws, kv_len=klh, causal=cfg.mask == MASK_CAUSAL, scale=cfg.scale, stream=s)
    s.synchronize()
    assert torch.equal(out, o.cpu())


# ------------------------------------------------------------------ regression: pipeline deadlocks
@pytest.mark.timeout(240)
@pytest.mark.parametrize("name,batch", [("bert_base_pad", 32), ("bert_large_384", 32), ("bert_large_512", 8)])
def test_back_to_back_launches_do_not_hang(name, batch):
    """Many items per persistent CTA, many launches back to back: exercises the K/V ring release
    (each MMA warp commits once per entry) and the L_FULL / L_EMPTY hand-off that used to run two
    phases ahead when items are a single step long.  A hang fails this test by timeout."""
    cfg = CONFIGS[name].with_(batch=batch)
    q, k, v, kl = make_fmha_inputs(cfg)
    qd, kd, vd = q.to(DEV), k.to(DEV), v.to(DEV)
    kld = None if kl is None else torch.from_numpy(kl).to(DEV)
    out = torch.empty_like(qd)
    first = None
    for i in range(30):
        fm.fmha_fwd(qd, kd, vd, kv_len=kld, scale=cfg.scale, out=out)
        if i == 0:
            torch.cuda.synchronize()
            first = out.clone()
    torch.cuda.synchronize()
    assert torch.equal(out, first)


# ------------------------------------------------------------------ programmatic dependent launch
@pytest.mark.timeout(240)
def test_pdl_chained_launches_keep_stream_order():
    """Launches overlap their prologue with the previous kernel (PDL), but every global access sits
    behind griddepcontrol.wait.  RAW: the second FMHA reads the first one's output as its Q.  WAR:
    the third writes its output into the buffer the second one read.  Both must match the same
    computations separated by full synchronisations, bit for bit, on every repetition."""
    cfg = CONFIGS["bert_large_512"].with_(batch=4)
    q, k, v, _ = make_fmha_inputs(cfg)
    qd, kd, vd = q.to(DEV), k.to(DEV), v.to(DEV)
    # reference: one launch at a time
    o1_ref = fm.fmha_fwd(qd, kd, vd, scale=cfg.scale)
    torch.cuda.synchronize()
    o2_ref = fm.fmha_fwd(o1_ref.clone(), kd, vd, scale=cfg.scale)
    torch.cuda.synchronize()
    o3_ref = fm.fmha_fwd(vd, qd, kd, scale=cfg.scale)
    torch.cuda.synchronize()
    for _ in range(20):
        o1 = torch.empty_like(qd)
        fm.fmha_fwd(qd, kd, vd, scale=cfg.scale, out=o1)          # writes o1
        o2 = fm.fmha_fwd(o1, kd, vd, scale=cfg.scale)             # RAW on o1
        fm.fmha_fwd(vd, qd, kd, scale=cfg.scale, out=o1)          # WAR on o1 (read by the previous launch)
        torch.cuda.synchronize()
        assert torch.equal(o2, o2_ref)
        assert torch.equal(o1, o3_ref)


@pytest.mark.timeout(240)
def test_pdl_gemm_feeds_fmha():
    """GEMM (PDL) -> FMHA (PDL) -> GEMM (PDL) on one stream: the FMHA's Q is the GEMM output and
    the last GEMM reads the FMHA output; equal to the same chain with a sync after every launch."""
    g = torch.Generator().manual_seed(7)
    b, h, s, d = 2, 4, 256, 64
    a = (torch.randn(b * h * s, 64, generator=g) * 0.5).half().to(DEV)
    w = (torch.randn(64, 64, generator=g) * 0.125).half().to(DEV)
    k = torch.randn(b, h, s, d, generator=g).half().to(DEV)
    v = torch.rand(b, h, s, d, generator=g).half().to(DEV)

    def chain(sync):
        x = fm.gemm_bias_act(a, w)
        if sync:
            torch.cuda.synchronize()
        o = fm.fmha_fwd(x.view(b, h, s, d), k, v, scale=0.125)
        if sync:
            torch.cuda.synchronize()
        y = fm.gemm_bias_act(o.view(b * h * s, d), w, act="relu")
        torch.cuda.synchronize()
        return y

    ref = chain(True)
    for _ in range(10):
        assert torch.equal(chain(False), ref)
