"""GPU parity of the packed variable-length path (fmha_fwd_varlen: the MLPerf BERT
inference layout QKV [T,3,H,D] + cu_seqlens) against oracle.attention_varlen_fp64.
Tolerances as tests/test_fmha_gpu.py (R10)."""

import numpy as np
import pytest
import torch

import paper_conf_asplos_hagedornfccgg23_b200 as fm
from oracle import attention_varlen_fp64
from workloads import VARLEN_CONFIGS, VarlenConfig, make_varlen_inputs

pytestmark = pytest.mark.gpu
DEV = torch.device("cuda:0") if torch.cuda.is_available() else None
TOL = {"fp16": (2e-3, 1e-3), "bf16": (8e-3, 3e-3)}


def check(got, ref, dtype, what=""):
    got = got.double().cpu().numpy()
    assert np.all(np.isfinite(got)), f"{what}: non-finite output"
    err = np.abs(got - ref).max()
    rel = np.linalg.norm(got - ref) / np.linalg.norm(ref)
    amax, rmax = TOL[dtype]
    assert err <= amax and rel <= rmax, f"{what}: max|err|={err:.3e} rel-L2={rel:.3e}"


def run(cfg, x, cu, max_seqlen=None, out=None):
    o = fm.fmha_fwd_varlen(x.to(DEV), torch.from_numpy(cu).to(DEV), max_seqlen or cfg.max_seqlen,
                           causal=cfg.causal, scale=cfg.scale, out=out)
    torch.cuda.synchronize()
    return o


LENGTHS = [
    [1],
    [128],
    [129, 1, 255, 256, 257],
    [0, 77, 0, 300, 5],
    [384, 200, 31, 128, 129, 383],
    [513, 2, 640],
    # odd levels 1, 3, 5 with several sequences each: last q-tiles paired across (sequence, head)
    [1, 130, 260, 390, 5, 300, 129, 0, 384, 383, 600, 77, 520, 31],
]


@pytest.mark.parametrize("dtype,d", [("fp16", 64), ("bf16", 64), ("fp16", 128), ("bf16", 128)])
@pytest.mark.parametrize("causal", [False, True])
@pytest.mark.parametrize("lens", LENGTHS, ids=lambda l: "-".join(map(str, l)))
def test_varlen_parity(dtype, d, causal, lens):
    cfg = VarlenConfig("vsweep", 21, len(lens), 3, max(max(lens), 1), d, dtype, causal)
    x, cu = make_varlen_inputs(cfg, lengths=lens)
    o = run(cfg, x, cu)
    check(o, attention_varlen_fp64(x, cu, cfg.scale, causal), dtype, f"lens={lens} d={d} causal={causal}")


def test_varlen_rows_outside_sequences_untouched_and_max_seqlen_slack():
    """Partial tiles are stored row by row: tokens of a neighbouring sequence are never overwritten
    (each sequence's rows are checked against the oracle in a buffer pre-filled with a sentinel),
    and a max_seqlen larger than every length gives the same result."""
    cfg = VarlenConfig("vslack", 22, 4, 2, 300, 64)
    lens = [130, 3, 300, 129]
    x, cu = make_varlen_inputs(cfg, lengths=lens)
    out = torch.full((int(cu[-1]), 2, 64), 7.0, dtype=torch.float16, device=DEV)
    o1 = run(cfg, x, cu, out=out)
    check(o1, attention_varlen_fp64(x, cu, cfg.scale), "fp16", "sentinel")
    o2 = run(cfg, x, cu, max_seqlen=1000)
    assert torch.equal(o1, o2)


@pytest.mark.parametrize("seq", [256, 512, 384])
def test_varlen_equal_lengths_matches_dense_kernel(seq):
    """Equal lengths: with an odd q-tile count (384 = 3 tiles) the dense [B,H,S,D] path runs the
    cross-unit pair instance, whose exp2 arithmetic (every exp2 on MUFU, ExpShape) is the varlen
    instances' one, so the outputs are bitwise equal (the pre-turn chunk count only reorders work).
    An even count runs the dense instance, which takes 2 of 8 exp2 pairs on the FMA-pipe polynomial:
    there both sides are held to the oracle tolerance and to each other within fp16 rounding."""
    cfg = VarlenConfig("veq", 23, 3, 4, seq, 64)
    x, cu = make_varlen_inputs(cfg, lengths=[seq] * 3)
    o = run(cfg, x, cu)
    xs = x.view(3, seq, 3, 4, 64).permute(2, 0, 3, 1, 4).contiguous().to(DEV)  # [3,B,H,S,D]
    od = fm.fmha_fwd(xs[0], xs[1], xs[2], scale=cfg.scale)
    torch.cuda.synchronize()
    od = od.permute(0, 2, 1, 3).reshape(3 * seq, 4, 64)
    if (seq // 128) % 2 == 1:
        assert torch.equal(o, od)
    else:
        ref = attention_varlen_fp64(x, cu, cfg.scale)
        check(o, ref, "fp16", "varlen")
        check(od, ref, "fp16", "dense instance")
        assert (o.float() - od.float()).abs().max().item() <= 2e-3


def test_varlen_bert_large_full_size():
    """BASELINE-size MLPerf-style batch (32 sequences, 16 heads, max 384) in the bench's launch
    configuration, against the full oracle."""
    cfg = VARLEN_CONFIGS["bert_large_varlen"]
    x, cu = make_varlen_inputs(cfg)
    o = run(cfg, x, cu)
    check(o, attention_varlen_fp64(x, cu, cfg.scale), "fp16", "bert_large_varlen")


def test_varlen_rejects_bad_args():
    x = torch.zeros((8, 3, 2, 64), dtype=torch.float16, device=DEV)
    cu = torch.tensor([0, 8], dtype=torch.int32, device=DEV)
    with pytest.raises(fm.FmhaError):
        fm.fmha_fwd_varlen(x, cu, 8, scale=-1.0)
    x96 = torch.zeros((8, 3, 2, 96), dtype=torch.float16, device=DEV)
    with pytest.raises(fm.FmhaError):
        fm.fmha_fwd_varlen(x96, cu, 8)
    # zero sequences / zero max_seqlen: no launch, OK
    fm.fmha_fwd_varlen(x, torch.zeros(1, dtype=torch.int32, device=DEV), 0)
