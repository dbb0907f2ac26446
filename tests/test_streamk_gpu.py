"""GPU parity for the stream-K tail FMHA (fmha_fwd_streamk) against the fp64 oracle.

The full rounds of the persistent schedule run fmha_fwd's items; the last, partial round's items are
cut into key ranges whose online-softmax states are merged in the kernel by the piece that finishes
last.  Splitting the keys is an implementation choice, not part of the method (PAPER.md L487 defines
O = softmax(scale Q K^T + mask) V), so the tolerances are the dense path's (R10).  Shapes
are chosen so the plan on a 148-SM B200 really splits (asserted through fmha_streamk_plan)."""

import numpy as np
import pytest
import torch

import paper_conf_asplos_hagedornfccgg23_b200 as fm
from oracle import attention_fp64
from workloads import CONFIGS, MASK_CAUSAL, MASK_KEY_PADDING, MASK_NONE, FmhaConfig, add_score_ramp, make_fmha_inputs

pytestmark = pytest.mark.gpu
DEV = torch.device("cuda:0") if torch.cuda.is_available() else None
TOL = {"fp16": (2e-3, 1e-3), "bf16": (8e-3, 3e-3)}


def sms():
    return torch.cuda.get_device_properties(0).multi_processor_count


def check(got, ref, dtype, what):
    got = got.double().cpu().numpy()
    assert np.all(np.isfinite(got)), what
    err = np.abs(got - ref).max()
    nrm = np.linalg.norm(ref)
    rel = np.linalg.norm(got - ref) / nrm if nrm > 0 else np.linalg.norm(got)
    amax, rmax = TOL[dtype]
    assert err <= amax and rel <= rmax, f"{what}: max|err|={err:.3e} rel-L2={rel:.3e}"


def run(cfg, q, k, v, kl):
    kld = None if kl is None else torch.from_numpy(np.asarray(kl, dtype=np.int32)).to(DEV)
    o = fm.fmha_fwd_streamk(q.to(DEV), k.to(DEV), v.to(DEV), kv_len=kld, causal=cfg.mask == MASK_CAUSAL,
                            scale=cfg.scale)
    torch.cuda.synchronize()
    return o


# (b, h, sq, skv) with >= 5 KV tiles (the plan splits only when that saves >= 4 KV steps): all-tail
# small problems (every item is split), cross-unit pairs (3 q-tiles), ragged tiles, Sq != Skv, and
# shapes with full rounds plus a tail
SHAPES = [(1, 3, 384, 1024), (2, 4, 512, 700), (1, 5, 300, 1300), (2, 3, 200, 700), (3, 2, 129, 1000),
          (5, 31, 256, 1024), (3, 50, 256, 2100)]


@pytest.mark.parametrize("dtype", ["fp16", "bf16"])
@pytest.mark.parametrize("d", [64, 128])
@pytest.mark.parametrize("mask", [MASK_NONE, MASK_CAUSAL, MASK_KEY_PADDING])
@pytest.mark.parametrize("shape", SHAPES)
def test_streamk_parity(dtype, d, mask, shape):
    b, h, sq, skv = shape
    cfg = FmhaConfig("streamk", 31, b, h, sq, skv, d, dtype, mask)
    s, tail = fm.streamk_plan(b, h, sq, skv, sms(), mask)
    if mask != MASK_CAUSAL:
        assert s >= 2 and tail > 0, f"plan does not split {shape}: {(s, tail)}"
    q, k, v, kl = make_fmha_inputs(cfg)
    if mask == MASK_KEY_PADDING:  # an empty row set, a row shorter than one piece, a full row
        kl = np.array([[0, 90, skv][i % 3] for i in range(b)], dtype=np.int32)
    o = run(cfg, q, k, v, kl)
    ref = attention_fp64(q, k, v, cfg.scale, kl, causal=mask == MASK_CAUSAL)
    check(o, ref, dtype, f"{dtype} d={d} mask={mask} shape={shape} plan={s, tail}")


@pytest.mark.parametrize("dtype", ["fp16", "bf16"])
@pytest.mark.parametrize("d", [64, 128])
def test_streamk_rescale_in_pieces(dtype, d):
    """Score-ramp inputs (the row max grows by > 8 in log2 per KV tile): every piece rescales lazily
    inside its own key range, and the merge rescales across pieces."""
    cfg = FmhaConfig("streamk_ramp", 32, 1, 3, 384, 1024, d, dtype)
    q, k, v, _ = make_fmha_inputs(cfg)
    q, k = add_score_ramp(q, k, cfg.scale)
    assert fm.streamk_plan(1, 3, 384, 1024, sms())[0] >= 2
    o = run(cfg, q, k, v, None)
    check(o, attention_fp64(q, k, v, cfg.scale), dtype, f"ramp d={d} {dtype}")


def test_streamk_full_rounds_plus_tail_bitwise():
    """A shape with two full rounds and a split tail (3 x 50 units x 2 q-tile pairs = 300 items = 2 x 148
    + 4, 32 KV tiles: 4 pieces of 8): every row against the fp64 oracle, the rows of the full rounds
    bitwise equal to fmha_fwd (same item arithmetic), the tail rows within the tolerance of it."""
    cfg = FmhaConfig("streamk_long", 36, 3, 50, 512, 4096, 64, "fp16")
    s, tail = fm.streamk_plan(cfg.batch, cfg.heads, cfg.seq_q, cfg.seq_kv, sms())
    assert s >= 2
    q, k, v, _ = make_fmha_inputs(cfg)
    o = run(cfg, q, k, v, None)
    check(o, attention_fp64(q, k, v, cfg.scale), cfg.dtype, "full rounds + tail")
    od = fm.fmha_fwd(q.to(DEV), k.to(DEV), v.to(DEV), scale=cfg.scale)
    torch.cuda.synchronize()
    # pair_mode 0: item i = (unit i // 2, q-tile pair i % 2); the last `tail` items are split
    items = cfg.batch * cfg.heads * 2
    fo = o.reshape(items, 256, cfg.head_dim)
    fd = od.reshape(items, 256, cfg.head_dim)
    assert torch.equal(fo[: items - tail], fd[: items - tail])
    assert (fo[items - tail:].float() - fd[items - tail:].float()).abs().max().item() <= 2e-3


def test_streamk_repeated_launches_reset_counters():
    """The merging piece resets its counter: back-to-back launches on one workspace (also inside a
    CUDA graph, as the bench replays it) give bitwise identical results (the merge order is fixed)."""
    cfg = FmhaConfig("streamk_rep", 33, 2, 4, 384, 1024, 64, "fp16")
    q, k, v, _ = make_fmha_inputs(cfg)
    qd, kd, vd = q.to(DEV), k.to(DEV), v.to(DEV)
    ws = torch.zeros(fm._lib.load().fmha_streamk_workspace_bytes(64, 0), dtype=torch.uint8, device=DEV)
    outs = [fm.fmha_fwd_streamk(qd, kd, vd, scale=cfg.scale, workspace=ws) for _ in range(5)]
    torch.cuda.synchronize()
    for o in outs[1:]:
        assert torch.equal(o, outs[0])
    cnt = ws[: 4 * sms()].view(torch.int32)
    assert torch.count_nonzero(cnt).item() == 0
    out = torch.empty_like(qd)
    g = torch.cuda.CUDAGraph()
    s = torch.cuda.Stream()
    s.wait_stream(torch.cuda.current_stream())
    with torch.cuda.stream(s):
        fm.fmha_fwd_streamk(qd, kd, vd, scale=cfg.scale, out=out, workspace=ws)
        torch.cuda.synchronize()
        with torch.cuda.graph(g, stream=s):
            for _ in range(3):
                fm.fmha_fwd_streamk(qd, kd, vd, scale=cfg.scale, out=out, workspace=ws)
    for _ in range(3):
        g.replay()
    torch.cuda.synchronize()
    assert torch.equal(out, outs[0])
    check(outs[0], attention_fp64(q, k, v, cfg.scale), "fp16", "repeated")


def test_streamk_workspace_errors():
    cfg = FmhaConfig("streamk_err", 34, 1, 3, 384, 1024, 64, "fp16")
    q, k, v, _ = make_fmha_inputs(cfg)
    qd, kd, vd = q.to(DEV), k.to(DEV), v.to(DEV)
    small = torch.zeros(1024, dtype=torch.uint8, device=DEV)
    with pytest.raises(fm.FmhaError, match="INVALID_ARG"):
        fm.fmha_fwd_streamk(qd, kd, vd, workspace=small)
    need = fm._lib.load().fmha_streamk_workspace_bytes(64, 0)
    big = torch.zeros(need + 512, dtype=torch.uint8, device=DEV)
    with pytest.raises(fm.FmhaError, match="MISALIGNED"):
        fm.fmha_fwd_streamk(qd, kd, vd, workspace=big[16:])
    # a shape the plan does not split runs fmha_fwd's kernel and schedule: bitwise equal, no workspace use
    cfg1 = FmhaConfig("streamk_nosplit", 35, 1, 2, 128, 128, 64, "fp16")
    assert fm.streamk_plan(1, 2, 128, 128, sms())[0] == 1
    q, k, v, _ = make_fmha_inputs(cfg1)
    o = fm.fmha_fwd_streamk(q.to(DEV), k.to(DEV), v.to(DEV), scale=cfg1.scale, workspace=small)
    od = fm.fmha_fwd(q.to(DEV), k.to(DEV), v.to(DEV), scale=cfg1.scale)
    torch.cuda.synchronize()
    assert torch.equal(o, od)
