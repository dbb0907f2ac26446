"""Multi-process (gloo, world size 2, CPU) checks of the multi-GPU orchestration bench.py runs
(multigpu.py): per-rank shards of a config reproduce the global problem exactly,
the one all-gather reassembles O in the global layout, rank 0's check finds it bitwise equal to the
single-process result, and the timing reduction is a max over ranks.  The per-(b, h) arithmetic here
is the oracle's, rounded to fp16 like the kernel's output (the GPU path's shard invariance is covered
by test_fmha_gpu.py::test_determinism_and_shard_consistency)."""

import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import multigpu
from workloads import CONFIGS, make_fmha_inputs, shard


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


BASE = CONFIGS["bert_base_pad"].with_(batch=4, heads=2, seq_q=24, seq_kv=24)


def _shard_output(cfg, offset):
    """Stand-in for one rank's kernel: O of its shard, per (b, h) independent, rounded to fp16."""
    from oracle import attention_fp64
    q, k, v, kl = make_fmha_inputs(cfg, batch_offset=offset)
    return torch.from_numpy(attention_fp64(q, k, v, cfg.scale, kl)).half()


def _worker(rank, world, port, scaling, q_out):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from oracle import attention_rows_fp64
        cfg, off = shard(BASE, rank, world, scaling)
        o = _shard_output(cfg, off)
        o_full = multigpu.gather_output(o, world, dist)           # bench.py's reassembly
        tmax = multigpu.max_over_ranks(float(rank + 1) * 1.5, world, dist, "cpu")
        if rank == 0:
            glob = multigpu.global_config(BASE, world, scaling)
            o_one = _shard_output(glob, 0)                          # "the same problem on one GPU"
            gq, gk, gv, gkl = make_fmha_inputs(glob)
            units = [(0, 0, 0), (glob.batch - 1, 1, 23), (glob.batch // 2, 0, 5)]
            rows = attention_rows_fp64(gq, gk, gv, glob.scale, units, gkl)
            chk = multigpu.check_gathered(o_full, o_one, rows, units)
            q_out.put((o_full.numpy(), tmax, chk))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("scaling", ["weak", "strong"])
def test_two_rank_bench_gather_and_check(scaling):
    world = 2
    ctx = mp.get_context("spawn")
    q_out = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, scaling, q_out)) for r in range(world)]
    for p in procs:
        p.start()
    gathered, tmax, chk = q_out.get(timeout=120)
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    from oracle import attention_fp64
    glob = BASE.with_(batch=BASE.batch * world) if scaling == "weak" else BASE
    assert multigpu.global_config(BASE, world, scaling) == glob
    q, k, v, kl = make_fmha_inputs(glob)
    np.testing.assert_array_equal(gathered, attention_fp64(q, k, v, glob.scale, kl).astype(np.float16))
    assert chk["bitwise_equal_1gpu"] and chk["max_abs_diff_1gpu"] == 0.0
    assert chk["oracle_rows_max_err"] <= 1e-3  # fp16 rounding of the stand-in
    assert tmax == 3.0  # max over ranks, not rank 0's


def test_check_gathered_detects_a_wrong_shard():
    a = torch.zeros(4, 2, 3, 8, dtype=torch.float16)
    b = a.clone()
    b[3, 1, 2, 7] = 1.0
    chk = multigpu.check_gathered(a, b)
    assert not chk["bitwise_equal_1gpu"] and chk["max_abs_diff_1gpu"] == 1.0


def test_shard_rules():
    cfg = CONFIGS["gpt_causal"]
    assert shard(cfg, 3, 8, "weak") == (cfg, 3 * cfg.batch)
    c2, off = shard(cfg, 3, 8, "strong")
    assert c2.batch == 1 and off == 3
    with pytest.raises(ValueError):
        shard(cfg, 0, 3, "strong")
