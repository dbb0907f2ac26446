"""Multi-process (gloo, world size 2, CPU) checks of the multi-GPU partition used by bench.py:
per-rank shards of a config reproduce the global problem exactly, and the timing reduction is a
max over ranks.  The FMHA arithmetic here is the oracle's (the GPU path is covered by
test_fmha_gpu.py::test_determinism_and_shard_consistency)."""

import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from workloads import CONFIGS, make_fmha_inputs, shard


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _worker(rank, world, port, scaling, q_out):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from oracle import attention_fp64
        base = CONFIGS["bert_base_pad"].with_(batch=4, heads=2, seq_q=24, seq_kv=24)
        cfg, off = shard(base, rank, world, scaling)
        q, k, v, kl = make_fmha_inputs(cfg, batch_offset=off)
        o = torch.from_numpy(attention_fp64(q, k, v, cfg.scale, kl))
        parts = [torch.empty_like(o) for _ in range(world)]
        dist.all_gather(parts, o)
        t = torch.tensor([float(rank + 1) * 1.5])
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        if rank == 0:
            q_out.put((torch.cat(parts).numpy(), float(t.item())))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("scaling", ["weak", "strong"])
def test_two_rank_shards_reassemble_global_problem(scaling):
    world = 2
    ctx = mp.get_context("spawn")
    q_out = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, scaling, q_out)) for r in range(world)]
    for p in procs:
        p.start()
    gathered, tmax = q_out.get(timeout=120)
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    from oracle import attention_fp64
    base = CONFIGS["bert_base_pad"].with_(batch=4, heads=2, seq_q=24, seq_kv=24)
    glob = base.with_(batch=base.batch * world) if scaling == "weak" else base
    q, k, v, kl = make_fmha_inputs(glob)
    ref = attention_fp64(q, k, v, glob.scale, kl)
    np.testing.assert_array_equal(gathered, ref)
    assert tmax == 3.0  # max over ranks, not rank 0's


def test_shard_rules():
    cfg = CONFIGS["gpt_causal"]
    assert shard(cfg, 3, 8, "weak") == (cfg, 3 * cfg.batch)
    c2, off = shard(cfg, 3, 8, "strong")
    assert c2.batch == 1 and off == 3
    with pytest.raises(ValueError):
        shard(cfg, 0, 3, "strong")
