"""Multi-GPU orchestration of bench.py's FMHA runs: shard, gather, check.

The path partitions by (batch x head): rank r of W owns a contiguous batch range (workloads.shard),
runs the kernel on it with no collective on the data path, and after the timed region ONE
all-gather reassembles O so rank 0 can check it:

  * bitwise against the same computation on one GPU (shard assignment must not change the per-(b, h)
    arithmetic -- SURVEY.md §8(e) "Check");
  * against the fp64 oracle on sampled rows (bench.py passes the oracle's row function in; this
    module does no attention arithmetic itself).

Scaling definitions:
  strong  the config as written is split over the W ranks (batch / W each); speedup = t_1 / max_r t_r
  weak    every rank runs the whole config on its own batch (global batch = W x batch)

Everything here works with any torch.distributed backend (NCCL on the GPU box, gloo in the CPU
tests), so tests/test_dist.py runs exactly this code at world size 2.
"""

from __future__ import annotations

import torch


def global_config(cfg, world: int, scaling: str):
    """The whole job's problem: the config itself (strong) or W copies of its batch (weak)."""
    if scaling == "strong":
        return cfg
    if scaling == "weak":
        return cfg.with_(batch=cfg.batch * world)
    raise ValueError(scaling)


def gather_output(o_local: torch.Tensor, world: int, dist) -> torch.Tensor:
    """All-gather every rank's O shard [b, ...] along the batch dimension -> the global O on every rank
    (one collective; ranks own equal, contiguous batch ranges, so concatenation is the global layout)."""
    if world == 1 or dist is None:
        return o_local
    o_local = o_local.contiguous()
    out = torch.empty((world * o_local.shape[0],) + tuple(o_local.shape[1:]), dtype=o_local.dtype,
                      device=o_local.device)
    try:
        dist.all_gather_into_tensor(out, o_local)
    except (RuntimeError, NotImplementedError, AttributeError):  # backends without the fused form
        parts = [torch.empty_like(o_local) for _ in range(world)]
        dist.all_gather(parts, o_local)
        out = torch.cat(parts)
    return out


def max_over_ranks(x: float, world: int, dist, device) -> float:
    """The job's time is the slowest rank's."""
    if world == 1 or dist is None:
        return x
    t = torch.tensor([x], dtype=torch.float64, device=device)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


def check_gathered(o_gathered: torch.Tensor, o_single: torch.Tensor, oracle_rows=None, units=None) -> dict:
    """Rank 0's check of the reassembled O: bitwise equality with the one-GPU O and, if given, the
    max |err| against oracle rows (units = [(b, h, i)], oracle_rows = float64 [len(units), D])."""
    a, b = o_gathered.detach().cpu(), o_single.detach().cpu()
    res = {"bitwise_equal_1gpu": bool(a.shape == b.shape and torch.equal(a, b)),
           "max_abs_diff_1gpu": float((a.double() - b.double()).abs().max()) if a.shape == b.shape else None,
           "gathered_bytes": int(a.numel() * a.element_size())}
    if oracle_rows is not None:
        got = torch.stack([a[bb, hh, ii].double() for bb, hh, ii in units]).numpy()
        res["oracle_rows"] = len(units)
        res["oracle_rows_max_err"] = float(abs(got - oracle_rows).max())
    return res
