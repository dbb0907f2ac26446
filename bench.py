#!/usr/bin/env python
"""Benchmark: FMHA forward TFLOP/s at BERT-large shapes (BASELINE.json metric) on N GPUs.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference] [--workload NAME]

A step is one pass of the whole hot path (one fmha_fwd launch through the C ABI) over one batch
of the workload (default bert_large_512: B=32, H=16, S=512, D=64, fp16).  N > 1 runs under
torchrun, one process per GPU; the config's batch is split over the ranks by (batch x head) shards
(--scaling strong, the default; --scaling weak gives every rank its own full batch), with no
collective on the data path; value = all ranks' algorithmic flops / max-over-ranks device time.
After the timed region one all-gather reassembles O and rank 0 checks it bitwise against the same
problem on one GPU plus sampled fp64 oracle rows (multigpu.py).

Rank 0 prints ONE JSON line.  See DESIGN.md §6 for every field.
"""

from __future__ import annotations

import argparse
import json
import os
import statistics
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

from workloads import (CONFIGS, FUSED_MLP_CONFIGS, SPLITKV_CONFIGS, LAYER_CONFIGS, MASK_CAUSAL, MASK_KEY_PADDING, VARLEN_CONFIGS,  # noqa: E402
                       make_fmha_inputs, make_layer_inputs, make_varlen_inputs, shard)

METRIC = "FMHA fwd TFLOP/s & % of B200 fp16 tensor peak at BERT-large shapes, 1/2/4/8 GPU"
SPEC_TFLOPS = 2250.0
L2_BYTES = 126 * 1024 * 1024


def alg_flops(cfg, kv_len) -> float:
    """4*D per visible (query, key) pair — SURVEY §8(d); masked pairs are not counted."""
    b, h, sq, skv, d = cfg.batch, cfg.heads, cfg.seq_q, cfg.seq_kv, cfg.head_dim
    if cfg.mask == MASK_CAUSAL:
        off = skv - sq
        i = np.arange(sq)
        pairs = int(np.clip(np.minimum(skv, i + off + 1), 0, None).sum()) * b * h
    elif cfg.mask == MASK_KEY_PADDING:
        pairs = int(sum(sq * min(int(x), skv) for x in kv_len)) * h
    else:
        pairs = b * h * sq * skv
    return 4.0 * d * pairs


def alg_bytes(cfg) -> float:
    e = 2
    return float(e * cfg.batch * cfg.heads * cfg.head_dim * (2 * cfg.seq_q + 2 * cfg.seq_kv))


def measured_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return d["bf16_tflops"], d.get("bf16_tflops_sustained"), d["hbm_gbs"], "measured"
    return 1590.0, 1400.0, 6650.0, "fallback"


def fmha_roofline(achieved_tf, ai, ms_step, bytes_step, traffic, peak_tf, hbm_gbs, peak_src) -> dict:
    """Roofline of the dense FMHA kernel: arithmetic intensity AI = algorithmic flops /
    algorithmic bytes (Q + K + V + O).  Below the measured ridge (peak TFLOP/s / HBM GB/s, ~258 flop/B)
    the bound is HBM and the line reports GB/s against the measured copy bandwidth (BERT-base padded,
    AI <= 64; BERT-large-384, AI 192); at or above it (BERT-large-512, AI 256 -- 1% below the ridge,
    where the two roofs coincide within 1%; GPT causal) the tensor peak."""
    kernel = "fmha_fwd_kernel"
    if ai * hbm_gbs / 1e3 < 0.97 * peak_tf:
        gbs = bytes_step / (ms_step * 1e-3) / 1e9
        return {"bound": "hbm", "achieved": round(gbs, 1), "peak": hbm_gbs, "unit": "GB/s",
                "frac": round(gbs / hbm_gbs, 4), "traffic": traffic, "arith_intensity": round(ai, 1),
                "peak_source": f"{peak_src} HBM copy bandwidth", "kernel": kernel,
                "tensor_frac": round(achieved_tf / peak_tf, 4)}
    return {"bound": "tensor", "achieved": round(achieved_tf, 2), "peak": peak_tf, "unit": "TFLOP/s",
            "frac": round(achieved_tf / peak_tf, 4), "traffic": traffic, "arith_intensity": round(ai, 1),
            "peak_source": f"{peak_src} bf16 dense burst (fp16 = bf16 rate)", "kernel": kernel}


class ClockSampler:
    """Samples SM clock and throttle reasons through NVML while the timed region runs."""

    REASONS = {
        "gpu_idle": 0x1, "applications_clocks_setting": 0x2, "sw_power_cap": 0x4, "hw_slowdown": 0x8,
        "sync_boost": 0x10, "sw_thermal_slowdown": 0x20, "hw_thermal_slowdown": 0x40,
        "hw_power_brake_slowdown": 0x80, "display_clock_setting": 0x100,
    }

    def __init__(self, index: int):
        self.samples, self.reasons, self.ok = [], set(), False
        self._stop = threading.Event()
        try:
            import pynvml
            pynvml.nvmlInit()
            self.nv = pynvml
            self.h = pynvml.nvmlDeviceGetHandleByIndex(index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
            self.ok = True
        except Exception:
            self.max_mhz = None

    def _run(self):
        while not self._stop.is_set():
            try:
                self.samples.append(self.nv.nvmlDeviceGetClockInfo(self.h, self.nv.NVML_CLOCK_SM))
                r = self.nv.nvmlDeviceGetCurrentClocksThrottleReasons(self.h)
                for k, bit in self.REASONS.items():
                    if r & bit and k != "gpu_idle":
                        self.reasons.add(k)
            except Exception:
                pass
            time.sleep(0.0005)

    def __enter__(self):
        if self.ok:
            self.t = threading.Thread(target=self._run, daemon=True)
            self.t.start()
        return self

    def __exit__(self, *a):
        if self.ok:
            self._stop.set()
            self.t.join()

    def summary(self):
        if not self.samples:
            return {"sm_mhz": None, "sm_max_mhz": self.max_mhz, "reasons": sorted(self.reasons), "samples": 0}
        return {"sm_mhz": statistics.median(self.samples), "sm_max_mhz": self.max_mhz,
                "reasons": sorted(self.reasons), "samples": len(self.samples)}


def exp_roofline(pairs: float, ms_step: float, sampler) -> dict:
    """Second roofline for the FMHA kernel: one exponential per visible (query, key)
    pair against the MUFU ex2 rate, 16 per clock per SM (B300_MICROARCH / profiles/ubench.txt) x 148
    SMs x the SM clock sampled during the timed region.  At D = 64 this unit, not the tensor core,
    bounds the kernel; 2 of every 8 exp2 pairs run as FMA-pipe polynomials, so frac may exceed 1."""
    mhz = (sampler.summary() or {}).get("sm_mhz") or 1965
    peak = 148 * 16 * mhz * 1e6
    achieved = pairs / (ms_step * 1e-3)
    return {"bound": "alu", "unit": "Gexp/s", "achieved": round(achieved / 1e9, 1), "peak": round(peak / 1e9, 1),
            "frac": round(achieved / peak, 4),
            "peak_source": "MUFU.EX2 16/clk/SM x 148 SMs x sampled SM clock (derived, DESIGN.md §6)"}


def cpu_oracle_sample(cfg, q, k, v, kv_len, budget_s: float):
    """Times the CPU oracle (as it stands) on whole (b,h) units of this workload until ~budget_s."""
    from oracle import attention_fp64
    try:
        from threadpoolctl import threadpool_info
        cores = max([t.get("num_threads", 1) for t in threadpool_info()] or [1])
    except Exception:
        cores = os.cpu_count()
    done_flops, units, t0 = 0.0, 0, time.perf_counter()
    causal = cfg.mask == MASK_CAUSAL
    while True:
        b, h = divmod(units % cfg.units, cfg.heads)
        kl = None if kv_len is None else [int(kv_len[b])]
        attention_fp64(q[b:b + 1, h:h + 1], k[b:b + 1, h:h + 1], v[b:b + 1, h:h + 1], cfg.scale, kl, causal)
        done_flops += alg_flops(cfg.with_(batch=1, heads=1), kl)
        units += 1
        el = time.perf_counter() - t0
        if el >= budget_s:
            break
    return {"value": done_flops / el / 1e12, "unit": "TFLOP/s", "cores": int(cores), "kind": "oracle",
            "sample": f"{units} (b,h) units (cycling over the {cfg.units} of {cfg.name}), numpy fp64, {el:.1f} s"}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=50)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", choices=["ours", "reference"], default="ours")
    ap.add_argument("--workload", default="bert_large_512", choices=sorted(CONFIGS) + sorted(VARLEN_CONFIGS) + sorted(LAYER_CONFIGS) + ["mlp", "lstm_cell"] + sorted(FUSED_MLP_CONFIGS) + sorted(SPLITKV_CONFIGS))
    ap.add_argument("--cpu-budget", type=float, default=15.0, help="seconds of CPU oracle timing")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--sustained", type=float, default=1.0,
                    help="seconds of back-to-back replays of the timed graph for the sustained-clock variant (0: off)")
    ap.add_argument("--stream-k", choices=["auto", "on", "off"], default="auto",
                    help="FMHA workloads: time fmha_fwd_streamk (the last partial round split along the keys, "
                         "merged in the kernel) instead of fmha_fwd; auto = when its plan splits and N = 1")
    ap.add_argument("--scaling", choices=["weak", "strong"], default="strong",
                    help="strong: ranks split the config's batch (SURVEY §8(e)); weak: each rank runs the whole config on its own batch")
    args = ap.parse_args()
    args.warmup = max(args.warmup, 3)

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if args.workload == "mlp":
        return run_mlp(args, world, rank, local)
    if args.workload == "lstm_cell":
        return run_lstm(args, world, rank, local)
    if args.workload in FUSED_MLP_CONFIGS:
        return run_mlp_fused(args, world, rank, local)
    if args.workload in SPLITKV_CONFIGS:
        return run_splitkv(args, world, rank, local)
    if args.workload in VARLEN_CONFIGS:
        return run_varlen(args, world, rank, local)
    if args.workload in LAYER_CONFIGS:
        return run_layer(args, world, rank, local)
    cfg = CONFIGS[args.workload]

    if args.impl == "reference":
        return run_reference(args, cfg, world, rank)

    # B200_BENCH_ONE_DEVICE=1 (testing only): every rank on cuda:0 with gloo collectives, so the
    # world > 1 path (sharding, max-over-ranks timing, the O all-gather and its check) runs on a
    # one-GPU box; the ranks then share one GPU, so its numbers are not scaling measurements.
    one_dev = os.environ.get("B200_BENCH_ONE_DEVICE") == "1"
    if one_dev:
        local = 0
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    dist = None
    if world > 1:
        import torch.distributed as dist
        if one_dev:
            dist.init_process_group("gloo")
        else:
            dist.init_process_group("nccl", device_id=dev)

    import paper_conf_asplos_hagedornfccgg23_b200 as fm
    import multigpu

    cfg_global = multigpu.global_config(cfg, world, args.scaling)
    cfg, offset = shard(cfg, rank, world, args.scaling)  # weak: own batch; strong: a slice of it
    q, k, v, kv_len = make_fmha_inputs(cfg, batch_offset=offset)
    set_bytes = alg_bytes(cfg)
    n_sets = max(1, int(np.ceil(3 * L2_BYTES / set_bytes)))  # rotate > 3x L2 of inputs+outputs
    qd, kd, vd = q.to(dev), k.to(dev), v.to(dev)
    sets = [(qd, kd, vd, torch.empty_like(qd))] + [
        (qd.clone(), kd.clone(), vd.clone(), torch.empty_like(qd)) for _ in range(n_sets - 1)]
    kl_dev = None if kv_len is None else torch.from_numpy(kv_len).to(dev)
    causal = cfg.mask == MASK_CAUSAL
    stream = torch.cuda.current_stream(dev)

    # stream-K tail: one launch of fmha_fwd_streamk when its plan splits the last round
    sms = torch.cuda.get_device_properties(dev).multi_processor_count
    sk_plan = fm.streamk_plan(cfg.batch, cfg.heads, cfg.seq_q, cfg.seq_kv, sms, cfg.mask)
    use_sk = args.stream_k == "on" or (args.stream_k == "auto" and world == 1 and sk_plan[0] > 1)
    sk_ws = fm.streamk_workspace(dev, cfg.head_dim) if use_sk else None

    def step(i):
        s = sets[i % n_sets]
        if use_sk:
            fm.fmha_fwd_streamk(s[0], s[1], s[2], kv_len=kl_dev, causal=causal, scale=cfg.scale, out=s[3],
                                workspace=sk_ws)
        else:
            fm.fmha_fwd(s[0], s[1], s[2], kv_len=kl_dev, causal=causal, scale=cfg.scale, out=s[3])

    for i in range(args.warmup):
        step(i)
    torch.cuda.synchronize()
    # The K timed steps are captured once into a CUDA graph (K kernel launches, rotating input sets)
    # so host-side launch overhead cannot starve a ~tens-of-microseconds kernel.  One untimed replay
    # uploads the graph before the timed replay.
    graph = torch.cuda.CUDAGraph()
    with torch.cuda.graph(graph):
        for i in range(args.steps):
            step(i)
    # (the NVML sampler is initialised before the upload replay, so the device is not left idle for the
    # NVML start-up between that replay and the timed one: an idle gap costs the first launches after it
    # a few % -- DESIGN.md §7)
    sampler = ClockSampler(local)
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    graph.replay()
    torch.cuda.synchronize()
    with sampler:
        if dist:
            dist.barrier()
        torch.cuda.synchronize()
        lead_in(stream)
        for _ in range(int(os.environ.get("B200_BENCH_WARM_REPLAYS", "0"))):  # (A/B of device warm-up)
            graph.replay()
        ev0.record(stream)
        graph.replay()
        ev1.record(stream)
        torch.cuda.synchronize()
        if dist:
            dist.barrier()
    ms = multigpu.max_over_ranks(ev0.elapsed_time(ev1), world, dist, "cpu" if one_dev else dev)
    flops_rank = alg_flops(cfg, kv_len)
    ms_step = ms / args.steps
    value = flops_rank * world / (ms_step * 1e-3) / 1e12

    # ---- sustained-clock variant: the same graph replayed back to back for >= args.sustained seconds
    # (a seconds-long job runs at the power-capped clock, not the burst clock of a ~1 ms region)
    sustained = None
    if args.sustained > 0:
        reps = max(1, int(np.ceil(args.sustained * 1e3 / max(ms, 1e-3))))
        ssampler = ClockSampler(local)
        s0, s1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        with ssampler:
            if dist:
                dist.barrier()
            torch.cuda.synchronize()
            lead_in(stream)
            s0.record(stream)
            for _ in range(reps):
                graph.replay()
            s1.record(stream)
            torch.cuda.synchronize()
        sus_ms = multigpu.max_over_ranks(s0.elapsed_time(s1), world, dist, "cpu" if one_dev else dev)
        sms_step = sus_ms / (reps * args.steps)
        sustained = {"value": round(flops_rank * world / (sms_step * 1e-3) / 1e12, 2), "unit": "TFLOP/s",
                     "ms_per_step": round(sms_step, 5), "steps": reps * args.steps, "seconds": round(sus_ms / 1e3, 3),
                     "clocks": ssampler.summary()}

    # ---- end to end through the C ABI with pinned HOST buffers (copies inside the timed region)
    e2e = None
    if not args.no_e2e:
        pq, pk, pv = q.pin_memory(), k.pin_memory(), v.pin_memory()
        po = torch.empty_like(pq).pin_memory()
        ws = torch.empty(fm.workspace_bytes(cfg.batch, cfg.heads, cfg.seq_q, cfg.seq_kv, cfg.head_dim),
                         dtype=torch.uint8, device=dev)
        klh = None if kv_len is None else torch.from_numpy(kv_len).pin_memory()
        e2e_steps = max(3, min(args.steps, 20))
        for _ in range(2):
            fm.fmha_fwd_from_host(pq, pk, pv, po, ws, kv_len=klh, causal=causal, scale=cfg.scale, stream=stream)
        torch.cuda.synchronize()
        if dist:
            dist.barrier()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        for _ in range(e2e_steps):
            fm.fmha_fwd_from_host(pq, pk, pv, po, ws, kv_len=klh, causal=causal, scale=cfg.scale, stream=stream)
        e1.record(stream)
        torch.cuda.synchronize()
        ems = multigpu.max_over_ranks(e0.elapsed_time(e1), world, dist, "cpu" if one_dev else dev)
        in_bytes = (pq.numel() + pk.numel() + pv.numel()) * pq.element_size() + (0 if klh is None else klh.numel() * 4)
        e2e = {"value": flops_rank * world / (ems / e2e_steps * 1e-3) / 1e12, "unit": "TFLOP/s",
               "h2d_bytes_per_step": int(in_bytes), "d2h_bytes_per_step": int(po.numel() * po.element_size()),
               "ms_per_step": ems / e2e_steps}

    # ---- check this rank's last output against sampled oracle rows (cheap sanity, not timed)
    from oracle import attention_rows_fp64
    units = [(0, 0, 0), (cfg.batch - 1, cfg.heads - 1, cfg.seq_q - 1),
             (cfg.batch // 2, min(1, cfg.heads - 1), cfg.seq_q // 3)]
    ref = attention_rows_fp64(q, k, v, cfg.scale, units, kv_len, causal)
    o_last = sets[(args.steps - 1) % n_sets][3]
    got = np.stack([o_last[b, h, i].double().cpu().numpy() for b, h, i in units])
    check_err = float(np.abs(got - ref).max())

    # ---- N > 1: one all-gather reassembles O (untimed); rank 0 checks it bitwise against the whole
    # problem on one GPU and against oracle rows spread over every rank's shard
    mgpu = None
    if world > 1:
        o_full = multigpu.gather_output(o_last.cpu() if one_dev else o_last, world, dist)
        if rank == 0:
            gq, gk, gv, gkl = make_fmha_inputs(cfg_global)
            gkl_dev = None if gkl is None else torch.from_numpy(gkl).to(dev)
            o_one = fm.fmha_fwd(gq.to(dev), gk.to(dev), gv.to(dev), kv_len=gkl_dev, causal=causal, scale=cfg.scale)
            torch.cuda.synchronize()
            gb = cfg_global.batch
            gunits = [(r * gb // world + (r % 2) * (gb // world - 1), r % cfg.heads, (37 * r) % cfg.seq_q)
                      for r in range(world)] + [(gb - 1, cfg.heads - 1, cfg.seq_q - 1)]
            gref = attention_rows_fp64(gq, gk, gv, cfg.scale, gunits, gkl, causal)
            mgpu = multigpu.check_gathered(o_full, o_one, gref, gunits)
            mgpu["collective"] = "all_gather_into_tensor (after the timed region)"
            del gq, gk, gv, o_one

    peak_burst, peak_sust, hbm, peak_src = measured_peaks()
    if dist:
        dist.barrier()
    if rank == 0:
        cpu = None
        if world == 1 and not args.no_cpu_baseline:
            cpu = cpu_oracle_sample(cfg, q, k, v, kv_len, args.cpu_budget)
        traffic = None
        tp = os.path.join(ROOT, "profiles", "traffic.json")
        if os.path.exists(tp):
            traffic = json.load(open(tp)).get(cfg.name)
        achieved = flops_rank / (ms_step * 1e-3) / 1e12  # per-GPU kernel throughput (1 launch / step)
        line = {
            "metric": METRIC, "value": round(value, 2), "unit": "TFLOP/s", "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(ms_step, 5),
            "higher_is_better": True, "scaling": args.scaling, "vs_baseline": None,
            "dtype": "f16" if cfg.dtype == "fp16" else "bf16", "data": "synthetic",
            "config": {"workload": cfg.name, "batch_per_gpu": cfg.batch, "heads": cfg.heads, "seq_q": cfg.seq_q,
                       "seq_kv": cfg.seq_kv, "head_dim": cfg.head_dim,
                       "mask": ["none", "key_padding", "causal"][cfg.mask], "parallelism": f"{args.scaling} dp{world} (b x h shards)",
                       "kernel": (f"fmha_fwd_streamk (last round: {sk_plan[1]} items x {sk_plan[0]} key pieces)"
                                  if use_sk else "fmha_fwd"),
                       "l2": f"rotating {n_sets} input/output sets ({n_sets * set_bytes / 1e6:.0f} MB > 126 MB L2)"},
            "pct_of_spec_2250": round(100 * achieved / SPEC_TFLOPS, 2),
            "pct_of_measured_peak": round(100 * achieved / peak_burst, 2),
            "achieved_gbs": round(alg_bytes(cfg) / (ms_step * 1e-3) / 1e9, 1),
            "clocks": sampler.summary(),
            "e2e": e2e,
            "gpu_launches": args.steps,
            "roofline": fmha_roofline(achieved, flops_rank / alg_bytes(cfg), ms_step, alg_bytes(cfg),
                                      traffic, peak_burst, hbm, peak_src),
            "roofline_exp": exp_roofline(alg_flops(cfg, kv_len) / (4.0 * cfg.head_dim), ms_step, sampler),
            "cpu_baseline": cpu,
            "check_max_abs_err": check_err,
            "multi_gpu_check": mgpu,
        }
        if sustained is not None:
            ach = flops_rank / (sustained["ms_per_step"] * 1e-3) / 1e12
            sustained["roofline"] = {"bound": "tensor", "achieved": round(ach, 2), "peak": peak_sust,
                                     "frac": round(ach / peak_sust, 4) if peak_sust else None,
                                     "peak_source": "measured bf16 dense sustained (MEASURED_PEAKS.json)"}
            line["sustained"] = sustained
        if world > 1:
            line["config"]["global_batch"] = cfg_global.batch
        print(json.dumps(line), flush=True)
    if dist:
        dist.destroy_process_group()


def run_mlp(args, world, rank, local):
    """BASELINE.json config 5: Transformer MLP block, tokens=16384, 1024 -> 4096 (+bias, GELU) -> 1024
    (+bias), fp16, two gemm_bias_act launches per step."""
    from workloads import MLP_CONFIG, make_mlp_inputs
    import paper_conf_asplos_hagedornfccgg23_b200 as fm
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    cfg = MLP_CONFIG
    x, w1, b1, w2, b2 = (t.to(dev) for t in make_mlp_inputs(cfg))
    h = torch.empty((cfg.tokens, cfg.d_ff), dtype=torch.float16, device=dev)
    y = torch.empty((cfg.tokens, cfg.d_model), dtype=torch.float16, device=dev)

    def step():
        fm.gemm_bias_act(x, w1, b1, act="gelu", out=h)
        fm.gemm_bias_act(h, w2, b2, act="none", out=y)

    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()
    graph = torch.cuda.CUDAGraph()
    with torch.cuda.graph(graph):
        for _ in range(args.steps):
            step()
    stream = torch.cuda.current_stream(dev)
    sampler = ClockSampler(local)  # (before the upload replay: no idle NVML start-up gap before timing)
    graph.replay()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with sampler:
        torch.cuda.synchronize()
        lead_in(stream)
        e0.record(stream)
        graph.replay()
        e1.record(stream)
        torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / args.steps
    flops = 2.0 * cfg.tokens * cfg.d_model * cfg.d_ff * 2
    peak_burst, _, _, src = measured_peaks()
    val = flops / (ms * 1e-3) / 1e12
    if rank == 0:
        print(json.dumps({"metric": "MLP block (GEMM+bias+GELU, GEMM+bias) TFLOP/s", "value": round(val, 2),
                          "unit": "TFLOP/s", "n_gpus": 1, "steps": args.steps, "warmup": args.warmup,
                          "ms_per_step": round(ms, 5), "higher_is_better": True, "dtype": "f16", "data": "synthetic",
                          "config": {"workload": "mlp", "tokens": cfg.tokens, "d_model": cfg.d_model, "d_ff": cfg.d_ff},
                          "clocks": sampler.summary(), "gpu_launches": 2 * args.steps,
                          "roofline": {"bound": "tensor", "achieved": round(val, 2), "peak": peak_burst,
                                       "unit": "TFLOP/s", "frac": round(val / peak_burst, 4),
                                       "peak_source": f"{src} bf16 dense burst"}}), flush=True)


def varlen_flops(lens, heads, d, causal) -> float:
    pairs = sum(int(n) * (int(n) + 1) // 2 if causal else int(n) * int(n) for n in lens)
    return 4.0 * d * heads * pairs


def run_varlen(args, world, rank, local):
    """packed variable-length MLPerf-style batch through fmha_fwd_varlen.  Weak
    scaling: rank r processes its own batch of sequences (global sequence index offset r * n)."""
    import paper_conf_asplos_hagedornfccgg23_b200 as fm
    cfg = VARLEN_CONFIGS[args.workload]
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    dist = None
    if world > 1:
        import torch.distributed as dist
        dist.init_process_group("nccl", device_id=dev)
    x, cu = make_varlen_inputs(cfg, seq_offset=rank * cfg.num_seqs)
    lens = np.diff(cu)
    set_bytes = 2.0 * x.numel() * 4 / 3  # Q, K, V in + O out
    n_sets = max(1, int(np.ceil(3 * L2_BYTES / set_bytes)))
    xd = x.to(dev)
    cud = torch.from_numpy(cu).to(dev)
    sets = [(xd if i == 0 else xd.clone(), torch.empty((x.shape[0], cfg.heads, cfg.head_dim), dtype=x.dtype,
                                                       device=dev)) for i in range(n_sets)]

    def step(i):
        s = sets[i % n_sets]
        fm.fmha_fwd_varlen(s[0], cud, cfg.max_seqlen, causal=cfg.causal, scale=cfg.scale, out=s[1])

    for i in range(args.warmup):
        step(i)
    torch.cuda.synchronize()
    graph = torch.cuda.CUDAGraph()
    with torch.cuda.graph(graph):
        for i in range(args.steps):
            step(i)
    stream = torch.cuda.current_stream(dev)
    sampler = ClockSampler(local)  # (before the upload replay: no idle NVML start-up gap before timing)
    graph.replay()
    torch.cuda.synchronize()
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with sampler:
        if dist:
            dist.barrier()
        torch.cuda.synchronize()
        lead_in(stream)
        ev0.record(stream)
        graph.replay()
        ev1.record(stream)
        torch.cuda.synchronize()
        if dist:
            dist.barrier()
    ms = ev0.elapsed_time(ev1)
    if dist:
        t = torch.tensor([ms], device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ms = float(t.item())
    ms_step = ms / args.steps
    flops_rank = varlen_flops(lens, cfg.heads, cfg.head_dim, cfg.causal)
    value = flops_rank * world / (ms_step * 1e-3) / 1e12

    e2e = None
    if not args.no_e2e:  # pinned host QKV + cu_seqlens -> device, kernel, O -> pinned host, one stream
        hx, hcu = x.pin_memory(), torch.from_numpy(cu).pin_memory()
        ho = torch.empty((x.shape[0], cfg.heads, cfg.head_dim), dtype=x.dtype).pin_memory()
        dx, dcu, do = torch.empty_like(xd), torch.empty_like(cud), torch.empty_like(sets[0][1])

        def e2e_step():
            dx.copy_(hx, non_blocking=True)
            dcu.copy_(hcu, non_blocking=True)
            fm.fmha_fwd_varlen(dx, dcu, cfg.max_seqlen, causal=cfg.causal, scale=cfg.scale, out=do)
            ho.copy_(do, non_blocking=True)
        for _ in range(2):
            e2e_step()
        torch.cuda.synchronize()
        n = max(3, min(args.steps, 20))
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        for _ in range(n):
            e2e_step()
        e1.record(stream)
        torch.cuda.synchronize()
        ems = e0.elapsed_time(e1)
        if dist:
            t = torch.tensor([ems], device=dev)
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            ems = float(t.item())
        e2e = {"value": flops_rank * world / (ems / n * 1e-3) / 1e12, "unit": "TFLOP/s",
               "h2d_bytes_per_step": int(hx.numel() * hx.element_size() + hcu.numel() * 4),
               "d2h_bytes_per_step": int(ho.numel() * ho.element_size()), "ms_per_step": ems / n}

    # sampled check of this rank's output against the oracle (three whole sequences)
    from oracle import attention_varlen_fp64
    o_last = sets[(args.steps - 1) % n_sets][1]
    err = 0.0
    for s_ in (0, len(lens) // 2, len(lens) - 1):
        a, b = int(cu[s_]), int(cu[s_ + 1])
        ref = attention_varlen_fp64(x[a:b], np.array([0, b - a]), cfg.scale, cfg.causal)
        err = max(err, float(np.abs(o_last[a:b].double().cpu().numpy() - ref).max()))
    peak_burst, _, hbm, peak_src = measured_peaks()
    if dist:
        dist.barrier()
    if rank == 0:
        cpu = None
        if world == 1 and not args.no_cpu_baseline:
            t0, done, k = time.perf_counter(), 0.0, 0
            while time.perf_counter() - t0 < args.cpu_budget:
                s_ = k % len(lens)
                a, b = int(cu[s_]), int(cu[s_ + 1])
                attention_varlen_fp64(x[a:b], np.array([0, b - a]), cfg.scale, cfg.causal)
                done += varlen_flops([b - a], cfg.heads, cfg.head_dim, cfg.causal)
                k += 1
            el = time.perf_counter() - t0
            cpu = {"value": done / el / 1e12, "unit": "TFLOP/s", "cores": os.cpu_count(), "kind": "oracle",
                   "sample": f"{k} whole sequences (all heads) of {cfg.name}, numpy fp64, {el:.1f} s"}
        achieved = flops_rank / (ms_step * 1e-3) / 1e12
        vl_bytes = 4.0 * int(cu[-1]) * cfg.heads * cfg.head_dim * 2  # packed Q, K, V read + O written
        line = {
            "metric": METRIC, "value": round(value, 2), "unit": "TFLOP/s", "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(ms_step, 5),
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None,
            "dtype": "f16" if cfg.dtype == "fp16" else "bf16", "data": "synthetic",
            "config": {"workload": cfg.name, "num_seqs_per_gpu": cfg.num_seqs, "tokens_per_gpu": int(cu[-1]),
                       "heads": cfg.heads, "max_seqlen": cfg.max_seqlen, "mean_seqlen": float(lens.mean()),
                       "head_dim": cfg.head_dim, "layout": "packed QKV [T,3,H,D] + cu_seqlens",
                       "causal": cfg.causal, "parallelism": f"dp{world} (sequence shards)",
                       "l2": f"rotating {n_sets} input/output sets ({n_sets * set_bytes / 1e6:.0f} MB > 126 MB L2)"},
            "pct_of_spec_2250": round(100 * achieved / SPEC_TFLOPS, 2),
            "clocks": sampler.summary(), "e2e": e2e, "gpu_launches": args.steps,
            "roofline": dict(fmha_roofline(achieved, flops_rank / vl_bytes, ms_step, vl_bytes, None, peak_burst, hbm,
                                           peak_src), kernel="fmha_fwd_kernel (varlen)"),
            "cpu_baseline": cpu, "check_max_abs_err": err,
        }
        print(json.dumps(line), flush=True)
    if dist:
        dist.destroy_process_group()


def traffic_for(name):
    """ncu DRAM bytes per launch of the workload's dominant kernel (profiles/traffic.json) or None."""
    tp = os.path.join(ROOT, "profiles", "traffic.json")
    try:
        return json.load(open(tp)).get(name)
    except Exception:
        return None


def lead_in(stream):
    """Keep the stream busy (a ~0.3 ms device spin) while the host enqueues the timed graph replay, so
    the start event is not followed by an idle gap of host-side graph-launch latency.  The spin runs
    before the start event, outside the timed region.  (The per-step time still falls with K -- 54.9 us
    at K = 10, 50.4 at K = 200 on BERT-large-512, profiles/r02c_ksweep_leadin.txt, 55.5 / 50.4 without
    the spin, r02c_ksweep.txt -- so that K dependence is device-side, not launch latency.)"""
    with torch.cuda.stream(stream):
        torch.cuda._sleep(600_000)


def _time_graph(fn, steps, stream):
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g):
        for _ in range(steps):
            fn()
    g.replay()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    lead_in(stream)
    e0.record(stream)
    g.replay()
    e1.record(stream)
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / steps


def run_layer(args, world, rank, local):
    """the synthetic Transformer layer (QKV GEMM -> varlen FMHA -> out GEMM -> MLP) as
    one transformer_layer_fwd call per step; the same layer composed from torch ops (cuBLAS linear,
    SDPA, GELU) is timed beside it as context.  Weak scaling over ranks (own batch per rank)."""
    import torch.nn.functional as F
    import paper_conf_asplos_hagedornfccgg23_b200 as fm
    cfg = LAYER_CONFIGS[args.workload]
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    dist = None
    if world > 1:
        import torch.distributed as dist
        dist.init_process_group("nccl", device_id=dev)
    tensors, cu = make_layer_inputs(cfg)
    x, wqkv, bqkv, wo, bo, w1, b1, w2, b2 = (t.to(dev) for t in tensors)
    cud = torch.from_numpy(cu).to(dev)
    t_, d, f = x.shape[0], cfg.d_model, cfg.d_ff
    lens = np.diff(cu)
    y = torch.empty((t_, d), dtype=torch.float16, device=dev)
    ws = torch.empty(fm.layer_workspace_bytes(t_, d, f), dtype=torch.uint8, device=dev)
    maxlen = int(lens.max())

    def step():
        fm.transformer_layer(x, wqkv, bqkv, wo, bo, w1, b1, w2, b2, cud, maxlen, cfg.heads, causal=cfg.causal,
                             scale=cfg.scale, out=y, workspace=ws)

    attn_flops = varlen_flops(lens, cfg.heads, cfg.head_dim, cfg.causal)
    gemm_flops = 2.0 * t_ * d * (3 * d + d + 2 * f)
    flops = attn_flops + gemm_flops
    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()
    stream = torch.cuda.current_stream(dev)
    graph = torch.cuda.CUDAGraph()
    with torch.cuda.graph(graph):
        for _ in range(args.steps):
            step()
    sampler = ClockSampler(local)  # (before the upload replay: no idle NVML start-up gap before timing)
    graph.replay()
    torch.cuda.synchronize()
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with sampler:
        if dist:
            dist.barrier()
        torch.cuda.synchronize()
        lead_in(stream)
        ev0.record(stream)
        graph.replay()
        ev1.record(stream)
        torch.cuda.synchronize()
        if dist:
            dist.barrier()
    ms = ev0.elapsed_time(ev1)
    if dist:
        tt = torch.tensor([ms], device=dev)
        dist.all_reduce(tt, op=dist.ReduceOp.MAX)
        ms = float(tt.item())
    ms_step = ms / args.steps
    value = flops * world / (ms_step * 1e-3) / 1e12

    # per-stage device times (each stage alone, same stream, CUDA graph of `steps` launches)
    qkv = ws[: t_ * 3 * d * 2].view(torch.float16).view(t_, 3 * d)
    a = torch.empty((t_, d), dtype=torch.float16, device=dev)
    z = torch.empty_like(a)
    h = torch.empty((t_, f), dtype=torch.float16, device=dev)
    fm.gemm_bias_act(x, wqkv, bqkv, out=qkv)
    stages = {
        "qkv_gemm": lambda: fm.gemm_bias_act(x, wqkv, bqkv, out=qkv),
        "fmha_varlen": lambda: fm.fmha_fwd_varlen(qkv.view(t_, 3, cfg.heads, cfg.head_dim), cud, maxlen,
                                                  causal=cfg.causal, scale=cfg.scale, out=a.view(t_, cfg.heads, -1)),
        "out_gemm": lambda: fm.gemm_bias_act(a, wo, bo, out=z),
        "mlp_gemm1_gelu": lambda: fm.gemm_bias_act(z, w1, b1, act="gelu", out=h),
        "mlp_gemm2": lambda: fm.gemm_bias_act(h, w2, b2, out=y),
    }
    stage_ms = {k: round(_time_graph(fn, args.steps, stream), 5) for k, fn in stages.items()}

    # context: the same layer from torch ops (cuBLAS GEMMs, SDPA, GELU) on the same device
    def torch_layer():
        q_ = F.linear(x, wqkv, bqkv).view(cfg.num_seqs, cfg.seq_len, 3, cfg.heads, cfg.head_dim)
        qh, kh, vh = (q_[:, :, i].transpose(1, 2) for i in range(3))
        o_ = F.scaled_dot_product_attention(qh, kh, vh, is_causal=cfg.causal, scale=cfg.scale)
        z_ = F.linear(o_.transpose(1, 2).reshape(t_, d), wo, bo)
        return F.linear(F.gelu(F.linear(z_, w1, b1)), w2, b2)
    torch_ms = None
    if all(int(n) == cfg.seq_len for n in lens):
        for _ in range(3):
            torch_layer()
        torch.cuda.synchronize()
        torch_ms = _time_graph(torch_layer, args.steps, stream)

    e2e = None
    if not args.no_e2e:  # pinned host X -> device, layer, Y -> pinned host (weights stay resident)
        hx = tensors[0].pin_memory()
        hy = torch.empty((t_, d), dtype=torch.float16).pin_memory()
        dx = torch.empty_like(x)

        def e2e_step():
            dx.copy_(hx, non_blocking=True)
            fm.transformer_layer(dx, wqkv, bqkv, wo, bo, w1, b1, w2, b2, cud, maxlen, cfg.heads,
                                 causal=cfg.causal, scale=cfg.scale, out=y, workspace=ws)
            hy.copy_(y, non_blocking=True)
        for _ in range(2):
            e2e_step()
        torch.cuda.synchronize()
        n = max(3, min(args.steps, 20))
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        for _ in range(n):
            e2e_step()
        e1.record(stream)
        torch.cuda.synchronize()
        ems = e0.elapsed_time(e1) / n
        e2e = {"value": flops * world / (ems * 1e-3) / 1e12, "unit": "TFLOP/s",
               "h2d_bytes_per_step": int(hx.numel() * 2), "d2h_bytes_per_step": int(hy.numel() * 2),
               "ms_per_step": ems}

    # sampled check: the last sequence against the oracle
    from oracle import transformer_layer_fp64
    step()
    torch.cuda.synchronize()
    lo, hi = int(cu[-2]), int(cu[-1])
    ref = transformer_layer_fp64(tensors[0][lo:hi], *tensors[1:], np.array([0, hi - lo]), cfg.heads, cfg.scale,
                                 cfg.causal)
    err = float(np.abs(y[lo:hi].double().cpu().numpy() - ref).max())
    peak_burst, _, _, peak_src = measured_peaks()
    if dist:
        dist.barrier()
    if rank == 0:
        cpu = None
        if world == 1 and not args.no_cpu_baseline:
            t0, done, k = time.perf_counter(), 0.0, 0
            while time.perf_counter() - t0 < args.cpu_budget:
                transformer_layer_fp64(tensors[0][lo:hi], *tensors[1:], np.array([0, hi - lo]), cfg.heads,
                                       cfg.scale, cfg.causal)
                n_ = hi - lo
                done += varlen_flops([n_], cfg.heads, cfg.head_dim, cfg.causal) + 2.0 * n_ * d * (4 * d + 2 * f)
                k += 1
            el = time.perf_counter() - t0
            cpu = {"value": done / el / 1e12, "unit": "TFLOP/s", "cores": os.cpu_count(), "kind": "oracle",
                   "sample": f"{k} x one {hi - lo}-token sequence through the whole layer, numpy fp64, {el:.1f} s"}
        line = {
            "metric": "Transformer layer (QKV GEMM, FMHA, out GEMM, MLP) TFLOP/s", "value": round(value, 2),
            "unit": "TFLOP/s", "n_gpus": world, "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": round(ms_step, 5), "higher_is_better": True, "scaling": "weak", "vs_baseline": None,
            "dtype": "f16", "data": "synthetic",
            "config": {"workload": cfg.name, "tokens_per_gpu": t_, "num_seqs": cfg.num_seqs, "seq_len": cfg.seq_len,
                       "d_model": d, "heads": cfg.heads, "d_ff": f, "causal": cfg.causal,
                       "parallelism": f"dp{world}", "l2": "inputs 34 MB + weights 25 MB + intermediates 235 MB "
                       "per step > 126 MB L2 (no flush between steps)"},
            "stage_ms": stage_ms, "attn_flops": attn_flops, "gemm_flops": gemm_flops,
            "context_torch_composition": None if torch_ms is None else {
                "ms_per_step": round(torch_ms, 5), "tflops": round(flops / (torch_ms * 1e-3) / 1e12, 2),
                "what": "F.linear (cuBLAS) + F.scaled_dot_product_attention + F.gelu, same shapes, fp16"},
            "clocks": sampler.summary(), "e2e": e2e, "gpu_launches": 5 * args.steps,
            "roofline": {"bound": "tensor", "achieved": round(flops / (ms_step * 1e-3) / 1e12, 2), "peak": peak_burst,
                         "unit": "TFLOP/s", "frac": round(flops / (ms_step * 1e-3) / 1e12 / peak_burst, 4),
                         "traffic": None, "peak_source": f"{peak_src} bf16 dense burst (fp16 = bf16 rate)",
                         "kernel": "whole layer step (gemm_bias_act x4 + fmha varlen)"},
            "cpu_baseline": cpu, "check_max_abs_err": err,
        }
        print(json.dumps(line), flush=True)
    if dist:
        dist.destroy_process_group()


def run_lstm(args, world, rank, local):
    """the paper's simplified LSTM cell (Fig. 12) as one
    dual_gemm_bias_act launch per step: relu(X Wx^T + H Wh^T + b), tokens 16384, input = hidden = 1024,
    4 gates (N = 4096).  The unfused torch composition (two cuBLAS GEMMs, add, ReLU) is timed beside it."""
    import torch.nn.functional as F
    import paper_conf_asplos_hagedornfccgg23_b200 as fm
    from workloads import make_gemm_inputs
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    m, n, k1, k2 = 16384, 4096, 1024, 1024
    x, wx, b = (t.to(dev) for t in make_gemm_inputs(m, n, k1, cfg_id=12))
    h, wh, _ = (t.to(dev) for t in make_gemm_inputs(m, n, k2, cfg_id=13))
    y = torch.empty((m, n), dtype=torch.float16, device=dev)
    stream = torch.cuda.current_stream(dev)
    step = lambda: fm.dual_gemm_bias_act(x, wx, h, wh, b, act="relu", out=y)
    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()
    sampler = ClockSampler(local)
    with sampler:
        ms = _time_graph(step, args.steps, stream)
    unfused = lambda: (F.linear(x, wx) + F.linear(h, wh, b)).relu_()
    for _ in range(3):
        unfused()
    torch.cuda.synchronize()
    torch_ms = _time_graph(unfused, args.steps, stream)
    flops = 2.0 * m * n * (k1 + k2)
    peak_burst, _, _, src = measured_peaks()
    from oracle import dual_gemm_bias_act_fp64
    rows = np.array([0, 1, m // 2, m - 1])
    ref = dual_gemm_bias_act_fp64(x[rows].cpu(), wx.cpu(), h[rows].cpu(), wh.cpu(), b.cpu(), 1)
    err = float(np.abs(y[torch.from_numpy(rows).to(dev)].double().cpu().numpy() - ref).max())
    val = flops / (ms * 1e-3) / 1e12
    if rank == 0:
        print(json.dumps({
            "metric": "simplified LSTM cell relu(X Wx^T + H Wh^T + b) TFLOP/s", "value": round(val, 2),
            "unit": "TFLOP/s", "n_gpus": 1, "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(ms, 5),
            "higher_is_better": True, "dtype": "f16", "data": "synthetic",
            "config": {"workload": "lstm_cell", "tokens": m, "input": k1, "hidden": k2, "gates_n": n},
            "context_torch_unfused": {"ms_per_step": round(torch_ms, 5), "speedup": round(torch_ms / ms, 3),
                                      "what": "F.linear + F.linear(+bias) + add + relu_ (cuBLAS + elementwise)"},
            "clocks": sampler.summary(), "gpu_launches": args.steps,
            "roofline": {"bound": "tensor", "achieved": round(val, 2), "peak": peak_burst, "unit": "TFLOP/s",
                         "frac": round(val / peak_burst, 4), "peak_source": f"{src} bf16 dense burst"},
            "check_max_abs_err": err}), flush=True)


def run_mlp_fused(args, world, rank, local):
    """the paper's fused multi-layer MLP (Fig. 11): L = 20
    layers of GEMM + bias + ReLU, N = K = 128 (or 64), M = 65536 rows, ONE mlp_fused_fwd launch per
    step.  The paper's comparator -- one cuBLASLt GEMM+bias+ReLU call per layer (torch's
    _addmm_activation, the cublasLt RELU_BIAS epilogue), intermediates through HBM -- is timed beside
    it.  Inputs rotate over sets larger than 3x L2; the weights (L x N x N fp16) stay resident."""
    import paper_conf_asplos_hagedornfccgg23_b200 as fm
    from workloads import make_fused_mlp_inputs
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    cfg = FUSED_MLP_CONFIGS[args.workload]
    x, w, b = make_fused_mlp_inputs(cfg.m, cfg.width, cfg.layers, cfg_id=cfg.cfg_id)
    xd, wd, bd = x.to(dev), w.to(dev), b.to(dev)
    set_bytes = 2 * xd.numel() * 2
    n_sets = max(1, int(np.ceil(3 * L2_BYTES / set_bytes)))
    sets = [(xd, torch.empty_like(xd))] + [(xd.clone(), torch.empty_like(xd)) for _ in range(n_sets - 1)]
    stream = torch.cuda.current_stream(dev)
    it = [0]

    def step():
        xs, ys = sets[it[0] % n_sets]
        it[0] += 1
        fm.mlp_fused(xs, wd, bd, act="relu", out=ys)

    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()
    sampler = ClockSampler(local)
    with sampler:
        ms = _time_graph(step, args.steps, stream)
    wt = [wd[l].t() for l in range(cfg.layers)]

    def cublaslt():
        h = sets[it[0] % n_sets][0]
        it[0] += 1
        for l in range(cfg.layers):
            h = torch._addmm_activation(bd[l], h, wt[l])  # cublasLt GEMM + bias + ReLU epilogue
        return h

    for _ in range(3):
        cublaslt()
    torch.cuda.synchronize()
    lt_ms = _time_graph(cublaslt, args.steps, stream)
    flops = 2.0 * cfg.m * cfg.width * cfg.width * cfg.layers
    peak_burst, _, _, src = measured_peaks()
    from oracle import mlp_fused_rows_fp64
    rows = np.array([0, 1, cfg.m // 2, cfg.m - 1])
    y = fm.mlp_fused(xd, wd, bd, act="relu")
    torch.cuda.synchronize()
    ref = mlp_fused_rows_fp64(x, w, b, rows)
    err = float(np.abs(y[torch.from_numpy(rows).to(dev)].double().cpu().numpy() - ref).max())
    val = flops / (ms * 1e-3) / 1e12
    if rank == 0:
        print(json.dumps({
            "metric": f"fused {cfg.layers}-layer MLP (GEMM+bias+ReLU, N=K={cfg.width}) TFLOP/s", "value": round(val, 2),
            "unit": "TFLOP/s", "n_gpus": 1, "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(ms, 5),
            "higher_is_better": True, "dtype": "f16", "data": "synthetic",
            "config": {"workload": cfg.name, "m": cfg.m, "width": cfg.width, "layers": cfg.layers,
                       "l2": f"rotating {n_sets} X/Y sets ({n_sets * set_bytes / 1e6:.0f} MB > 3x L2); W resident"},
            "context_cublaslt_per_layer": {"ms_per_step": round(lt_ms, 5), "speedup": round(lt_ms / ms, 3),
                                           "what": f"{cfg.layers} x torch._addmm_activation (cublasLt GEMM+bias+ReLU epilogue)"},
            "clocks": sampler.summary(), "gpu_launches": args.steps,
            "roofline": {"bound": "tensor", "achieved": round(val, 2), "peak": peak_burst, "unit": "TFLOP/s",
                         "frac": round(val / peak_burst, 4), "peak_source": f"{src} bf16 dense burst",
                         "kernel": "mlp_fused_kernel", "traffic": traffic_for(cfg.name)},
            "check_max_abs_err": err}), flush=True)


def run_splitkv(args, world, rank, local):
    """split-KV FMHA on a decode-like shape (few (b, h) units, a 16-row query block,
    16k keys): one fmha_fwd_splitkv call per step (split kernel + merge kernel, default split
    count).  The dense fmha_fwd kernel on the same inputs (one work item per (b, h): 32 of 148 SMs
    busy) is timed beside it.  HBM-bound: the roofline is the algorithmic bytes (Q + K + V + O) per
    step over the measured HBM bandwidth."""
    import paper_conf_asplos_hagedornfccgg23_b200 as fm
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    cfg = SPLITKV_CONFIGS[args.workload]
    q, k, v, _ = make_fmha_inputs(cfg)
    set_bytes = alg_bytes(cfg)
    n_sets = max(1, int(np.ceil(3 * L2_BYTES / set_bytes)))
    qd, kd, vd = q.to(dev), k.to(dev), v.to(dev)
    sets = [(qd, kd, vd, torch.empty_like(qd))] + [
        (qd.clone(), kd.clone(), vd.clone(), torch.empty_like(qd)) for _ in range(n_sets - 1)]
    lib = fm._lib.load()
    splits = lib.fmha_splitkv_default_splits(cfg.batch, cfg.heads, cfg.seq_q, cfg.seq_kv)
    ws = torch.empty(max(16, lib.fmha_splitkv_workspace_bytes(cfg.batch, cfg.heads, cfg.seq_q, cfg.head_dim, splits)),
                     dtype=torch.uint8, device=dev)
    stream = torch.cuda.current_stream(dev)
    it = [0]

    def step():
        a, b_, c, o = sets[it[0] % n_sets]
        it[0] += 1
        fm.fmha_fwd_splitkv(a, b_, c, scale=cfg.scale, num_splits=splits, out=o, workspace=ws)

    def dense():
        a, b_, c, o = sets[it[0] % n_sets]
        it[0] += 1
        fm.fmha_fwd(a, b_, c, scale=cfg.scale, out=o)

    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()
    sampler = ClockSampler(local)
    with sampler:
        ms = _time_graph(step, args.steps, stream)
    for _ in range(3):
        dense()
    torch.cuda.synchronize()
    dense_ms = _time_graph(dense, args.steps, stream)
    _, _, hbm, src = measured_peaks()
    gbs = set_bytes / (ms * 1e-3) / 1e9
    from oracle import attention_rows_fp64
    o = sets[0][3]
    step_ok = fm.fmha_fwd_splitkv(qd, kd, vd, scale=cfg.scale, num_splits=splits, out=o, workspace=ws)
    torch.cuda.synchronize()
    units = [(0, 0, 0), (cfg.batch - 1, cfg.heads - 1, cfg.seq_q - 1)]
    ref = attention_rows_fp64(q, k, v, cfg.scale, units)
    err = float(np.abs(torch.stack([step_ok[b, h, i] for b, h, i in units]).double().cpu().numpy() - ref).max())
    if rank == 0:
        print(json.dumps({
            "metric": "split-KV FMHA fwd achieved HBM GB/s (decode-like shape)", "value": round(gbs, 1),
            "unit": "GB/s", "n_gpus": 1, "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(ms, 5),
            "higher_is_better": True, "dtype": "bf16" if cfg.dtype == "bf16" else "f16", "data": "synthetic",
            "config": {"workload": cfg.name, "batch": cfg.batch, "heads": cfg.heads, "seq_q": cfg.seq_q,
                       "seq_kv": cfg.seq_kv, "head_dim": cfg.head_dim, "num_splits": splits,
                       "l2": f"rotating {n_sets} input/output sets ({n_sets * set_bytes / 1e6:.0f} MB > 3x L2)"},
            "tflops": round(alg_flops(cfg, None) / (ms * 1e-3) / 1e12, 2),
            "context_dense_fmha_fwd": {"ms_per_step": round(dense_ms, 5), "speedup": round(dense_ms / ms, 3),
                                       "what": "fmha_fwd (one work item per (b, h, q-tile pair)) on the same inputs"},
            "clocks": sampler.summary(), "gpu_launches": 2 * args.steps,
            "roofline": {"bound": "hbm", "achieved": round(gbs, 1), "peak": hbm, "unit": "GB/s",
                         "frac": round(gbs / hbm, 4), "peak_source": f"{src} HBM copy bandwidth",
                         "kernel": "fmha_fwd_kernel (split) + fmha_splitkv_combine_kernel",
                         "traffic": traffic_for(cfg.name)},
            "check_max_abs_err": err}), flush=True)


def run_reference(args, cfg, world, rank):
    """Reference arm for this tier = the CPU oracle, as it stands, on the host cores (rank 0 only)."""
    if rank != 0:
        return
    q, k, v, kv_len = make_fmha_inputs(cfg)
    from oracle import attention_fp64
    causal = cfg.mask == MASK_CAUSAL
    # each step: a bounded sample of the workload (a fixed number of whole (b,h) units)
    per_unit = None
    t0 = time.perf_counter()
    attention_fp64(q[:1, :1], k[:1, :1], v[:1, :1], cfg.scale, None if kv_len is None else kv_len[:1], causal)
    per_unit = time.perf_counter() - t0
    per_step_s = min(2.0, 90.0 / max(1, args.steps + min(args.warmup, 3)))  # whole run ~<= 1.5 min
    n_units = int(max(1, min(cfg.units, per_step_s / max(per_unit, 1e-6))))
    sub = cfg.with_(batch=max(1, n_units // cfg.heads) if n_units >= cfg.heads else 1,
                    heads=cfg.heads if n_units >= cfg.heads else n_units)
    qs, ks, vs = q[:sub.batch, :sub.heads], k[:sub.batch, :sub.heads], v[:sub.batch, :sub.heads]
    kls = None if kv_len is None else kv_len[:sub.batch]
    for _ in range(args.warmup if args.warmup <= 3 else 3):
        attention_fp64(qs, ks, vs, cfg.scale, kls, causal)
    t0 = time.perf_counter()
    for _ in range(args.steps):
        attention_fp64(qs, ks, vs, cfg.scale, kls, causal)
    el = time.perf_counter() - t0
    val = alg_flops(sub, kls) * args.steps / el / 1e12
    try:
        from threadpoolctl import threadpool_info
        cores = max([t.get("num_threads", 1) for t in threadpool_info()] or [1])
    except Exception:
        cores = os.cpu_count()
    line = {"impl": "reference", "metric": METRIC, "value": val, "unit": "TFLOP/s", "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": el / args.steps * 1e3,
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None,
            "dtype": "f64", "data": "synthetic",
            "config": {"workload": cfg.name, "batch_per_gpu": cfg.batch, "heads": cfg.heads, "seq_q": cfg.seq_q,
                       "seq_kv": cfg.seq_kv, "head_dim": cfg.head_dim,
                       "mask": ["none", "key_padding", "causal"][cfg.mask]},
            "cpu_baseline": {"value": val, "unit": "TFLOP/s", "cores": int(cores), "kind": "oracle",
                             "sample": f"{sub.batch * sub.heads} of {cfg.units} (b,h) units of {cfg.name} per step"},
            "e2e": {"value": val, "unit": "TFLOP/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


if __name__ == "__main__":
    main()
