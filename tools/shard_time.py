"""Projected strong scaling of BERT-large-512: the per-GPU kernel of an N-way (b x h)
shard is fmha_fwd on batch 32/N; with no data-path collective the N-GPU step time is the max over
ranks of that kernel, so t(32)/t(32/N) is the speedup the kernels allow (one GPU, rotating inputs
larger than L2 as in bench.py, CUDA graph of K launches after a device spin, median of 5)."""
import sys

import torch

sys.path.insert(0, ".")
import paper_conf_asplos_hagedornfccgg23_b200 as fm  # noqa: E402
from workloads import CONFIGS, make_fmha_inputs  # noqa: E402

dev = torch.device("cuda:0")
cfg0 = CONFIGS["bert_large_512"]
res = {}
for n in (1, 2, 4, 8):
    cfg = cfg0.with_(batch=cfg0.batch // n)
    q, k, v, _ = make_fmha_inputs(cfg)
    nset = max(3, int(3 * 126e6 / (4 * q.numel() * 2)) + 1)
    sets = [(q.to(dev), k.to(dev), v.to(dev), torch.empty_like(q, device=dev)) for _ in range(nset)]
    K = 50
    s = torch.cuda.Stream()
    s.wait_stream(torch.cuda.current_stream())
    with torch.cuda.stream(s):
        for i in range(nset):
            a = sets[i]
            fm.fmha_fwd(a[0], a[1], a[2], scale=cfg.scale, out=a[3])
        torch.cuda.synchronize()
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g, stream=s):
            for i in range(K):
                a = sets[i % nset]
                fm.fmha_fwd(a[0], a[1], a[2], scale=cfg.scale, out=a[3])
        g.replay()
        torch.cuda.synchronize()
        ts = []
        for _ in range(5):
            torch.cuda._sleep(600_000)
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            g.replay()
            e1.record()
            torch.cuda.synchronize()
            ts.append(e0.elapsed_time(e1) / K * 1e3)
    res[n] = sorted(ts)[2]
    print(f"N={n}: batch {cfg.batch} per GPU, {nset} rotating sets: {res[n]:.2f} us per launch; "
          f"projected speedup t1/tN = {res[1] / res[n]:.2f}x", flush=True)
