"""Per-step device times inside one timed graph replay of the BERT-large-512 bench (events captured
between the launches, external=True), to locate the K-dependent part of the per-step time."""
import sys

import numpy as np
import torch

sys.path.insert(0, ".")
import paper_conf_asplos_hagedornfccgg23_b200 as fm  # noqa: E402
from workloads import CONFIGS, make_fmha_inputs  # noqa: E402

dev = torch.device("cuda:0")
cfg = CONFIGS["bert_large_512"]
q, k, v, _ = make_fmha_inputs(cfg)
sets = [(q.to(dev), k.to(dev), v.to(dev), torch.empty_like(q, device=dev)) for _ in range(3)]
K = int(sys.argv[1]) if len(sys.argv) > 1 else 20
evs = [torch.cuda.Event(enable_timing=True, external=True) for _ in range(K + 1)]
s = torch.cuda.Stream()
s.wait_stream(torch.cuda.current_stream())
with torch.cuda.stream(s):
    for i in range(5):
        a = sets[i % 3]
        fm.fmha_fwd(a[0], a[1], a[2], scale=cfg.scale, out=a[3])
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=s):
        for i in range(K):
            evs[i].record()
            a = sets[i % 3]
            fm.fmha_fwd(a[0], a[1], a[2], scale=cfg.scale, out=a[3])
        evs[K].record()
    g.replay()
    torch.cuda.synchronize()
    for rep in range(3):
        torch.cuda._sleep(600_000)
        g.replay()
        torch.cuda.synchronize()
        t = np.array([evs[i].elapsed_time(evs[i + 1]) * 1e3 for i in range(K)])
        print(f"rep {rep}: total {t.sum():.1f} us, per step: " + " ".join(f"{x:.1f}" for x in t), flush=True)
