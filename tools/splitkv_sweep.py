"""Split-KV FMHA time vs num_splits on the decode_splitkv bench shape (run via gpurun). Tuning aid."""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_asplos_hagedornfccgg23_b200 as fm  # noqa: E402
from workloads import SPLITKV_CONFIGS, make_fmha_inputs  # noqa: E402

cfg = SPLITKV_CONFIGS["decode_splitkv"]
for name, c in [("bench", cfg), ("b1h8", cfg.with_(batch=1)), ("sq1", cfg.with_(seq_q=1))]:
    q, k, v, _ = make_fmha_inputs(c)
    q, k, v = q.cuda(), k.cuda(), v.cuda()
    ws = torch.empty(1 << 28, dtype=torch.uint8, device="cuda")
    o = torch.empty_like(q)
    lib = fm._lib.load()
    d = lib.fmha_splitkv_default_splits(c.batch, c.heads, c.seq_q, c.seq_kv)
    line = []
    for s in [1, 2, 3, 4, 5, 6, 8, 9, 11, 13, 16, 22, 32, 43, 64]:
        for _ in range(3):
            fm.fmha_fwd_splitkv(q, k, v, scale=c.scale, num_splits=s, out=o, workspace=ws)
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(20):
            fm.fmha_fwd_splitkv(q, k, v, scale=c.scale, num_splits=s, out=o, workspace=ws)
        e1.record()
        torch.cuda.synchronize()
        line.append(f"{s}:{e0.elapsed_time(e1) / 20 * 1e3:.0f}")
    print(f"{name} (default {d}) us: " + " ".join(line), flush=True)
