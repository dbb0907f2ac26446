import torch, numpy as np, sys, os
sys.path.insert(0, os.getcwd())
import paper_conf_asplos_hagedornfccgg23_b200 as fm
from workloads import CONFIGS, make_fmha_inputs
for name in ["bert_large_384", "bert_large_512"]:
    cfg = CONFIGS[name]
    q, k, v, _ = make_fmha_inputs(cfg)
    q, k, v = q.cuda(), k.cuda(), v.cuda()
    kb = torch.zeros(cfg.batch, cfg.seq_kv, device="cuda")
    o = torch.empty_like(q)
    res = {}
    for mode in ["none", "bias"]:
        f = (lambda: fm.fmha_fwd(q, k, v, scale=cfg.scale, out=o)) if mode == "none" else (lambda: fm.fmha_fwd(q, k, v, scale=cfg.scale, out=o, key_bias=kb))
        for _ in range(5): f()
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(50): f()
        e1.record(); torch.cuda.synchronize()
        res[mode] = e0.elapsed_time(e1) / 50 * 1e3
    print(name, {k: round(v, 1) for k, v in res.items()}, "us")
