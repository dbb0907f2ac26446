"""A few back-to-back launches of one FMHA workload (for ncu under gpurun; not a timing tool).
usage: python tools/fmha_prof.py [workload] [launches]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_asplos_hagedornfccgg23_b200 as fm  # noqa: E402
from workloads import CONFIGS, MASK_CAUSAL, VARLEN_CONFIGS, make_fmha_inputs, make_varlen_inputs  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else "bert_large_512"
n = int(sys.argv[2]) if len(sys.argv) > 2 else 5
dev = torch.device("cuda:0")
if name in CONFIGS:
    cfg = CONFIGS[name]
    q, k, v, kl = make_fmha_inputs(cfg)
    q, k, v = q.to(dev), k.to(dev), v.to(dev)
    kld = None if kl is None else torch.from_numpy(kl).to(dev)
    run = lambda: fm.fmha_fwd(q, k, v, kv_len=kld, causal=cfg.mask == MASK_CAUSAL, scale=cfg.scale)
else:
    cfg = VARLEN_CONFIGS[name]
    qkv, cu = make_varlen_inputs(cfg)
    qkv, cu_d = qkv.to(dev), torch.from_numpy(cu).to(dev)
    run = lambda: fm.fmha_fwd_varlen(qkv, cu_d, int(max(cu[1:] - cu[:-1])), scale=cfg.scale)
for _ in range(n):
    run()
torch.cuda.synchronize()
print("ok", name, n)
