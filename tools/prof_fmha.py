"""Per-phase cycle profile of the FMHA softmax warps (build: make variant NAME=prof DEFS=-DFMHA_PROF=1).
usage: python tools/prof_fmha.py [workload]   (run via gpurun)"""
import ctypes
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
os.environ.setdefault("B200FMHA_LIB", os.path.join(ROOT, "paper_conf_asplos_hagedornfccgg23_b200", "lib", "libb200fmha_prof.so"))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_asplos_hagedornfccgg23_b200 as fm  # noqa: E402
from paper_conf_asplos_hagedornfccgg23_b200 import _lib  # noqa: E402
from workloads import CONFIGS, MASK_CAUSAL, VARLEN_CONFIGS, make_fmha_inputs, make_varlen_inputs  # noqa: E402

NAMES = ["turnaround", "S_FULL wait", "S TMEM load", "mask+max", "decision+PV_DONE", "pre-turn exp",
         "turn wait", "exp in turn", "O rescale", "P store drain", "item end (L_EMPTY)", "tail"]
name = sys.argv[1] if len(sys.argv) > 1 else "bert_large_512"
lib = _lib.load()
lib.fmha_trace_set.argtypes = [ctypes.c_void_p]
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
buf = torch.zeros(148 * 16 * 16, dtype=torch.int64, device=dev)
for _ in range(3):
    buf.zero_()
    lib.fmha_trace_set(buf.data_ptr())
    run()
    torch.cuda.synchronize()
a = buf.cpu().numpy().reshape(148, 16, 16)[:, :8, :].astype(np.float64)  # softmax warps 0-7
steps = a[:, :, 15].sum()
tot = a[:, :, :12].sum()
per_cta = a[:, :, 15].sum(1) / 8
print(f"{name}: {steps / a.shape[0] / 8:.1f} steps per softmax warp (max over CTAs {per_cta.max():.0f}); "
      f"softmax-warp cycles per CTA: mean {a[:, :, :12].sum((1, 2)).mean() / 8:.0f}, max {a[:, :, :12].sum((1, 2)).max() / 8:.0f}; cycles per step:")
for i, nm in enumerate(NAMES):
    print(f"  {nm:20s} {a[:, :, i].sum() / steps:8.0f}  ({100 * a[:, :, i].sum() / tot:4.1f}%)")
print(f"  {'total':20s} {tot / steps:8.0f}")
m = buf.cpu().numpy().reshape(148, 16, 16)[:, 12:14, :].astype(np.float64)  # MMA warps 12, 13
MN = ["K ring wait", "Q wait", "S_FREE wait", "QK issue", "V ring wait", "O_EMPTY wait", "P_FULL wait", "PV issue",
      "between", "tail"]
msteps = m[:, :, 15].sum()
mtot = m[:, :, :10].sum()
print(f"MMA warps: {msteps / m.shape[0] / 2:.1f} QKs per warp; cycles per step:")
for i, nm in enumerate(MN):
    print(f"  {nm:20s} {m[:, :, i].sum() / msteps:8.0f}  ({100 * m[:, :, i].sum() / mtot:4.1f}%)")
