"""Timeline of CTA 0 of the FMHA kernel (debug build lib/libb200fmha_trace.so; run via gpurun).
usage: python tools/trace_fmha.py [workload] > gpurun_out/trace.txt"""
import ctypes
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

from paper_conf_asplos_hagedornfccgg23_b200 import _lib  # noqa: E402
from workloads import CONFIGS, MASK_CAUSAL, make_fmha_inputs  # noqa: E402

_lib.LIB_PATH = os.path.join(ROOT, "paper_conf_asplos_hagedornfccgg23_b200", "lib", "libb200fmha_trace.so")
import paper_conf_asplos_hagedornfccgg23_b200 as fm  # noqa: E402

lib = _lib.load()
lib.fmha_trace_set.argtypes = [ctypes.c_void_p]
lib.fmha_trace_count.restype = ctypes.c_uint
EV = {1: "S_WAIT", 2: "S_READY", 3: "MAX_DONE", 4: "XCHG", 5: "EXP_DONE", 6: "MMA_P", 7: "MMA_O", 8: "MMA_PV",
      9: "MMA_QK", 10: "COR_ST", 11: "COR_PV", 12: "COR_ORDY", 13: "EPI", 14: "TMA_KV", 15: "ITEM"}

name = sys.argv[1] if len(sys.argv) > 1 else "bert_large_512"
dev = torch.device("cuda:0")
buf = torch.zeros(24 * 2048, dtype=torch.int64, device=dev)
if name in CONFIGS:
    cfg = CONFIGS[name]
    q, k, v, kl = make_fmha_inputs(cfg)
    q, k, v = q.to(dev), k.to(dev), v.to(dev)
    kld = None if kl is None else torch.from_numpy(kl).to(dev)
    run = lambda: fm.fmha_fwd(q, k, v, kv_len=kld, causal=cfg.mask == MASK_CAUSAL, scale=cfg.scale)
else:  # packed variable-length workload
    from workloads import VARLEN_CONFIGS, make_varlen_inputs
    cfg = VARLEN_CONFIGS[name]
    qkv, cu = make_varlen_inputs(cfg)
    qkv, cu_d = qkv.to(dev), torch.from_numpy(cu).to(dev)
    run = lambda: fm.fmha_fwd_varlen(qkv, cu_d, int(max(cu[1:] - cu[:-1])), scale=cfg.scale)
for it in range(3):
    buf.zero_()
    lib.fmha_trace_set(buf.data_ptr())
    run()
    torch.cuda.synchronize()
recs = [r for r in buf.cpu().tolist() if r != 0]
n = len(recs)
ev = []
for r in recs:
    r &= (1 << 64) - 1
    ev.append((r >> 24, (r >> 18) & 63, (r >> 12) & 63, r & 0xFFF))
ev.sort()
t0 = ev[0][0]
print(f"# {n} events, workload {name}; columns: cycle, warp, event, aux")
for c, w, e, a in ev:
    print(f"{c - t0:9d}  w{w:02d}  {EV.get(e, e):9s} {a}")
