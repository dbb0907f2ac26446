"""Timeline of CTA 0 of the fused MLP kernel (debug build lib/libb200fmha_trace.so; run via gpurun).
usage: B200_MLP_SLOTS=S python tools/trace_mlp.py N M > gpurun_out/trace_mlp.txt"""
import ctypes
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

from paper_conf_asplos_hagedornfccgg23_b200 import _lib  # noqa: E402

_lib.LIB_PATH = os.path.join(ROOT, "paper_conf_asplos_hagedornfccgg23_b200", "lib", "libb200fmha_trace.so")
import paper_conf_asplos_hagedornfccgg23_b200 as fm  # noqa: E402

lib = _lib.load()
lib.fmha_trace_set.argtypes = [ctypes.c_void_p]
EV = {1: "EPI_ACC", 2: "EPI_LDTM", 3: "EPI_STS", 4: "EPI_ARRIVE", 5: "MMA_GO", 6: "MMA_COMMIT", 7: "EPI_MATH"}
n, m = int(sys.argv[1]), int(sys.argv[2])
L = 20
x = torch.randn(m, n, device="cuda", dtype=torch.float16)
w = (torch.randn(L, n, n, device="cuda") * (2 / n) ** 0.5).half()
b = torch.zeros(L, n, device="cuda", dtype=torch.float16)
buf = torch.zeros(24 * 2048, dtype=torch.int64, device="cuda")
for it in range(3):
    buf.zero_()
    lib.fmha_trace_set(buf.data_ptr())
    fm.mlp_fused(x, w, b)
    torch.cuda.synchronize()
ev = []
for r in buf.cpu().tolist():
    if r == 0:
        continue
    r &= (1 << 64) - 1
    ev.append((r >> 24, (r >> 18) & 63, (r >> 12) & 63, r & 0xFFF))
ev.sort()
t0 = ev[0][0]
print(f"# {len(ev)} events N={n} M={m}; cycle, warp, event, slot, layer")
for c, wp, e, a in ev:
    print(f"{c - t0:9d}  w{wp:02d}  {EV.get(e, e):11s} r{a // 64} l{a % 64}")
