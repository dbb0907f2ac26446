"""Per-layer time of the fused MLP kernel vs slots (S) and M (run via gpurun).  Tuning aid only.
usage: python tools/mlp_sweep.py"""
import os
import subprocess
import sys

if len(sys.argv) == 1:
    for n in (128, 64):
        for s in (["1", "2", "4"] if n == 128 else ["1", "2", "4", "8"]):
            for m in (128 * 148, 128 * 148 * 4):
                env = dict(os.environ, B200_MLP_SLOTS=s)
                out = subprocess.run([sys.executable, __file__, str(n), str(m)], env=env, capture_output=True, text=True)
                print(f"N={n} S={s} M={m}: {out.stdout.strip()} {out.stderr.strip()[-200:]}", flush=True)
    sys.exit(0)

import torch  # noqa: E402
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_asplos_hagedornfccgg23_b200 as fm  # noqa: E402

n, m = int(sys.argv[1]), int(sys.argv[2])
L = 20
x = torch.randn(m, n, device="cuda", dtype=torch.float16)
w = (torch.randn(L, n, n, device="cuda") * (2 / n) ** 0.5).half()
b = torch.zeros(L, n, device="cuda", dtype=torch.float16)
y = torch.empty_like(x)
for _ in range(3):
    fm.mlp_fused(x, w, b, out=y)
torch.cuda.synchronize()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record()
for _ in range(20):
    fm.mlp_fused(x, w, b, out=y)
e1.record()
torch.cuda.synchronize()
ms = e0.elapsed_time(e1) / 20
tiles = (m + 127) // 128
print(f"{ms * 1e3:.1f} us  {2 * m * n * n * L / ms / 1e9:.0f} TF/s  per-layer {ms * 1e3 / L:.2f} us")
