"""Is the GELU epilogue's cost power (clock) or time?  gemm_bias_act at 8192^3 and at the MLP shape,
with and without GELU: one launch cold (after 1 s idle) and a 2 s back-to-back run, with the SM clock
sampled through NVML (bench.ClockSampler)."""
import sys
import time

import torch

sys.path.insert(0, ".")
import paper_conf_asplos_hagedornfccgg23_b200 as fm  # noqa: E402
from bench import ClockSampler  # noqa: E402

dev = torch.device("cuda:0")
for (m, n, k) in [(8192, 8192, 8192), (16384, 4096, 1024)]:
    a = torch.randn(m, k, device=dev, dtype=torch.float16)
    w = torch.randn(n, k, device=dev, dtype=torch.float16) * 0.03
    b = torch.randn(n, device=dev, dtype=torch.float16)
    c = torch.empty(m, n, device=dev, dtype=torch.float16)
    for act in ("none", "gelu", "none", "gelu"):
        fm.gemm_bias_act(a, w, b, act=act, out=c)
        torch.cuda.synchronize()
        time.sleep(1.0)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        fm.gemm_bias_act(a, w, b, act=act, out=c)
        e1.record()
        torch.cuda.synchronize()
        cold = e0.elapsed_time(e1)
        reps = max(1, int(2000 / max(cold, 0.01)))
        smp = ClockSampler(0)
        with smp:
            e0.record()
            for _ in range(reps):
                fm.gemm_bias_act(a, w, b, act=act, out=c)
            e1.record()
            torch.cuda.synchronize()
        hot = e0.elapsed_time(e1) / reps
        fl = 2.0 * m * n * k
        print(f"{(m, n, k)} {act}: cold {cold * 1e3:.1f} us ({fl / cold / 1e9:.0f} TF/s)  sustained {hot * 1e3:.1f} us "
              f"({fl / hot / 1e9:.0f} TF/s) clocks {smp.summary()}", flush=True)
