"""Context measurement (not our path): the MLP block's GEMM shapes (config 5) through cuBLAS (torch.matmul,
fp16, no epilogue) and through gemm_bias_act (ours, with and without the bias + activation epilogue).
CUDA graph of 10 launches, median of 5 replays."""
import sys

import torch

sys.path.insert(0, ".")
import paper_conf_asplos_hagedornfccgg23_b200 as fm  # noqa: E402

dev = torch.device("cuda:0")


def time_fn(fn, n=10):
    s = torch.cuda.Stream()
    s.wait_stream(torch.cuda.current_stream())
    with torch.cuda.stream(s):
        fn()
        torch.cuda.synchronize()
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g, stream=s):
            for _ in range(n):
                fn()
    g.replay()
    torch.cuda.synchronize()
    ts = []
    for _ in range(5):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        g.replay()
        e1.record()
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1) / n)
    return sorted(ts)[2]


for (m, n, k) in [(16384, 4096, 1024), (16384, 1024, 4096), (8192, 8192, 8192)]:
    a = torch.randn(m, k, device=dev, dtype=torch.float16)
    w = torch.randn(n, k, device=dev, dtype=torch.float16) * 0.03
    b = torch.randn(n, device=dev, dtype=torch.float16)
    c = torch.empty(m, n, device=dev, dtype=torch.float16)
    fl = 2.0 * m * n * k
    res = {"cublas": time_fn(lambda: torch.matmul(a, w.t(), out=c)),
           "ours_none": time_fn(lambda: fm.gemm_bias_act(a, w, b, act="none", out=c)),
           "ours_gelu": time_fn(lambda: fm.gemm_bias_act(a, w, b, act="gelu", out=c))}
    print((m, n, k), ", ".join(f"{k_}: {v_ * 1e3:.1f} us = {fl / v_ / 1e9:.0f} TFLOP/s" for k_, v_ in res.items()), flush=True)
