"""Context measurement (not our path): library attention kernels at the bench shapes on this B200 --
torch SDPA with its cuDNN / flash / efficient backends, fp16, CUDA graph of 20 launches, median of 5."""
import sys

import torch
from torch.nn.attention import SDPBackend, sdpa_kernel

dev = torch.device("cuda:0")


def time_fn(fn, n=20):
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


sys.path.insert(0, ".")
import paper_conf_asplos_hagedornfccgg23_b200 as fm  # noqa: E402

for (b, h, s, d, dt, causal) in [(32, 16, 512, 64, torch.float16, False), (32, 16, 384, 64, torch.float16, False),
                                 (8, 32, 2048, 128, torch.bfloat16, True), (8, 32, 2048, 128, torch.bfloat16, False),
                                 (4, 32, 4096, 128, torch.bfloat16, True), (8, 32, 2048, 64, torch.float16, True)]:
    q = torch.randn(b, h, s, d, device=dev, dtype=dt)
    k = torch.randn(b, h, s, d, device=dev, dtype=dt)
    v = torch.randn(b, h, s, d, device=dev, dtype=dt)
    flops = 4.0 * b * h * s * s * d * (0.5 if causal else 1.0)
    out = torch.empty_like(q)
    res = {"ours": time_fn(lambda: fm.fmha_fwd(q, k, v, causal=causal, out=out))}
    for name, be in [("cudnn", SDPBackend.CUDNN_ATTENTION), ("flash", SDPBackend.FLASH_ATTENTION),
                     ("efficient", SDPBackend.EFFICIENT_ATTENTION)]:
        try:
            with sdpa_kernel(be):
                res[name] = time_fn(lambda: torch.nn.functional.scaled_dot_product_attention(q, k, v, is_causal=causal))
        except Exception as e:  # backend not available for this shape / build
            res[name] = f"n/a ({type(e).__name__})"
    line = ", ".join(f"{k_}: {v_:.4f} ms = {flops / v_ / 1e9:.0f} TFLOP/s" if isinstance(v_, float) else f"{k_}: {v_}"
                     for k_, v_ in res.items())
    print(f"{(b, h, s, d, str(dt)[6:], 'causal' if causal else 'full')}: {line}", flush=True)
