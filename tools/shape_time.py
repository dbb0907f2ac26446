"""Times fmha_fwd (the library B200FMHA_LIB points at) on a few shapes: CUDA graph of 20 launches,
median of 5 replays.  usage: python tools/shape_time.py [tag]"""
import sys

import torch

sys.path.insert(0, ".")
import paper_conf_asplos_hagedornfccgg23_b200 as fm  # noqa: E402

dev = torch.device("cuda:0")
tag = sys.argv[1] if len(sys.argv) > 1 else ""


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


for (b, h, s, d, dt, causal) in [(8, 32, 2048, 128, torch.bfloat16, True), (8, 32, 2048, 128, torch.bfloat16, False),
                                 (4, 32, 4096, 128, torch.bfloat16, True), (32, 16, 512, 64, torch.float16, False)]:
    torch.manual_seed(0)
    q = torch.randn(b, h, s, d, device=dev, dtype=dt)
    k = torch.randn(b, h, s, d, device=dev, dtype=dt)
    v = torch.randn(b, h, s, d, device=dev, dtype=dt)
    flops = 4.0 * b * h * s * s * d * (0.5 if causal else 1.0)
    out = torch.empty_like(q)
    t = time_fn(lambda: fm.fmha_fwd(q, k, v, causal=causal, out=out))
    print(f"{tag} {(b, h, s, d, 'causal' if causal else 'full')}: {t:.4f} ms = {flops / t / 1e9:.0f} TFLOP/s", flush=True)
