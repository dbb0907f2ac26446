"""Timing probe: fmha_fwd vs fmha_fwd_streamk on a few shapes (CUDA graph of 20 launches, median of 5)."""
import sys

import torch

sys.path.insert(0, ".")
import paper_conf_asplos_hagedornfccgg23_b200 as fm

dev = torch.device("cuda:0")
sms = torch.cuda.get_device_properties(dev).multi_processor_count


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
        ts.append(e0.elapsed_time(e1) / n * 1e3)
    return sorted(ts)[2]


for (b, h, sq, skv, d) in [(32, 16, 384, 384, 64), (1, 3, 384, 1024, 64), (2, 4, 512, 1024, 64),
                           (3, 50, 512, 4096, 64), (3, 50, 512, 2048, 64), (8, 14, 384, 1024, 64), (2, 24, 384, 8192, 128)]:
    q = torch.randn(b, h, sq, d, device=dev, dtype=torch.float16)
    k = torch.randn(b, h, skv, d, device=dev, dtype=torch.float16)
    v = torch.randn(b, h, skv, d, device=dev, dtype=torch.float16)
    o1, o2 = torch.empty_like(q), torch.empty_like(q)
    ws = fm.streamk_workspace(dev, d)
    t1 = time_fn(lambda: fm.fmha_fwd(q, k, v, out=o1))
    t2 = time_fn(lambda: fm.fmha_fwd_streamk(q, k, v, out=o2, workspace=ws))
    err = (o1.float() - o2.float()).abs().max().item()
    print(f"{(b, h, sq, skv, d)} plan={fm.streamk_plan(b, h, sq, skv, sms)} fmha_fwd {t1:.2f} us  streamk {t2:.2f} us  "
          f"max|diff| {err:.2e}", flush=True)
