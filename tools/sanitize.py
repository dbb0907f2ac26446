"""Small invocations of every kernel for compute-sanitizer (run via gpurun):
    compute-sanitizer --tool {memcheck,racecheck,synccheck} python tools/sanitize.py"""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_asplos_hagedornfccgg23_b200 as fm  # noqa: E402

dev = torch.device("cuda:0")
PART = os.environ.get("SAN_PART", "all")  # all | base | strided | bias2d | streamk | rest
want = lambda part: PART in ("all", part)
g = torch.Generator(device="cpu").manual_seed(0)
r = lambda *s, dt=torch.float16: torch.randn(*s, generator=g).to(dt).to(dev)
for d in (64, 128):
    for dt in (torch.float16, torch.bfloat16):
        q, k, v = r(1, 2, 200, d, dt=dt), r(1, 2, 300, d, dt=dt), r(1, 2, 300, d, dt=dt)
        if want("base"):
            fm.fmha_fwd(q, k, v)
            fm.fmha_fwd(q, k, v, causal=True)
            fm.fmha_fwd(q, k, v, kv_len=torch.tensor([150], dtype=torch.int32, device=dev))
            q3 = r(2, 2, 384, d, dt=dt)
            fm.fmha_fwd(q3, q3, q3)  # pair_mode 1 (odd q-tile count)
            fm.fmha_fwd_splitkv(q[:, :, :16].contiguous(), k, v, num_splits=3)
        # key bias (MODE_BIAS) with stride == seq_kv = 300: the clamped bias loads of the ragged last
        # KV tile must stay inside the row (run with PYTORCH_NO_CUDA_MEMORY_CACHING=1 so the bias
        # allocation ends exactly at the last row)
        if want("base"):
            fm.fmha_fwd(q, k, v, key_bias=torch.randn(1, 300, generator=g).to(dev))
        # round 2: strided [B,S,H,D] views (fmha_fwd_strided, 4-D TMA maps) and the general additive
        # mask (MODE_BIAS2D) with its row stride == seq_kv rounded to 8, broadcast over heads
        qs = r(1, 200, 2, d, dt=dt).transpose(1, 2)
        ks = r(1, 300, 2, d, dt=dt).transpose(1, 2)
        if want("strided"):
            fm.fmha_fwd(qs, ks, ks)
        ab = torch.randn(1, 1, 200, 304, generator=g).to(dt).to(dev)[..., :300]
        if want("bias2d"):
            fm.fmha_fwd(q, k, v, attn_bias=ab)
        # round 2: the stream-K tail (MODE_DENSE_TAIL / MODE_PAIRX_TAIL): every item of these small
        # problems is split along the keys, counted with atomics and merged by the last piece through
        # bulk copies into the idle Q/K/V region; run twice so the counters' reset is exercised
        if want("streamk"):
            kl = r(1, 2, 1000, d, dt=dt)
            for _ in range(2):
                fm.fmha_fwd_streamk(q, kl, kl)                 # dense pairs (2 q-tiles), 8 KV tiles -> 4 pieces
                k3 = torch.cat([kl, kl[:, :1]], dim=1)      # 3 heads
                fm.fmha_fwd_streamk(r(1, 3, 384, d, dt=dt), k3, k3)  # cross-unit pairs
                fm.fmha_fwd_streamk(q, kl, kl, causal=True)
qkv = r(300, 3, 4, 64)
cu = torch.tensor([0, 100, 100, 300], dtype=torch.int32, device=dev)
a, w, b = r(300, 136), r(264, 136) * 0.1, r(264)
if want("rest"):
    fm.fmha_fwd_varlen(qkv, cu, 200)
    fm.fmha_fwd_varlen(qkv, cu, 200, causal=True)
    fm.gemm_bias_act(a, w, b, act="gelu")
    fm.gemm_bias_act(r(600, 1024), r(1024, 1024) * 0.03, b.new_zeros(1024), act="relu")  # CTA-pair kernel
    fm.dual_gemm_bias_act(a, w, a, w, b, act="tanh")
    for n in (64, 128):
        fm.mlp_fused(r(700, n), r(3, n, n) * 0.1, r(3, n))
# the opt-in key-split kernel (B200_FMHA_KS=1) is covered by running this script with that variable
torch.cuda.synchronize()
print("sanitize workload done")
