"""Launches fmha_fwd_streamk on a long-key shape whose last round is split (3 x 50 x 512 x 4096, fp16:
300 items = 2 rounds of 148 + 4 items x 4 key pieces) a few times, for ncu under gpurun."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_asplos_hagedornfccgg23_b200 as fm  # noqa: E402

dev = torch.device("cuda:0")
q = torch.randn(3, 50, 512, 64, device=dev, dtype=torch.float16)
k = torch.randn(3, 50, 4096, 64, device=dev, dtype=torch.float16)
v = torch.randn(3, 50, 4096, 64, device=dev, dtype=torch.float16)
for _ in range(4):
    fm.fmha_fwd_streamk(q, k, v)
torch.cuda.synchronize()
print("ok", fm.streamk_plan(3, 50, 512, 4096, torch.cuda.get_device_properties(dev).multi_processor_count))
