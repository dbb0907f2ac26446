"""Launch the MLP block's two GEMMs (config 5) a few times, plus the GEMM1 shape without activation
(for ncu under gpurun; not a timing tool).  usage: python tools/gemm_prof.py [n]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_asplos_hagedornfccgg23_b200 as fm  # noqa: E402
from workloads import make_mlp_inputs  # noqa: E402

n = int(sys.argv[1]) if len(sys.argv) > 1 else 3
dev = torch.device("cuda:0")
x, w1, b1, w2, b2 = (t.to(dev) for t in make_mlp_inputs())
for _ in range(n):
    h = fm.gemm_bias_act(x, w1, b1, act="gelu")
    y = fm.gemm_bias_act(h, w2, b2, act="none")
    h0 = fm.gemm_bias_act(x, w1, b1, act="none")
torch.cuda.synchronize()
print("ok")
