"""Pure-Python scalar FMHA — brute force for tiny shapes (S, D <= ~16).

TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).

Same steps as oracle/fmha.py (GEMM -> softmax(max, exp, sum, divide) ->
GEMM) but written as explicit scalar loops with ``math.fsum`` (exactly rounded
sums) and ``math.exp``, so it shares no library routine with the numpy oracle.
Used by tests/test_oracle.py to pin the numpy oracle (pin P11).
"""

from __future__ import annotations

import math


def attention_brute(q, k, v, scale: float, kv_len=None, causal: bool = False, key_bias=None, attn_bias=None):
    """q: nested lists [B][H][Sq][D] of floats; k, v: [B][H][Skv][D]; key_bias None or
    [B][Skv] additive bias (R20; -inf excludes the key); attn_bias None or nested
    lists [B][H][Sq][Skv] (R21; -inf excludes the pair).
    Returns nested lists [B][H][Sq][D]."""
    import struct
    scale = struct.unpack("f", struct.pack("f", scale))[0]  # fp32 value (R1)
    out = []
    for b in range(len(q)):
        ob = []
        for h in range(len(q[b])):
            qb, kb, vb = q[b][h], k[b][h], v[b][h]
            sq, skv, d = len(qb), len(kb), len(qb[0])
            limit = skv if kv_len is None else max(0, min(int(kv_len[b]), skv))
            oh = []
            for i in range(sq):
                vis = [j for j in range(skv)
                       if j < limit and (not causal or j <= i + (skv - sq))
                       and (key_bias is None or key_bias[b][j] != -math.inf)
                       and (attn_bias is None or attn_bias[b][h][i][j] != -math.inf)]
                if not vis:
                    oh.append([0.0] * d)
                    continue
                s = {j: math.fsum(qb[i][t] * kb[j][t] for t in range(d)) * scale
                     + (0.0 if key_bias is None else key_bias[b][j])
                     + (0.0 if attn_bias is None else attn_bias[b][h][i][j]) for j in vis}
                m = max(s.values())
                e = {j: math.exp(s[j] - m) for j in vis}
                l = math.fsum(e.values())
                oh.append([math.fsum(e[j] / l * vb[j][t] for j in vis) for t in range(d)])
            ob.append(oh)
        out.append(ob)
    return out
