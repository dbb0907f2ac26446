"""Executed warp-instructions and stall samples per kernel role, from an ncu report.
Each SASS instruction is attributed to the fmha_kernel.cuh line it came from, or (for code inlined
from helper headers) to the nearest preceding kernel-file instruction in address order.
usage: python tools/ncu_roles.py rep.ncu-rep"""
import csv
import io
import subprocess
import sys

ROLES = [(282, 326, "tma"), (326, 484, "mma"), (484, 643, "softmax"), (643, 684, "corr-loop"),
         (684, 741, "corr-epilogue")]

out = subprocess.run(["ncu", "-i", sys.argv[1], "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True, errors="replace").stdout
rows = list(csv.reader(io.StringIO(out)))
insts = []  # (addr, file_is_kernel, line, executed, samples)
fname, line = "", 0
hdr = None
for r in rows:
    if len(r) == 2 and r[0] == "File Path":
        fname = r[1]
        continue
    if r and r[0] == "Line No":
        hdr = r
        continue
    if hdr is None or len(r) < 8:
        continue
    if r[0]:
        line = int(r[0])
        continue
    if r[2] in ("...", "-") or not r[2].startswith("0x"):
        continue
    ex = int(r[hdr.index("Instructions Executed", 4)] or 0)
    sm = int(r[hdr.index("Warp Stall Sampling (All Samples)", 4)] or 0)
    insts.append((int(r[2], 16), fname.endswith("fmha_kernel.cuh"), line, ex, sm, r[3].strip()))
# an instruction can be listed under several (inlined) source lines: keep one entry per address,
# preferring the kernel-file attribution
best = {}
for t in insts:
    if t[0] not in best or (t[1] and not best[t[0]][1]):
        best[t[0]] = t
insts = sorted(best.values())
role_of = lambda ln: next((n for a, b, n in ROLES if a <= ln < b), "other")
cur = "other"
tot = {}
for addr, k, ln, ex, sm, src in insts:
    if k:
        cur = role_of(ln)
    e = tot.setdefault(cur, [0, 0])
    e[0] += ex
    e[1] += sm
T = sum(v[0] for v in tot.values())
S = sum(v[1] for v in tot.values())
print(f"{'role':15s} {'warp-inst':>12s} {'%':>6s} {'samples':>8s} {'%':>6s}")
for n, (ex, sm) in sorted(tot.items(), key=lambda x: -x[1][0]):
    print(f"{n:15s} {ex:12d} {100 * ex / T:6.1f} {sm:8d} {100 * sm / max(S, 1):6.1f}")
