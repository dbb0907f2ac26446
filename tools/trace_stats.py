"""Per-phase cycle statistics of a trace dump (tools/trace_fmha.py output) for the key-split kernel:
softmax warps 0-15 (S wait, TMEM load + max, exponentials, rescale + P-store drain, loop turnaround,
item merge), MMA warps 16/17 (P_FULL waits per stream, ring waits).
usage: python tools/trace_stats.py gpurun_out/trace.txt"""
import collections
import sys

rows = []
for line in open(sys.argv[1]):
    if line.startswith("#") or not line.strip():
        continue
    c, w, e, a = line.split()
    rows.append((int(c), int(w[1:]), e, int(a)))
by = collections.defaultdict(list)
for r in rows:
    by[r[1]].append(r)
span = max(r[0] for r in rows) - min(r[0] for r in rows)
print(f"span {span} cycles, {len(rows)} events")
acc = collections.defaultdict(list)
for w, evs in by.items():
    prev = None
    for c, _, e, a in evs:
        if prev is not None:
            acc[(w < 16, prev[2], e)].append(c - prev[0])
        prev = (c, w, e, a)
print(f"{'role':8s} {'from':10s} {'to':10s} {'n':>6s} {'mean':>8s} {'p50':>8s} {'sum/warp':>9s}")
nw = {True: 16, False: 2}
for (sm, a, b), v in sorted(acc.items(), key=lambda kv: -sum(kv[1])):
    v = sorted(v)
    print(f"{'softmax' if sm else 'other':8s} {a:10s} {b:10s} {len(v):6d} {sum(v)/len(v):8.0f} {v[len(v)//2]:8d} "
          f"{sum(v)/nw[sm]:9.0f}")
