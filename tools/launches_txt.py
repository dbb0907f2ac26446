"""Format an ncu --csv launch list (gpu__time_duration.sum) as profiles/*_launches.txt.
usage: python tools/launches_txt.py <csv> "<command/comment>" [kernel-substring ...]"""
import csv
import sys

path, comment = sys.argv[1], sys.argv[2]
keys = sys.argv[3:]
rows = [r for r in csv.reader(open(path)) if len(r) > 10]
hdr = rows[0]
ik, iname, iv, iu = hdr.index("ID"), hdr.index("Kernel Name"), hdr.index("Metric Value"), hdr.index("Metric Unit")
ig, ib = hdr.index("Grid Size"), hdr.index("Block Size")
print(f"# {comment}")
print("# per-launch device time (cold-cache, serialised by the profiler; compare shares, not absolutes)")
tot, ours = 0.0, {k: 0.0 for k in keys}
for r in rows[1:]:
    t = float(r[iv].replace(",", "")) * {"ns": 1e-3, "nsecond": 1e-3, "us": 1.0, "usecond": 1.0, "ms": 1e3, "msecond": 1e3}[r[iu]]
    tot += t
    for k in keys:
        if k in r[iname]:
            ours[k] += t
    print(f"{r[ik]:>3} {t:10.3f} us  grid {r[ig]:>14} block {r[ib]:>14}  {r[iname][:110]}")
spin = sum(float(r[iv].replace(",", "")) * {"ns": 1e-3, "nsecond": 1e-3, "us": 1.0, "usecond": 1.0, "ms": 1e3,
                                             "msecond": 1e3}[r[iu]] for r in rows[1:] if "spin_kernel" in r[iname])
for k in keys:
    print(f"# {k} share of listed device time: {100 * ours[k] / tot:.1f}%"
          + (f"; {100 * ours[k] / (tot - spin):.1f}% without bench.lead_in's spin_kernel (run before each timed"
             f" region, outside it)" if spin > 0 else ""))
