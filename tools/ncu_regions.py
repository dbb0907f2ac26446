"""Per-instruction warp-stall samples from an ncu source page (csv, --print-source sass), grouped
into regions delimited by barrier waits; prints the top-N instructions with stall columns.
usage: ncu -i rep --page source --csv --print-source sass > src.csv; python tools/ncu_regions.py src.csv"""
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
hdr, data = rows[1], rows[2:]
i_s = hdr.index("Warp Stall Sampling (All Samples)")
i_src = hdr.index("Source")
i_ex = hdr.index("Instructions Executed")
stall_cols = [i for i, h in enumerate(hdr) if h.startswith("stall_") or "Stall" in h and "Sampling" not in h]
tot = sum(int(r[i_s] or 0) for r in data)
print("total samples", tot)
top = sorted(range(len(data)), key=lambda n: -int(data[n][i_s] or 0))[: int(sys.argv[2]) if len(sys.argv) > 2 else 25]
for n in sorted(top):
    r = data[n]
    ctx = ""
    # nearest preceding barrier instruction (to know what a branch spins on)
    for m in range(n, max(0, n - 4), -1):
        if "SYNCS" in data[m][i_src] or "BAR" in data[m][i_src]:
            ctx = data[m][i_src].strip()[:70]
            break
    print(f"[{n:5d}] {int(r[i_s]):6d} {100 * int(r[i_s]) / tot:5.1f}% ex={r[i_ex]:>8s}  {r[i_src].strip()[:60]:60s} | {ctx}")
