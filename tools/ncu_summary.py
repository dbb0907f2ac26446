"""Summarise an ncu report (run here, no GPU): key throughput metrics + top stall reasons.
usage: python tools/ncu_summary.py gpurun_out/<rep>.ncu-rep [--source]"""
import csv
import io
import subprocess
import sys

KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "dram__throughput.avg.pct_of_peak_sustained_elapsed", "sm__cycles_elapsed.avg.per_second",
        "launch__registers_per_thread", "launch__grid_size", "launch__block_size",
        "sm__inst_executed_pipe_xu.avg.pct_of_peak_sustained_active",
        "sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__inst_executed_pipe_fmaheavy.avg.pct_of_peak_sustained_active",
        "sm__inst_executed_pipe_fmalite.avg.pct_of_peak_sustained_active",
        "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__pipe_tc_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__pipe_tmem_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__pipe_shared_cycles_active.avg.pct_of_peak_sustained_active",
        "smsp__issue_active.avg.pct_of_peak_sustained_active",
        "sm__throughput.avg.pct_of_peak_sustained_elapsed",
        "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum",
        "local_load", "lts__t_bytes.sum", "smsp__thread_inst_executed_per_inst_executed.ratio"]


def main(path, source=False):
    raw = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(raw)))
    hdr, units, vals = rows[0], rows[1], rows[2:]
    for v in vals:
        print("kernel:", v[hdr.index("Kernel Name")][:90])
        for i, h in enumerate(hdr):
            if any(h == k or (k in h and "pct" not in k and k in ("local_load",)) for k in KEYS):
                print(f"  {h:75s} {units[i]:>12s} {v[i]}")
        stalls = [(h, v[i]) for i, h in enumerate(hdr)
                  if h.startswith("smsp__average_warps_issue_stalled_") and h.endswith("_per_issue_active.ratio")]
        stalls = sorted(((float(x or 0), h) for h, x in stalls), reverse=True)[:10]
        print("  top stalls (warps per issue-active cycle):")
        for x, h in stalls:
            print(f"    {h.replace('smsp__average_warps_issue_stalled_', '').replace('_per_issue_active.ratio', ''):30s} {x:.3f}")


if __name__ == "__main__":
    main(sys.argv[1], "--source" in sys.argv)
