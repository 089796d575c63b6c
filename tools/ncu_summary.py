"""Summarise an ncu report (raw page) for the kernels in it: time, DRAM bytes,
issue activity, warp stall breakdown.  Usage: python tools/ncu_summary.py rep.ncu-rep"""
import csv
import io
import subprocess
import sys

KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed",
        "smsp__issue_active.avg.pct_of_peak_sustained_active", "smsp__inst_executed.sum",
        "sm__warps_active.avg.pct_of_peak_sustained_active", "launch__registers_per_thread",
        "launch__occupancy_limit_registers", "launch__occupancy_limit_shared_mem",
        "l1tex__t_sector_hit_rate.pct", "lts__t_sector_hit_rate.pct",
        "sm__inst_executed_pipe_fp64.avg.pct_of_peak_sustained_active",
        "sm__cycles_elapsed.avg.per_second", "launch__grid_size", "launch__block_size"]
STALLS = ["long_scoreboard", "short_scoreboard", "mio_throttle", "lg_throttle", "wait", "barrier",
          "math_pipe_throttle", "no_instruction", "not_selected", "selected", "branch_resolving",
          "dispatch_stall", "tex_throttle", "drain", "membar", "sleeping", "imc_miss", "misc"]


def main(path):
    out = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr, units = rows[0], rows[1]
    ix = {h: i for i, h in enumerate(hdr)}
    for r in rows[2:]:
        name = r[ix["Kernel Name"]][:60]
        print(f"== {name}  (id {r[ix['ID']]})")
        for k in KEYS:
            if k in ix:
                print(f"   {k:60s} {r[ix[k]]:>18s} {units[ix[k]]}")
        st = []
        for s in STALLS:
            k = f"smsp__average_warps_issue_stalled_{s}_per_issue_active.ratio"
            if k in ix and r[ix[k]]:
                st.append((float(r[ix[k]]), s))
        st.sort(reverse=True)
        print("   stalls per issue: " + ", ".join(f"{s}={v:.2f}" for v, s in st[:8]))


if __name__ == "__main__":
    main(sys.argv[1])
