"""Build profiles/<tag>_<config>_summary.md from the gpurun_out artefacts of
tools/ncu_capture.sh and a bench JSON line.
Usage: python tools/summarize_round.py <tag> <config> <bench.json>"""
import collections
import csv
import io
import json
import os
import subprocess
import sys


def launches(path):
    lines = [l for l in open(path) if l.startswith('"')]   # skip ncu's ==WARNING==/==PROF== lines
    rows = list(csv.reader(lines))
    hdr = rows[0]
    ix = {h: i for i, h in enumerate(hdr)}
    per = collections.defaultdict(list)
    for r in rows[1:]:
        if len(r) != len(hdr) or r[ix["Metric Name"]] != "gpu__time_duration.sum":
            continue
        name = r[ix["Kernel Name"]].split("(")[0].replace("void ", "")
        per[name].append(float(r[ix["Metric Value"]]) / 1e6)   # ns -> ms
    return per


def ncu_raw(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    return rows[0], rows[1], rows[2:]


def main(tag, cfg, bench_path):
    os.makedirs("profiles", exist_ok=True)
    bench = json.loads(open(bench_path).read().strip().splitlines()[-1])
    lines = [f"# Profile summary — round tag `{tag}`, workload `{cfg}`", ""]
    lines += ["Bench line (device-timed, CUDA events on the library stream):", "", "```json",
              json.dumps(bench, indent=1), "```", ""]
    per = launches(f"gpurun_out/launches_{tag}_{cfg}.csv")
    lines += ["## Launch list (ncu `gpu__time_duration.sum`, `--clock-control none`; cold-cache, serialised)", "",
              "The first launches are corpus load (init, recount, θ build); the rest are the sweeps.", "",
              "| kernel | launches | mean ms | share of sweep kernels |", "|---|---|---|---|"]
    sweep_kernels = {"sweep_kernel", "sweep_tile_kernel", "sweep_quad_kernel", "word_table_kernel", "prologue_kernel", "zero_rows_kernel", "gather_z_kernel", "theta_kernel",
                     "recount_kernel"}
    tot = sum(sum(v) for k, v in per.items() if any(s in k for s in sweep_kernels))
    for k, v in sorted(per.items(), key=lambda kv: -sum(kv[1])):
        share = sum(v) / tot if any(s in k for s in sweep_kernels) and tot else 0.0
        lines.append(f"| `{k}` | {len(v)} | {sum(v) / len(v):.3f} | {share * 100:.1f} % |")
    rep = f"gpurun_out/prof_{tag}_{cfg}.ncu-rep"
    if os.path.exists(rep):
        hdr, units, rows = ncu_raw(rep)
        ix = {h: i for i, h in enumerate(hdr)}
        keys = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
                "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed",
                "smsp__issue_active.avg.pct_of_peak_sustained_active", "smsp__inst_executed.sum",
                "sm__warps_active.avg.pct_of_peak_sustained_active", "launch__registers_per_thread",
                "l1tex__data_pipe_lsu_wavefronts.avg.pct_of_peak_sustained_elapsed",
                "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum.pct_of_peak_sustained_elapsed",
                "smsp__thread_inst_executed_per_inst_executed.ratio",
                "lts__t_sector_hit_rate.pct", "l1tex__t_sector_hit_rate.pct"]
        lines += ["", f"## `ncu --set full` ({os.path.basename(rep)})", ""]
        for r in rows:
            lines += [f"### `{r[ix['Kernel Name']][:80]}`", "", "| metric | value |", "|---|---|"]
            for k in keys:
                if k in ix:
                    lines.append(f"| {k} | {r[ix[k]]} {units[ix[k]]} |")
            st = []
            for k in hdr:
                if k.startswith("smsp__average_warps_issue_stalled_") and k.endswith("_per_issue_active.ratio"):
                    try:
                        st.append((float(r[ix[k]]), k[len("smsp__average_warps_issue_stalled_"):-len("_per_issue_active.ratio")]))
                    except ValueError:
                        pass
            st.sort(reverse=True)
            lines.append("| top stalls (per issue) | " + ", ".join(f"{n} {v:.2f}" for v, n in st[:5]) + " |")
            lines.append("")
    out = f"profiles/{tag}_{cfg}_summary.md"
    open(out, "w").write("\n".join(lines) + "\n")
    print(out)


if __name__ == "__main__":
    main(*sys.argv[1:4])
