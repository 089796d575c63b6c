"""Record, in profiles/traffic.json (one entry per bench config), the DRAM
traffic of the sampling kernel from an ncu --set full report:
dram__bytes_read.sum + dram__bytes_write.sum per launch (bench.py reports it
as roofline.traffic for that config).
Usage: python tools/write_traffic.py <report.ncu-rep> <config-name> <round-tag>"""
import csv
import io
import json
import os
import subprocess
import sys


def main(rep, config, tag):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr, units = rows[0], rows[1]
    ix = {h: i for i, h in enumerate(hdr)}
    scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12}
    for r in rows[2:]:
        if "sweep" not in r[ix["Kernel Name"]]:
            continue
        rd = float(r[ix["dram__bytes_read.sum"]]) * scale[units[ix["dram__bytes_read.sum"]]]
        wr = float(r[ix["dram__bytes_write.sum"]]) * scale[units[ix["dram__bytes_write.sum"]]]
        t = float(r[ix["gpu__time_duration.sum"]])
        doc = {"config": config, "round": tag, "kernel": r[ix["Kernel Name"]],
               "sweep_kernel_dram_bytes_per_launch": rd + wr, "dram_read": rd, "dram_write": wr,
               "ncu_duration_" + units[ix["gpu__time_duration.sum"]]: t, "report": os.path.basename(rep)}
        os.makedirs("profiles", exist_ok=True)
        path = os.path.join("profiles", "traffic.json")
        allc = json.load(open(path)) if os.path.exists(path) else {}
        allc[config] = doc
        with open(path, "w") as f:
            json.dump(allc, f, indent=1, sort_keys=True)
        print(json.dumps(doc))
        return


if __name__ == "__main__":
    main(*sys.argv[1:4])
