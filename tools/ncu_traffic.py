#!/usr/bin/env python
"""Write profiles/ncu_traffic_<config>.json from an ncu raw-page CSV export (one --set full
capture of one step's kernels, taken by tools/gpurun_suite.sh) and the bench JSON line of
the same code: per kernel, DRAM bytes read + written per launch (the roofline's `traffic`),
its duration under ncu, and the build parameters the line reports, stamped with the git
commit the capture was taken at.  bench.py reads the file and uses the traffic only when the
parameters match its own handle.

  python tools/ncu_traffic.py --raw gpurun_out/X_raw.csv --bench gpurun_out/X_bench.log \
      --config c5 --commit <sha> [--out profiles/ncu_traffic_c5.json]
"""
import argparse
import csv
import datetime
import json
import os
import subprocess

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def short_name(kernel: str) -> str:
    for k in ("panel_kernel", "spmv_bccoo_s2_kernel", "spmv_bccoo_kernel", "combine_kernel"):
        if k in kernel:
            return k
    return kernel.split("(")[0].split("::")[-1]


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--raw", required=True)
    ap.add_argument("--bench", required=True, help="log whose last JSON line is the bench line")
    ap.add_argument("--config", default="c5")
    ap.add_argument("--commit", default=None)
    ap.add_argument("--out", default=None)
    a = ap.parse_args()
    rows = list(csv.reader(open(a.raw)))
    hdr = rows[0]
    kernels = {}
    for vals in rows[2:]:
        d = dict(zip(hdr, vals))
        if "dram__bytes_read.sum" not in d:
            continue
        unit = rows[1][hdr.index("dram__bytes_read.sum")]
        scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}.get(unit, 1)
        rd = float(d["dram__bytes_read.sum"].replace(",", "")) * scale
        wunit = rows[1][hdr.index("dram__bytes_write.sum")]
        wr = float(d["dram__bytes_write.sum"].replace(",", "")) * {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6,
                                                                     "Gbyte": 1e9}.get(wunit, 1)
        dunit = rows[1][hdr.index("gpu__time_duration.sum")]
        dur = float(d["gpu__time_duration.sum"].replace(",", "")) * {"ms": 1, "us": 1e-3, "ns": 1e-6,
                                                                      "s": 1e3}.get(dunit, 1)
        kernels[short_name(d.get("Kernel Name", ""))] = {"dram_bytes_per_launch": rd + wr, "dram_read": rd,
                                                         "dram_write": wr, "ncu_duration_ms": dur}
    line = None
    for ln in open(a.bench):
        ln = ln.strip()
        if ln.startswith("{") and '"metric"' in ln:
            line = json.loads(ln)
    params = line["config"]["params"] if line else {}
    for k in kernels.values():
        k["params"] = params
    commit = a.commit or subprocess.run(["git", "-C", ROOT, "rev-parse", "--short", "HEAD"], capture_output=True,
                                        text=True).stdout.strip()
    out = {"config": a.config, "commit": commit, "captured": datetime.date.today().isoformat(),
           "source": os.path.relpath(a.raw, ROOT), "kernels": kernels,
           "how": "ncu --set full --clock-control none, one launch per kernel of a bench.py step; "
                  "dram__bytes_read.sum + dram__bytes_write.sum"}
    path = a.out or os.path.join(ROOT, "profiles", f"ncu_traffic_{a.config}.json")
    with open(path, "w") as f:
        json.dump(out, f, indent=1)
    print(json.dumps(out, indent=1))


if __name__ == "__main__":
    main()
