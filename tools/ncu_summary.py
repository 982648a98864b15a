"""Summarise ncu outputs into profiles/ (tracked): key metrics of one `--set full`
capture, the kernel's top stall lines, and per-kernel shares of a launch list.

  python tools/ncu_summary.py --rep gpurun_out/prof.ncu-rep --launches gpurun_out/launches.csv \
      --alg-bytes 8547844000 --out profiles/r01_c5
"""
import argparse
import csv
import io
import json
import subprocess
from collections import defaultdict

KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "dram__throughput.avg.pct_of_peak_sustained_elapsed", "lts__throughput.avg.pct_of_peak_sustained_elapsed",
        "lts__t_sector_hit_rate.pct", "l1tex__t_sector_hit_rate.pct",
        "l1tex__m_l1tex2xbar_req_cycles_active.avg.pct_of_peak_sustained_elapsed",
        "l1tex__data_pipe_lsu_wavefronts.avg.pct_of_peak_sustained_elapsed",
        "sm__throughput.avg.pct_of_peak_sustained_elapsed", "sm__warps_active.avg.per_cycle_active",
        "launch__registers_per_thread", "launch__grid_size", "launch__block_size",
        "launch__occupancy_limit_registers", "smsp__issue_active.avg.pct_of_peak_sustained_active"]


def ncu_csv(args):
    out = subprocess.run(["ncu"] + args, capture_output=True, text=True).stdout
    return list(csv.reader(io.StringIO(out)))


def to_bytes(v, unit):
    f = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12}.get(unit)
    return v * f if f else v


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--rep")
    ap.add_argument("--launches")
    ap.add_argument("--alg-bytes", type=float, default=0)
    ap.add_argument("--out", required=True)
    ap.add_argument("--title", default="")
    a = ap.parse_args()
    summ = {"title": a.title}
    lines = [f"# {a.title}", ""]
    if a.rep:
        rows = ncu_csv(["-i", a.rep, "--page", "raw", "--csv"])
        hdr, units, vals = rows[0], rows[1], rows[2]
        m = {}
        for i, h in enumerate(hdr):
            if h in KEYS:
                try:
                    m[h] = (float(vals[i].replace(",", "")), units[i])
                except ValueError:
                    m[h] = (vals[i], units[i])
        kname = vals[hdr.index("Kernel Name")] if "Kernel Name" in hdr else ""
        summ["kernel"] = kname
        summ["metrics"] = {k: {"value": v, "unit": u} for k, (v, u) in m.items()}
        dur_ms = m["gpu__time_duration.sum"][0] * {"ms": 1, "us": 1e-3, "ns": 1e-6}.get(m["gpu__time_duration.sum"][1], 1)
        rd = to_bytes(*m["dram__bytes_read.sum"])
        wr = to_bytes(*m["dram__bytes_write.sum"])
        summ["dram_bytes_per_launch"] = rd + wr
        summ["duration_ms_ncu"] = dur_ms
        lines += [f"kernel: `{kname}`", "", "| metric | value |", "|---|---|"]
        for k in KEYS:
            if k in m:
                lines.append(f"| {k} | {m[k][0]} {m[k][1]} |")
        lines += ["", f"DRAM traffic per launch: {(rd + wr) / 1e9:.3f} GB (read {rd / 1e9:.3f}, write {wr / 1e9:.3f})"]
        if a.alg_bytes:
            summ["alg_bytes"] = a.alg_bytes
            lines.append(f"algorithmic bytes per launch: {a.alg_bytes / 1e9:.3f} GB -> traffic/alg = {(rd + wr) / a.alg_bytes:.2f}")
            lines.append(f"ncu (cold, serialised) achieved alg GB/s: {a.alg_bytes / (dur_ms * 1e-3) / 1e9:.1f}")
        # stall breakdown
        src = ncu_csv(["-i", a.rep, "--page", "source", "--csv", "--print-source", "sass"])
        shdr = src[1]
        data = src[2:]
        ix = {h: i for i, h in enumerate(shdr)}
        S = "Warp Stall Sampling (All Samples)"
        if S in ix:
            tot = sum(float(r[ix[S]] or 0) for r in data) or 1.0
            stalls = [h for h in shdr if h.startswith("stall_") and "Not Issued" not in h]
            agg = {h: sum(float(r[ix[h]] or 0) for r in data) / tot for h in stalls}
            top = sorted(agg.items(), key=lambda kv: -kv[1])[:8]
            summ["stalls"] = dict(top)
            lines += ["", "## warp stall reasons (share of samples)", ""]
            lines += [f"- {k}: {v * 100:.1f}%" for k, v in top]
            lines += ["", "## top SASS lines by stall samples", "", "| share | sass | top reason |", "|---|---|---|"]
            for r in sorted(data, key=lambda r: -float(r[ix[S]] or 0))[:12]:
                s = float(r[ix[S]] or 0) / tot
                rs = max(stalls, key=lambda h: float(r[ix[h]] or 0))
                lines.append(f"| {s * 100:.1f}% | `{r[1][:70]}` | {rs} |")
    if a.launches:
        rows = list(csv.reader(open(a.launches)))
        hi = [i for i, r in enumerate(rows) if "Kernel Name" in r][0]
        hdr = rows[hi]
        ix = {h: i for i, h in enumerate(hdr)}
        agg = defaultdict(lambda: [0, 0.0])
        for r in rows[hi + 1:]:
            if r[ix["Metric Name"]] != "gpu__time_duration.sum":
                continue
            v = float(r[ix["Metric Value"]].replace(",", ""))
            v *= {"ms": 1e3, "us": 1.0, "ns": 1e-3}.get(r[ix["Metric Unit"]], 1.0)
            k = r[ix["Kernel Name"]].split("(")[0][:90]
            agg[k][0] += 1
            agg[k][1] += v
        tot = sum(v[1] for v in agg.values()) or 1.0
        summ["launch_shares"] = {k: {"launches": n, "us": us, "share": us / tot} for k, (n, us) in agg.items()}
        lines += ["", "## launch list (ncu, cold-cache, serialised: compare shares)", "",
                  "| launches | total us | share | kernel |", "|---|---|---|---|"]
        for k, (n, us) in sorted(agg.items(), key=lambda kv: -kv[1][1]):
            lines.append(f"| {n} | {us:.1f} | {us / tot * 100:.1f}% | `{k}` |")
    open(a.out + ".md", "w").write("\n".join(lines) + "\n")
    json.dump(summ, open(a.out + ".json", "w"), indent=1)
    print("\n".join(lines))


if __name__ == "__main__":
    main()
