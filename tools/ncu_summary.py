#!/usr/bin/env python
"""Summarise ncu output into profiles/ (tracked).

    python tools/ncu_summary.py --launches gpurun_out/launches.csv \
        --full gpurun_out/prof.ncu-rep --out profiles/ncu_summary.json --tag r01_ycsb_c3

launches: CSV of `ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file ...`
          (cold-cache, serialised per-launch times: compare SHARES of the step, not absolutes)
full:     one `ncu --set full` capture; per kernel DRAM bytes, duration, throughput
"""
import argparse
import collections
import csv
import io
import json
import os
import subprocess

NCU = "/usr/local/cuda/bin/ncu"


def _rows(text):
    lines = [ln for ln in text.splitlines() if ln.startswith('"')]
    return list(csv.reader(io.StringIO("\n".join(lines))))


def parse_launches(path):
    rows = _rows(open(path).read())
    hdr = rows[0]
    ki = hdr.index("Kernel Name")
    mi = hdr.index("Metric Name")
    vi = hdr.index("Metric Value")
    ui = hdr.index("Metric Unit")
    agg = collections.OrderedDict()
    for r in rows[1:]:
        if len(r) <= vi or r[mi] != "gpu__time_duration.sum":
            continue
        v = float(r[vi].replace(",", ""))
        unit = r[ui]
        ns = v * TIME_UNITS.get(unit, 1.0)
        name = r[ki].split("(")[0]
        a = agg.setdefault(name, {"launches": 0, "total_ns": 0.0})
        a["launches"] += 1
        a["total_ns"] += ns
    tot = sum(a["total_ns"] for a in agg.values()) or 1.0
    for a in agg.values():
        a["share"] = a["total_ns"] / tot
        a["mean_ns"] = a["total_ns"] / a["launches"]
    return dict(sorted(agg.items(), key=lambda kv: -kv[1]["total_ns"])), tot


BYTE_UNITS = {"byte": 1.0, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12}
TIME_UNITS = {"ns": 1.0, "nsecond": 1.0, "us": 1e3, "usecond": 1e3, "ms": 1e6, "msecond": 1e6, "s": 1e9, "second": 1e9}

WANT = ["lts__t_sectors.sum", "lts__t_sectors_srcunit_ltcfabric.sum", "dram__sectors_read.sum",
        "dram__bytes_read.sum", "dram__bytes_write.sum", "gpu__time_duration.sum",
        "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "dram__throughput.avg.pct_of_peak_sustained_elapsed",
        "lts__t_bytes.sum", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
        "sm__warps_active.avg.pct_of_peak_sustained_active", "launch__registers_per_thread",
        "launch__grid_size", "launch__block_size", "l1tex__t_bytes.sum",
        "lts__t_sectors_srcunit_tex_op_red.sum", "lts__t_sectors_srcunit_tex_op_atom.sum",
        "smsp__inst_executed.sum"]


def parse_full(rep):
    text = subprocess.check_output([NCU, "-i", rep, "--page", "raw", "--csv"]).decode()
    rows = _rows(text)
    hdr, units = rows[0], rows[1]
    out = {}
    for r in rows[2:]:
        name = r[hdr.index("Kernel Name")].split("(")[0]
        d = {}
        for m in WANT:
            if m in hdr:
                i = hdr.index(m)
                try:
                    v = float(r[i].replace(",", ""))
                except ValueError:
                    continue
                u = units[i]
                v *= BYTE_UNITS.get(u, 1.0) * TIME_UNITS.get(u, 1.0)
                if u == "sector":
                    d[m + ".bytes"] = v * 32
                d[m] = v
        if "dram__bytes_read.sum" in d:
            d["dram_bytes"] = d["dram__bytes_read.sum"] + d.get("dram__bytes_write.sum", 0.0)
        out.setdefault(name, d)
    return out


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--launches")
    ap.add_argument("--full", nargs="*", default=[])
    ap.add_argument("--out", required=True)
    ap.add_argument("--tag", default="")
    ap.add_argument("--note", default="")
    ap.add_argument("--fresh", action="store_true", help="drop kernels of an existing summary")
    a = ap.parse_args()
    res = {"tag": a.tag, "note": a.note}
    if os.path.exists(a.out) and not a.fresh:
        old = json.load(open(a.out))
        res["kernels"] = old.get("kernels", {})
    else:
        res["kernels"] = {}
    if a.launches:
        res["launch_list"], res["launch_total_ns"] = parse_launches(a.launches)
    for rep in a.full:
        for k, v in parse_full(rep).items():
            res["kernels"][k] = v
    json.dump(res, open(a.out, "w"), indent=1, sort_keys=True)
    # human-readable companion
    md = [f"# ncu summary {a.tag}", "", a.note, ""]
    if a.launches:
        md += ["| kernel | launches | mean us | share of listed time |", "|---|---|---|---|"]
        for k, v in res["launch_list"].items():
            md.append(f"| {k} | {v['launches']} | {v['mean_ns'] / 1e3:.1f} | {100 * v['share']:.1f}% |")
    if res["kernels"]:
        md += ["", "| kernel (--set full) | dram bytes | duration us | dram % peak | L2 bytes |", "|---|---|---|---|---|"]
        for k, v in res["kernels"].items():
            md.append("| %s | %.3g | %.1f | %s | %.3g |" % (
                k, v.get("dram_bytes", float("nan")), v.get("gpu__time_duration.sum", 0) / 1e3,
                v.get("gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed",
                      v.get("dram__throughput.avg.pct_of_peak_sustained_elapsed", "?")),
                v.get("lts__t_sectors.sum", float("nan")) * 32))
    open(os.path.splitext(a.out)[0] + ".md", "w").write("\n".join(md) + "\n")
    print("\n".join(md))


if __name__ == "__main__":
    main()
