#!/usr/bin/env python
"""Per-source-line stall-sample share of one kernel from an ncu report (compiled with -lineinfo).

    python tools/ncu_lines.py REPORT.ncu-rep KERNEL_INDEX [TOP]

KERNEL_INDEX: position of the launch in the report (0-based; ncu's csv repeats the first
function name on every section, so launches are told apart by order).
"""
import csv
import io
import subprocess
import sys


def main():
    rep, want = sys.argv[1], int(sys.argv[2])
    top = int(sys.argv[3]) if len(sys.argv) > 3 else 25
    text = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                          capture_output=True, text=True).stdout
    sec, hdr, agg, cur = -1, None, {}, None
    for r in csv.reader(io.StringIO(text)):
        if r and r[0] == "Line No":
            sec += 1
            hdr = r
            continue
        if sec != want or not hdr or not r:
            continue
        if r[0] and r[0].isdigit():  # a CUDA source line; following rows (empty line no) are its SASS
            cur = (int(r[0]), r[1][:110])
            continue
        if r[0] or cur is None:
            continue
        try:
            s = int(float(r[hdr.index("Warp Stall Sampling (All Samples)")]))
            lsb = int(float(r[hdr.index("stall_long_sb")]))
        except (ValueError, IndexError):
            continue
        a = agg.setdefault(cur, [0, 0])
        a[0] += s
        a[1] += lsb
    tot = sum(v[0] for v in agg.values()) or 1
    print("== launch", want, "samples", tot)
    for (ln, src), (s, l) in sorted(agg.items(), key=lambda kv: -kv[1][0])[:top]:
        print(f"{100 * s / tot:5.1f}% (long_sb {100 * l / tot:4.1f}%) L{ln}: {src.strip()}")


if __name__ == "__main__":
    main()
