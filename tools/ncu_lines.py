#!/usr/bin/env python
"""Per-source-line stall-sample share of one kernel from an ncu report (compiled with -lineinfo).

    python tools/ncu_lines.py REPORT.ncu-rep KERNEL_SUBSTRING [TOP]
"""
import csv
import io
import subprocess
import sys


def main():
    rep, want = sys.argv[1], sys.argv[2]
    top = int(sys.argv[3]) if len(sys.argv) > 3 else 25
    text = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                          capture_output=True, text=True).stdout
    fn, hdr, agg = None, None, {}
    for r in csv.reader(io.StringIO(text)):
        if len(r) >= 2 and r[0] == "Function Name":
            fn = r[1]
            continue
        if r and r[0] == "Line No":
            hdr = r
            continue
        if hdr and r and r[0] and fn:
            try:
                si = hdr.index("Warp Stall Sampling (All Samples)") if "Warp Stall Sampling (All Samples)" in hdr else 4
                s = int(float(r[si]))
            except (ValueError, IndexError):
                continue
            agg.setdefault(fn, []).append((s, int(r[0]), r[1][:110]))
    for f, v in agg.items():
        if want not in f:
            continue
        tot = sum(x[0] for x in v) or 1
        print("==", f[:80], "samples", tot)
        for s, ln, src in sorted(v, reverse=True)[:top]:
            print(f"{100 * s / tot:5.1f}% L{ln}: {src.strip()}")


if __name__ == "__main__":
    main()
