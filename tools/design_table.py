#!/usr/bin/env python
"""Markdown table of bench lines for DESIGN.md:  python tools/design_table.py TAG [DIR]
(reads DIR/bench_TAG_<workload>.json, DIR defaults to profiles/)."""
import json
import os
import sys

ROWS = [("default", "tpcc_c4 strict — **default** (2²⁰ txns, 64 wh, full mix)"),
        ("tpcc_c4_delayed", "tpcc_c4 delayed"), ("tpcc_c4_opt", "tpcc_c4 delayed + reorder (NEXT-1)"),
        ("tpcc_c5", "tpcc_c5 shape on 1 GPU (512 wh, NO/Pay, 2²⁰)"),
        ("ycsb_c3", "ycsb_c3 (10⁷ rows, 2²⁰×10 ops, θ=0.99)"), ("ycsb_c3_4ops", "ycsb_c3, 4 ops"),
        ("ycsb_c3_sparse", "ycsb_c3 sparse keys (hash-index probes)"),
        ("tpcc_c2", "tpcc_c2 (1 wh, NO/Pay, 16 k) — single launch"),
        ("tpcc_c2_opt", "tpcc_c2 delayed + reorder — single launch"),
        ("ycsb_c1", "ycsb_c1 (10⁴ rows, 1024×4) — single launch"), ("ycsb_e", "ycsb_e (NEXT-4, 2¹⁶ txns)")]


def si(v):
    for d, s in ((1e9, " G"), (1e6, " M"), (1e3, " K")):
        if abs(v) >= d:
            return "%.3g%s" % (v / d, s)
    return "%.3g" % v


def main():
    tag = sys.argv[1]
    d0 = sys.argv[2] if len(sys.argv) > 2 else "profiles"
    print("| workload | ms/step | committed txn/s | e2e txn/s | closed loop e2e | processed txn/s | commit rate | dominant kernel (ms) | roofline frac |")
    print("|---|---|---|---|---|---|---|---|---|")
    for w, label in ROWS:
        p = os.path.join(d0, "bench_%s_%s.json" % (tag, w))
        if not os.path.exists(p):
            continue
        d = json.load(open(p))
        r = d.get("roofline") or {}
        e = (d.get("e2e") or {}).get("value")
        c = (d.get("closed_loop_e2e") or {}).get("value")
        single = "small" in r.get("kernel", "")
        frac = ("%.3f (execute bytes / whole launch; latency-bound, §6b)" % r["frac"]) if single else "%.3f" % r.get("frac", 0)
        kern = "`%s` %.3f" % (r.get("kernel", "?"), r.get("kernel_ms", 0))
        print("| %s | %.4f | %s | %s | %s | %s | %.3g | %s | %s |" % (
            label, d["ms_per_step"], si(d["value"]), si(e) if e else "—", si(c) if c else "—",
            si(d.get("processed_txns_per_s", 0)), d.get("commit_rate", 0), kern, frac))


if __name__ == "__main__":
    main()
