#!/usr/bin/env python
"""Table VIII on our store: share of the conflict-mark memory held by large-sized
buckets (LTPG_FLAG_LARGE_BUCKETS, NEXT-3) vs standard-sized marks, per warehouse count and batch
size, from what the library allocated (ltpg_mark_memory).  Needs a GPU.
    python tools/table8.py > profiles/table8_r02.json"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    import torch
    import paper_conf_icde_wei0l0lzj024_b200 as ltpg
    from workloads import tpcc
    from workloads.formats import TPCC_TABLE_NAMES
    torch.cuda.set_device(0)
    rows = []
    for W in (8, 16, 32, 64):
        wl = tpcc.TpccWorkload(W, seed=0x17C0 + W, mode="strict", mix=tpcc.MIX_NO_PAY)
        tables = wl.initial_tables()
        for B in (1 << 14, 1 << 16, 1 << 20):
            g = ltpg.tpcc_database(wl, max_txns=B, tables=tables, append_batches=1, flags=ltpg.LTPG_FLAG_LARGE_BUCKETS)
            std = large = 0
            per = {}
            for t in range(9):
                a, b, su = g.mark_memory(t)
                std += a
                large += b
                if b:
                    per[TPCC_TABLE_NAMES[t]] = {"s_u": su, "large_bytes": b}
            g.close()
            rows.append({"warehouses": W, "batch": B, "standard_bytes": std, "large_bytes": large,
                         "large_pct": 100.0 * large / (std + large), "standard_pct": 100.0 * std / (std + large),
                         "popular_tables": per})
            print("W=%d B=%d large %.3f%% (%s)" % (W, B, rows[-1]["large_pct"], per), file=sys.stderr)
    print(json.dumps({"table": "VIII", "note": "mark memory as allocated by ltpg_load_table with "
                      "LTPG_FLAG_LARGE_BUCKETS (buckets for tables with max_txns / rows > 1, <= 64 MB each); "
                      "standard = one 4-byte word per unit and kind (capacity rows incl. append regions)",
                      "rows": rows}, indent=1))


if __name__ == "__main__":
    main()
