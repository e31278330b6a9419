#!/usr/bin/env python
"""Mutation check of the oracle's pins (test infrastructure).

Applies plausible one-line mistakes to oracle/ltpg_oracle.cpp, one at a time, builds each
mutant into a scratch .so, and runs the oracle's CPU pins (tests/test_oracle_*.py) against it
through LTPG_ORACLE_LIB.  A mutant the pins do not catch ("SURVIVED") means part of the oracle
is not pinned by anything independent of it.  Exit status 1 if any mutant survives or the
unmutated oracle fails its pins.

    python tools/mutate_oracle.py [--only NAME,...] [--list]
"""
import argparse
import concurrent.futures
import os
import subprocess
import sys
import tempfile

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
SRC = os.path.join(ROOT, "oracle", "ltpg_oracle.cpp")
PINS = ["tests/test_oracle_tpcc_pins.py", "tests/test_oracle_tpcc.py", "tests/test_oracle_ops.py"]

# (name, what the mistake is, exact source text, replacement)
MUTATIONS = [
    # the five mistakes the round-1 review found unpinned
    ("sl_threshold_le", "StockLevel counts S_QUANTITY <= threshold",
     "if (x.get(TS, sk, S_QUANTITY) < thr) ++low;", "if (x.get(TS, sk, S_QUANTITY) <= thr) ++low;"),
    ("sl_window_shift", "StockLevel window [nx-21, nx-1) instead of [nx-20, nx)",
     "for (int64_t o = nx - 20; o < nx; ++o) {", "for (int64_t o = nx - 21; o < nx - 1; ++o) {"),
    ("by_name_position", "by-name customer at position (n+2)/2 instead of ceil(n/2)",
     "size_t pos = (v.size() + 1) / 2;", "size_t pos = (v.size() + 2) / 2;"),
    ("os_sum_plus_one", "OrderStatus sum of OL_DELIVERY_D off by one",
     "res[3] = sum_dd;", "res[3] = sum_dd + 1;"),
    ("dl_total_plus_delivered", "Delivery total adds the delivered count",
     "res[1] = total;", "res[1] = total + delivered;"),
    # more of the same kind
    ("sl_no_distinct", "StockLevel counts repeated items once per line",
     "items.erase(std::unique(items.begin(), items.end()), items.end());", ""),
    ("sl_result_nx", "StockLevel second slot reports nx - 1",
     "res[1] = nx;", "res[1] = nx - 1;"),
    ("os_carrier_slot", "OrderStatus reports O_OL_CNT as the carrier",
     "int64_t carrier = x.get(TO, ok, O_CARRIER_ID);", "int64_t carrier = x.get(TO, ok, O_OL_CNT);"),
    ("os_lines_short", "OrderStatus skips the order's last line",
     "for (int64_t l = 1; l <= cnt; ++l) {\n    uint64_t lk = key_ol(w, d, o, uint64_t(l));\n    sum_dd",
     "for (int64_t l = 1; l < cnt; ++l) {\n    uint64_t lk = key_ol(w, d, o, uint64_t(l));\n    sum_dd"),
    ("by_name_tie_desc", "by-name ties on C_FIRST broken by descending c_id",
     "std::sort(v.begin(), v.end());\n    size_t pos",
     "std::sort(v.begin(), v.end(), [](const std::pair<int64_t, int64_t>& a, const std::pair<int64_t, int64_t>& b) "
     "{ return a.first != b.first ? a.first < b.first : a.second > b.second; });\n    size_t pos"),
    ("dl_cursor_stays", "Delivery leaves the cursor on the delivered order",
     "x.set(TD, dk, D_NEXT_DELIV_O_ID, o + 1);", "x.set(TD, dk, D_NEXT_DELIV_O_ID, o);"),
    ("dl_no_delivery_cnt", "Delivery does not count the customer's deliveries",
     "x.upd_add(TC, ck, C_DELIVERY_CNT, 1);", "x.upd_add(TC, ck, C_DELIVERY_CNT, 0);"),
    ("dl_date", "Delivery stamps OL_DELIVERY_D with clock + 1",
     "x.set(TOL, lk, OL_DELIVERY_D, x.clock);", "x.set(TOL, lk, OL_DELIVERY_D, x.clock + 1);"),
    ("dl_empty_no_read", "Delivery on an empty queue does not read the D_NEXT_O_ID unit",
     "x.acc(TD, dk, x.grp(TD, D_NEXT_O_ID), ACC_R);\n      x.set", "x.set"),
    ("no_total_disc", "NewOrder total ignores the customer discount",
     "res[1] = sum_amount * (10000 - disc) * (10000 + w_tax + d_tax) / 100000000;",
     "res[1] = sum_amount * 10000 * (10000 + w_tax + d_tax) / 100000000;"),
    ("pay_no_history_tid", "Payment HISTORY row stores 0 as the TID",
     "int64_t(x.tid), 0}});", "0, 0}});"),
    # commit rule (R1) and delayed update (R7)
    ("rule_raw_ignores_adds", "a read ignores smaller-rank ADDs (RAW on adds missed)",
     "if (a.acc == ACC_R) {\n        if (std::min(w, ad) < r) raw = true;",
     "if (a.acc == ACC_R) {\n        if (w < r) raw = true;"),
    ("rule_add_vs_write", "an ADD ignores a smaller-rank plain write",
     "} else {\n        if (w < r) waw = true;", "} else {\n        if (false) waw = true;"),
    ("rule_le", "a txn conflicts with its own marks (<= instead of <)",
     "} else if (a.acc == ACC_W) {\n        if (std::min(w, ad) < r) waw = true;",
     "} else if (a.acc == ACC_W) {\n        if (std::min(w, ad) <= r) waw = true;"),
    ("fetch_add_order", "o_id pre-image taken after the increment",
     "results[4ull * r] = o;", "results[4ull * r] = o + 1;"),
]


def build(src_text, out):
    with tempfile.NamedTemporaryFile("w", suffix=".cpp", delete=False) as f:
        f.write(src_text)
        path = f.name
    try:
        subprocess.check_call(["g++", "-O1", "-std=c++17", "-shared", "-fPIC", path, "-o", out])
    finally:
        os.unlink(path)


def run_pins(lib, pins):
    env = dict(os.environ, LTPG_ORACLE_LIB=lib)
    p = subprocess.run([sys.executable, "-m", "pytest", "-x", "-q", "-p", "no:cacheprovider"] + pins,
                       cwd=ROOT, env=env, capture_output=True, text=True)
    tail = [ln for ln in p.stdout.splitlines() if ln.strip()][-1:] or [""]
    first_fail = next((ln for ln in p.stdout.splitlines() if ln.startswith("FAILED")), "")
    return p.returncode, tail[0], first_fail


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--only", default="")
    ap.add_argument("--list", action="store_true")
    ap.add_argument("--jobs", type=int, default=max(1, (os.cpu_count() or 2) // 2))
    ap.add_argument("--pins", default=",".join(PINS), help="test files to run against each mutant")
    args = ap.parse_args()
    if args.list:
        for name, what, _, _ in MUTATIONS:
            print("%-24s %s" % (name, what))
        return 0
    src = open(SRC).read()
    only = set(filter(None, args.only.split(",")))
    tmp = tempfile.mkdtemp(prefix="ltpg_mut_")
    base = os.path.join(tmp, "base.so")
    build(src, base)
    pins = args.pins.split(",")
    rc, tail, _ = run_pins(base, pins)
    print("%-24s %-8s %s" % ("(unmutated)", "PASS" if rc == 0 else "FAIL", tail), flush=True)
    bad = rc != 0
    todo = [m for m in MUTATIONS if not only or m[0] in only]

    def one(m):
        name, what, old, new = m
        n = src.count(old)
        if n != 1:
            return name, "BROKEN", "pattern found %d times" % n
        lib = os.path.join(tmp, name + ".so")
        build(src.replace(old, new), lib)
        rc, tail, first = run_pins(lib, pins)
        return name, "CAUGHT" if rc != 0 else "SURVIVED", "%s | %s" % (what, first.replace("FAILED ", "") or tail)

    with concurrent.futures.ThreadPoolExecutor(max_workers=args.jobs) as ex:
        for name, verdict, msg in ex.map(one, todo):
            bad |= verdict != "CAUGHT"
            print("%-24s %-8s %s" % (name, verdict, msg), flush=True)
    return 1 if bad else 0


if __name__ == "__main__":
    sys.exit(main())
