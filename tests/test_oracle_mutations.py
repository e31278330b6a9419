"""The oracle's TPC-C read / result paths are pinned: every plausible one-line mistake of
tools/mutate_oracle.py in them turns tests/test_oracle_tpcc_pins.py red.  CPU only (g++).
(The full list, including the commit-rule mutants the other oracle pins catch, is run by
`python tools/mutate_oracle.py`; its output is committed as profiles/mutation_r02.txt.)"""
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

READ_PATH = ["sl_threshold_le", "sl_window_shift", "by_name_position", "os_sum_plus_one",
             "dl_total_plus_delivered", "sl_no_distinct", "sl_result_nx", "os_carrier_slot", "os_lines_short",
             "by_name_tie_desc", "dl_cursor_stays", "dl_no_delivery_cnt", "dl_date", "dl_empty_no_read",
             "pay_no_history_tid"]


def test_read_path_mutants_are_caught():
    p = subprocess.run([sys.executable, os.path.join(ROOT, "tools", "mutate_oracle.py"), "--only",
                        ",".join(READ_PATH), "--pins", "tests/test_oracle_tpcc_pins.py"],
                       cwd=ROOT, capture_output=True, text=True, timeout=900)
    lines = p.stdout.splitlines()
    assert lines and lines[0].split()[1] == "PASS", p.stdout + p.stderr
    verdict = {ln.split()[0]: ln.split()[1] for ln in lines[1:]}
    assert set(verdict) == set(READ_PATH), p.stdout
    assert all(v == "CAUGHT" for v in verdict.values()), p.stdout
    assert p.returncode == 0
