"""NEXT-4: YCSB core workloads A-E (Zipf alpha = 2.5, 10 ops per txn) on the GPU
OPS path -- reads, RMW updates, inserts of fresh keys, read-latest and short scans --
closed loop with retries, bit-exact against the oracle (status, reads, final table)."""
import numpy as np
import pytest

import oracle
from tests.test_gpu_ops import check_batch, concat, select
from workloads.formats import ST_CONFLICT
from workloads.ycsb import ycsb_letter

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("letter", ["A", "B", "C", "D", "E"])
def test_ycsb_letter_closed_loop(letter):
    import paper_conf_icde_wei0l0lzj024_b200 as lib
    wl = ycsb_letter(letter, 10_000, seed=0x17C0 + ord(letter))
    keys, cols = wl.initial_table()
    B = 2000
    g = lib.ycsb_database(wl, max_txns=B, max_ops=B * 10, capacity=len(keys) + 8 * B)
    o = oracle.ycsb_db(wl)
    pending, tid = None, 1
    for bno in range(5):
        fresh = wl.batch(B - (0 if pending is None else len(pending["tid"])), tid, bno)
        tid += len(fresh["tid"])
        batch = fresh if pending is None else concat(pending, fresh)
        st = check_batch(g, o, batch, {0: (keys, cols)})
        ab = np.nonzero(st == ST_CONFLICT)[0]
        pending = select(batch, ab) if len(ab) else None
