"""NewOrder rollback (R11: an unused item id -> user abort, status 2; its marks still count,
P:106 / R2; it is not retried) on the CUDA path == oracle: strict and delayed mode, with and
without NEXT-1 reordering, one and two (loopback) partitions, rollback rates 1% and 100%.
Status precedence: a conflict-aborted txn reports 0 even if it would also
user-abort."""
import numpy as np
import pytest

import oracle
from tests import tpcc_cc
from tests.test_gpu_tpcc import compare, compare_tables
from workloads import tpcc
from workloads.formats import ST_CONFLICT, ST_USER_ABORT, NEW_ORDER

pytestmark = pytest.mark.gpu


def L():
    import paper_conf_icde_wei0l0lzj024_b200 as lib
    return lib


@pytest.mark.parametrize("parts", [1, 2])
@pytest.mark.parametrize("reorder", [False, True])
@pytest.mark.parametrize("mode", ["strict", "delayed"])
@pytest.mark.parametrize("frac", [0.01, 1.0])
def test_neworder_rollback_closed_loop(frac, mode, reorder, parts):
    lib = L()
    W, B = 2, 2000
    wl = tpcc.TpccWorkload(W, seed=41, mode=mode, mix=tpcc.MIX_FULL, rollback_frac=frac,
                           remote_line_frac=0.1)
    tables = wl.initial_tables()
    g = lib.tpcc_database(wl, max_txns=B, tables=tables, append_batches=5, loopback=parts,
                          flags=lib.LTPG_FLAG_REORDER if reorder else 0)
    o = oracle.tpcc_db(wl, tables)
    o.set_reorder(reorder)
    pending, tid, n_ua = None, 1, 0
    for bno in range(4):
        fresh = wl.batch(B - (0 if pending is None else len(pending["tid"])), tid, bno)
        tid += len(fresh["tid"])
        batch = fresh if pending is None else {k: np.concatenate([pending[k], fresh[k]]) for k in fresh}
        st = compare(g, o, batch, 2 + bno)
        ua = st == ST_USER_ABORT
        n_ua += int(ua.sum())
        assert (batch["type"][ua] == NEW_ORDER).all()   # only NewOrder rolls back
        ab = np.nonzero(st == ST_CONFLICT)[0]
        pending = {k: v[ab] for k, v in batch.items()} if len(ab) else None
    assert n_ua > 0
    dumps = compare_tables(g, o)
    assert all(tpcc_cc.check(dumps).values())


def test_rollback_every_neworder_rank0_user_aborts():
    """Rank 0 is a rolled-back NewOrder: status 2 (it conflicts with nothing smaller), o_id 0,
    and its stock marks still abort a later NewOrder on the same stock row (R2)."""
    lib = L()
    wl = tpcc.TpccWorkload(1, seed=4, rollback_frac=1.0)
    tables = wl.initial_tables()
    g = lib.tpcc_database(wl, max_txns=64, tables=tables, append_batches=2)
    o = oracle.tpcc_db(wl, tables)
    b = wl.batch(2, 1, 0, types=[NEW_ORDER, NEW_ORDER])
    b["params"][1, 3] = 1                                      # txn 1: a single line ...
    b["params"][1, 8:16] = b["params"][0, 8:16]                # ... on txn 0's first stock row
    b["params"][1, 6] = 0                                      # no rollback flag (its item exists)
    st = compare(g, o, b, 2)
    assert list(st) == [ST_USER_ABORT, ST_CONFLICT]
    compare_tables(g, o)
