"""Inter-batch pipeline: LTPG_BATCH_ASYNC keeps two batches in flight;
aborted txns of batch n re-run in batch n+2 (the paper's schedule).  Results of every batch
must equal the oracle run on the same batch sequence."""
import numpy as np
import pytest

import oracle
from tests.test_gpu_ops import concat, select
from workloads import tpcc
from workloads.formats import ST_COMMIT, ST_CONFLICT
from workloads.ycsb import YcsbWorkload

pytestmark = pytest.mark.gpu


def L():
    import paper_conf_icde_wei0l0lzj024_b200 as lib
    return lib


def test_ycsb_pipeline_n_plus_2():
    wl = YcsbWorkload(20_000, theta=0.8, ops_per_txn=6, seed=44)
    keys, cols = wl.initial_table()
    g = L().ycsb_database(wl, max_txns=4096, max_ops=4096 * 6)
    o = oracle.ycsb_db(wl)
    B, tid = 3000, 1
    inflight, retry = [], {}
    for bno in range(10):
        pend = retry.pop(bno, None)
        fresh = wl.batch(B - (0 if pend is None else len(pend["tid"])), tid, bno)
        tid += len(fresh["tid"])
        batch = fresh if pend is None else concat(pend, fresh)
        inflight.append((bno, batch, g.run_ops(batch, wait=False)))
        if len(inflight) == 2 or bno == 9:
            while inflight and (len(inflight) == 2 or bno == 9):
                k, bk, p = inflight.pop(0)
                out = p.wait()
                rc, st, rd = o.run_ops(bk)
                assert rc == 0
                assert (out["status"] == st).all() and (out["reads"] == rd).all()
                assert (out["abort_idx"] == np.nonzero(st == ST_CONFLICT)[0]).all()
                ab = np.nonzero(st == ST_CONFLICT)[0]
                if len(ab):
                    retry[k + 2] = select(bk, ab)  # n+2: batch n+1 was already submitted
    gk, gc = g.dump_table(0)
    ok, oc = o.dump_table(0)
    assert (gk == ok).all() and (gc == oc).all()


def test_tpcc_pipeline_full_mix():
    wl = tpcc.TpccWorkload(2, seed=8, mode="strict", mix=tpcc.MIX_FULL)
    tables = wl.initial_tables()
    g = L().tpcc_database(wl, max_txns=2048, tables=tables, append_batches=10)
    o = oracle.tpcc_db(wl, tables)
    inflight = []
    for bno in range(8):
        b = wl.batch(2000, 1 + 2000 * bno, bno)
        inflight.append((b, 2 + bno, g.run_tpcc(b, 2 + bno, wait=False)))
        while len(inflight) == 2 or (bno == 7 and inflight):
            bk, clk, p = inflight.pop(0)
            out = p.wait()
            rc, st, res = o.run_tpcc(bk, clk)
            assert rc == 0 and (out["status"] == st).all()
            assert (out["reads"].reshape(-1, 4) == res).all()
    for t in range(9):
        gk, gc = g.dump_table(t)
        ok, oc = o.dump_table(t)
        assert (gc == oc).all(), t


def test_four_in_flight_rejected():
    wl = YcsbWorkload(1000, theta=0.5, ops_per_txn=4, seed=2)
    g = L().ycsb_database(wl, max_txns=512, max_ops=2048)
    b = [wl.batch(256, 1 + 256 * i, i) for i in range(4)]
    ps = [g.run_ops(b[i], wait=False) for i in range(3)]
    with pytest.raises(L().LtpgError):
        g.run_ops(b[3], wait=False)
    for p_ in ps:
        p_.wait()
    g.run_ops(b[3]).get("status")
