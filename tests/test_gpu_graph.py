"""GPU: batch graphs (capi.cu) -- a batch's device work captured once per shape and replayed
with the next batches' epoch / clock from device memory -- give exactly the results of
kernel-by-kernel enqueueing (the default) and of the oracle, across replays, shape
changes, the slot rotation of the pipeline and device-resident buffers that are reused."""
import numpy as np
import pytest

import oracle
from tests.test_gpu_fullsize import _retry_batch
from workloads import tpcc
from workloads.formats import ST_COMMIT
from workloads.ycsb import YcsbWorkload

pytestmark = pytest.mark.gpu


def L():
    import paper_conf_icde_wei0l0lzj024_b200 as lib
    return lib


def _host(out, n):
    return {k: (v.cpu().numpy() if hasattr(v, "cpu") else v) for k, v in out.items() if k != "stats"}


def test_ycsb_graph_replay_device_buffers():
    """Fixed-shape closed loop with device inputs staged in two reused buffers (the graph key
    repeats, so slots replay), one shape change in the middle (recapture), vs direct enqueueing + oracle."""
    import torch
    wl = YcsbWorkload(20_000, theta=0.5, ops_per_txn=4, seed=11)
    dbs = [L().ycsb_database(wl, max_txns=2048, max_ops=8192, flags=f) for f in (L().LTPG_FLAG_GRAPH, 0)]
    o = oracle.ycsb_db(wl)
    dev = torch.device("cuda", 0)
    bufs = [{k: torch.empty(n, dtype=torch.uint8, device=dev)
             for k, n in (("tid", 8 * 2048), ("op_begin", 4 * 2049), ("ops", 16 * 8192), ("args", 8 * 8192))}
            for _ in range(2)]
    B = 1024
    batch, tid = wl.batch(B, 1, 0), 1 + B
    kern = []
    for bno in range(14):
        if bno == 7:  # shape change: a smaller batch, then back
            B = 900
        if bno == 9:
            B = 1024
        rc, ost, ores = o.run_ops(batch)
        assert rc == 0
        buf = bufs[bno % 2]
        n, m = len(batch["tid"]), len(batch["args"])
        for k in ("tid", "op_begin", "ops", "args"):
            a = np.ascontiguousarray(batch[k]).view(np.uint8)
            buf[k][:len(a)].copy_(torch.from_numpy(a))
        for db in dbs:
            out = db.run_ops(buf, n_txns=n, n_ops=m, device_out=False, stats=True)
            assert (out["status"] == ost).all(), (bno, np.nonzero(out["status"] != ost)[0][:5])
            assert (out["reads"] == ores).all(), bno
            kern.append(out["stats"]["n_kernels"])
        assert kern[-1] == kern[-2]  # replay counts the captured launches
        batch, tid = _retry_batch(wl, batch, ost, B, tid, bno + 1)
    gk, gc = dbs[0].dump_table(0)
    ok, oc = o.dump_table(0)
    assert (gk == ok).all() and (gc == oc).all()
    dk, dc = dbs[1].dump_table(0)
    assert (dk == ok).all() and (dc == oc).all()


@pytest.mark.parametrize("mode", ["strict", "delayed"])
def test_tpcc_graph_replay_closed_loop(mode):
    """TPC-C full mix, fixed batch size (replays on every slot), host inputs, stats on and
    off (one graph serves both), vs direct enqueueing and the oracle; CC on the final state."""
    from tests.test_gpu_tpcc import compare_tables
    from tests import tpcc_cc
    wl = tpcc.TpccWorkload(2, seed=9, mode=mode, mix=tpcc.MIX_FULL)
    tables = wl.initial_tables()
    dbs = [L().tpcc_database(wl, max_txns=2048, tables=tables, append_batches=12, flags=f)
           for f in (L().LTPG_FLAG_GRAPH, 0)]
    o = oracle.tpcc_db(wl, tables)
    B = 2048
    batch, tid = wl.batch(B, 1, 0), 1 + B
    for bno in range(10):
        rc, ost, ores = o.run_tpcc(batch, 2 + bno)
        assert rc == 0
        for db in dbs:
            out = db.run_tpcc(batch, 2 + bno, stats=bool(bno % 3))
            assert (out["status"] == ost).all(), (bno, np.nonzero(out["status"] != ost)[0][:5])
            assert (out["reads"] == ores).all(), bno
        assert 0 < (ost == ST_COMMIT).sum()
        batch, tid = _retry_batch(wl, batch, ost, B, tid, bno + 1)
    dumps = compare_tables(dbs[0], o)
    compare_tables(dbs[1], o)
    cc = tpcc_cc.check(dumps)
    assert all(cc.values()), cc
