"""GPU parity at BASELINE.json's full sizes, in the launch configuration bench.py times.

The database is opened by `bench.open_database` (same append capacities and flags as the
bench), inputs and outputs are device-resident tensors handed to the C-ABI exactly as the
bench's timed leg does, and the batch shapes are the bench's: 2^20 txns.  The CPU oracle is
fast enough to compute every output of these batches, so the comparison is complete
(not sampled): status, commit bitmask, abort list and every result slot of two consecutive
batches (a fresh batch, then its aborted txns + fresh txns, with the state of the first
carried over), then every table's canonical dump -- bit-exact.

configs[0] (YCSB 10k rows, 1024 x 4 ops) and configs[1] (TPC-C 1 warehouse, 16k; strict and
delayed + NEXT-1) -- one cooperative launch each in the bench --, configs[2] (YCSB 10M rows, 2^20
x 10 ops, zipf 0.99) and configs[3] (TPC-C 64 warehouses, full mix, 2^20; strict, delayed,
delayed + NEXT-1) against the oracle; configs[4] (512 warehouses, 2^20) by the partition
invariance PIN-8 at full size (one partition vs eight loopback partitions, every output and the
WAREHOUSE / DISTRICT state equal) plus CC1, and -- opt-in, LTPG_FULL_C5=1 on a box with the host
RAM for it -- against the oracle like the others.
"""
import numpy as np
import pytest

import bench
import oracle
from tests import tpcc_cc
from workloads.formats import ST_COMMIT, ST_CONFLICT, T_WAREHOUSE, T_DISTRICT

pytestmark = pytest.mark.gpu


def _to_dev(batch):
    import torch
    dev = torch.device("cuda", torch.cuda.current_device())
    return {k: (torch.from_numpy(np.ascontiguousarray(v).view(np.uint8).copy()).to(dev)
                if isinstance(v, np.ndarray) else v) for k, v in batch.items()}


def _run_dev(db, kind, batch, clock):
    """One batch the way bench.py's device-resident leg runs it; outputs copied back."""
    import torch
    n = len(batch["tid"])
    n_reads = len(batch["args"]) if kind == "ycsb" else 4 * n
    out = db._outputs(n, n_reads, True)
    bd = _to_dev(batch)
    s = torch.cuda.current_stream().cuda_stream
    if kind == "ycsb":
        db.run_ops(bd, stream=s, want_reads=True, device_out=True, n_txns=n, n_ops=n_reads, out=out)
    else:
        db.run_tpcc(bd, clock, stream=s, want_reads=True, device_out=True, n_txns=n, out=out)
    torch.cuda.synchronize()
    na = int(out["n_aborted"].cpu()[0])
    h = {"status": out["status"].cpu().numpy(), "commit_bits": out["commit_bits"].cpu().numpy().view(np.uint32),
         "abort_idx": out["abort_idx"].cpu().numpy().view(np.uint32)[:na],
         "reads": out["reads"].cpu().numpy()[:n_reads]}
    if kind == "tpcc":
        h["reads"] = h["reads"].reshape(n, 4)
    return h


def _check_outputs(g, ost, ores):
    bad = np.nonzero(g["status"] != ost)[0]
    assert len(bad) == 0, ("status", bad[:10], g["status"][bad[:10]], ost[bad[:10]])
    exp_bits = np.packbits((ost == ST_COMMIT).astype(np.uint8), bitorder="little")
    exp_bits = np.pad(exp_bits, (0, 4 * len(g["commit_bits"]) - len(exp_bits))).view(np.uint32)
    assert (g["commit_bits"] == exp_bits).all()
    assert (g["abort_idx"] == np.nonzero(ost == ST_CONFLICT)[0]).all()
    diff = np.nonzero(g["reads"] != ores)[0]
    assert len(diff) == 0, ("reads", diff[:10])


def _select_ops(batch, idx):
    """Txns idx of an OPS batch (CSR op lists), vectorised."""
    ob = batch["op_begin"].astype(np.int64)
    lens = ob[idx + 1] - ob[idx]
    starts = np.concatenate([[0], np.cumsum(lens)])
    sel = np.repeat(ob[idx] - starts[:-1], lens) + np.arange(starts[-1])
    return {"tid": batch["tid"][idx], "ops": batch["ops"][sel], "args": batch["args"][sel],
            "op_begin": starts.astype(np.uint32)}


def _retry_batch(wl, batch, status, B, tid, bno):
    """Next batch of the closed loop (a9): this batch's conflict aborts, original TIDs first,
    then fresh txns up to B."""
    ab = np.nonzero(status == ST_CONFLICT)[0]
    fresh = wl.batch(B - len(ab), tid, bno)
    if "op_begin" in batch:
        a = _select_ops(batch, ab)
        nxt = {"tid": np.concatenate([a["tid"], fresh["tid"]]), "ops": np.concatenate([a["ops"], fresh["ops"]]),
               "args": np.concatenate([a["args"], fresh["args"]]),
               "op_begin": np.concatenate([a["op_begin"], fresh["op_begin"][1:] + a["op_begin"][-1]]).astype(np.uint32)}
    else:
        nxt = {k: np.concatenate([batch[k][ab], fresh[k]]) for k in fresh}
    return nxt, tid + len(fresh["tid"])


def _c5_enabled():
    """configs[4] against the oracle needs ~35 GB of host RAM and ~10 minutes: opt-in
    (LTPG_FULL_C5=1; its log is committed as profiles/fullsize_c5_r02.txt)."""
    import os
    if os.environ.get("LTPG_FULL_C5") != "1":
        return False
    try:
        return os.sysconf("SC_PAGE_SIZE") * os.sysconf("SC_PHYS_PAGES") > 100 << 30
    except (ValueError, OSError):
        return False


# (ycsb_c1 / tpcc_c2 / tpcc_c2_opt: BASELINE configs[0] and [1], which the bench runs as ONE
# cooperative launch -- the single-launch path in the bench's own launch configuration)
@pytest.mark.parametrize("name", ["ycsb_c1", "tpcc_c2", "tpcc_c2_opt", "ycsb_c3", "tpcc_c4", "tpcc_c4_delayed",
                                  "tpcc_c4_opt",
                                  pytest.param("tpcc_c5", marks=pytest.mark.skipif(
                                      not _c5_enabled(), reason="opt-in: LTPG_FULL_C5=1 and > 100 GB host RAM"))])
def test_full_size_equals_oracle(name):
    w = bench.WORKLOADS[name]
    kind, B = w["kind"], w["batch"]
    wl = bench.make_workload(name)
    db = bench.open_database(name, wl, 4)
    if kind == "ycsb":
        o = oracle.ycsb_db(wl)
        tables = [0]
    else:
        o = oracle.tpcc_db(wl, wl.initial_tables())
        tables = list(range(9))
    if w.get("reorder"):
        o.set_reorder(True)
    batch = wl.batch(B, 1, 0)
    tid = 1 + B
    for bno in range(2):
        if kind == "ycsb":
            rc, ost, ores = o.run_ops(batch)
        else:
            rc, ost, ores = o.run_tpcc(batch, 2 + bno)
        assert rc == 0
        g = _run_dev(db, kind, batch, 2 + bno)
        _check_outputs(g, ost, ores)
        if bno == 0:
            assert 0 < (ost == ST_COMMIT).sum() < B  # both paths exercised at full size
            batch, tid = _retry_batch(wl, batch, ost, B, tid, bno + 1)
    dumps = {}
    for t in tables:
        gk, gc = db.dump_table(t)
        ok, oc = o.dump_table(t)
        assert gc.shape == oc.shape, (t, gc.shape, oc.shape)
        if ok is not None:
            assert (gk == ok).all(), t
        assert (gc == oc).all(), (t, np.nonzero((gc != oc).any(axis=0))[0][:5])
        dumps[t] = (gk, gc)
        del ok, oc
    if kind == "tpcc":
        cc = tpcc_cc.check(dumps)
        assert all(cc.values()), cc
    db.close()
    o.close()


def test_c5_full_size_partition_invariance():
    """configs[4] shape (512 warehouses, NewOrder/Payment, 2^20 txns): one partition and
    eight loopback partitions (the multi-GPU gating and exchange, §8(e)) give identical
    verdicts, results and WAREHOUSE / DISTRICT state on two consecutive batches; CC1 holds."""
    name = "tpcc_c5"
    B = bench.WORKLOADS[name]["batch"]
    wl = bench.make_workload(name)
    outs = []
    for loop in (1, 8):
        db = bench.open_database(name, wl, 3, loopback=loop)
        batch = wl.batch(B, 1, 0)
        tid = 1 + B
        got = []
        for bno in range(2):
            g = _run_dev(db, "tpcc", batch, 2 + bno)
            got.append(g)
            if bno == 0:
                batch, tid = _retry_batch(wl, batch, g["status"], B, tid, bno + 1)
        got.append({t: db.dump_table(t) for t in (T_WAREHOUSE, T_DISTRICT)})
        db.close()
        outs.append(got)
    a, b = outs
    for bno in range(2):
        for k in ("status", "commit_bits", "abort_idx", "reads"):
            assert (a[bno][k] == b[bno][k]).all(), (bno, k)
    # fresh 50/50 batch: ~63.5% of the NewOrders commit, Payments <= W
    assert 0.28 < (a[0]["status"] == ST_COMMIT).mean() < 0.36
    for t in (T_WAREHOUSE, T_DISTRICT):
        assert (a[2][t][0] == b[2][t][0]).all() and (a[2][t][1] == b[2][t][1]).all(), t
    # CC1 (TPC-C 3.3.2.1): W_YTD = sum of the warehouse's D_YTD
    Wd, Dd = tpcc_cc._df(a[2], T_WAREHOUSE), tpcc_cc._df(a[2], T_DISTRICT)
    s = Dd.groupby((Dd["key"].astype(np.int64) - 1) // 10)["D_YTD"].sum()
    assert (Wd["W_YTD"].values == s.reindex(Wd["key"].astype(np.int64)).values).all()
    assert (Wd["W_YTD"].values > 30_000_000).all()  # every warehouse took committed Payments

