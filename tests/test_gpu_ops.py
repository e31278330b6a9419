"""GPU parity, OPS mode: the CUDA path (through the C-ABI) vs the CPU oracle,
element by element, bit-exact (all state is integer).  Needs a B200."""
import numpy as np
import pytest

import oracle
from tests import opscases
from workloads.formats import (SELECT, UPDATE, ADD, INSERT, DELETE, SCAN, ST_COMMIT, ST_CONFLICT)
from workloads.ycsb import YcsbWorkload

pytestmark = pytest.mark.gpu


def L():
    import paper_conf_icde_wei0l0lzj024_b200 as lib
    return lib


def make_pair(descs, tables, max_txns, max_ops, extra_rows=64, flags=0, layout=0):
    g = L().Database(max(descs) + 1, max_txns, max_ops, flags=flags)
    o = oracle.OracleDB(max(descs) + 1)
    for t, (grp, add, ng) in descs.items():
        k, c = tables[t]
        lay = layout if isinstance(layout, int) else layout[t % len(layout)]
        g.load_table(t, grp, add, ng, k, c, capacity=c.shape[1] + extra_rows, layout=lay)
        o.define_table(t, grp, add, ng, True)
        o.load_table(t, k, c)
    return g, o


def check_batch(g, o, batch, tables):
    rc, ost, ord_ = o.run_ops(batch)
    assert rc == 0
    out = g.run_ops(batch)
    assert (out["status"] == ost).all(), np.nonzero(out["status"] != ost)[0][:10]
    assert (out["reads"] == ord_).all(), np.nonzero(out["reads"] != ord_)[0][:10]
    exp_bits = np.packbits((ost == ST_COMMIT).astype(np.uint8), bitorder="little")
    exp_bits = np.pad(exp_bits, (0, 4 * len(out["commit_bits"]) - len(exp_bits))).view(np.uint32)
    assert (out["commit_bits"] == exp_bits).all()
    assert (out["abort_idx"] == np.nonzero(ost == ST_CONFLICT)[0]).all()
    for t in tables:
        gk, gc = g.dump_table(t)
        ok, oc = o.dump_table(t)
        assert gk.shape == ok.shape and (gk == ok).all(), t
        assert gc.shape == oc.shape and (gc == oc).all(), t
    return ost


@pytest.mark.parametrize("encoding", ["row_level_no_optimizations", "split_only_write",
                                      "split_and_delayed_update"])
def test_example3_gpu(encoding):
    descs, tables, batch, gold = opscases.example3(encoding)
    g, o = make_pair(descs, tables, 16, 16)
    st = check_batch(g, o, batch, tables)
    assert [i + 1 for i, s in enumerate(st) if s == ST_COMMIT] == gold["expected_commits"][encoding]["value"]


@pytest.mark.parametrize("flags", [0, 1, 2, 3, 8, 10])
@pytest.mark.parametrize("seed", range(12))
def test_random_tiny_batches_all_kinds(seed, flags):
    """Every op kind incl. INSERT claims, DELETE, SCAN over absent keys; grouping and
    mark-filter on/off (PIN-8 invariance)."""
    rng = np.random.default_rng(500 + seed)
    tables = opscases.rand_tables(rng)
    g, o = make_pair(opscases.RAND_DESCS, tables, 64, 256, extra_rows=2048, flags=flags)
    for b in range(6):
        batch = opscases.rand_batch(rng, int(rng.integers(1, 60)), tid_start=1 + 100 * b)
        check_batch(g, o, batch, tables)


@pytest.mark.parametrize("layout", [1, (0, 1)])
@pytest.mark.parametrize("seed", range(4))
def test_random_tiny_batches_layouts(seed, layout):
    """Column placement is result-invisible: columnar and mixed row-block/columnar tables."""
    rng = np.random.default_rng(900 + seed)
    tables = opscases.rand_tables(rng)
    g, o = make_pair(opscases.RAND_DESCS, tables, 64, 256, extra_rows=2048, layout=layout)
    for b in range(6):
        batch = opscases.rand_batch(rng, int(rng.integers(1, 60)), tid_start=1 + 100 * b)
        check_batch(g, o, batch, tables)


def test_epoch_tag_wrap_600_batches():
    """Mark words carry an 8-bit epoch tag that repeats every 255 batches (all marks are
    reset at the wrap): 600 consecutive small batches on hot keys stay oracle-identical."""
    wl = YcsbWorkload(64, theta=0.9, ops_per_txn=4, seed=77)
    keys, cols = wl.initial_table()
    descs = {0: tuple(wl.table_desc()[:3])}
    g, o = make_pair(descs, {0: (keys, cols)}, 64, 256)
    tid = 1
    for bno in range(600):
        batch = wl.batch(int(1 + bno % 48), tid, bno)
        tid += len(batch["tid"])
        rc, ost, ord_ = o.run_ops(batch)
        out = g.run_ops(batch)
        assert rc == 0 and (out["status"] == ost).all() and (out["reads"] == ord_).all(), bno
    gk, gc = g.dump_table(0)
    ok, oc = o.dump_table(0)
    assert (gc == oc).all()


def test_ycsb_c1_closed_loop():
    """BASELINE configs[0]: YCSB-A 10k rows, 1024 txns x 4 ops, zipf 0.5, retries."""
    wl = YcsbWorkload(10_000, theta=0.5, ops_per_txn=4, seed=0x17C0)
    keys, cols = wl.initial_table()
    descs = {0: tuple(wl.table_desc()[:3])}
    tables = {0: (keys, cols)}
    g, o = make_pair(descs, tables, 2048, 8192)
    pending = None
    tid = 1
    rates = []
    for b in range(30):
        fresh = wl.batch(1024 - (0 if pending is None else len(pending["tid"])), tid, b)
        tid += len(fresh["tid"])
        batch = fresh if pending is None else concat(pending, fresh)
        st = check_batch(g, o, batch, tables)
        rates.append((st == ST_COMMIT).mean())
        ab = np.nonzero(st == ST_CONFLICT)[0]
        pending = select(batch, ab) if len(ab) else None
    assert 0.3 < rates[0] < 0.8


def test_validation_and_atomicity_gpu():
    descs = {0: ([0, 0], [0, 0], 1)}
    tables = {0: (np.arange(8, dtype=np.uint64), np.arange(16, dtype=np.int64).reshape(2, 8))}
    g, o = make_pair(descs, tables, 16, 128)
    lib = L()
    bad = opscases.make_batch([[(1, UPDATE, 0, 0, 0, 1), (1, SELECT, 0, 1, 0, 0)]])
    with pytest.raises(lib.LtpgError) as e:
        g.run_ops(bad)
    assert e.value.rc == lib.LTPG_EINVAL
    b = opscases.make_batch([[(1, UPDATE, 0, 0, 0, 5)], [(2, UPDATE, 0, 0, 0, 5)]])
    b["tid"] = np.array([3, 2], np.uint64)
    with pytest.raises(lib.LtpgError):
        g.run_ops(b)
    k, c = g.dump_table(0)
    assert (c == tables[0][1]).all()  # nothing changed
    # capacity: more inserts than the append region holds -> ECAPACITY, nothing changed
    many = opscases.make_batch([[(100 + i, INSERT, 0, 0, 0, 7) for i in range(80)]])
    with pytest.raises(lib.LtpgError) as e:
        g.run_ops(many)
    assert e.value.rc == lib.LTPG_ECAPACITY
    k, c = g.dump_table(0)
    assert (c == tables[0][1]).all() and len(k) == 8
    # the db still works afterwards
    ok = opscases.make_batch([[(1, UPDATE, 0, 0, 0, 5)], [(100, INSERT, 0, 0, 0, 9)]])
    check_batch(g, o, ok, tables)


def test_device_resident_inputs_and_outputs():
    import torch
    wl = YcsbWorkload(5000, theta=0.8, ops_per_txn=10, seed=7)
    keys, cols = wl.initial_table()
    descs = {0: tuple(wl.table_desc()[:3])}
    g, o = make_pair(descs, {0: (keys, cols)}, 4096, 40960)
    batch = wl.batch(4000, 1, 0)
    rc, ost, ord_ = o.run_ops(batch)
    dev = {"tid": torch.from_numpy(batch["tid"].view(np.int64)).cuda(),
           "op_begin": torch.from_numpy(batch["op_begin"].view(np.int32)).cuda(),
           "ops": torch.from_numpy(batch["ops"].view(np.uint8)).cuda(),
           "args": torch.from_numpy(batch["args"]).cuda()}
    out = g.run_ops(dev, stream=torch.cuda.current_stream().cuda_stream)
    torch.cuda.synchronize()
    assert (out["status"].cpu().numpy() == ost).all()
    assert (out["reads"][:len(ord_)].cpu().numpy() == ord_).all()
    na = int(out["n_aborted"].item())
    assert (out["abort_idx"][:na].cpu().numpy().view(np.uint32) == np.nonzero(ost == ST_CONFLICT)[0]).all()
    gk, gc = g.dump_table(0)
    ok_, oc = o.dump_table(0)
    assert (gc == oc).all()


def select(batch, idx):
    ob = batch["op_begin"]
    parts = [np.arange(ob[i], ob[i + 1]) for i in idx]
    sel = np.concatenate(parts) if parts else np.zeros(0, np.int64)
    lens = np.array([ob[i + 1] - ob[i] for i in idx], dtype=np.uint32)
    return {"tid": batch["tid"][idx], "ops": batch["ops"][sel], "args": batch["args"][sel],
            "op_begin": np.concatenate([[0], np.cumsum(lens)]).astype(np.uint32)}


def concat(a, b):
    return {"tid": np.concatenate([a["tid"], b["tid"]]), "ops": np.concatenate([a["ops"], b["ops"]]),
            "args": np.concatenate([a["args"], b["args"]]),
            "op_begin": np.concatenate([a["op_begin"], b["op_begin"][1:] + a["op_begin"][-1]]).astype(np.uint32)}


def test_closed_loop_with_compose_retry():
    """a9 through the library: every next batch is ltpg_compose_retry(previous batch, its abort
    list, fresh txns); GPU == oracle on every batch, and the retried txns keep their TIDs."""
    wl = YcsbWorkload(10_000, theta=0.9, ops_per_txn=4, seed=0x17C0)
    keys, cols = wl.initial_table()
    descs = {0: tuple(wl.table_desc()[:3])}
    tables = {0: (keys, cols)}
    g, o = make_pair(descs, tables, 1024, 4096)
    batch = wl.batch(1024, 1, 0)
    tid = 1025
    for b in range(12):
        st = check_batch(g, o, batch, tables)
        ab = np.nonzero(st == ST_CONFLICT)[0].astype(np.uint32)
        fresh = wl.batch(1024, tid, b + 1)
        nxt, nf = L().compose_retry(batch, ab, fresh, 1024, 4096)
        assert (nxt["tid"][:len(ab)] == batch["tid"][ab]).all() and nf == 1024 - len(ab)
        tid += nf
        batch = nxt


@pytest.mark.parametrize("theta", [0.5, 0.99])
def test_ycsb_sparse_keys_hash_probe(theta):
    """Sparse u64 keys (splitmix64 of the row number): no dense key -> row mapping, every op goes
    through the PK hash index (linear probing); closed loop with retries == oracle."""
    wl = YcsbWorkload(50_000, theta=theta, ops_per_txn=10, seed=0x5A1, sparse_keys=True)
    keys, cols = wl.initial_table()
    descs = {0: tuple(wl.table_desc()[:3])}
    tables = {0: (keys, cols)}
    g, o = make_pair(descs, tables, 4096, 40960)
    pending, tid = None, 1
    for b in range(6):
        fresh = wl.batch(4096 - (0 if pending is None else len(pending["tid"])), tid, b)
        tid += len(fresh["tid"])
        batch = fresh if pending is None else concat(pending, fresh)
        st = check_batch(g, o, batch, tables)
        ab = np.nonzero(st == ST_CONFLICT)[0]
        pending = select(batch, ab) if len(ab) else None
