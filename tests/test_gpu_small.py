"""GPU parity of the single-launch path for small OPS batches (k_ops_small: a2..a8 in one
cooperative kernel with grid-wide barriers, used for single-partition OPS batches of at most
16384 txns) -- against the oracle, and against the multi-kernel path it replaces
(LTPG_FLAG_NO_SINGLE_LAUNCH), across the size boundary and with INSERT / SCAN / DELETE."""
import numpy as np
import pytest

import oracle
from tests import opscases
from tests.test_gpu_ops import check_batch, make_pair
from workloads.ycsb import YcsbWorkload

pytestmark = pytest.mark.gpu

SMALL_MAX = 16384


def L():
    import paper_conf_icde_wei0l0lzj024_b200 as lib
    return lib


@pytest.mark.parametrize("n", [1, 31, 256, 257, 4097, SMALL_MAX, SMALL_MAX + 1])
def test_single_launch_ycsb_equals_oracle(n):
    """YCSB-E-like mix (SCAN 45%, INSERT 5%, zipf 0.9): sizes on both sides of the boundary,
    three batches so append cursors and INSERT claims carry over."""
    wl = YcsbWorkload(20_000, theta=0.9, ops_per_txn=4, seed=0x5E + n, scan_frac=0.45, insert_frac=0.05)
    keys, cols = wl.initial_table()
    descs = {0: tuple(wl.table_desc()[:3])}
    tables = {0: (keys, cols)}
    g, o = make_pair(descs, tables, SMALL_MAX + 1, 4 * (SMALL_MAX + 1), extra_rows=4 * n + 64)
    tid = 1
    for b in range(3):
        batch = wl.batch(n, tid, b)
        tid += n
        check_batch(g, o, batch, tables)


@pytest.mark.parametrize("flags", [0, 2, 4])  # (+ no mark filter, + NEXT-1 reordering)
@pytest.mark.parametrize("seed", range(8))
def test_single_launch_equals_multi_kernel(seed, flags):
    """Every op kind (incl. duplicate-key INSERT user aborts, DELETE, SCAN over absent keys):
    the single launch and the multi-kernel path give the same verdicts, reads and tables."""
    rng = np.random.default_rng(7100 + seed)
    tables = opscases.rand_tables(rng)
    g1, o = make_pair(opscases.RAND_DESCS, tables, 64, 256, extra_rows=2048, flags=flags)
    g2, _ = make_pair(opscases.RAND_DESCS, tables, 64, 256, extra_rows=2048,
                      flags=flags | L().LTPG_FLAG_NO_SINGLE_LAUNCH)
    if flags & 4:
        o.set_reorder(True)
    for b in range(8):
        batch = opscases.rand_batch(rng, int(rng.integers(1, 60)), tid_start=1 + 100 * b)
        st = check_batch(g1, o, batch, tables)
        out = g2.run_ops(batch)
        assert (out["status"] == st).all()
    for t in tables:
        a, b_ = g1.dump_table(t), g2.dump_table(t)
        assert (a[0] == b_[0]).all() and (a[1] == b_[1]).all()


def test_single_launch_graph_replay():
    """LTPG_FLAG_GRAPH captures the cooperative launch; replays see the new batch scalars."""
    wl = YcsbWorkload(10_000, theta=0.5, ops_per_txn=4, seed=0x17C0)
    keys, cols = wl.initial_table()
    descs = {0: tuple(wl.table_desc()[:3])}
    tables = {0: (keys, cols)}
    g, o = make_pair(descs, tables, 2048, 8192, flags=L().LTPG_FLAG_GRAPH)
    for b in range(6):
        check_batch(g, o, wl.batch(1024, 1 + 1024 * b, b), tables)



# malformed batches (EINVAL inside the single launch, nothing applied) and the epoch-tag wrap
# over 600 batches: test_gpu_ops.test_validation_and_atomicity_gpu / test_epoch_tag_wrap_600_batches
# run small single-partition batches, i.e. this path


# ---- TPC-C: k_tpcc_small (single-partition batches of <= 16384 txns, <= 64 warehouses) -------
def _tpcc_pair(W, mode, mix, max_txns, batches, seed, flags=0, rollback=0.0):
    from workloads import tpcc
    wl = tpcc.TpccWorkload(W, seed=seed, mode=mode, mix=mix, rollback_frac=rollback)
    tables = wl.initial_tables()
    g = L().tpcc_database(wl, max_txns=max_txns, tables=tables, append_batches=batches + 1, flags=flags)
    o = oracle.tpcc_db(wl, tables)
    if flags & L().LTPG_FLAG_REORDER:
        o.set_reorder(True)
    return wl, tables, g, o


def _tpcc_loop(wl, g, o, sizes, others=()):
    """closed loop (aborts re-run first): every db (g and `others`, other flags) gives the
    oracle's verdicts, results and abort list for every batch"""
    from workloads.formats import ST_CONFLICT
    pending, tid = None, 1
    for bno, n in enumerate(sizes):
        k = 0 if pending is None else len(pending["tid"])
        fresh = wl.batch(max(n - k, 1), tid, bno)
        tid += len(fresh["tid"])
        batch = fresh if pending is None else {key: np.concatenate([pending[key], fresh[key]]) for key in fresh}
        rc, st, res = o.run_tpcc(batch, 2 + bno)
        assert rc == 0
        for h in (g,) + tuple(others):
            out = h.run_tpcc(batch, 2 + bno)
            bad = np.nonzero(out["status"] != st)[0]
            assert len(bad) == 0, ("status", bno, bad[:10], batch["type"][bad[:10]], out["status"][bad[:10]], st[bad[:10]])
            assert (out["reads"] == res).all(), ("results", bno)
            assert (out["abort_idx"] == np.nonzero(st == ST_CONFLICT)[0]).all()
        ab = np.nonzero(st == ST_CONFLICT)[0]
        pending = {key: v[ab] for key, v in batch.items()} if len(ab) else None


@pytest.mark.parametrize("mode", ["strict", "delayed"])
@pytest.mark.parametrize("n", [1, 33, 257, 3000, SMALL_MAX])
def test_single_launch_tpcc_full_mix_equals_oracle(n, mode):
    """Full mix (StockLevel districts claimed in the grouping stage, Delivery leaders and
    followers), closed loop over 3 batches, 2 warehouses: verdicts, results, tables, CC."""
    from tests import tpcc_cc
    from tests.test_gpu_tpcc import compare_tables
    from workloads import tpcc
    wl, _, g, o = _tpcc_pair(2, mode, tpcc.MIX_FULL, SMALL_MAX + 1, 4, seed=0x5A11 + n)
    _tpcc_loop(wl, g, o, [n, n, n])
    dumps = compare_tables(g, o)
    cc = tpcc_cc.check(dumps)
    assert all(cc.values()), cc


@pytest.mark.parametrize("flags", [0, 2, 4])  # (+ no mark filter, + NEXT-1 reordering)
@pytest.mark.parametrize("mode", ["strict", "delayed"])
def test_single_launch_tpcc_equals_multi_kernel_across_boundary(mode, flags):
    """Batch sizes alternating across the 16384 boundary (single launch <-> multi-kernel: the
    batch scratch's rest state is restored after each multi-kernel batch); a twin db on the
    multi-kernel path only (LTPG_FLAG_NO_SINGLE_LAUNCH) gives the same verdicts; tables == oracle."""
    from tests.test_gpu_tpcc import compare_tables
    from workloads import tpcc
    wl, tables, g, o = _tpcc_pair(3, mode, tpcc.MIX_FULL, 20000, 8, seed=0x5A12, flags=flags)
    g2 = L().tpcc_database(wl, max_txns=20000, tables=tables, append_batches=9,
                           flags=flags | L().LTPG_FLAG_NO_SINGLE_LAUNCH)
    _tpcc_loop(wl, g, o, [700, 17000, 5000, SMALL_MAX, 20000, 64, 9000], others=[g2])
    compare_tables(g, o)
    for t in range(9):
        a, b_ = g.dump_table(t), g2.dump_table(t)
        assert (a[1] == b_[1]).all(), t


@pytest.mark.parametrize("mode", ["strict", "delayed"])
def test_single_launch_tpcc_c2_rollback(mode):
    """BASELINE configs[1] shape (1 warehouse, NewOrder + Payment, 16k) with 1% NewOrder
    rollbacks (R11: user abort, status 2) on the single launch."""
    from tests.test_gpu_tpcc import compare_tables
    from workloads import tpcc
    wl, _, g, o = _tpcc_pair(1, mode, tpcc.MIX_NO_PAY, SMALL_MAX, 4, seed=0x17C1, rollback=0.01)
    _tpcc_loop(wl, g, o, [SMALL_MAX] * 3)
    compare_tables(g, o)


def test_single_launch_tpcc_graph_replay_and_compact_params():
    """LTPG_FLAG_GRAPH captures the single launch (with its scratch clears) and replays it;
    compact parameter records are expanded ahead of it; == oracle."""
    from tests.test_gpu_tpcc import compare, compare_tables
    from workloads import tpcc
    wl, _, g, o = _tpcc_pair(2, "strict", tpcc.MIX_FULL, 4096, 8, seed=0x5A13, flags=L().LTPG_FLAG_GRAPH)
    tid = 1
    for bno in range(6):
        batch = wl.batch(2048 if bno % 3 else 4096, tid, bno)
        tid += len(batch["tid"])
        if bno % 2:
            packed, offs = L().pack_params_compact(batch["type"], batch["params"])
            rc, ost, ores = o.run_tpcc(batch, 2 + bno)
            out = g.run_tpcc({"tid": batch["tid"], "type": batch["type"], "params": packed, "offsets": offs,
                              "compact": True}, 2 + bno)
            assert (out["status"] == ost).all() and (out["reads"] == ores).all()
        else:
            compare(g, o, batch, 2 + bno)
    compare_tables(g, o)


def test_single_launch_tpcc_einval_applies_nothing():
    """An invalid NewOrder line (found by the execute stage of the single launch) rejects the
    whole batch with EINVAL, nothing applied; the next batch runs normally."""
    from tests.test_gpu_tpcc import compare, compare_tables
    from workloads import tpcc
    from workloads.formats import NEW_ORDER
    wl, _, g, o = _tpcc_pair(1, "strict", tpcc.MIX_NO_PAY, 4096, 4, seed=0x5A14)
    batch = wl.batch(4096, 1, 0)
    bad = {k: v.copy() for k, v in batch.items()}
    r = int(np.nonzero(bad["type"] == NEW_ORDER)[0][7])
    bad["params"][r, 8:12] = np.frombuffer(np.uint32(200000).tobytes(), np.uint8)  # item id out of range
    with pytest.raises(L().LtpgError):
        g.run_tpcc(bad, 2)
    compare(g, o, batch, 2)
    compare_tables(g, o)


def test_single_launch_dispatch_rule():
    """The documented dispatch: single-partition TPC-C / OPS batches of <= 16384 txns run as ONE
    kernel launch (ltpg_stats.n_kernels == 1); larger batches and LTPG_FLAG_NO_SINGLE_LAUNCH run
    the multi-kernel path."""
    from workloads import tpcc
    lib = L()
    wl = tpcc.TpccWorkload(2, seed=0x5A15, mode="strict", mix=tpcc.MIX_FULL)
    tables = wl.initial_tables()
    g = lib.tpcc_database(wl, max_txns=SMALL_MAX + 64, tables=tables, append_batches=4)
    g2 = lib.tpcc_database(wl, max_txns=SMALL_MAX + 64, tables=tables, append_batches=4,
                           flags=lib.LTPG_FLAG_NO_SINGLE_LAUNCH)
    g.run_tpcc(wl.batch(1000, 1, 0), 2)  # (a db's first TPC-C batch also builds the ORDER -> lines map)
    assert g.run_tpcc(wl.batch(1000, 1001, 5), 2, stats=True)["stats"]["n_kernels"] == 1
    assert g.run_tpcc(wl.batch(SMALL_MAX, 2001, 1), 3, stats=True)["stats"]["n_kernels"] == 1
    assert g.run_tpcc(wl.batch(SMALL_MAX + 1, 30000, 2), 4, stats=True)["stats"]["n_kernels"] > 5
    assert g2.run_tpcc(wl.batch(1000, 1, 0), 2, stats=True)["stats"]["n_kernels"] > 5
    y = YcsbWorkload(10_000, theta=0.5, ops_per_txn=4, seed=0x17C0)
    keys, cols = y.initial_table()
    gy, _ = make_pair({0: tuple(y.table_desc()[:3])}, {0: (keys, cols)}, 2048, 8192)
    gy.run_ops(y.batch(1024, 1, 0))
    assert gy.run_ops(y.batch(1024, 1025, 1), stats=True)["stats"]["n_kernels"] == 1


def test_single_launch_graph_replay_after_multi_kernel_batch():
    """LTPG_FLAG_GRAPH: a captured single-launch batch is replayed after a multi-kernel batch left
    the batch scratch dirty (the captured graph carries the scratch clears) -- == oracle."""
    from tests.test_gpu_tpcc import compare_tables
    from workloads import tpcc
    wl, _, g, o = _tpcc_pair(2, "strict", tpcc.MIX_FULL, 20000, 8, seed=0x5A16, flags=L().LTPG_FLAG_GRAPH)
    _tpcc_loop(wl, g, o, [700, 700, 17000, 700, 700, 17000, 700])
    compare_tables(g, o)
