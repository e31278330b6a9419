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
