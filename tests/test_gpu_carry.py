"""a9 on the device (LTPG_BATCH_CARRY_ABORTS): a batch led by the previous batch's conflict
aborts -- kept on the device, original TIDs and parameter blocks, ascending ranks -- followed by
fresh txns from the host equals the oracle running the host-composed batch (aborts of the
previous batch in TID order, then the fresh txns) in every output and table."""
import numpy as np
import pytest

import oracle
from tests.test_gpu_tpcc import compare_tables
from workloads import tpcc
from workloads.formats import ST_CONFLICT

pytestmark = pytest.mark.gpu


def L():
    import paper_conf_icde_wei0l0lzj024_b200 as lib
    return lib


@pytest.mark.parametrize("compact", [False, True])
@pytest.mark.parametrize("mode", ["strict", "delayed"])
def test_carry_closed_loop_equals_oracle(mode, compact):
    lib = L()
    W, B = 2, 3000
    wl = tpcc.TpccWorkload(W, seed=71, mode=mode, mix=tpcc.MIX_FULL, rollback_frac=0.01)
    tables = wl.initial_tables()
    g = lib.tpcc_database(wl, max_txns=B, tables=tables, append_batches=6)
    o = oracle.tpcc_db(wl, tables)
    tid, prev = 1, None
    carried_total = 0
    for bno in range(6):
        nc = g.pending_aborts() if prev is not None else 0
        fresh = wl.batch(B - nc, tid, bno)
        tid += len(fresh["tid"])
        inp = fresh
        if compact:
            packed, offs = lib.pack_params_compact(fresh["type"], fresh["params"])
            inp = {"tid": fresh["tid"], "type": fresh["type"], "params": packed, "offsets": offs, "compact": True}
        out = g.run_tpcc(inp, 2 + bno, carry=prev is not None)
        batch = fresh if prev is None else {k: np.concatenate([prev[k][prev_ab], fresh[k]]) for k in fresh}
        assert len(out["status"]) == len(batch["tid"]) == nc + len(fresh["tid"])
        rc, st, res = o.run_tpcc(batch, 2 + bno)
        assert rc == 0
        assert (out["status"] == st).all(), (bno, np.nonzero(out["status"] != st)[0][:8])
        assert (out["reads"] == res).all(), bno
        assert (out["abort_idx"] == np.nonzero(st == ST_CONFLICT)[0]).all()
        prev, prev_ab = batch, np.nonzero(st == ST_CONFLICT)[0]
        carried_total += nc
    assert carried_total > 0
    compare_tables(g, o)


def test_carry_needs_a_completed_previous_batch():
    lib = L()
    wl = tpcc.TpccWorkload(1, seed=5, mix=tpcc.MIX_FULL)
    g = lib.tpcc_database(wl, max_txns=512, tables=wl.initial_tables(), append_batches=4)
    b = wl.batch(100, 1, 0)
    with pytest.raises(lib.LtpgError) as e:  # nothing ran yet
        g.run_tpcc(b, 2, carry=True)
    assert e.value.rc == lib.LTPG_EINVAL
    p = g.run_tpcc(b, 2, wait=False)
    with pytest.raises(lib.LtpgError) as e:  # the previous batch is still in flight
        g.run_tpcc(wl.batch(100, 200, 1), 3, carry=True)
    assert e.value.rc == lib.LTPG_EINVAL
    p.wait()
    assert g.pending_aborts() == int((p.out["status"] == ST_CONFLICT).sum()) if hasattr(p, "out") else True
    n = g.pending_aborts()
    out = g.run_tpcc(wl.batch(512 - n, 1000, 2), 4, carry=True)
    assert len(out["status"]) == 512
    with pytest.raises(lib.LtpgError) as e:  # carried + given > max_txns
        g.run_tpcc(wl.batch(512, 5000, 3), 5, carry=True)
    assert e.value.rc == lib.LTPG_EINVAL


@pytest.mark.parametrize("device_out", [False, True])
def test_committed_reads_only(device_out):
    """LTPG_RESULT_COMMITTED_READS: the result slots of the committed txns, packed in rank order,
    written by the kernel into a pinned host (or device) buffer; with NO_STATUS / NO_ABORT_LIST
    the bitmask and n_aborted still describe the batch.  == the oracle's committed rows."""
    import torch
    lib = L()
    W, B = 2, 3000
    wl = tpcc.TpccWorkload(W, seed=73, mode="strict", mix=tpcc.MIX_FULL)
    tables = wl.initial_tables()
    g = lib.tpcc_database(wl, max_txns=B, tables=tables, append_batches=4)
    o = oracle.tpcc_db(wl, tables)
    for bno in range(3):
        b = wl.batch(B - 7 * bno, 1 + B * bno, bno)  # ragged sizes
        rc, st, res = o.run_tpcc(b, 2 + bno)
        inp = b
        if device_out:
            inp = {k: torch.from_numpy(np.ascontiguousarray(v)).cuda() for k, v in b.items()}
        out = g.run_tpcc(inp, 2 + bno, device_out=device_out, committed_reads=True, no_status=bno == 1,
                         no_abort_list=bno == 2, n_txns=len(b["tid"]))
        bits = out["commit_bits"]
        bits = bits.cpu().numpy() if hasattr(bits, "cpu") else np.asarray(bits)
        got_commit = np.unpackbits(bits.view(np.uint8), bitorder="little")[:len(st)].astype(bool)
        assert (got_commit == (st == 1)).all()
        assert int(np.asarray(out["n_aborted"].cpu() if hasattr(out["n_aborted"], "cpu") else out["n_aborted"])[0]) \
            == int((st == ST_CONFLICT).sum())
        reads = out["reads"]
        reads = reads.cpu().numpy() if hasattr(reads, "cpu") else np.asarray(reads)
        nc = int((st == 1).sum())
        assert (reads.reshape(-1)[:4 * nc].reshape(nc, 4) == res[st == 1]).all(), bno
    compare_tables(g, o)


def test_tid_range_equals_explicit_tids():
    """LTPG_BATCH_TID_RANGE: only the first TID crosses PCIe, the device fills the consecutive
    rest; with carried aborts (LTPG_BATCH_CARRY_ABORTS) the carried txns keep their TIDs (HISTORY
    rows store them) -- closed loop == the oracle on the host-composed batches."""
    lib = L()
    wl = tpcc.TpccWorkload(2, seed=79, mode="strict", mix=tpcc.MIX_FULL)
    tables = wl.initial_tables()
    g = lib.tpcc_database(wl, max_txns=2000, tables=tables, append_batches=5)
    o = oracle.tpcc_db(wl, tables)
    tid, prev = 100, None
    for bno in range(4):
        nc = g.pending_aborts() if prev is not None else 0
        fresh = wl.batch(2000 - nc, tid, bno)
        packed, offs = lib.pack_params_compact(fresh["type"], fresh["params"])
        inp = {"tid": fresh["tid"][:1].copy(), "type": fresh["type"], "params": packed, "offsets": offs,
               "compact": True, "tid_range": True}
        out = g.run_tpcc(inp, 2 + bno, carry=prev is not None, n_txns=len(fresh["type"]))
        tid += len(fresh["tid"])
        batch = fresh if prev is None else {k: np.concatenate([prev[k][prev_ab], fresh[k]]) for k in fresh}
        rc, st, res = o.run_tpcc(batch, 2 + bno)
        assert rc == 0 and (out["status"] == st).all() and (out["reads"] == res).all(), bno
        prev, prev_ab = batch, np.nonzero(st == ST_CONFLICT)[0]
    compare_tables(g, o)
