#!/usr/bin/env python
"""Test harness, not product code: small end-to-end runs of the library for compute-sanitizer
(memcheck / racecheck / synccheck), each checked against the oracle:
python tests/sanitize_run.py ycsb_c1|tpcc_c2|multirank
(multirank: 2 ranks on one GPU over CUDA IPC, gloo bootstrap; run under torch.distributed.run)."""
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def ycsb_c1(batches=3):
    import oracle
    import paper_conf_icde_wei0l0lzj024_b200 as ltpg
    from workloads.ycsb import YcsbWorkload
    wl = YcsbWorkload(10_000, theta=0.5, ops_per_txn=4, seed=0x17C0)
    g = ltpg.ycsb_database(wl, max_txns=1024, max_ops=4096)
    o = oracle.ycsb_db(wl)
    for b in range(batches):
        batch = wl.batch(1024, 1 + 1024 * b, b)
        out = g.run_ops(batch, stats=True)
        rc, st, rd = o.run_ops(batch)
        assert rc == 0 and (out["status"] == st).all() and (out["reads"] == rd).all()
    print("ycsb_c1 ok")


def tpcc_c2(batches=2, mode="strict", flags=0):
    import oracle
    import paper_conf_icde_wei0l0lzj024_b200 as ltpg
    from workloads import tpcc
    wl = tpcc.TpccWorkload(1, seed=0x17C1, mode=mode, mix=tpcc.MIX_FULL, rollback_frac=0.01)
    tables = wl.initial_tables()
    g = ltpg.tpcc_database(wl, max_txns=4096, tables=tables, append_batches=batches + 1, flags=flags)
    o = oracle.tpcc_db(wl, tables)
    o.set_reorder(bool(flags & ltpg.LTPG_FLAG_REORDER))
    for b in range(batches):
        batch = wl.batch(4096, 1 + 4096 * b, b)
        out = g.run_tpcc(batch, 2 + b, stats=True)
        rc, st, res = o.run_tpcc(batch, 2 + b)
        assert rc == 0 and (out["status"] == st).all() and (out["reads"] == res).all()
    for t in range(9):
        assert (g.dump_table(t)[1] == o.dump_table(t)[1]).all(), t
    print("tpcc_c2 (%s, flags %d) ok" % (mode, flags))


def ycsb_e(batches=3):
    """YCSB-E: INSERTs (the cooperative insert tail) and SCANs."""
    import oracle
    import paper_conf_icde_wei0l0lzj024_b200 as ltpg
    from workloads.ycsb import ycsb_letter
    wl = ycsb_letter("E", 20_000, seed=5)
    g = ltpg.ycsb_database(wl, max_txns=2048, max_ops=20480, capacity=20_000 + 20480 * batches)
    o = oracle.ycsb_db(wl)
    for b in range(batches):
        batch = wl.batch(2048, 1 + 2048 * b, b)
        out = g.run_ops(batch)
        rc, st, rd = o.run_ops(batch)
        assert rc == 0 and (out["status"] == st).all() and (out["reads"] == rd).all()
    print("ycsb_e ok")


def carry(batches=3):
    """TPC-C closed loop with the aborts carried on the device, consecutive TIDs, committed
    result slots written into pinned host memory by the kernel."""
    import oracle
    import paper_conf_icde_wei0l0lzj024_b200 as ltpg
    from workloads import tpcc
    wl = tpcc.TpccWorkload(1, seed=3, mix=tpcc.MIX_FULL)
    tables = wl.initial_tables()
    g = ltpg.tpcc_database(wl, max_txns=2048, tables=tables, append_batches=batches + 1)
    o = oracle.tpcc_db(wl, tables)
    tid, prev = 1, None
    for b in range(batches):
        nc = g.pending_aborts() if prev is not None else 0
        fresh = wl.batch(2048 - nc, tid, b)
        packed, offs = ltpg.pack_params_compact(fresh["type"], fresh["params"])
        inp = {"tid": fresh["tid"][:1].copy(), "type": fresh["type"], "params": packed, "offsets": offs,
               "compact": True, "tid_range": True}
        out = g.run_tpcc(inp, 2 + b, carry=prev is not None, n_txns=len(fresh["type"]), committed_reads=True)
        batch = fresh if prev is None else {k: np.concatenate([prev[k][pab], fresh[k]]) for k in fresh}
        rc, st, res = o.run_tpcc(batch, 2 + b)
        assert rc == 0 and (out["status"] == st).all() and (out["reads"] == res[st == 1]).all()
        tid += len(fresh["tid"])
        prev, pab = batch, np.nonzero(st == 0)[0]
    print("carry ok")


def multirank(sharded=False):
    import torch
    import torch.distributed as dist
    import oracle
    import paper_conf_icde_wei0l0lzj024_b200 as ltpg
    from workloads import tpcc
    dist.init_process_group("gloo")
    rank, world = dist.get_rank(), dist.get_world_size()
    torch.cuda.set_device(0)
    wl = tpcc.TpccWorkload(4, seed=7, mix=tpcc.MIX_FULL, remote_line_frac=0.2, remote_cust_frac=0.3)
    tables = wl.initial_tables()
    g = ltpg.tpcc_database(wl, max_txns=2048, tables=tables, append_batches=3, rank=rank, world=world)
    o = oracle.tpcc_db(wl, tables)
    for b in range(2):
        batch = wl.batch(2048, 1 + 2048 * b, b)
        rc, st, res = o.run_tpcc(batch, 2 + b)
        assert rc == 0
        if sharded:  # this rank's shard only (route_tpcc): its statuses == the oracle's
            shard = ltpg.route_tpcc(batch, wl.W, world, rank)
            out = g.run_tpcc(shard, 2 + b)
            assert (out["status"] == st[shard["grank"]]).all()
        else:
            out = g.run_tpcc(batch, 2 + b)
            assert (out["status"] == st).all() and (out["reads"] == res).all()
    dist.barrier()
    g.close()
    dist.barrier()
    print("multirank rank %d ok" % rank)


if __name__ == "__main__":
    what = sys.argv[1]
    if what == "tpcc_c2":
        tpcc_c2()
        tpcc_c2(mode="delayed", flags=4)  # + NEXT-1 reordering
    elif what == "multirank_sharded":
        multirank(sharded=True)
    else:
        globals()[what]()
