"""The real multi-rank path on one GPU: world = 2..4 PROCESSES, each one rank
of a partitioned db (its own key / warehouse range, loaded from its own rows), exchanging
per-txn verdicts and result slots through the peer-memory kernels (csrc/xchg.cu) over CUDA
IPC regions -- the same code that runs over NVLink on an 8xB200 box, here with every rank
on cuda:0 (CUDA IPC within one device).  torch.distributed (gloo, 127.0.0.1) carries only
the handle bootstrap.  Every rank's status / commit bits / abort list / read results must
equal the CPU oracle's on every batch of a closed loop with retries, and the union of the
ranks' final tables must equal the oracle's (PIN-8)."""
import multiprocessing as mp
import os
import socket

import numpy as np
import pytest

import oracle
from workloads import tpcc
from workloads.formats import ST_COMMIT, ST_CONFLICT

pytestmark = pytest.mark.gpu


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _concat(a, b):
    return {k: np.concatenate([a[k], b[k]]) for k in b}


def _select(batch, idx):
    """Sub-batch of txns idx (CSR-aware for OPS batches)."""
    if "op_begin" not in batch:
        return {k: v[idx] for k, v in batch.items()}
    ob = batch["op_begin"]
    sel = np.concatenate([np.arange(ob[i], ob[i + 1]) for i in idx]) if len(idx) else np.zeros(0, np.int64)
    cnt = (ob[1:] - ob[:-1])[idx]
    nob = np.zeros(len(idx) + 1, np.uint32)
    np.cumsum(cnt, out=nob[1:])
    return {"tid": batch["tid"][idx], "op_begin": nob, "ops": batch["ops"][sel], "args": batch["args"][sel]}


def _concat_ops(a, b):
    ob = np.concatenate([a["op_begin"][:-1], b["op_begin"] + a["op_begin"][-1]]).astype(np.uint32)
    return {"tid": np.concatenate([a["tid"], b["tid"]]), "op_begin": ob,
            "ops": np.concatenate([a["ops"], b["ops"]]), "args": np.concatenate([a["args"], b["args"]])}


def _make(kind, seed):
    if kind.startswith("tpcc"):
        mode = kind.split("_")[1]
        return tpcc.TpccWorkload(4, seed=seed, mode=mode, mix=tpcc.MIX_FULL, remote_line_frac=0.2,
                                 remote_cust_frac=0.3)
    from workloads.ycsb import ycsb_letter, YcsbWorkload
    if kind == "ycsb_e":  # inserts of fresh keys + short scans crossing key ranges
        return ycsb_letter("E", 6000, seed=seed)
    return YcsbWorkload(6000, theta=0.9, ops_per_txn=10, seed=seed)


def _loop(kind, wl, B, nb, run):
    """Closed loop with retries: run(batch, bno) -> status; aborted txns lead the next batch."""
    pending, tid, seq = None, 1, []
    ops = not kind.startswith("tpcc")
    for bno in range(nb):
        fresh = wl.batch(B - (0 if pending is None else len(pending["tid"])), tid, bno)
        tid += len(fresh["tid"])
        batch = fresh if pending is None else (_concat_ops(pending, fresh) if ops else _concat(pending, fresh))
        st = run(batch, bno)
        seq.append(st)
        ab = np.nonzero(st == ST_CONFLICT)[0]
        pending = _select(batch, ab) if len(ab) else None
    return seq


def _worker(rank, world, port, kind, seed, B, nb, q):
    import sys
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    import torch
    import torch.distributed as dist
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        torch.cuda.set_device(0)
        import paper_conf_icde_wei0l0lzj024_b200 as lib
        wl = _make(kind, seed)
        if kind.startswith("tpcc"):
            g = lib.tpcc_database(wl, max_txns=B, tables=wl.initial_tables(), append_batches=nb + 1, rank=rank,
                                  world=world)
        else:
            g = lib.ycsb_database(wl, max_txns=B, max_ops=10 * B, capacity=wl.n_rows + 10 * B * nb, rank=rank,
                                  world=world)
        outs = []

        def run(batch, bno):
            o = g.run_tpcc(batch, 2 + bno) if kind.startswith("tpcc") else g.run_ops(batch)
            outs.append((o["status"].copy(), np.asarray(o["reads"]).copy(), o["abort_idx"].copy(),
                         o["commit_bits"].copy()))
            return o["status"]

        _loop(kind, wl, B, nb, run)
        dumps = {t: g.dump_table(t) for t in range(9 if kind.startswith("tpcc") else 1)}
        dist.barrier()  # peers read this rank's exchange region during their batches
        g.close()
        q.put((rank, outs, dumps, None))
    except Exception as e:  # surface the failure in the parent
        import traceback
        q.put((rank, None, None, traceback.format_exc()))
    finally:
        dist.destroy_process_group()


def _union(parts, keyed):
    ks = [k for k, _ in parts]
    cs = [c for _, c in parts]
    c = np.concatenate(cs, axis=1)
    if keyed:
        k = np.concatenate(ks)
        o = np.argsort(k, kind="stable")
        return k[o], c[:, o]
    o = np.lexsort(c[::-1]) if c.shape[1] else np.zeros(0, np.int64)
    return None, c[:, o]


@pytest.mark.parametrize("kind,world", [("tpcc_strict", 2), ("tpcc_delayed", 3), ("ycsb", 2), ("ycsb_e", 4),
                                        ("tpcc_strict", 4), ("ycsb", 3)])
def test_multirank_processes_equal_oracle(kind, world):
    seed, B, nb = 0x5EED + world, 1500, 4
    port = _free_port()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_worker, args=(r, world, port, kind, seed, B, nb, q)) for r in range(world)]
    for p in procs:
        p.start()
    try:
        res = sorted([q.get(timeout=600) for _ in range(world)], key=lambda x: x[0])
    finally:
        for p in procs:
            p.join(timeout=120)
            if p.is_alive():
                p.kill()
    for r in res:
        assert r[3] is None, "rank %d failed:\n%s" % (r[0], r[3])

    # the oracle over the same closed loop (its own statuses drive the retries)
    wl = _make(kind, seed)
    if kind.startswith("tpcc"):
        tables = wl.initial_tables()
        o = oracle.tpcc_db(wl, tables)
    else:
        o = oracle.ycsb_db(wl)
    exp = []

    def orun(batch, bno):
        rc, st, rd = o.run_tpcc(batch, 2 + bno) if kind.startswith("tpcc") else o.run_ops(batch)
        assert rc == 0
        exp.append((st, rd))
        return st

    _loop(kind, wl, B, nb, orun)
    for rank, outs, _, _ in res:
        assert len(outs) == nb
        for bno, ((st, rd, ab, bits), (ost, ord_)) in enumerate(zip(outs, exp)):
            assert (st == ost).all(), (rank, bno, np.nonzero(st != ost)[0][:10])
            assert (rd.reshape(ord_.shape) == ord_).all(), (rank, bno)
            assert (ab == np.nonzero(ost == ST_CONFLICT)[0]).all(), (rank, bno)
            eb = np.packbits((ost == ST_COMMIT).astype(np.uint8), bitorder="little")
            eb = np.pad(eb, (0, 4 * len(bits) - len(eb))).view(np.uint32)
            assert (bits == eb).all(), (rank, bno)
    # union of the ranks' tables == the oracle's (ITEM is replicated: rank 0's copy)
    for t in res[0][2]:
        ok, oc = o.dump_table(t)
        if kind.startswith("tpcc") and t == 7:
            gk, gc = res[0][2][t]
        else:
            gk, gc = _union([r[2][t] for r in res], ok is not None)
        assert gc.shape == oc.shape, (t, gc.shape, oc.shape)
        if ok is not None:
            assert (gk == ok).all(), t
        assert (gc == oc).all(), t
    if kind != "ycsb_e":  # (E: short scans + fresh inserts at Zipf 2.5 rarely conflict)
        assert any((ost == ST_CONFLICT).any() for ost, _ in exp)  # the abort path was exercised


# ---- sharded TPC-C batches (include/ltpg.h "Sharded batches"): every rank receives only its shard
def _sharded_worker(rank, world, port, mode, seed, B, nb, q):
    import sys
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    import torch
    import torch.distributed as dist
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        torch.cuda.set_device(0)
        import paper_conf_icde_wei0l0lzj024_b200 as lib
        wl = _make("tpcc_" + mode, seed)
        g = lib.tpcc_database(wl, max_txns=B, tables=wl.initial_tables(), append_batches=nb + 1, rank=rank,
                              world=world)
        outs = []

        def run(batch, bno):
            shard = lib.route_tpcc(batch, wl.W, world, rank)
            o = g.run_tpcc(shard, 2 + bno)
            outs.append((shard["grank"].copy(), o["status"].copy(), np.asarray(o["reads"]).copy(),
                         o["abort_idx"].copy()))
            # the global verdicts (a coordinator's view): every txn's status from the ranks holding it
            parts = [None] * world
            dist.all_gather_object(parts, (shard["grank"], o["status"]))
            st = np.full(len(batch["tid"]), 255, np.uint8)
            for gr, s in parts:
                assert ((st[gr] == 255) | (st[gr] == s)).all()  # identical on every rank holding a txn
                st[gr] = s
            assert (st != 255).all()
            return st

        _loop("tpcc", wl, B, nb, run)
        dumps = {t: g.dump_table(t) for t in range(9)}
        dist.barrier()
        g.close()
        q.put((rank, outs, dumps, None))
    except Exception:
        import traceback
        q.put((rank, None, None, traceback.format_exc()))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("mode,world", [("strict", 2), ("delayed", 3), ("strict", 4)])
def test_multirank_sharded_equal_oracle(mode, world):
    """Each rank gets only the txns touching its warehouses (ltpg_route_tpcc); only the verdict
    bytes of cross-rank txns and remote-customer Payment results cross ranks.  Per shard: status
    == oracle, abort list == the shard's conflict aborts, result slots == oracle on the txn's
    home rank; union of the ranks' tables == oracle."""
    import paper_conf_icde_wei0l0lzj024_b200 as lib
    seed, B, nb = 0x5A4D + world, 1500, 4
    port = _free_port()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_sharded_worker, args=(r, world, port, mode, seed, B, nb, q)) for r in range(world)]
    for p in procs:
        p.start()
    try:
        res = sorted([q.get(timeout=600) for _ in range(world)], key=lambda x: x[0])
    finally:
        for p in procs:
            p.join(timeout=120)
            if p.is_alive():
                p.kill()
    for r in res:
        assert r[3] is None, "rank %d failed:\n%s" % (r[0], r[3])
    wl = _make("tpcc_" + mode, seed)
    o = oracle.tpcc_db(wl, wl.initial_tables())
    exp, batches = [], []

    def orun(batch, bno):
        rc, st, rd = o.run_tpcc(batch, 2 + bno)
        assert rc == 0
        exp.append((st, rd))
        batches.append(batch)
        return st

    _loop("tpcc", wl, B, nb, orun)
    n_shard = 0
    for rank, outs, _, _ in res:
        for bno, ((gr, st, rd, ab), (ost, ord_), batch) in enumerate(zip(outs, exp, batches)):
            n_shard += len(gr)
            assert (st == ost[gr]).all(), (rank, bno)
            assert (ab == np.nonzero(ost[gr] == ST_CONFLICT)[0]).all(), (rank, bno)
            p = batch["params"][gr]
            home = lib.part_of_w(p[:, 0].astype(np.int64) | (p[:, 1].astype(np.int64) << 8), wl.W, world) == rank
            assert (rd.reshape(-1, 4)[home] == ord_[gr][home]).all(), (rank, bno)
    assert n_shard < world * sum(len(b["tid"]) for b in batches)  # shards, not the global batch
    for t in res[0][2]:
        ok, oc = o.dump_table(t)
        gk, gc = res[0][2][t] if t == 7 else _union([r[2][t] for r in res], ok is not None)
        assert gc.shape == oc.shape, (t, gc.shape, oc.shape)
        if ok is not None:
            assert (gk == ok).all(), t
        assert (gc == oc).all(), t
