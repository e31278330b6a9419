"""Multi-rank host plumbing on CPU (world_size 2, gloo, 127.0.0.1): per-rank routing of a
global TPC-C batch into shards (ltpg_route_tpcc), per-rank partition loading (disjoint + complete, ITEM replicated), and
the verdict exchange semantics (max of conflict*2 | user_abort)."""
import multiprocessing as mp
import os
import socket

import numpy as np
import pytest


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    import sys
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    import torch
    import torch.distributed as dist
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from paper_conf_icde_wei0l0lzj024_b200 import dist as D
        from workloads import tpcc
        import paper_conf_icde_wei0l0lzj024_b200 as L
        wl = tpcc.TpccWorkload(4, seed=1)
        shard = L.route_tpcc(wl.batch(2000, 1, 0), 4, world, rank)
        parts = [None] * world
        dist.all_gather_object(parts, shard["grank"].tolist())
        uid = parts
        tables = wl.initial_tables()
        mine = D.tpcc_rank_tables(tables, 4, rank, world)
        keysets = {t: (None if k is None else k.tolist(), c.shape[1]) for t, (k, c) in mine.items()}
        # exchange semantics: local verdict flags -> MAX over ranks -> identical status everywhere
        rng = np.random.default_rng(rank)
        flags = torch.from_numpy(rng.integers(0, 4, 64).astype(np.uint8))
        local = flags.clone()
        dist.all_reduce(flags, op=dist.ReduceOp.MAX)
        status = np.where(flags.numpy() >= 2, 0, np.where(flags.numpy() == 1, 2, 1))
        q.put((rank, uid, keysets, local.numpy(), status, D.warehouse_ranges(4, world)))
    finally:
        dist.destroy_process_group()


def test_two_rank_gloo_plumbing():
    world = 2
    port = _free_port()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = sorted([q.get(timeout=300) for _ in range(world)], key=lambda x: x[0])
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    assert res[0][1] == res[1][1]                                      # every rank saw every shard
    covered = sorted(set(res[0][1][0]) | set(res[0][1][1]))
    assert covered == list(range(2000)) and len(res[0][1][0]) < 2000     # shards cover the batch
    assert res[0][5] == [(1, 3), (3, 5)]                               # warehouses 1-2 | 3-4
    from workloads import tpcc
    from workloads.formats import T_ITEM, T_HISTORY
    full = tpcc.TpccWorkload(4, seed=1).initial_tables()
    for t, (k, c) in full.items():
        n0, n1 = res[0][2][t][1], res[1][2][t][1]
        if t == T_ITEM:
            assert n0 == n1 == c.shape[1]                               # replicated
            continue
        assert n0 + n1 == c.shape[1] and n0 > 0 and n1 > 0              # disjoint + complete
        if k is not None:
            a, b = set(res[0][2][t][0]), set(res[1][2][t][0])
            assert not (a & b) and (a | b) == set(k.tolist())
    # status after the exchange is identical on both ranks and equals the host rule
    assert (res[0][4] == res[1][4]).all()
    mx = np.maximum(res[0][3], res[1][3])
    assert (res[0][4] == np.where(mx >= 2, 0, np.where(mx == 1, 2, 1))).all()


def test_key_ranges_match_part_of_key():
    import paper_conf_icde_wei0l0lzj024_b200 as L
    from paper_conf_icde_wei0l0lzj024_b200 import dist as D
    for ks, world in ((10_000_000, 8), (12, 3), (7, 4)):
        keys = np.arange(ks, dtype=np.uint64)
        p = L.part_of_key(keys, ks, world)
        for r, (lo, hi) in enumerate(D.key_ranges(ks, world)):
            assert ((keys >= lo) & (keys < hi) == (p == r)).all()


def _handles_worker(rank, world, port, q):
    import sys
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    import torch.distributed as dist
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from paper_conf_icde_wei0l0lzj024_b200 import dist as D
        mine = bytes([rank]) * 128  # stands in for ltpg_peer_handle's 128 bytes
        q.put((rank, D.gather_handles(mine)))
    finally:
        dist.destroy_process_group()


def test_peer_handle_allgather_rank_order():
    """Peer-memory bootstrap: every rank receives all handles, in rank order (what
    ltpg_connect_peers requires)."""
    world = 3
    port = _free_port()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_handles_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = sorted([q.get(timeout=300) for _ in range(world)], key=lambda x: x[0])
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    for rank, hs in res:
        assert hs == [bytes([r]) * 128 for r in range(world)]
