"""SURVEY §8(e) host routing (ltpg_route_tpcc, host code of the C-ABI; no GPU): every rank's
shard holds exactly the txns touching its warehouses (home, NewOrder supply, Payment customer),
in global order, with their global ranks; every txn lands on its home rank."""
import numpy as np
import pytest

from workloads import tpcc


def _parts(batch, W, world):
    import paper_conf_icde_wei0l0lzj024_b200 as L
    p = batch["params"]
    w = p[:, 0].astype(np.int64) | (p[:, 1].astype(np.int64) << 8)
    sets = [{int(L.part_of_w(x, W, world))} for x in w]
    for r in range(len(w)):
        if batch["type"][r] == 0:
            for l in range(p[r, 3]):
                sw = int(p[r, 12 + 8 * l]) | (int(p[r, 13 + 8 * l]) << 8)
                sets[r].add(int(L.part_of_w(sw, W, world)))
        elif batch["type"][r] == 1:
            sets[r].add(int(L.part_of_w(int(p[r, 4]) | (int(p[r, 5]) << 8), W, world)))
    return [int(L.part_of_w(x, W, world)) for x in w], sets


@pytest.mark.parametrize("world", [1, 2, 3, 5, 8])
def test_route_shards(world):
    import paper_conf_icde_wei0l0lzj024_b200 as L
    W = 8
    wl = tpcc.TpccWorkload(W, seed=11, mix=tpcc.MIX_FULL, remote_line_frac=0.2, remote_cust_frac=0.3)
    b = wl.batch(3000, 100, 0)
    home, sets = _parts(b, W, world)
    seen = np.zeros(len(b["tid"]), int)
    for rank in range(world):
        s = L.route_tpcc(b, W, world, rank)
        want = np.array([r for r in range(len(home)) if rank in sets[r]], np.uint32)
        assert (s["grank"] == want).all()
        assert s["n_global"] == len(b["tid"])
        assert (s["tid"] == b["tid"][want]).all() and (s["type"] == b["type"][want]).all()
        assert (s["params"] == b["params"][want]).all()
        seen[want] += 1
    assert (seen >= 1).all()
    cross = np.array([len(x) > 1 for x in sets])
    assert (seen[~cross] == 1).all()
    if world > 1:
        assert cross.any()
