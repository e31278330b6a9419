"""Host-side plumbing for the multi-GPU path; one process per GPU.

torch.distributed (any backend: nccl on the GPU box, gloo in CPU tests) only carries the
bootstrap -- the ranks' 128-byte exchange handles (CUDA IPC handles of their exchange
regions) -- and bench-side timing reductions.  The per-batch exchange itself is the library's
own peer-memory kernels (csrc/xchg.cu).  Host routing of sharded TPC-C batches:
paper_conf_icde_wei0l0lzj024_b200.route_tpcc (ltpg_route_tpcc).
"""
import numpy as np


def gather_handles(handle, group=None):
    """All ranks' exchange handles (bytes), in rank order of `group`."""
    import torch.distributed as dist
    out = [None] * dist.get_world_size(group)
    dist.all_gather_object(out, bytes(handle), group=group)
    return out


def connect_peers(db, group=None):
    """Bootstrap a multi-rank db's peer-memory exchange: every rank of `group` calls this."""
    db.connect_peers(gather_handles(db.peer_handle(), group))


def warehouse_ranges(n_warehouses, world):
    """[(lo, hi)) warehouse ids owned by each rank: the inverse of part_of_w (contiguous)."""
    from . import part_of_w
    w = np.arange(1, n_warehouses + 1)
    p = part_of_w(w, n_warehouses, world)
    return [(int(w[p == r].min()), int(w[p == r].max()) + 1) if (p == r).any() else (0, 0) for r in range(world)]


def key_ranges(key_space, world):
    chunk = (int(key_space) + world - 1) // world
    return [(min(r * chunk, key_space), min((r + 1) * chunk, key_space)) for r in range(world)]


def tpcc_rank_tables(tables, n_warehouses, rank, world):
    """Rows of every TPC-C table that rank owns (ITEM replicated) -- what a rank loads."""
    from . import part_of_w, tpcc_owner_w
    out = {}
    for t, (k, c) in tables.items():
        ow = tpcc_owner_w(t, k, c)
        if ow is None or world == 1:
            out[t] = (k, c)
            continue
        own = part_of_w(ow, n_warehouses, world) == rank
        out[t] = (None if k is None else k[own], c[:, own])
    return out
