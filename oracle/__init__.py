"""ctypes binding of the LTPG CPU oracle -- TEST INFRASTRUCTURE ONLY.

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl
reference legs may import this package.  The product path
(paper_conf_icde_wei0l0lzj024_b200) never does.
"""
import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "ltpg_oracle.cpp")
_LIB = os.path.join(_HERE, "libltpg_oracle.so")

ORC_OK, ORC_EINVAL, ORC_EINTERNAL = 0, -1, -7


def build(force=False):
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + ".tmp%d" % os.getpid()
        subprocess.check_call(["g++", "-O2", "-std=c++17", "-shared", "-fPIC", _SRC, "-o", tmp])
        os.replace(tmp, _LIB)
    return _LIB


_lib = None


def lib():
    global _lib
    if _lib is None:
        # LTPG_ORACLE_LIB: a deliberately mutated build (tools/mutate_oracle.py) -- tests only
        L = ctypes.CDLL(os.environ.get("LTPG_ORACLE_LIB") or build())
        vp, u32, u64, i64, ip = ctypes.c_void_p, ctypes.c_uint32, ctypes.c_uint64, ctypes.c_int64, ctypes.c_int
        L.orc_create.restype = vp
        L.orc_create.argtypes = [u32, u32]
        L.orc_destroy.argtypes = [vp]
        L.orc_set_reorder.argtypes = [vp, ip]
        L.orc_set_threads.argtypes = [vp, u32]
        L.orc_define_table.restype = ip
        L.orc_define_table.argtypes = [vp, u32, u32, vp, vp, u32, u32]
        L.orc_load_table.restype = ip
        L.orc_load_table.argtypes = [vp, u32, u64, vp, vp]
        L.orc_run_ops.restype = ip
        L.orc_run_ops.argtypes = [vp, u32, vp, vp, vp, vp, vp, vp]
        L.orc_run_tpcc.restype = ip
        L.orc_run_tpcc.argtypes = [vp, u32, vp, vp, vp, i64, vp, vp]
        L.orc_count_rows.restype = u64
        L.orc_count_rows.argtypes = [vp, u32]
        L.orc_n_cols.restype = u32
        L.orc_n_cols.argtypes = [vp, u32]
        L.orc_dump_table.restype = ip
        L.orc_dump_table.argtypes = [vp, u32, vp, vp]
        _lib = L
    return _lib


def _p(a):
    return None if a is None else a.ctypes.data_as(ctypes.c_void_p)


class OracleDB:
    """One oracle database (tables + PK indexes), run batch by batch."""

    def __init__(self, n_tables, n_warehouses=0):
        self.L = lib()
        self.h = self.L.orc_create(n_tables, n_warehouses)
        self.has_pk = {}

    def set_reorder(self, on=True):
        """NEXT-1 logical reordering: abort iff WAW or (RAW and WAR)."""
        self.L.orc_set_reorder(self.h, int(bool(on)))

    def set_threads(self, n):
        """SURVEY §8(d) secondary baseline: O1-O3 on n threads (1 = the plain oracle)."""
        self.L.orc_set_threads(self.h, int(n))

    def close(self):
        if self.h:
            self.L.orc_destroy(self.h)
            self.h = None

    __del__ = close

    def define_table(self, t, col_group, col_is_add, n_groups, has_pk=True):
        g = np.ascontiguousarray(col_group, dtype=np.uint8)
        a = np.ascontiguousarray(col_is_add, dtype=np.uint8)
        rc = self.L.orc_define_table(self.h, t, len(g), _p(g), _p(a), n_groups, int(bool(has_pk)))
        if rc:
            raise ValueError("orc_define_table rc=%d" % rc)
        self.has_pk[t] = bool(has_pk)

    def load_table(self, t, keys, cols):
        cols = np.ascontiguousarray(cols, dtype=np.int64)
        n = cols.shape[1] if cols.ndim == 2 else 0
        k = None if keys is None else np.ascontiguousarray(keys, dtype=np.uint64)
        rc = self.L.orc_load_table(self.h, t, n, _p(k), _p(cols))
        if rc:
            raise ValueError("orc_load_table rc=%d" % rc)

    def run_ops(self, batch):
        tid = np.ascontiguousarray(batch["tid"], dtype=np.uint64)
        ob = np.ascontiguousarray(batch["op_begin"], dtype=np.uint32)
        ops = np.ascontiguousarray(batch["ops"])
        args = np.ascontiguousarray(batch["args"], dtype=np.int64)
        n = len(tid)
        status = np.zeros(n, dtype=np.uint8)
        reads = np.zeros(len(ops), dtype=np.int64)
        rc = self.L.orc_run_ops(self.h, n, _p(tid), _p(ob), _p(ops), _p(args), _p(status), _p(reads))
        return rc, status, reads

    def run_tpcc(self, batch, clock):
        tid = np.ascontiguousarray(batch["tid"], dtype=np.uint64)
        ty = np.ascontiguousarray(batch["type"], dtype=np.uint8)
        params = np.ascontiguousarray(batch["params"], dtype=np.uint8)
        n = len(tid)
        status = np.zeros(n, dtype=np.uint8)
        res = np.zeros(4 * n, dtype=np.int64)
        rc = self.L.orc_run_tpcc(self.h, n, _p(tid), _p(ty), _p(params), int(clock), _p(status), _p(res))
        return rc, status, res.reshape(n, 4)

    def dump_table(self, t):
        n = int(self.L.orc_count_rows(self.h, t))
        nc = int(self.L.orc_n_cols(self.h, t))
        keys = np.zeros(n, dtype=np.uint64) if self.has_pk.get(t, True) else None
        cols = np.zeros((nc, n), dtype=np.int64)
        rc = self.L.orc_dump_table(self.h, t, _p(keys), _p(cols))
        if rc:
            raise ValueError("orc_dump_table rc=%d" % rc)
        return keys, cols


def ycsb_db(workload):
    db = OracleDB(1)
    g, a, ng, pk = workload.table_desc()
    db.define_table(0, g, a, ng, pk)
    keys, cols = workload.initial_table()
    db.load_table(0, keys, cols)
    return db


def tpcc_db(workload, tables=None):
    db = OracleDB(9, workload.W)
    for t, (g, a, ng, pk) in workload.table_descs().items():
        db.define_table(t, g, a, ng, pk)
    tables = tables if tables is not None else workload.initial_tables()
    for t, (k, c) in tables.items():
        db.load_table(t, k, c)
    return db
