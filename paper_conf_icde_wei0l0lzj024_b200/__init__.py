"""Thin Python binding of the B200 LTPG C-ABI (include/ltpg.h).

Argument marshalling only: every step of a batch (validation, warp division,
execute, marks, conflict detection, write-back, result compaction) runs in the
CUDA kernels of libltpg.so.  There is no CPU fallback: importing this package
fails if the shared library is missing, and every call that reaches a device
fails if there is no CUDA device.

Names follow the C-ABI: ltpg_create_db / ltpg_load_table / ltpg_run_batch /
ltpg_dump_table / ltpg_destroy_db / ltpg_last_error.  The ``Database`` class is
a convenience wrapper over them that accepts numpy arrays (host) or torch
tensors (host pinned or CUDA).
"""
import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libltpg.so")

if not os.path.exists(LIB_PATH):
    raise ImportError("libltpg.so not built: run `python paper_conf_icde_wei0l0lzj024_b200/build.py` "
                      "(or __graft_entry__.build()); there is no CPU fallback")

_lib = ctypes.CDLL(LIB_PATH)

# ---- constants (include/ltpg.h) ------------------------------------------------------
LTPG_OK, LTPG_EINVAL, LTPG_ENOMEM, LTPG_ECAPACITY = 0, -1, -2, -3
LTPG_ECUDA, LTPG_EPOISONED, LTPG_EINTERNAL = -4, -6, -7
ERR_NAMES = {0: "OK", -1: "EINVAL", -2: "ENOMEM", -3: "ECAPACITY", -4: "ECUDA", -6: "EPOISONED", -7: "EINTERNAL"}
LTPG_MODE_OPS, LTPG_MODE_TPCC = 0, 1
LTPG_FLAG_NO_GROUPING = 1 << 0
LTPG_FLAG_NO_MARK_FILTER = 1 << 1
LTPG_FLAG_REORDER = 1 << 2
LTPG_FLAG_UNFUSED = 1 << 3
LTPG_FLAG_LARGE_BUCKETS = 1 << 5
LTPG_FLAG_GRAPH = 1 << 6
LTPG_FLAG_L2_PERSIST_MARKS = 1 << 7
LTPG_FLAG_NO_SINGLE_LAUNCH = 1 << 12
LTPG_PEER_HANDLE_BYTES = 128
LTPG_PARAM_BYTES = 128
LTPG_LAYOUT_ROWBLOCK, LTPG_LAYOUT_COLUMNAR = 0, 1
LTPG_FLAG_LOOPBACK_SHIFT = 8
LTPG_ST_CONFLICT, LTPG_ST_COMMIT, LTPG_ST_USER_ABORT = 0, 1, 2

c_u32, c_u64, c_i64, c_int, c_vp = ctypes.c_uint32, ctypes.c_uint64, ctypes.c_int64, ctypes.c_int, ctypes.c_void_p


class ltpg_config(ctypes.Structure):
    _fields_ = [("device", c_int), ("rank", c_int), ("world", c_int),
                ("max_txns", c_u32), ("max_ops", c_u32), ("flags", c_u32), ("n_tables", c_u32),
                ("n_warehouses", c_u32), ("key_space", c_u64)]


class ltpg_table_desc(ctypes.Structure):
    _fields_ = [("n_cols", c_u32), ("col_group", c_vp), ("col_is_add", c_vp), ("n_groups", c_u32),
                ("capacity_rows", c_u64), ("has_pk", c_u32), ("owner_rule", c_u32), ("layout", c_u32)]


class ltpg_batch(ctypes.Structure):
    _fields_ = [("n_txns", c_u32), ("tid", c_vp), ("mode", c_u32), ("n_ops", c_u32), ("op_begin", c_vp),
                ("ops", c_vp), ("op_arg", c_vp), ("proc_type", c_vp), ("proc_params", c_vp),
                ("batch_clock", c_i64), ("inputs_on_device", c_int), ("stream", c_vp), ("flags", c_u32),
                ("proc_offsets", c_vp), ("grank", c_vp), ("n_global", c_u32)]


class ltpg_stats(ctypes.Structure):
    _fields_ = [("ms_upload", ctypes.c_float), ("ms_group", ctypes.c_float), ("ms_exec", ctypes.c_float),
                ("ms_detect", ctypes.c_float), ("ms_exchange", ctypes.c_float),
                ("ms_writeback", ctypes.c_float), ("ms_download", ctypes.c_float),
                ("n_commit", c_u32), ("n_conflict", c_u32), ("n_user_abort", c_u32), ("n_kernels", c_u32),
                ("popular_tables", c_u32)]

    def as_dict(self):
        return {k: getattr(self, k) for k, _ in self._fields_}


class ltpg_result(ctypes.Structure):
    _fields_ = [("commit_bits", c_vp), ("status", c_vp), ("abort_idx", c_vp), ("n_aborted", c_vp),
                ("reads", c_vp), ("outputs_on_device", c_int), ("stats", ctypes.POINTER(ltpg_stats)),
                ("flags", c_u32), ("reads_cap", c_u64)]


_lib.ltpg_create_db.restype = c_int
_lib.ltpg_create_db.argtypes = [ctypes.POINTER(ltpg_config), ctypes.POINTER(c_vp)]
_lib.ltpg_load_table.restype = c_int
_lib.ltpg_load_table.argtypes = [c_vp, c_u32, ctypes.POINTER(ltpg_table_desc), c_u64, c_vp, c_vp]
_lib.ltpg_run_batch.restype = c_int
_lib.ltpg_run_batch.argtypes = [c_vp, ctypes.POINTER(ltpg_batch), ctypes.POINTER(ltpg_result)]
_lib.ltpg_dump_table.restype = c_int
_lib.ltpg_dump_table.argtypes = [c_vp, c_u32, ctypes.POINTER(c_u64), c_vp, c_vp]
_lib.ltpg_destroy_db.restype = None
_lib.ltpg_destroy_db.argtypes = [c_vp]
_lib.ltpg_last_error.restype = ctypes.c_char_p
_lib.ltpg_last_error.argtypes = [c_vp]
_lib.ltpg_wait_batch.restype = c_int
_lib.ltpg_wait_batch.argtypes = [c_vp, ctypes.POINTER(ltpg_result)]
_lib.ltpg_peer_handle.restype = c_int
_lib.ltpg_peer_handle.argtypes = [c_vp, c_vp]
_lib.ltpg_connect_peers.restype = c_int
_lib.ltpg_connect_peers.argtypes = [c_vp, c_vp]
class ltpg_batch_buf(ctypes.Structure):
    _fields_ = [("cap_txns", c_u32), ("cap_ops", c_u32), ("tid", c_vp), ("op_begin", c_vp), ("ops", c_vp),
                ("op_arg", c_vp), ("proc_type", c_vp), ("proc_params", c_vp), ("n_txns", c_u32), ("n_ops", c_u32),
                ("n_retried", c_u32), ("n_fresh", c_u32)]


_lib.ltpg_compose_retry.restype = c_int
_lib.ltpg_compose_retry.argtypes = [ctypes.POINTER(ltpg_batch), c_vp, c_u32, ctypes.POINTER(ltpg_batch),
                                    ctypes.POINTER(ltpg_batch_buf)]
_lib.ltpg_pending_aborts.restype = c_int
_lib.ltpg_pending_aborts.argtypes = [c_vp, ctypes.POINTER(c_u32)]
_lib.ltpg_route_tpcc.restype = c_int
_lib.ltpg_route_tpcc.argtypes = [ctypes.POINTER(ltpg_batch), c_u32, c_u32, c_u32, ctypes.POINTER(ltpg_batch_buf), c_vp]
_lib.ltpg_mark_memory.restype = c_int
_lib.ltpg_mark_memory.argtypes = [c_vp, c_u32, ctypes.POINTER(c_u64), ctypes.POINTER(c_u64), ctypes.POINTER(c_u32)]
_lib.ltpg_version.restype = ctypes.c_char_p
_lib.ltpg_version.argtypes = []

# C-ABI names, re-exported unchanged
ltpg_create_db = _lib.ltpg_create_db
ltpg_load_table = _lib.ltpg_load_table
ltpg_run_batch = _lib.ltpg_run_batch
ltpg_dump_table = _lib.ltpg_dump_table
ltpg_destroy_db = _lib.ltpg_destroy_db
ltpg_last_error = _lib.ltpg_last_error
ltpg_version = _lib.ltpg_version
ltpg_wait_batch = _lib.ltpg_wait_batch
ltpg_peer_handle = _lib.ltpg_peer_handle
ltpg_connect_peers = _lib.ltpg_connect_peers
ltpg_compose_retry = _lib.ltpg_compose_retry
ltpg_mark_memory = _lib.ltpg_mark_memory
ltpg_route_tpcc = _lib.ltpg_route_tpcc
ltpg_pending_aborts = _lib.ltpg_pending_aborts
LTPG_BATCH_ASYNC = 1
LTPG_BATCH_COMPACT_PARAMS = 2
LTPG_BATCH_CARRY_ABORTS = 4
LTPG_BATCH_TID_RANGE = 8
LTPG_RESULT_COMMITTED_READS, LTPG_RESULT_NO_STATUS, LTPG_RESULT_NO_ABORT_LIST = 1, 2, 4

EXPORTED = ["ltpg_create_db", "ltpg_load_table", "ltpg_run_batch", "ltpg_wait_batch", "ltpg_dump_table",
            "ltpg_destroy_db", "ltpg_last_error", "ltpg_version", "ltpg_peer_handle", "ltpg_connect_peers",
            "ltpg_compose_retry", "ltpg_mark_memory", "ltpg_route_tpcc", "ltpg_pending_aborts"]


class LtpgError(RuntimeError):
    def __init__(self, rc, msg):
        super().__init__("%s (%d): %s" % (ERR_NAMES.get(rc, "?"), rc, msg))
        self.rc = rc


def _numel(x):
    return int(x.numel()) if hasattr(x, "numel") else int(np.asarray(x).size)


def _ptr(x):
    if x is None:
        return None
    if hasattr(x, "data_ptr"):  # torch tensor (host or CUDA)
        return c_vp(x.data_ptr())
    return x.ctypes.data_as(c_vp)


def _on_device(x):
    return bool(getattr(x, "is_cuda", False))


class Database:
    """One device database (tables + PK indexes + conflict marks) on one GPU."""

    def __init__(self, n_tables, max_txns, max_ops=0, device=0, flags=0, n_warehouses=0, rank=0, world=1,
                 key_space=0, loopback=1):
        self._keep = []
        flags |= (int(loopback) & 0xF) << LTPG_FLAG_LOOPBACK_SHIFT if loopback > 1 else 0
        cfg = ltpg_config(device=device, rank=rank, world=world, max_txns=max_txns,
                          max_ops=max_ops, flags=flags, n_tables=n_tables, n_warehouses=n_warehouses,
                          key_space=key_space)
        h = c_vp()
        rc = ltpg_create_db(ctypes.byref(cfg), ctypes.byref(h))
        self.h = h
        if rc:
            msg = ltpg_last_error(h).decode() if h.value else ""
            self.close()
            raise LtpgError(rc, msg)
        self.n_tables = n_tables
        self.max_txns = max_txns
        self.max_ops = max_ops
        self.n_cols = {}
        self.has_pk = {}
        self._out = None

    # -- multi-rank peer-memory exchange bootstrap (include/ltpg.h) ----------------------------
    def peer_handle(self):
        """This rank's LTPG_PEER_HANDLE_BYTES-byte exchange handle (bytes)."""
        buf = ctypes.create_string_buffer(LTPG_PEER_HANDLE_BYTES)
        self._check(ltpg_peer_handle(self.h, ctypes.cast(buf, c_vp)))
        return buf.raw

    def connect_peers(self, handles):
        """handles: every rank's peer_handle(), in rank order."""
        blob = b"".join(bytes(h) for h in handles)
        buf = ctypes.create_string_buffer(blob, len(blob))
        self._check(ltpg_connect_peers(self.h, ctypes.cast(buf, c_vp)))

    def close(self):
        if getattr(self, "h", None) is not None and self.h.value:
            ltpg_destroy_db(self.h)
        self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def _check(self, rc):
        if rc:
            raise LtpgError(rc, ltpg_last_error(self.h).decode())

    def load_table(self, t, col_group, col_is_add, n_groups, keys, cols, capacity=None, has_pk=True,
                   owner_rule=0, layout=0):
        g = np.ascontiguousarray(col_group, dtype=np.uint8)
        a = np.ascontiguousarray(col_is_add, dtype=np.uint8)
        cols = np.ascontiguousarray(cols, dtype=np.int64)
        n = cols.shape[1] if cols.ndim == 2 else 0
        k = None if (keys is None or not has_pk) else np.ascontiguousarray(keys, dtype=np.uint64)
        cap = int(capacity if capacity is not None else max(n, 1))
        d = ltpg_table_desc(n_cols=len(g), col_group=_ptr(g), col_is_add=_ptr(a), n_groups=n_groups,
                            capacity_rows=cap, has_pk=int(bool(has_pk)), owner_rule=owner_rule,
                            layout=layout)
        self._check(ltpg_load_table(self.h, t, ctypes.byref(d), n, _ptr(k), _ptr(cols)))
        self.n_cols[t] = len(g)
        self.has_pk[t] = bool(has_pk)

    # -- batches -------------------------------------------------------------------------
    def _outputs(self, n, n_reads, device_out, pinned=False):
        if device_out:
            import torch
            dev = torch.device("cuda", torch.cuda.current_device())
            return {"status": torch.empty(n, dtype=torch.uint8, device=dev),
                    "commit_bits": torch.empty((n + 31) // 32, dtype=torch.int32, device=dev),
                    "abort_idx": torch.empty(max(n, 1), dtype=torch.int32, device=dev),
                    "n_aborted": torch.zeros(1, dtype=torch.int32, device=dev),
                    "reads": torch.empty(max(n_reads, 1), dtype=torch.int64, device=dev)}
        if pinned:  # page-locked host memory the device can write (LTPG_RESULT_COMMITTED_READS)
            import torch
            o = {"status": torch.empty(n, dtype=torch.uint8), "commit_bits": torch.empty((n + 31) // 32, dtype=torch.int32),
                 "abort_idx": torch.empty(max(n, 1), dtype=torch.int32), "n_aborted": torch.zeros(1, dtype=torch.int32),
                 "reads": torch.empty(max(n_reads, 1), dtype=torch.int64)}
            return {k: v.pin_memory().numpy() for k, v in o.items()}
        return {"status": np.empty(n, np.uint8), "commit_bits": np.empty((n + 31) // 32, np.uint32),
                "abort_idx": np.empty(max(n, 1), np.uint32), "n_aborted": np.zeros(1, np.uint32),
                "reads": np.empty(max(n_reads, 1), np.int64)}

    def _run(self, bt, n, n_reads, want_reads, device_out, stats, out, wait=True, keep=None, rflags=0):
        if out is None:
            out = self._outputs(n, n_reads, device_out, pinned=bool(rflags & LTPG_RESULT_COMMITTED_READS))
        st = ltpg_stats() if stats else None
        res = ltpg_result(commit_bits=_ptr(out["commit_bits"]),
                          status=None if rflags & LTPG_RESULT_NO_STATUS else _ptr(out["status"]),
                          abort_idx=None if rflags & LTPG_RESULT_NO_ABORT_LIST else _ptr(out["abort_idx"]),
                          n_aborted=_ptr(out["n_aborted"]),
                          reads=_ptr(out["reads"]) if want_reads else None,
                          outputs_on_device=int(device_out),
                          stats=ctypes.pointer(st) if st is not None else None, flags=rflags,
                          reads_cap=_numel(out["reads"]) if want_reads else 0)
        if not wait:
            bt.flags |= LTPG_BATCH_ASYNC
            self._check(ltpg_run_batch(self.h, ctypes.byref(bt), ctypes.byref(res)))
            return Pending(self, res, bt, st, out, n, n_reads, want_reads, device_out, keep, rflags)
        self._check(ltpg_run_batch(self.h, ctypes.byref(bt), ctypes.byref(res)))
        return self._collect(out, n, n_reads, want_reads, device_out, st, rflags)

    def _collect(self, out, n, n_reads, want_reads, device_out, st, rflags=0):
        out = dict(out)
        if not device_out:
            na = int(out["n_aborted"][0])
            if not rflags & LTPG_RESULT_NO_ABORT_LIST:
                out["abort_idx"] = out["abort_idx"][:na]
            if rflags & LTPG_RESULT_NO_STATUS:
                out["status"] = None
            if want_reads and rflags & LTPG_RESULT_COMMITTED_READS:  # the committed txns' slots only
                bits = np.asarray(out["commit_bits"])[:(n + 31) // 32].view(np.uint32)
                nc = int(np.bitwise_count(bits).sum())
                out["reads"] = out["reads"][:4 * nc]
            else:
                out["reads"] = out["reads"][:n_reads] if want_reads else None
        if st is not None:
            out["stats"] = st.as_dict()
        return out

    def run_ops(self, batch, stream=None, want_reads=True, device_out=None, stats=False, out=None,
                n_txns=None, n_ops=None, wait=True):
        """batch: dict(tid u64[n], op_begin u32[n+1], ops OP_DTYPE/uint8[n_ops*16], args i64[n_ops]).
        Pass n_txns / n_ops when the arrays are raw byte views."""
        tid, ob, ops, args = batch["tid"], batch["op_begin"], batch["ops"], batch["args"]
        n = len(tid) if n_txns is None else n_txns
        n_ops = len(args) if n_ops is None else n_ops
        on_dev = _on_device(tid)
        if device_out is None:
            device_out = on_dev
        bt = ltpg_batch(n_txns=n, tid=_ptr(tid), mode=LTPG_MODE_OPS, n_ops=n_ops, op_begin=_ptr(ob),
                        ops=_ptr(ops), op_arg=_ptr(args), inputs_on_device=int(on_dev),
                        stream=c_vp(stream) if stream else None)
        return self._run(bt, n, n_ops, want_reads, device_out, stats, out, wait, keep=batch)

    def pending_aborts(self):
        """Conflict aborts a carry=True batch would lead with (ltpg_pending_aborts)."""
        n = c_u32(0)
        self._check(ltpg_pending_aborts(self.h, ctypes.byref(n)))
        return n.value

    def run_tpcc(self, batch, clock, stream=None, want_reads=True, device_out=None, stats=False, out=None,
                 n_txns=None, wait=True, carry=False, committed_reads=False, no_status=False, no_abort_list=False):
        """batch: dict(tid u64[n], type u8[n], params u8[n,128]) -- or packed blocks:
        params = used bytes back to back and offsets u32[n+1] (see pack_params), or compact
        records with compact=True (see pack_params_compact).  A rank's shard of a global batch
        (route_tpcc) also carries grank u32[n] and n_global.  carry=True: the batch is the previous
        batch's conflict aborts (kept on the device) followed by these txns
        (LTPG_BATCH_CARRY_ABORTS); the outputs cover pending_aborts() + n txns.  tid_range=True in
        the batch dict: tid holds only the first TID, the others are consecutive (LTPG_BATCH_TID_RANGE).  committed_reads:
        reads = the result slots of the committed txns only, in rank order (host outputs must
        then be pinned memory); no_status / no_abort_list skip those outputs."""
        tid, ty, params = batch["tid"], batch["type"], batch["params"]
        offsets = batch.get("offsets")
        grank = batch.get("grank")
        nf = len(tid) if n_txns is None else n_txns
        n = nf + (self.pending_aborts() if carry else 0)
        on_dev = _on_device(tid)
        if device_out is None:
            device_out = on_dev
        bt = ltpg_batch(n_txns=nf, tid=_ptr(tid), mode=LTPG_MODE_TPCC, proc_type=_ptr(ty),
                        proc_params=_ptr(params), batch_clock=int(clock), inputs_on_device=int(on_dev),
                        stream=c_vp(stream) if stream else None, proc_offsets=_ptr(offsets),
                        flags=(LTPG_BATCH_COMPACT_PARAMS if batch.get("compact") else 0) |
                        (LTPG_BATCH_CARRY_ABORTS if carry else 0) |
                        (LTPG_BATCH_TID_RANGE if batch.get("tid_range") else 0),
                        grank=_ptr(grank), n_global=int(batch.get("n_global", 0)))
        rflags = ((LTPG_RESULT_COMMITTED_READS if committed_reads else 0) | (LTPG_RESULT_NO_STATUS if no_status else 0)
                  | (LTPG_RESULT_NO_ABORT_LIST if no_abort_list else 0))
        out = self._run(bt, n, 4 * n, want_reads, device_out, stats, out, wait, keep=batch, rflags=rflags)
        if wait and not device_out and want_reads:
            out["reads"] = out["reads"].reshape(-1, 4)
        return out

    def mark_memory(self, t):
        """(standard bytes, large-bucket bytes, allocated s_u) of table t's conflict marks (Table VIII)."""
        a, b, su = c_u64(0), c_u64(0), c_u32(0)
        self._check(ltpg_mark_memory(self.h, t, ctypes.byref(a), ctypes.byref(b), ctypes.byref(su)))
        return a.value, b.value, su.value

    def dump_table(self, t):
        nr = c_u64(0)
        self._check(ltpg_dump_table(self.h, t, ctypes.byref(nr), None, None))
        n = nr.value
        nc = self.n_cols[t]
        keys = np.zeros(max(n, 1), np.uint64)
        cols = np.zeros((nc, max(n, 1)), np.int64) if n else np.zeros((nc, 0), np.int64)
        colbuf = np.zeros(max(nc * n, 1), np.int64)
        self._check(ltpg_dump_table(self.h, t, ctypes.byref(nr), _ptr(keys), _ptr(colbuf)))
        cols = colbuf[:nc * n].reshape(nc, n)
        return (keys[:n] if self.has_pk[t] else None), cols


# used prefix of each TPC-C parameter block (include/ltpg.h layouts)
_USED = {0: None, 1: 24, 2: 8, 3: 4, 4: 4}


def pack_params(types, params):
    """Pack 128-byte TPC-C parameter blocks to their used prefixes (client side).
    Returns (packed u8[total], offsets u32[n+1]); NewOrder uses 8 + 8 * n_lines bytes."""
    types = np.asarray(types)
    params = np.asarray(params, dtype=np.uint8).reshape(len(types), 128)
    used = np.zeros(len(types), np.int64)
    for t, u in _USED.items():
        m = types == t
        used[m] = 8 + 8 * params[m, 3].astype(np.int64) if u is None else u
    offs = np.zeros(len(types) + 1, np.int64)
    np.cumsum(used, out=offs[1:])
    mask = np.arange(128)[None, :] < used[:, None]
    return params[mask], offs.astype(np.uint32)


def pack_params_compact(types, params):
    """Compact TPC-C records (include/ltpg.h LTPG_BATCH_COMPACT_PARAMS): NewOrder lines as 22-bit
    fields (item, qty, remote flag) in a little-endian bit stream plus the supply warehouses of
    remote lines, Payment amounts as u32.
    Client-side encoding (vectorised); returns (packed u8[total], offsets u32[n+1])."""
    types = np.asarray(types)
    params = np.ascontiguousarray(params, dtype=np.uint8).reshape(len(types), 128)
    n = len(types)
    comp = np.zeros((n, 128), np.uint8)
    used = np.zeros(n, np.int64)
    for t, u in _USED.items():  # other types: the used prefix
        if u is not None and t != 1:
            m = types == t
            comp[m, :u] = params[m, :u]
            used[m] = u
    no = np.nonzero(types == 0)[0]
    if len(no):
        P = params[no]
        nl = P[:, 3].astype(np.int64)
        w = P[:, 0].astype(np.uint32) | (P[:, 1].astype(np.uint32) << 8)
        L = P[:, 8:128].reshape(len(no), 15, 8)
        item = L[:, :, :4].copy().view(np.uint32)[:, :, 0]
        sw = L[:, :, 4:6].copy().view(np.uint16)[:, :, 0].astype(np.uint32)
        qty = L[:, :, 6].astype(np.uint32)
        live = np.arange(15)[None, :] < nl[:, None]
        if (live & ((item >= (1 << 17)) | (qty < 1) | (qty > 16))).any():
            raise ValueError("NewOrder line not representable compactly (item >= 2^17 or qty outside 1..16)")
        remote = live & (sw != w[:, None])
        v = np.where(live, item | ((qty - 1) << 17) | (remote.astype(np.uint32) << 21), 0).astype(np.uint32)
        C = np.zeros((len(no), 132), np.uint8)  # (+4: the last line's 4-byte window)
        C[:, :7] = P[:, :7]
        nrem = remote.sum(axis=1)
        C[:, 7] = nrem
        # 22-bit lines, little-endian bit stream: line l at bits 22 l .. 22 l + 21
        for l in range(15):
            bit = 22 * l
            x = v[:, l].astype(np.uint64) << np.uint64(bit & 7)
            for j in range(4):
                C[:, 8 + (bit >> 3) + j] |= ((x >> np.uint64(8 * j)) & np.uint64(0xFF)).astype(np.uint8)
        lb = (22 * nl + 7) // 8
        # supply warehouses of remote lines at 8 + lb + 2 k (k-th remote line)
        k = np.cumsum(remote, axis=1) - 1
        ri, li = np.nonzero(remote)
        pos = 8 + lb[ri] + 2 * k[ri, li]
        C[ri, pos] = (sw[ri, li] & 0xFF).astype(np.uint8)
        C[ri, pos + 1] = (sw[ri, li] >> 8).astype(np.uint8)
        comp[no] = C[:, :128]
        used[no] = 8 + lb + 2 * nrem
    pay = np.nonzero(types == 1)[0]
    if len(pay):
        amount = params[pay, 16:24].copy().view(np.int64)[:, 0]
        if ((amount < 0) | (amount >= (1 << 32))).any():
            raise ValueError("Payment amount not representable compactly (outside [0, 2^32))")
        comp[pay, :12] = params[pay, :12]
        comp[pay, 12:16] = amount.astype(np.uint32).view(np.uint8).reshape(len(pay), 4)
        used[pay] = 16
    offs = np.zeros(n + 1, np.int64)
    np.cumsum(used, out=offs[1:])
    mask = np.arange(128)[None, :] < used[:, None]
    return comp[mask], offs.astype(np.uint32)


class Pending:
    """An asynchronously submitted batch (LTPG_BATCH_ASYNC): .wait() completes it."""

    def __init__(self, db, res, bt, st, out, n, n_reads, want_reads, device_out, keep, rflags=0):
        self.db, self.res, self.bt, self.st, self.out = db, res, bt, st, out
        self.args = (n, n_reads, want_reads, device_out)
        self.rflags = rflags
        self.keep = keep  # host buffers must stay alive until the batch completes

    def wait(self):
        self.db._check(ltpg_wait_batch(self.db.h, ctypes.byref(self.res)))
        return self.db._collect(self.out, *self.args, self.st, self.rflags)


def part_of_w(w, nw, nparts):
    """Owning partition of warehouse w (contiguous ranges; mirrors csrc part_of_w)."""
    return 0 if nparts <= 1 else ((np.asarray(w, dtype=np.int64) - 1) * nparts) // nw


def part_of_key(key, key_space, nparts):
    """Owning partition of a key of an owner_rule-2 table (mirrors csrc part_of_key)."""
    if nparts <= 1:
        return np.zeros_like(np.asarray(key, dtype=np.uint64), dtype=np.int64)
    chunk = (int(key_space) + nparts - 1) // nparts
    return np.minimum(np.asarray(key, dtype=np.uint64) // np.uint64(chunk), nparts - 1).astype(np.int64)


def ycsb_database(workload, max_txns, max_ops, capacity=None, device=0, flags=0, loopback=1, rank=0, world=1,
                  peer_group=None):
    """YCSB usertable, key-range partitioned (owner_rule 2) when world * loopback > 1; a
    multi-rank db loads only its own key range."""
    db = Database(1, max_txns, max_ops, device=device, flags=flags, key_space=workload.n_rows, loopback=loopback,
                  rank=rank, world=world)
    g, a, ng, pk = workload.table_desc()
    keys, cols = workload.initial_table()
    if world > 1:
        own = part_of_key(keys, workload.n_rows, world) == rank
        keys, cols = keys[own], cols[:, own]
    db.load_table(0, g, a, ng, keys, cols, capacity=capacity or max(len(keys), 1), has_pk=pk, owner_rule=2)
    _connect(db, world, flags, peer_group)
    return db


def _connect(db, world, flags, group):
    """Multi-rank db with the peer-memory exchange: all-gather the handles (torch.distributed)."""
    if world > 1:
        from .dist import connect_peers
        connect_peers(db, group)


def tpcc_owner_w(t, keys, cols):
    """Warehouse that owns each row of TPC-C table t (None: replicated ITEM)."""
    from workloads.formats import (T_WAREHOUSE, T_DISTRICT, T_CUSTOMER, T_HISTORY, T_NEW_ORDER, T_ORDER,
                                   T_ORDER_LINE, T_STOCK)
    if t == T_WAREHOUSE:
        return keys.astype(np.int64)
    if t == T_DISTRICT:
        return (keys.astype(np.int64) - 1) // 10
    if t == T_CUSTOMER:
        return ((keys.astype(np.int64) - 1) // 3000 - 1) // 10
    if t == T_HISTORY:
        return cols[2].astype(np.int64)  # H_C_W_ID: the customer's owner keeps the row
    if t in (T_NEW_ORDER, T_ORDER):
        return ((keys >> np.uint64(32)).astype(np.int64) - 1) // 10
    if t == T_ORDER_LINE:
        return (((keys >> np.uint64(4)) >> np.uint64(32)).astype(np.int64) - 1) // 10
    if t == T_STOCK:
        return (keys.astype(np.int64) - 1) // 100000
    return None


def tpcc_database(workload, max_txns, tables=None, append_batches=4, device=0, flags=0, capacity=None,
                  loopback=1, rank=0, world=1, max_ops=0, peer_group=None):
    """Load the TPC-C schema; append regions sized for ``append_batches`` batches of max_txns.
    A multi-rank db (world > 1) loads only the rows of its warehouses (ITEM replicated)."""
    from workloads.formats import T_ORDER, T_NEW_ORDER, T_ORDER_LINE, T_HISTORY, T_ITEM
    db = Database(9, max_txns, max_ops, device=device, flags=flags, n_warehouses=workload.W, loopback=loopback,
                  rank=rank, world=world)
    from .dist import tpcc_rank_tables
    tables = tables if tables is not None else workload.initial_tables()
    if world > 1:
        tables = tpcc_rank_tables(tables, workload.W, rank, world)
    extra = {T_ORDER: 1, T_NEW_ORDER: 1, T_ORDER_LINE: 15, T_HISTORY: 1}
    for t, (g, a, ng, pk) in workload.table_descs().items():
        k, c = tables[t]
        n = c.shape[1]
        cap = n + extra.get(t, 0) * max_txns * append_batches
        if capacity and t in capacity:
            cap = capacity[t]
        # append-heavy tables columnar (consecutive lanes append whole sectors); the randomly
        # accessed ones row-blocked (a STOCK / CUSTOMER update writes one sector)
        db.load_table(t, g, a, ng, k, c, capacity=max(cap, 1), has_pk=pk,
                      owner_rule=0 if t == T_ITEM else 1,
                      layout=LTPG_LAYOUT_COLUMNAR if t in (T_ORDER, T_ORDER_LINE) else LTPG_LAYOUT_ROWBLOCK)
    _connect(db, world, flags, peer_group)
    return db


def route_tpcc(batch, n_warehouses, world, rank):
    """SURVEY §8(e) host routing (ltpg_route_tpcc): rank's shard of a global TPC-C batch -- the
    txns touching its warehouses, in order -- as a batch dict with grank (global ranks) and
    n_global, ready for Database.run_tpcc."""
    b = {k: np.ascontiguousarray(batch[k]) for k in ("tid", "type", "params")}
    n = len(b["tid"])
    gb = ltpg_batch(n_txns=n, tid=_ptr(b["tid"]), mode=LTPG_MODE_TPCC, proc_type=_ptr(b["type"]),
                    proc_params=_ptr(b["params"]))
    out = {"tid": np.zeros(max(n, 1), np.uint64), "type": np.zeros(max(n, 1), np.uint8),
           "params": np.zeros((max(n, 1), LTPG_PARAM_BYTES), np.uint8)}
    grank = np.zeros(max(n, 1), np.uint32)
    buf = ltpg_batch_buf(cap_txns=n, tid=_ptr(out["tid"]), proc_type=_ptr(out["type"]),
                         proc_params=_ptr(out["params"]))
    rc = ltpg_route_tpcc(ctypes.byref(gb), n_warehouses, world, rank, ctypes.byref(buf), grank.ctypes.data_as(c_vp))
    if rc:
        raise LtpgError(rc, "ltpg_route_tpcc: invalid arguments")
    m = buf.n_txns
    return {"tid": out["tid"][:m], "type": out["type"][:m], "params": out["params"][:m], "grank": grank[:m],
            "n_global": n}


def compose_retry(prev, abort_idx, fresh, max_txns, max_ops=0):
    """a9, the host retry loop (ltpg_compose_retry): the next batch = the conflict aborts of
    `prev` (ascending ranks from run_ops / run_tpcc, original TIDs) followed by as many txns of
    `fresh` as fit in max_txns (and max_ops).  Host numpy batches in, a host numpy batch out;
    returns (batch, n_fresh_taken)."""
    ops = "op_begin" in prev
    abort_idx = np.ascontiguousarray(abort_idx, dtype=np.uint32)

    def desc(b):
        if ops:
            b = {k: np.ascontiguousarray(v) for k, v in b.items()}
            return b, ltpg_batch(n_txns=len(b["tid"]), tid=_ptr(b["tid"]), mode=LTPG_MODE_OPS,
                                 n_ops=len(b["args"]), op_begin=_ptr(b["op_begin"]), ops=_ptr(b["ops"]),
                                 op_arg=_ptr(b["args"]))
        b = {k: np.ascontiguousarray(v) for k, v in b.items()}
        return b, ltpg_batch(n_txns=len(b["tid"]), tid=_ptr(b["tid"]), mode=LTPG_MODE_TPCC,
                             proc_type=_ptr(b["type"]), proc_params=_ptr(b["params"]))

    pk, pd = desc(prev)
    fk, fd = desc(fresh)
    out = {"tid": np.zeros(max_txns, np.uint64)}
    if ops:
        out.update(op_begin=np.zeros(max_txns + 1, np.uint32), ops=np.zeros(max(max_ops, 1), pk["ops"].dtype),
                   args=np.zeros(max(max_ops, 1), np.int64))
        buf = ltpg_batch_buf(cap_txns=max_txns, cap_ops=max_ops, tid=_ptr(out["tid"]), op_begin=_ptr(out["op_begin"]),
                             ops=_ptr(out["ops"]), op_arg=_ptr(out["args"]))
    else:
        out.update(type=np.zeros(max_txns, np.uint8), params=np.zeros((max_txns, LTPG_PARAM_BYTES), np.uint8))
        buf = ltpg_batch_buf(cap_txns=max_txns, tid=_ptr(out["tid"]), proc_type=_ptr(out["type"]),
                             proc_params=_ptr(out["params"]))
    rc = ltpg_compose_retry(ctypes.byref(pd), abort_idx.ctypes.data_as(c_vp), len(abort_idx), ctypes.byref(fd),
                            ctypes.byref(buf))
    if rc:
        raise LtpgError(rc, "ltpg_compose_retry: invalid arguments")
    n, m = buf.n_txns, buf.n_ops
    if ops:
        res = {"tid": out["tid"][:n], "op_begin": out["op_begin"][:n + 1], "ops": out["ops"][:m], "args": out["args"][:m]}
    else:
        res = {"tid": out["tid"][:n], "type": out["type"][:n], "params": out["params"][:n]}
    return res, buf.n_fresh
