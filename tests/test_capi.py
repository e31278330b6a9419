"""CPU-only checks of the C-ABI boundary: the library loads and exports every
symbol include/ltpg.h declares; struct layouts match the header."""
import ctypes
import os
import re
import subprocess

import numpy as np
import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "ltpg.h")


def declared_functions():
    src = open(HEADER).read()
    return sorted(set(re.findall(r"LTPG_API\s+[\w\s\*]+?\b(ltpg_\w+)\s*\(", src)))


def test_header_declares_boundary():
    fns = declared_functions()
    for name in ("ltpg_create_db", "ltpg_load_table", "ltpg_run_batch", "ltpg_dump_table",
                 "ltpg_destroy_db", "ltpg_last_error"):
        assert name in fns


def test_library_exports_every_declared_symbol():
    import paper_conf_icde_wei0l0lzj024_b200 as L
    out = subprocess.check_output(["nm", "-D", "--defined-only", L.LIB_PATH]).decode()
    exported = set(re.findall(r"\sT\s(ltpg_\w+)", out))
    for name in declared_functions():
        assert name in exported, name
        assert hasattr(L, name)
    assert set(L.EXPORTED) == set(declared_functions())
    assert L.ltpg_version().decode().startswith("ltpg-b200")


def test_struct_layouts_match_header():
    """Compile a tiny C program against the header and compare sizes/offsets with ctypes."""
    import paper_conf_icde_wei0l0lzj024_b200 as L
    prog = r"""
#include <stdio.h>
#include <stddef.h>
#include "ltpg.h"
int main(void) {
  printf("%zu %zu %zu %zu %zu %zu\n", sizeof(ltpg_op), sizeof(ltpg_config), sizeof(ltpg_table_desc),
         sizeof(ltpg_batch), sizeof(ltpg_result), sizeof(ltpg_stats));
  printf("%zu %zu %zu\n", offsetof(ltpg_batch, batch_clock), offsetof(ltpg_batch, stream),
         offsetof(ltpg_result, stats));
  printf("%zu %zu\n", sizeof(ltpg_batch_buf), offsetof(ltpg_batch_buf, n_txns));
  return 0;
}
"""
    import tempfile
    with tempfile.TemporaryDirectory() as d:
        c = os.path.join(d, "t.c")
        exe = os.path.join(d, "t")
        open(c, "w").write(prog)
        subprocess.check_call(["gcc", "-I", os.path.join(ROOT, "include"), c, "-o", exe])
        lines = subprocess.check_output([exe]).decode().split("\n")
    sizes = [int(x) for x in lines[0].split()]
    offs = [int(x) for x in lines[1].split()]
    assert sizes == [16, ctypes.sizeof(L.ltpg_config), ctypes.sizeof(L.ltpg_table_desc),
                     ctypes.sizeof(L.ltpg_batch), ctypes.sizeof(L.ltpg_result), ctypes.sizeof(L.ltpg_stats)]
    assert offs == [L.ltpg_batch.batch_clock.offset, L.ltpg_batch.stream.offset, L.ltpg_result.stats.offset]
    assert [int(x) for x in lines[2].split()] == [ctypes.sizeof(L.ltpg_batch_buf), L.ltpg_batch_buf.n_txns.offset]


def test_op_record_matches_generator_format():
    from workloads.formats import OP_DTYPE
    assert OP_DTYPE.itemsize == 16
    assert [OP_DTYPE.fields[f][1] for f in ("key", "kind", "table", "col", "aux")] == [0, 8, 9, 10, 12]


def test_create_without_gpu_fails_cleanly(has_gpu):
    if has_gpu:
        pytest.skip("GPU present")
    import paper_conf_icde_wei0l0lzj024_b200 as L
    with pytest.raises(L.LtpgError):
        L.Database(1, 16, 16)


def test_sm100a_cubin_present():
    import paper_conf_icde_wei0l0lzj024_b200 as L
    out = subprocess.check_output(["/usr/local/cuda/bin/cuobjdump", "--list-elf", L.LIB_PATH]).decode()
    assert "sm_100a" in out


def _unpack_compact_model(types, packed, offs):
    """Independent reading of include/ltpg.h's compact record layout (test model)."""
    out = np.zeros((len(types), 128), np.uint8)
    for r, t in enumerate(types):
        q = packed[offs[r]:offs[r + 1]]
        if t == 0:
            nl, nrem = int(q[3]), int(q[7])
            lb = (22 * nl + 7) // 8
            assert len(q) == 8 + lb + 2 * nrem
            out[r, :7] = q[:7]
            w = int(q[0]) | int(q[1]) << 8
            stream = int.from_bytes(bytes(q[8:8 + lb]), "little")  # the lines' bit stream
            k = 0
            for li in range(nl):
                v = (stream >> (22 * li)) & ((1 << 22) - 1)
                sw = w
                if (v >> 21) & 1:
                    a = 8 + lb + 2 * k
                    sw = int(q[a]) | int(q[a + 1]) << 8
                    k += 1
                rec = (v & 0x1FFFF).to_bytes(4, "little") + sw.to_bytes(2, "little") + bytes([((v >> 17) & 15) + 1, 0])
                out[r, 8 + 8 * li:16 + 8 * li] = np.frombuffer(rec, np.uint8)
            assert k == nrem
        elif t == 1:
            assert len(q) == 16
            out[r, :12] = q[:12]
            out[r, 16:20] = q[12:16]
        else:
            out[r, :len(q)] = q
    return out


def test_compact_params_roundtrip_and_size():
    """pack_params_compact: the used prefix of every TPC-C block is recovered by an independent
    decoder of the documented layout (22-bit lines in a bit stream), with about half the bytes
    of used prefixes."""
    import paper_conf_icde_wei0l0lzj024_b200 as L
    from workloads import tpcc
    wl = tpcc.TpccWorkload(8, seed=5, mix=tpcc.MIX_FULL, remote_line_frac=0.2)
    b = wl.batch(3000, 1, 0)
    packed, offs = L.pack_params_compact(b["type"], b["params"])
    pref, poffs = L.pack_params(b["type"], b["params"])
    assert packed.nbytes < 0.6 * pref.nbytes
    dec = _unpack_compact_model(b["type"], packed, offs)
    used = np.diff(poffs.astype(np.int64))
    for r in range(len(b["type"])):
        assert (dec[r, :used[r]] == b["params"][r, :used[r]]).all(), r


# ---- a9: the host retry loop (ltpg_compose_retry; host-only, runs without a GPU) ---------------
def _np_retry_ops(prev, ab, fresh, cap_txns, cap_ops):
    """Plain reference: aborted txns (ascending ranks) then the fresh prefix that fits."""
    ob = prev["op_begin"]
    txns = [(prev["tid"][r], prev["ops"][ob[r]:ob[r + 1]], prev["args"][ob[r]:ob[r + 1]]) for r in ab]
    nops = sum(len(t[1]) for t in txns)
    fb = fresh["op_begin"]
    for j in range(len(fresh["tid"])):
        k = fb[j + 1] - fb[j]
        if len(txns) == cap_txns or nops + k > cap_ops:
            break
        txns.append((fresh["tid"][j], fresh["ops"][fb[j]:fb[j + 1]], fresh["args"][fb[j]:fb[j + 1]]))
        nops += k
    lens = np.array([len(t[1]) for t in txns], np.uint32)
    return {"tid": np.array([t[0] for t in txns], np.uint64),
            "op_begin": np.concatenate([[0], np.cumsum(lens)]).astype(np.uint32),
            "ops": np.concatenate([t[1] for t in txns]), "args": np.concatenate([t[2] for t in txns])}


@pytest.mark.parametrize("seed", range(6))
def test_compose_retry_ops_equals_reference(seed):
    import paper_conf_icde_wei0l0lzj024_b200 as L
    from workloads.ycsb import YcsbWorkload
    wl = YcsbWorkload(5000, theta=0.8, ops_per_txn=3 + seed % 3, seed=seed)
    prev = wl.batch(300, 1, 0)
    fresh = wl.batch(400, 301, 1)
    rng = np.random.default_rng(seed)
    ab = np.sort(rng.choice(300, size=rng.integers(0, 300), replace=False)).astype(np.uint32)
    cap_t, cap_o = 350, (350 * (3 + seed % 3)) - 7 * seed
    got, nf = L.compose_retry(prev, ab, fresh, cap_t, cap_o)
    exp = _np_retry_ops(prev, ab, fresh, cap_t, cap_o)
    assert nf == len(exp["tid"]) - len(ab)
    for k in exp:
        assert (got[k] == exp[k]).all(), k
    assert (np.diff(got["tid"].astype(np.int64)) > 0).all()  # TID order preserved


def test_compose_retry_tpcc_and_errors():
    import paper_conf_icde_wei0l0lzj024_b200 as L
    from workloads import tpcc
    wl = tpcc.TpccWorkload(2, seed=3, mode="strict", mix=tpcc.MIX_FULL)
    prev = wl.batch(200, 1, 0)
    fresh = wl.batch(200, 201, 1)
    ab = np.array([0, 5, 17, 199], np.uint32)
    got, nf = L.compose_retry(prev, ab, fresh, 150)
    assert nf == 146 and len(got["tid"]) == 150
    assert (got["tid"][:4] == prev["tid"][ab]).all() and (got["tid"][4:] == fresh["tid"][:146]).all()
    assert (got["type"][:4] == prev["type"][ab]).all() and (got["params"][:4] == prev["params"][ab]).all()
    assert (got["params"][4:] == fresh["params"][:146]).all()
    for bad in (np.array([5, 5], np.uint32), np.array([7, 3], np.uint32), np.array([200], np.uint32)):
        with pytest.raises(L.LtpgError):
            L.compose_retry(prev, bad, fresh, 150)  # not ascending / out of range
    with pytest.raises(L.LtpgError):
        L.compose_retry(fresh, np.array([0], np.uint32), prev, 150)  # fresh TIDs must follow the retried
    with pytest.raises(L.LtpgError):
        L.compose_retry(prev, np.arange(151, dtype=np.uint32), fresh, 150)  # aborts alone overflow
