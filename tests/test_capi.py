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
            assert len(q) == 8 + 4 * nl + 2 * nrem
            out[r, :7] = q[:7]
            w = int(q[0]) | int(q[1]) << 8
            k = 0
            for li in range(nl):
                v = int.from_bytes(bytes(q[8 + 4 * li:12 + 4 * li]), "little")
                sw = w
                if (v >> 21) & 1:
                    a = 8 + 4 * nl + 2 * k
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
    decoder of the documented layout, with ~1/3 fewer bytes than used prefixes."""
    import paper_conf_icde_wei0l0lzj024_b200 as L
    from workloads import tpcc
    wl = tpcc.TpccWorkload(8, seed=5, mix=tpcc.MIX_FULL, remote_line_frac=0.2)
    b = wl.batch(3000, 1, 0)
    packed, offs = L.pack_params_compact(b["type"], b["params"])
    pref, poffs = L.pack_params(b["type"], b["params"])
    assert packed.nbytes < 0.8 * pref.nbytes
    dec = _unpack_compact_model(b["type"], packed, offs)
    used = np.diff(poffs.astype(np.int64))
    for r in range(len(b["type"])):
        assert (dec[r, :used[r]] == b["params"][r, :used[r]]).all(), r
