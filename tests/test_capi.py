"""CPU-only checks of the C-ABI boundary: the library loads and exports every
symbol include/ltpg.h declares; struct layouts match the header."""
import ctypes
import os
import re
import subprocess

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
