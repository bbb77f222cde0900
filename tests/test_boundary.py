"""The C-ABI boundary (include/bc.h) without a GPU: the library loads, exports every
symbol the header declares, agrees with the header on struct layouts, and refuses to
run without an sm_100 device (no CPU fallback)."""
import ctypes
import os
import re

import numpy as np
import pytest

import bcgen
import paper_conf_pldi_eizenbergppmd17_b200 as bc

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "bc.h")


def declared_functions():
    src = open(HEADER).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(bc_[a-z_]+)\s*\(", src)))


def test_library_exports_every_declared_symbol():
    L = bc.lib()
    decl = declared_functions()
    assert set(decl) >= {"bc_init", "bc_load_trace", "bc_detect", "bc_races", "bc_destroy",
                         "bc_status_string"}
    for name in decl:
        assert hasattr(L, name), name
    assert sorted(bc.EXPORTS) == decl


def test_struct_layouts_match_header():
    assert bcgen.RECORD_DTYPE.itemsize == 272 == bc.RECORD_BYTES
    assert bc.RACE_DTYPE.itemsize == 32
    assert bc.RACE_DTYPE == np.dtype(bcgen.RACE_DTYPE)
    # compile the header with the host C compiler and compare the layouts ctypes uses
    import subprocess, tempfile
    with tempfile.TemporaryDirectory() as d:
        c = os.path.join(d, "sz.c")
        open(c, "w").write('#include <stdio.h>\n#include <stddef.h>\n#include "bc.h"\n'
                           'int main(){printf("%zu %zu %zu %zu %zu\\n", sizeof(bc_record), sizeof(bc_race),'
                           ' sizeof(bc_config), sizeof(bc_stats), offsetof(bc_stats, ms_total));return 0;}\n')
        exe = os.path.join(d, "sz")
        subprocess.check_call(["gcc", "-I", os.path.join(ROOT, "include"), c, "-o", exe])
        got = [int(x) for x in subprocess.check_output([exe]).split()]
    assert got == [272, 32, ctypes.sizeof(bc._Config), ctypes.sizeof(bc._Stats), bc._Stats.ms_total.offset]
    src = open(HEADER).read()
    for name, val in [("BC_OP_LD", 0), ("BC_OP_ATOM", 2), ("BC_OP_AR_GLB", 8), ("BC_OP_FI", 13)]:
        assert re.search(rf"{name} = {val}\b", src), name
    assert bcgen.OP_AR_GLB == 8 and bcgen.OP_FI == 13


def test_status_strings():
    L = bc.lib()
    for code in range(0, -9, -1):
        assert L.bc_status_string(code)
    assert bc.phase_names()[:3] == ["header", "partition", "replay"]


def test_no_cpu_fallback():
    import torch
    if torch.cuda.is_available():
        pytest.skip("a GPU is present")
    with pytest.raises(bc.BcError) as e:
        bc.Context(dict(grid=(1,), block=(32,), smem_bytes=0))
    assert e.value.status == -4  # BC_ERR_CUDA


def test_invalid_args():
    with pytest.raises(bc.BcError) as e:
        bc.Context(dict(grid=(1,), block=(2048,), smem_bytes=0))
    assert e.value.status == -1
    with pytest.raises(bc.BcError) as e:
        bc.Context(dict(grid=(1,), block=(32,), granule_log2=5))
    assert e.value.status == -1
