"""C-ABI library checks that need no GPU (-m "not gpu"): the .so builds/loads, exports every
symbol include/spgemm.h declares, answers host-only queries, and fails cleanly (no crash,
no fallback) when no sm_100 device is present."""
import ctypes
import os
import re

import numpy as np
import pytest
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "spgemm.h")


@pytest.fixture(scope="module")
def lib():
    from paper_conf_icpp_nagasakanm17_b200 import build
    build.build()
    from paper_conf_icpp_nagasakanm17_b200 import _lib
    return _lib.load()


def _declared():
    txt = open(HEADER).read()
    return sorted(set(re.findall(r"SPGEMM_API[^;(]*?\b(spgemm_\w+)\s*\(", txt)))


def test_header_declares_abi():
    names = _declared()
    for must in ("spgemm_create", "spgemm_symbolic", "spgemm_numeric", "spgemm_destroy"):
        assert must in names


def test_exports_every_declared_symbol(lib):
    from paper_conf_icpp_nagasakanm17_b200 import _lib
    names = _declared()
    assert sorted(_lib.EXPORTS) == names
    for nm in names:
        assert hasattr(lib, nm), nm
    # nothing else leaks (kernels and helpers are hidden)
    out = os.popen(f"nm -D --defined-only {_lib.LIB_PATH}").read()
    exported = sorted(set(re.findall(r"\bT (spgemm_\w+)", out)))
    assert exported == names


def test_library_is_sm100a(lib):
    from paper_conf_icpp_nagasakanm17_b200 import _lib
    out = os.popen(f"/usr/local/cuda/bin/cuobjdump --list-elf {_lib.LIB_PATH}").read()
    assert "sm_100a" in out
    assert b"sm_100a" in lib.spgemm_version()


def test_host_queries(lib):
    from paper_conf_icpp_nagasakanm17_b200 import group_bounds
    for phase in (1, 2):
        b = group_bounds(phase)
        assert len(b) >= 7 and b == sorted(b) and len(set(b)) == len(b)
    assert lib.spgemm_status_string(0) == b"SPGEMM_OK"
    assert lib.spgemm_status_string(5) == b"SPGEMM_ERR_INDEX_OVERFLOW"
    arr = (ctypes.c_int64 * 24)()
    n = ctypes.c_int32()
    assert lib.spgemm_group_bounds(3, arr, ctypes.byref(n)) == 1  # INVALID_ARG
    assert lib.spgemm_set_option(None, 0, 0) == 1
    assert lib.spgemm_symbolic(None, 0, 0, 0, None, None, None, None, None, None, None) == 1
    assert lib.spgemm_numeric(None, 0, None, None, None, None) == 1
    assert lib.spgemm_destroy(None) == 1


def test_group_bounds_match_oracle_grouping():
    """The library's group table, fed to the oracle's grouping rule, reproduces Table I's
    shape: PWARP-size rows land in group 0 and the largest keys in the overflow group."""
    import oracle
    from paper_conf_icpp_nagasakanm17_b200 import group_bounds
    up = group_bounds(1)
    assert oracle.bin_of([1], up)[0] == 0
    assert oracle.bin_of([up[-1] + 1], up)[0] == len(up)
    assert up[0] <= 32  # Table I group 6 is "0-32"; PWARP rows are small


@pytest.mark.skipif(torch.cuda.is_available(), reason="checks the no-GPU error path")
def test_create_without_gpu_fails_cleanly(lib):
    h = ctypes.c_void_p()
    st = lib.spgemm_create(ctypes.byref(h), 0, None, None)
    assert st in (4, 6)  # ERR_CUDA or NOT_SUPPORTED, never OK on a GPU-less box
    if h.value:
        assert len(lib.spgemm_last_error(h)) > 0
        assert lib.spgemm_destroy(h) == 0


def test_product_path_has_no_oracle_import():
    """The package must not import or reference the oracle (no CPU fallback)."""
    pkg = os.path.join(ROOT, "paper_conf_icpp_nagasakanm17_b200")
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".h")):
                txt = open(os.path.join(dirpath, f)).read()
                assert "import oracle" not in txt and "from oracle" not in txt, f
                assert "gustavson" not in txt.lower(), f


def test_binding_matches_header_enums_and_stats_layout(tmp_path):
    """The Python binding's option ids, kernel-family ids and spgemm_stats_t layout agree with
    include/spgemm.h (compiled with gcc: sizeof and offsetof of every field)."""
    import subprocess
    from paper_conf_icpp_nagasakanm17_b200 import _lib
    txt = open(HEADER).read()
    opts = {m.group(1).lower(): int(m.group(2)) for m in re.finditer(r"SPGEMM_OPT_(\w+)\s*=\s*(\d+)", txt)}
    assert opts == _lib.OPTIONS
    kinds = {int(m.group(2)): m.group(1).lower() for m in re.finditer(r"SPGEMM_KERNEL_(\w+)\s*=\s*(\d+)", txt)}
    assert kinds == _lib.KERNELS
    fields = [f for f, _ in _lib.Stats._fields_]
    src = tmp_path / "layout.c"
    src.write_text("#include <stdio.h>\n#include <stddef.h>\n#include \"spgemm.h\"\nint main(void){\n"
                   "printf(\"%zu\\n\", sizeof(spgemm_stats_t));\n" +
                   "".join(f"printf(\"%zu\\n\", offsetof(spgemm_stats_t, {f}));\n" for f in fields) + "return 0;}\n")
    exe = tmp_path / "layout"
    subprocess.check_call(["gcc", "-std=c99", f"-I{os.path.dirname(HEADER)}", str(src), "-o", str(exe)])
    out = [int(x) for x in subprocess.check_output([str(exe)]).split()]
    assert out[0] == ctypes.sizeof(_lib.Stats)
    assert out[1:] == [getattr(_lib.Stats, f).offset for f in fields]
