"""The C-ABI library loads and exports every symbol include/ecl_mst.h declares
(no compute calls: this runs without a GPU)."""
import ctypes
import os
import re
import subprocess

import pytest

from paper_conf_sc_fallingsb23_b200 import _native, build

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def lib():
    build.build()
    return _native.load()


def declared_functions():
    src = open(os.path.join(ROOT, "include", "ecl_mst.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(ecl_mst\w*)\s*\(", src)))


def test_exports_every_declared_symbol(lib):
    names = declared_functions()
    assert len(names) >= 8
    for name in names:
        assert hasattr(lib, name), name
    assert sorted(_native.EXPORTED) == names


def _c_layout(tmp_path, struct, fields):
    """sizeof and offsetof(field) of a header struct, as gcc lays it out."""
    src = tmp_path / "layout.c"
    lines = ["#include <stdio.h>", "#include <stddef.h>", '#include "ecl_mst.h"', "int main(void) {",
             f'printf("%zu\\n", sizeof({struct}));']
    lines += [f'printf("%zu\\n", offsetof({struct}, {f}));' for f in fields]
    lines += ["return 0; }"]
    src.write_text("\n".join(lines))
    exe = tmp_path / "layout"
    subprocess.check_call(["gcc", "-std=c11", "-I", os.path.join(ROOT, "include"), "-o", str(exe), str(src)])
    out = [int(x) for x in subprocess.check_output([str(exe)]).split()]
    return out[0], out[1:]


@pytest.mark.parametrize("struct,cls", [("ecl_mst_options", "EclMstOptions"), ("ecl_mst_stats", "EclMstStats")])
def test_struct_layouts_match_header(tmp_path, struct, cls):
    """The ctypes mirrors of the header structs have gcc's size and field offsets."""
    C = getattr(_native, cls)
    names = [f[0] for f in C._fields_]
    size, offs = _c_layout(tmp_path, struct, names)
    assert ctypes.sizeof(C) == size
    assert [getattr(C, f).offset for f in names] == offs


def test_workspace_bytes(lib):
    b = _native.ecl_mst_workspace_bytes(1000, 5000)
    assert b >= 1000 * (4 + 16) + 5000 * 16
    assert lib.ecl_mst_workspace_bytes(-1, 10) == 0
    assert lib.ecl_mst_workspace_bytes(10, 1 << 33) == 0
    # C5-sized graph fits comfortably in one B200 (180 GB)
    assert _native.ecl_mst_workspace_bytes(1 << 26, 2_000_000_000) < 70e9


def test_argument_validation_without_gpu(lib):
    o = _native.default_options()
    assert o.filter == -1 and o.path_halving == 1 and o.atomic_guards == -1 and o.flatten == 1
    assert o.seed == 0x5EED and o.threshold_samples == 1024 and o.refilter == -1 and o.filter_c == 0
    rc = lib.ecl_mst_device(-1, 0, None, None, None, None, None, None, 0, None, None)
    assert rc == _native.ERR_INVALID
    assert b"negative" in lib.ecl_mst_last_error()
    rc = lib.ecl_mst_device(5, 1 << 33, None, None, None, None, None, None, 0, None, None)
    assert rc == _native.ERR_TOO_LARGE
    buf = ctypes.create_string_buffer(64)
    rc = lib.ecl_mst_device(5, 10, buf, buf, buf, buf, buf, buf, 8, None, None)
    assert rc == _native.ERR_WORKSPACE


def test_no_oracle_in_product_path():
    pkg = os.path.join(ROOT, "paper_conf_sc_fallingsb23_b200")
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".h", ".c")):
                text = open(os.path.join(dirpath, f)).read()
                assert "import oracle" not in text and "from oracle" not in text, f
                assert "oracle_kruskal" not in text, f
