"""CPU-side checks of the C ABI: the library builds/loads, exports every symbol
include/dbc.h declares, and rejects bad input on the host (no GPU needed)."""

from __future__ import annotations

import ctypes
import os
import re

import numpy as np
import pytest

import workloads as W

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "dbc.h")


def _declared_functions():
    src = open(HEADER).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    names = re.findall(r"^\s*(?:const\s+)?[a-z_0-9]+\s*\*?\s*(dbc_[a-z_0-9]+)\s*\(", src, flags=re.M)
    return sorted(set(names))


@pytest.fixture(scope="module")
def lib():
    from paper_conf_ipps_mclaughlinb14_b200 import dbc

    if not os.path.exists(dbc.LIB_PATH):
        import __graft_entry__

        __graft_entry__.build()
    return dbc.load_library()


def test_header_declares_the_survey_entry_points():
    names = _declared_functions()
    for f in ["dbc_create", "dbc_static_compute", "dbc_insert_edges", "dbc_get_bc",
              "dbc_get_bc_partial_device", "dbc_get_root_state", "dbc_destroy",
              "dbc_insert_edges_device", "dbc_strerror", "dbc_last_error"]:
        assert f in names


def test_library_exports_every_declared_symbol(lib):
    from paper_conf_ipps_mclaughlinb14_b200 import dbc

    names = _declared_functions()
    assert names, "no declarations parsed"
    for f in names:
        assert hasattr(lib, f), f"libdbc.so does not export {f}"
        assert f in dbc.SIGNATURES, f"binding lacks {f}"


def test_built_for_sm100a():
    from paper_conf_ipps_mclaughlinb14_b200 import dbc
    import subprocess

    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", dbc.LIB_PATH],
                         capture_output=True, text=True).stdout
    assert "sm_100a" in out


def test_abi_version_and_strerror(lib):
    assert lib.dbc_abi_version() == 2
    assert lib.dbc_strerror(-6) == b"invalid edge in batch"
    assert lib.dbc_strerror(0) == b"ok"


def _create(lib, n, rp, col, roots):
    from paper_conf_ipps_mclaughlinb14_b200 import dbc

    out = ctypes.c_void_p()
    rp = np.ascontiguousarray(rp, np.int64)
    col = np.ascontiguousarray(col, np.int32)
    roots = np.ascontiguousarray(roots, np.int32)
    rc = lib.dbc_create(ctypes.byref(out), n, dbc._np_ptr(rp), dbc._np_ptr(col),
                        dbc._np_ptr(roots), roots.size, None)
    return rc, out


@pytest.mark.parametrize("case", ["asym", "selfloop", "dup", "range", "rp0", "roots_dup", "root_range", "n0"])
def test_create_rejects_bad_input_on_host(lib, case):
    g = W.path_graph(4)
    rp, col, roots, n = g.row_ptr.copy(), g.col.copy(), np.array([0, 1], np.int32), 4
    if case == "asym":
        col[0] = 2  # row 0: [2] but row 2 has no 0
    elif case == "selfloop":
        col[0] = 0
    elif case == "dup":
        col[1:3] = 0  # row 1 = [0, 0]
    elif case == "range":
        col[0] = 9
    elif case == "rp0":
        rp = rp + 1
    elif case == "roots_dup":
        roots = np.array([1, 1], np.int32)
    elif case == "root_range":
        roots = np.array([7], np.int32)
    elif case == "n0":
        n = 0
    rc, out = _create(lib, n, rp, col, roots)
    assert rc == -1 and not out.value
    assert lib.dbc_last_error(None)


def test_python_binding_raises_without_fallback(monkeypatch, tmp_path):
    from paper_conf_ipps_mclaughlinb14_b200 import dbc

    monkeypatch.setattr(dbc, "_lib", None)
    monkeypatch.setattr(dbc, "LIB_PATH", str(tmp_path / "missing.so"))
    with pytest.raises(ImportError):
        dbc.load_library()


def test_product_never_imports_oracle():
    pkg = os.path.join(ROOT, "paper_conf_ipps_mclaughlinb14_b200")
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".h", ".cpp")):
                txt = open(os.path.join(dirpath, f)).read()
                assert "import oracle" not in txt and "from oracle" not in txt, f
                assert "oracle/" not in txt.replace("oracle/ ", ""), f


def test_binding_struct_layouts_match_the_header(tmp_path):
    """dbc_options / dbc_tuning / dbc_insert_stats / dbc_timings: the ctypes
    mirrors have the C sizes and field offsets (compiled against include/dbc.h)."""
    import subprocess

    from paper_conf_ipps_mclaughlinb14_b200 import dbc

    structs = {"dbc_options": dbc.Options, "dbc_tuning": dbc.Tuning,
               "dbc_insert_stats": dbc.InsertStats, "dbc_timings": dbc.Timings}
    lines = ['#include <stdio.h>', '#include <stddef.h>', '#include "dbc.h"', "int main(void) {"]
    for cname, py in structs.items():
        lines.append(f'printf("{cname} size %zu\\n", sizeof({cname}));')
        for fname, _ in py._fields_:
            lines.append(f'printf("{cname} {fname} %zu\\n", offsetof({cname}, {fname}));')
    lines.append("return 0; }")
    src = tmp_path / "layout.c"
    src.write_text("\n".join(lines))
    exe = tmp_path / "layout"
    subprocess.check_call(["gcc", "-I", os.path.join(ROOT, "include"), str(src), "-o", str(exe)])
    out = subprocess.run([str(exe)], capture_output=True, text=True, check=True).stdout.split("\n")
    got = {tuple(l.split()[:2]): int(l.split()[2]) for l in out if l}
    for cname, py in structs.items():
        assert got[(cname, "size")] == ctypes.sizeof(py), cname
        for fname, _ in py._fields_:
            assert got[(cname, fname)] == getattr(py, fname).offset, (cname, fname)
