"""The C-ABI library loads and exports every symbol include/louvain.h declares,
and the host-side validation path reports the documented error codes (no GPU
compute is called here)."""
import ctypes
import os
import re

import numpy as np
import pytest

import paper_conf_ipps_naimmht17_b200 as lvb

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def declared_functions():
    names = []
    for hdr in sorted(os.listdir(os.path.join(ROOT, "include"))):
        if not hdr.endswith(".h"):
            continue
        text = open(os.path.join(ROOT, "include", hdr)).read()
        text = re.sub(r"/\*.*?\*/", "", text, flags=re.S)
        names += re.findall(r"^\s*(?:const\s+)?\w+\s*\*?\s*(louvain_\w+)\s*\(", text, flags=re.M)
    return sorted(set(names))


def test_header_declares_north_star_entry_points():
    names = declared_functions()
    for must in ("louvain_create_csr", "louvain_sweep", "louvain_aggregate", "louvain_run", "louvain_modularity"):
        assert must in names


def test_every_declared_symbol_is_exported():
    L = ctypes.CDLL(lvb.LIB_PATH)
    missing = [n for n in declared_functions() if not hasattr(L, n)]
    assert not missing, missing
    assert set(declared_functions()) == set(lvb.FUNCS)  # the binding covers the whole ABI


def test_struct_layouts_match_header(tmp_path):
    # compile a probe against the real header and compare sizes/offsets with the binding
    src = tmp_path / "probe.c"
    src.write_text("""
#include <stdio.h>
#include <stddef.h>
#include "louvain.h"
int main(void) {
  printf("%zu %zu %zu %zu %zu %zu %zu\\n", sizeof(louvain_params_t), sizeof(louvain_qnum_t),
         sizeof(louvain_stats_t), offsetof(louvain_params_t, size_limit), offsetof(louvain_params_t, max_levels),
         offsetof(louvain_stats_t, edges_swept), offsetof(louvain_stats_t, q));
  return 0;
}
""")
    exe = tmp_path / "probe"
    import subprocess
    subprocess.run(["gcc", "-I", os.path.join(ROOT, "include"), "-o", str(exe), str(src)], check=True)
    got = [int(x) for x in subprocess.run([str(exe)], capture_output=True, text=True).stdout.split()]
    assert got == [ctypes.sizeof(lvb.Params), ctypes.sizeof(lvb.QNum), ctypes.sizeof(lvb.Stats),
                   lvb.Params.size_limit.offset, lvb.Params.max_levels.offset,
                   lvb.Stats.edges_swept.offset, lvb.Stats.q.offset]


def test_params_default_are_the_papers():
    p = lvb.params()
    assert (p.mode, p.singleton_rule, p.revert_on_decrease) == (0, 1, 1)
    assert (p.th_bin_exp, p.th_final_exp, p.size_limit) == (2, 6, 100000)
    assert list(p.deg_bounds) == [4, 8, 16, 32, 84, 319]


def _create(rowptr, col, w=None, flags=lvb.VALIDATE):
    h = ctypes.c_void_p()
    rowptr = np.ascontiguousarray(rowptr, dtype=np.int64)
    col = np.ascontiguousarray(col, dtype=np.int32)
    wp = None
    if w is not None:
        w = np.ascontiguousarray(w, dtype=np.uint32)
        wp = w.ctypes.data
    rc = lvb.lib().louvain_create_csr(len(rowptr) - 1, len(col), rowptr.ctypes.data,
                                      col.ctypes.data if len(col) else None, wp, flags, None, ctypes.byref(h))
    if rc == 0:
        lvb.lib().louvain_destroy(h)
    return rc


@pytest.mark.parametrize("case,rowptr,col,w,code", [
    ("rowptr0", [1, 2], [0], None, lvb.E_INVALID_GRAPH),
    ("rowptr_end", [0, 1, 3], [1, 0], None, lvb.E_INVALID_GRAPH),
    ("non_monotone", [0, 2, 1, 2], [1, 2], None, lvb.E_INVALID_GRAPH),
    ("col_range", [0, 1, 2], [5, 0], None, lvb.E_INVALID_GRAPH),
    ("zero_weight", [0, 1, 2], [1, 0], [0, 0], lvb.E_INVALID_GRAPH),
    ("asymmetric", [0, 1, 1], [1], None, lvb.E_INVALID_GRAPH),
    ("asym_weight", [0, 1, 2], [1, 0], [2, 3], lvb.E_INVALID_GRAPH),
    ("overflow", [0, 1, 2], [1, 0], [1_600_000_000, 1_600_000_000], lvb.E_OVERFLOW),
])
def test_validation_error_codes(case, rowptr, col, w, code):
    assert _create(rowptr, col, w) == code, lvb.lib().louvain_last_error()


def test_null_arguments():
    h = ctypes.c_void_p()
    assert lvb.lib().louvain_create_csr(-1, 0, None, None, None, 0, None, ctypes.byref(h)) == lvb.E_INVALID_ARG
    assert lvb.lib().louvain_create_csr(1, 0, None, None, None, 0, None, ctypes.byref(h)) == lvb.E_INVALID_ARG
    assert lvb.lib().louvain_get_info(None, None, None, None) == lvb.E_INVALID_ARG
    assert lvb.lib().louvain_sweep(None, None, None, None) == lvb.E_INVALID_ARG
    assert lvb.lib().louvain_run(None, None, None, None, None) == lvb.E_INVALID_ARG
    assert lvb.lib().louvain_destroy(None) == 0
    assert lvb.lib().louvain_last_error() is not None


def test_product_package_does_not_import_oracle():
    # the product path never imports, links or includes anything under oracle/
    pkg = os.path.join(ROOT, "paper_conf_ipps_naimmht17_b200")
    bad = re.compile(r"^\s*(import\s+oracle|from\s+oracle|#\s*include\s*[<\"].*oracle)|louvain_oracle|liblouvain_oracle",
                     re.M)
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".h", ".cpp")):
                text = open(os.path.join(dirpath, f)).read()
                text = re.sub(r"//.*", "", text)
                assert not bad.search(text), f
    out = __import__("subprocess").run(["nm", "-D", lvb.LIB_PATH], capture_output=True, text=True).stdout
    assert "orc_" not in out
