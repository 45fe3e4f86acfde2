"""The C-ABI boundary without a GPU: libmf.so loads, exports every symbol include/mf.h declares,
the Python struct mirrors match the header, and compute calls fail loudly (no CPU fallback)."""
import ctypes as C
import os
import re

import numpy as np
import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def header_functions():
    src = open(os.path.join(ROOT, "include", "mf.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"^\s*(?:mf_status|void|const char\s*\*|int32_t)\s+(mf_\w+)\s*\(", src, flags=re.M)))


@pytest.fixture(scope="module")
def mf():
    import paper_conf_sc_yangznjs0t024_b200 as m
    m.build()
    return m


def test_header_declares_the_paper_calls():
    fns = header_functions()
    for name in ("mf_tile_matrix_from_csr", "mf_cg_solve", "mf_bicgstab_solve", "mf_precond_create",
                 "mf_spmv", "mf_levels", "mf_dot", "mf_cg_update_xr", "mf_cg_update_p"):
        assert name in fns


def test_every_declared_symbol_is_exported(mf):
    L = C.CDLL(mf.LIB_PATH)
    missing = [f for f in header_functions() if not hasattr(L, f)]
    assert not missing
    assert sorted(mf.SYMBOLS) == header_functions()


def test_library_is_sm100a_only(mf):
    out = os.popen(f"cuobjdump --list-elf {mf.LIB_PATH} 2>&1").read()
    assert "sm_100a" in out
    assert "sm_90" not in out and "sm_80" not in out


def test_status_strings_and_defaults(mf):
    L = mf.lib()
    for code, name in mf.STATUS.items():
        assert L.mf_status_string(code).decode() == name
    o = mf.SolveOpts()
    L.mf_default_solve_opts(C.byref(o))
    assert (o.tol, o.max_iter, o.mode, o.switch_eps, o.range_guard, o.sticky) == (1e-10, 1000, 2, -1.0, 1, 0)
    c = mf.ConvertOpts()
    L.mf_default_convert_opts(C.byref(c))
    assert (c.classify, c.loss_tol, c.grid_ctas, c.block_threads, c.layout) == (1, 1e-15, 0, 0, 0)
    assert L.mf_abi_version() == 2


def test_struct_sizes_match_header(mf, tmp_path):
    """Compile a tiny C program against include/mf.h and compare sizeof/offsetof with ctypes."""
    prog = tmp_path / "sz.c"
    prog.write_text('#include <stdio.h>\n#include <stddef.h>\n#include "mf.h"\nint main(){'
                    'printf("%zu %zu %zu %zu %zu\\n", sizeof(mf_convert_opts), sizeof(mf_tile_info),'
                    'sizeof(mf_tile_export), sizeof(mf_solve_opts), sizeof(mf_solve_info));'
                    'printf("%zu %zu\\n", offsetof(mf_solve_opts, collect_stats), offsetof(mf_tile_info, layout));'
                    'return 0;}')
    exe = tmp_path / "sz"
    assert os.system(f"gcc -I{ROOT}/include -o {exe} {prog}") == 0
    sizes = os.popen(str(exe)).read().split()
    assert [int(s) for s in sizes[:5]] == [C.sizeof(mf.ConvertOpts), C.sizeof(mf.TileInfo), C.sizeof(mf.TileExport),
                                          C.sizeof(mf.SolveOpts), C.sizeof(mf.SolveInfo)]
    assert int(sizes[5]) == mf.SolveOpts.collect_stats.offset
    assert int(sizes[6]) == mf.TileInfo.layout.offset


def test_compute_calls_fail_loudly_without_gpu(mf):
    torch = pytest.importorskip("torch")
    if torch.cuda.is_available():
        pytest.skip("a GPU is present")
    L = mf.lib()
    h = C.c_void_p()
    st = L.mf_tile_matrix_from_csr(4, 4, 0, C.c_void_p(16), None, None, None, None, C.byref(h))
    assert st in (5, 10)            # MF_ERR_CUDA / MF_ERR_UNSUPPORTED_DEVICE, never a silent success
    assert not h.value
    th = np.zeros(4)
    st = L.mf_levels(C.c_void_p(16), 4, C.c_void_p(th.ctypes.data), C.c_void_p(16), None)
    assert st in (5, 10)
