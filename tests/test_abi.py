"""The C-ABI library builds, loads and exports every symbol include/mst.h declares (CPU)."""
import ctypes
import os
import re

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def header_symbols(name="mst.h"):
    txt = open(os.path.join(ROOT, "include", name)).read()
    txt = re.sub(r"/\*.*?\*/", "", txt, flags=re.S)
    return sorted(set(re.findall(r"\b(mst_[a-z_]+)\s*\(", txt)))


def test_header_symbols_listed_in_binding():
    import paper_conf_ppopp_nasrebp13_b200 as p
    assert header_symbols() == sorted(p.EXPORTS)
    assert header_symbols("mst_debug.h") == sorted(p.mst.DEBUG_EXPORTS)


def test_library_exports_every_declared_symbol():
    import paper_conf_ppopp_nasrebp13_b200 as p
    L = p.load()
    for name in header_symbols() + header_symbols("mst_debug.h"):
        assert hasattr(L, name), name
    assert "sm_100a" in p.mst_version()


def test_library_is_sm100a_only():
    import subprocess
    import paper_conf_ppopp_nasrebp13_b200 as p
    p.load()
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", p.lib_path()],
                         capture_output=True, text=True).stdout
    assert "sm_100a" in out


def test_no_device_fails_loudly():
    torch = pytest.importorskip("torch")
    if torch.cuda.is_available():
        pytest.skip("a GPU is present")
    import numpy as np
    import paper_conf_ppopp_nasrebp13_b200 as p
    with pytest.raises(p.MSTError) as ei:
        p.mst_solve_host(3, np.array([0, 1]), np.array([1, 2]), np.array([1, 1]))
    assert ei.value.status in (3,)  # MST_ECUDA: no CPU fallback


def test_product_path_does_not_import_oracle():
    pkg = os.path.join(ROOT, "paper_conf_ppopp_nasrebp13_b200")
    bad = re.compile(r"import\s+oracle|from\s+oracle|_oracle\.so|oracle_kruskal|kruskal\.cpp")
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".h", ".cpp")):
                txt = open(os.path.join(dirpath, f)).read()
                assert not bad.search(txt), f


def test_stats_struct_and_options_match_the_header(tmp_path):
    """the ctypes mirror of mst_stats and the option numbers agree with include/mst.h (a
    plain C compile of the header measures the struct)"""
    import subprocess
    import ctypes as C
    import paper_conf_ppopp_nasrebp13_b200 as p
    src = tmp_path / "probe.c"
    src.write_text('#include <stdio.h>\n#include <stddef.h>\n#include "mst.h"\n'
                   'int main(void){printf("%zu %zu %zu %d %d %d %d %d\\n", sizeof(mst_stats),'
                   ' offsetof(mst_stats, light_switch_round), offsetof(mst_stats, light_t),'
                   ' MST_OPT_DENSE, MST_OPT_KEEP_EDGES, MST_OPT_DEVICE_TAIL, MST_OPT_COMPACT_TAU,'
                   ' MST_OPT_LIGHT_FIRST); return 0;}\n')
    exe = tmp_path / "probe"
    r = subprocess.run(["gcc", "-I", os.path.join(ROOT, "include"), "-I", "/usr/local/cuda/include",
                        str(src), "-o", str(exe)], capture_output=True, text=True)
    assert r.returncode == 0, r.stderr
    vals = subprocess.run([str(exe)], capture_output=True, text=True).stdout.split()
    size, off_sw, off_t = (int(x) for x in vals[:3])
    S = p.mst.mst_stats
    assert C.sizeof(S) == size
    assert S.light_switch_round.offset == off_sw and S.light_t.offset == off_t
    m = p.mst
    assert [int(x) for x in vals[3:]] == [m.MST_OPT_DENSE, m.MST_OPT_KEEP_EDGES,
                                          m.MST_OPT_DEVICE_TAIL, m.MST_OPT_COMPACT_TAU,
                                          m.MST_OPT_LIGHT_FIRST]


def test_argument_errors_before_any_device_work():
    """include/mst.h error conventions on the host-side checks: MST_EINVAL with a message for
    out-of-range sizes, null pointers and null handles — decided before any CUDA call, so they
    hold on a machine without a GPU too; mst_destroy(NULL) is a no-op"""
    import ctypes as C
    import paper_conf_ppopp_nasrebp13_b200 as p
    L = p.load()
    EINVAL = 1
    g = C.c_void_p()
    buf = (C.c_int32 * 4)(0, 1, 1, 2)
    wb = (C.c_uint32 * 2)(1, 1)
    cases = [
        (1 << 31, 2, buf, buf, wb, "n ="),            # n > 2^31 - 1
        (-1, 2, buf, buf, wb, "n ="),
        (4, 1 << 31, buf, buf, wb, "m ="),            # m > 2^31 - 1
        (4, -5, buf, buf, wb, "m ="),
        (4, 2, None, buf, wb, "null input pointer"),
        (4, 2, buf, buf, None, "null input pointer"),
        (0, 2, buf, buf, wb, "n = 0"),                # edges on no vertices
    ]
    for create in (L.mst_create, L.mst_create_host):
        for n, m, s, d, w, msg in cases:
            st = create(n, m, s, d, w, C.byref(g))
            assert st == EINVAL, (create, n, m, st)
            assert msg in L.mst_last_error().decode(), L.mst_last_error()
            assert not g.value  # *out is NULL after a failed create
        assert create(4, 2, buf, buf, wb, None) == EINVAL  # out == NULL
    ne, tw = C.c_int64(), C.c_uint64()
    assert L.mst_run(None, None, buf, C.byref(ne), C.byref(tw)) == EINVAL
    assert L.mst_run_host(None, None, buf, C.byref(ne), C.byref(tw)) == EINVAL
    assert L.mst_set_option(None, p.mst.MST_OPT_DENSE, 1) == EINVAL
    assert L.mst_set_profiling(None, 1) == EINVAL
    assert L.mst_get_stats(None, C.byref(p.mst.mst_stats())) == EINVAL
    L.mst_destroy(None)
    out_ids = (C.c_int32 * 4)()
    assert L.mst_solve_host(-1, 0, None, None, None, out_ids, C.byref(ne), C.byref(tw)) == EINVAL
    assert L.mst_create_sim(4, 2, buf, buf, wb, 0, C.byref(g)) == EINVAL  # nshards < 1
    assert L.mst_create_sim(4, 2, buf, buf, wb, 65, C.byref(g)) == EINVAL  # nshards > 64
