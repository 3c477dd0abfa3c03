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
