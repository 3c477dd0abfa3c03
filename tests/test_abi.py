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
