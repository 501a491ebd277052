"""CPU-side checks of the boundary: libamgt.so loads and exports every entry point that
include/amgt.h declares (no compute calls — there is no GPU here)."""
import ctypes
import os
import re

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _header_functions():
    src = open(os.path.join(ROOT, "include", "amgt.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(amgt_[a-z0-9_]+)\s*\(", src)))


def test_library_exports_every_header_symbol():
    import paper_conf_sc_luzwflcy0c024_b200 as amgt
    lib = ctypes.CDLL(amgt.LIB_PATH)
    names = _header_functions()
    assert len(names) >= 20
    missing = [n for n in names if not hasattr(lib, n)]
    assert not missing, missing
    # and the binding declares a signature for each
    assert set(names) <= set(amgt.EXPORTED) | {"amgt_hierarchy_nlev"}, set(names) - set(amgt.EXPORTED)


def test_version_and_no_cpu_fallback():
    import paper_conf_sc_luzwflcy0c024_b200 as amgt
    assert "sm_100a" in amgt.version()
    # the product package must not reference the oracle
    pkg = os.path.join(ROOT, "paper_conf_sc_luzwflcy0c024_b200")
    for dp, _, fs in os.walk(pkg):
        for f in fs:
            if f.endswith((".py", ".cu", ".cuh", ".h")):
                txt = open(os.path.join(dp, f)).read()
                assert "import oracle" not in txt and "from oracle" not in txt and "oracle_" not in txt, f


def test_sm100a_code_in_library():
    import shutil
    import subprocess
    import paper_conf_sc_luzwflcy0c024_b200 as amgt
    if not shutil.which("cuobjdump"):
        pytest.skip("cuobjdump not available")
    out = subprocess.run(["cuobjdump", "-lelf", amgt.LIB_PATH], capture_output=True, text=True).stdout
    assert "sm_100a" in out
