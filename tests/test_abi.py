"""The C-ABI library loads and exports every symbol include/gfsl.h declares (CPU only:
no compute call is made without a GPU)."""
import ctypes
import os
import re

from paper_conf_ppopp_moscovicicp17_b200 import build as gbuild
from paper_conf_ppopp_moscovicicp17_b200 import gfsl as G

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def declared_functions():
    src = open(os.path.join(ROOT, "include", "gfsl.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(gfsl_[a-z_]+)\s*\(", src)))


def test_header_declares_the_north_star_calls():
    names = declared_functions()
    for f in ["gfsl_create", "gfsl_batch", "gfsl_validate", "gfsl_destroy"]:
        assert f in names
    assert sorted(G.EXPORTS) == names


def test_library_exports_every_declared_symbol():
    gbuild.build()
    lib = ctypes.CDLL(gbuild.LIB)
    for name in declared_functions():
        assert hasattr(lib, name), name
    # the binding's loader declares the same set
    lib2 = G.load_library()
    assert lib2.gfsl_last_error() is not None


def test_sm100a_code_in_library():
    import subprocess
    gbuild.build()
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", gbuild.LIB],
                         capture_output=True, text=True).stdout
    assert "sm_100a" in out
