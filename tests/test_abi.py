"""CPU-side checks of the C-ABI library: it loads, exports every declared symbol,
and rejects bad calls without touching the GPU."""
import ctypes
import os
import re

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "cuts.h")
LIB = os.path.join(ROOT, "paper_conf_sc_xiangkshs21_b200", "libcuts.so")


def _declared():
    text = open(HEADER).read()
    text = re.sub(r"/\*.*?\*/", "", text, flags=re.S)
    return sorted(set(re.findall(r"\b(cuts_[a-z0-9_]+)\s*\(", text)))


@pytest.fixture(scope="module")
def lib():
    import importlib.util
    spec = importlib.util.spec_from_file_location("_b", os.path.join(ROOT, "paper_conf_sc_xiangkshs21_b200", "build.py"))
    b = importlib.util.module_from_spec(spec)
    spec.loader.exec_module(b)
    b.build()
    return ctypes.CDLL(LIB)


def test_header_declares_the_boundary():
    names = _declared()
    for must in ["cuts_create", "cuts_destroy", "cuts_last_error", "cuts_load_graph", "cuts_set_query",
                 "cuts_count", "cuts_enumerate", "cuts_set_root_range", "cuts_set_dist", "cuts_get_stats"]:
        assert must in names


def test_library_exports_every_declared_symbol(lib):
    for name in _declared():
        assert hasattr(lib, name), name
    from paper_conf_sc_xiangkshs21_b200 import _lib as L
    assert sorted(L.EXPORTED) == _declared()


def test_version_and_null_args(lib):
    lib.cuts_version.restype = ctypes.c_int
    assert lib.cuts_version() == 3
    lib.cuts_create.restype = ctypes.c_int
    lib.cuts_create.argtypes = [ctypes.c_void_p, ctypes.c_void_p]
    assert lib.cuts_create(None, None) == -1                  # CUTS_EINVAL, no CUDA call
    lib.cuts_count.restype = ctypes.c_int
    lib.cuts_count.argtypes = [ctypes.c_void_p, ctypes.c_int, ctypes.c_void_p]
    assert lib.cuts_count(None, 0, None) == -1
    lib.cuts_last_error.restype = ctypes.c_char_p
    lib.cuts_last_error.argtypes = [ctypes.c_void_p]
    assert lib.cuts_last_error(None) == b"null context"
    lib.cuts_destroy.argtypes = [ctypes.c_void_p]
    lib.cuts_destroy(None)                                     # NULL-safe


def test_stats_struct_layout():
    from paper_conf_sc_xiangkshs21_b200 import _lib as L
    # u32 k + u32[8] -> 36 B, padded to 40 before the u64 level sizes
    assert L.cuts_stats.level_size.offset == 40
    assert ctypes.sizeof(L.cuts_opts) == 40


def test_sass_is_sm100a(lib):
    """The shipped cubin targets sm_100a (checked with cuobjdump, no GPU needed)."""
    import shutil
    import subprocess
    exe = shutil.which("cuobjdump") or "/usr/local/cuda/bin/cuobjdump"
    if not os.path.exists(exe):
        pytest.skip("cuobjdump not available")
    out = subprocess.run([exe, "--list-elf", LIB], capture_output=True, text=True).stdout
    assert "sm_100a" in out


def test_product_does_not_import_oracle():
    """The product path never imports, links or loads the oracle (rule 3)."""
    pkg = os.path.join(ROOT, "paper_conf_sc_xiangkshs21_b200")
    pat = re.compile(r"import\s+oracle|from\s+oracle|liboracle|cuts_oracle")
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".h", ".cpp")):
                assert not pat.search(open(os.path.join(dirpath, f)).read()), f
