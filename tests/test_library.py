"""CPU-only checks of the boundary: the C-ABI library builds for sm_100a,
loads, and exports every function include/mce.h declares; the binding's
option struct matches the header; the product path has no CPU fallback."""

import ctypes
import os
import re
import subprocess

import pytest

from paper_conf_ipps_geilpo23_b200 import _lib

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def header_functions():
    src = open(_lib.HEADER).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    names = re.findall(r"^\s*(?:const\s+)?[\w]+\s*\*?\s*(mce_\w+)\s*\(", src, flags=re.M)
    return sorted(set(names))


@pytest.fixture(scope="module")
def built():
    if not os.path.exists(_lib.LIB_PATH):
        _lib.build()
    return _lib.LIB_PATH


def test_header_declares_the_north_star_calls():
    names = header_functions()
    for need in ("mce_load_csr", "mce_enumerate", "mce_find_one"):
        assert need in names
    assert set(names) == set(_lib.EXPORTS)


def test_library_exports_every_symbol(built):
    out = subprocess.check_output(["nm", "-D", "--defined-only", built]).decode()
    exported = set(re.findall(r" T (mce_\w+)", out))
    missing = set(header_functions()) - exported
    assert not missing, missing


def test_library_loads_and_reports_version(built):
    L = _lib.lib()
    assert b"sm_100a" in L.mce_version()
    o = _lib.Options()
    L.mce_default_options(ctypes.byref(o))
    assert o.bound == 1 and o.heuristic == 3 and o.shard_count == 1 and o.orientation == 0


def test_sm100a_code_only(built):
    out = subprocess.check_output(["/usr/local/cuda/bin/cuobjdump", "--list-elf", built]).decode()
    assert "sm_100a" in out
    assert not re.search(r"sm_(?!100a)\d+", out)


def test_options_struct_layout(tmp_path):
    """ctypes mirror of mce_options == the C compiler's layout of include/mce.h."""
    fields = [f for f, _ in _lib.Options._fields_]
    prog = "#include <stdio.h>\n#include <stddef.h>\n#include \"mce.h\"\nint main(void){\n"
    prog += 'printf("%zu\\n", sizeof(mce_options));\n'
    for f in fields:
        prog += f'printf("%zu\\n", offsetof(mce_options, {f}));\n'
    prog += "return 0;}\n"
    c = tmp_path / "layout.c"
    c.write_text(prog)
    exe = tmp_path / "layout"
    subprocess.check_call(["gcc", "-I", os.path.dirname(_lib.HEADER), str(c), "-o", str(exe)])
    vals = [int(x) for x in subprocess.check_output([str(exe)]).split()]
    assert vals[0] == ctypes.sizeof(_lib.Options)
    assert vals[1:] == [getattr(_lib.Options, f).offset for f in fields]


def test_no_gpu_means_loud_failure(built):
    import torch

    if torch.cuda.is_available():
        pytest.skip("a GPU is present")
    import numpy as np

    from paper_conf_ipps_geilpo23_b200 import Graph, MCEError

    with pytest.raises(MCEError):
        Graph(np.array([0, 1, 2], np.int64), np.array([1, 0], np.int32))


def test_product_never_imports_oracle():
    pkg = os.path.join(ROOT, "paper_conf_ipps_geilpo23_b200")
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".h", ".cpp")):
                txt = open(os.path.join(dirpath, f)).read()
                assert "import oracle" not in txt and "from oracle" not in txt and "mce_oracle" not in txt, f
