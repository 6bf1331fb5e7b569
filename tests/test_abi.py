"""CPU checks of the C-ABI boundary: libbk.so loads, exports every symbol include/bk.h declares,
its struct sizes match the binding, and it fails loudly (no fallback) without a GPU."""
import ctypes as C
import os
import re
import subprocess

import pytest

from paper_conf_ipps_mokhtaris14_b200 import bk

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def header_functions():
    src = open(os.path.join(ROOT, "include", "bk.h")).read()
    return sorted(set(re.findall(r"BK_API\s+[\w\s\*]+?\b(bk_\w+)\s*\(", src)))


def test_header_declares_the_north_star_entry_points():
    fns = header_functions()
    for f in ("bk_create", "bk_register_segments", "bk_run", "bk_destroy"):
        assert f in fns
    assert sorted(bk.EXPORTS) == fns


def test_library_exports_every_declared_symbol():
    out = subprocess.run(["nm", "-D", "--defined-only", bk.LIB_PATH], capture_output=True, text=True, check=True).stdout
    exported = sorted(set(re.findall(r" T (bk_\w+)", out)))
    assert exported == header_functions()  # and nothing else leaks (visibility=hidden)
    lib = bk.lib()
    for f in header_functions():
        assert getattr(lib, f) is not None


def test_abi_struct_sizes_match_binding():
    assert bk.abi_sizes() == [C.sizeof(s) for s in bk.ABI_STRUCTS]


def test_library_is_built_for_sm100a_only():
    out = subprocess.run(["cuobjdump", "--list-elf", bk.LIB_PATH], capture_output=True, text=True).stdout
    arches = set(re.findall(r"sm_(\d+a?)", out))
    assert arches == {"100a"}, out


def test_no_gpu_fails_loudly_and_null_safety():
    import torch
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    with pytest.raises(bk.BkError) as e:
        bk.bk_create(device=0)
    assert e.value.status == bk.BK_E_CUDA
    assert bk.lib().bk_destroy(None) == bk.BK_OK
    assert bk.lib().bk_strerror(bk.BK_E_RANGE) == b"record exceeds chunk budget"


def test_product_package_never_imports_the_oracle():
    pkg = os.path.join(ROOT, "paper_conf_ipps_mokhtaris14_b200")
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".cpp", ".h")):
                txt = open(os.path.join(dirpath, f)).read()
                assert "oracle" not in txt.replace("never imports the oracle", "").replace("never the oracle", ""), f


def test_header_is_plain_c_and_links(tmp_path):
    """include/bk.h compiles as C99 and C++17, and a plain C program links against libbk.so and calls
    the GPU-free entry points (no torch, no CUDA headers in the signatures)."""
    import shutil
    if not shutil.which("gcc"):
        pytest.skip("no gcc")
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    src = tmp_path / "abi.c"
    src.write_text(
        '#include "bk.h"\n#include <stdio.h>\n'
        "int main(void) { unsigned s[12]; int v = bk_abi_sizes(s, 12);\n"
        '  printf("%d %u %s\\n", v, s[0], bk_strerror(BK_E_RANGE));\n'
        "  return bk_destroy(NULL); }\n")
    exe = tmp_path / "abi"
    libdir = os.path.join(root, "paper_conf_ipps_mokhtaris14_b200")
    subprocess.check_call(["gcc", "-std=c99", "-Wall", "-Werror", "-I", os.path.join(root, "include"), str(src),
                           "-L", libdir, "-l:libbk.so", "-Wl,-rpath," + libdir, "-o", str(exe)])
    subprocess.check_call(["g++", "-std=c++17", "-Wall", "-Werror", "-fsyntax-only", "-x", "c++",
                           os.path.join(root, "include", "bk.h")])
    out = subprocess.run([str(exe)], capture_output=True, text=True, check=True).stdout.split()
    assert int(out[1]) == bk.abi_sizes()[0] and "record" in " ".join(out[2:])
