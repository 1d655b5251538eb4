"""CPU checks of the C-ABI library: it builds, loads, exports every symbol
include/dsp.h declares, and fails loudly (no CPU fallback) without a GPU."""
import os
import re
import subprocess

import pytest

import paper_conf_ppopp_caiz0zszck23_b200 as pkg
from paper_conf_ppopp_caiz0zszck23_b200 import _build

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def libpath():
    return _build.build()


def header_functions():
    src = open(os.path.join(ROOT, "include", "dsp.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(dsp_[a-z_]+)\s*\(", src)))


def test_header_declares_the_binding_names():
    assert header_functions() == sorted(pkg.ABI_SYMBOLS)


def test_library_exports_every_symbol(libpath):
    out = subprocess.check_output(["nm", "-D", "--defined-only", libpath], text=True)
    exported = {line.split()[-1] for line in out.splitlines() if line.strip()}
    for name in header_functions():
        assert name in exported, name
    lib = pkg.lib(libpath)
    for name in header_functions():
        assert hasattr(lib, name)


def test_sm100a_only(libpath):
    out = subprocess.check_output(["/usr/local/cuda/bin/cuobjdump", "--list-elf", libpath], text=True)
    assert "sm_100a" in out
    assert not re.search(r"sm_(?!100a)\d+", out)


def test_static_entry_points(libpath):
    assert pkg.dsp_abi_version() == 1
    assert pkg.dsp_status_str(-3) == "DSP_ERR_DUPLICATE_SEED"
    assert pkg.dsp_status_str(0) == "DSP_OK"


def test_no_cpu_fallback_without_gpu(libpath):
    import torch
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    with pytest.raises(pkg.DSPError) as e:
        pkg.dsp_create(0, 1, 0)
    assert e.value.status == pkg.dsp.DSP_ERR_CUDA


def test_invalid_world_rejected(libpath):
    with pytest.raises(pkg.DSPError) as e:
        pkg.dsp_create(0, 9, 0)
    assert e.value.status == pkg.dsp.DSP_ERR_INVALID_ARG
    with pytest.raises(pkg.DSPError):
        pkg.dsp_create(2, 2, 0)


def test_product_never_imports_oracle():
    pkgdir = os.path.join(ROOT, "paper_conf_ppopp_caiz0zszck23_b200")
    for dirpath, _, files in os.walk(pkgdir):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".h")):
                txt = open(os.path.join(dirpath, f)).read()
                assert not re.search(r"^\s*(import|from)\s+oracle", txt, re.M), f
                assert "oracle.c" not in txt and "liboracle" not in txt, f


def test_no_environment_switches_in_the_library():
    """Every behaviour switch of libdsp.so is an ABI argument or a documented
    dsp_set_option (include/dsp.h); the library reads no environment."""
    csrc = os.path.join(ROOT, "paper_conf_ppopp_caiz0zszck23_b200", "csrc")
    for f in os.listdir(csrc):
        txt = open(os.path.join(csrc, f)).read()
        assert "getenv" not in txt and "environ" not in txt, f
