"""CPU checks of the boundary: the C-ABI library loads and exports every function that
include/warpdrive.h declares (no compute calls), and the Python binding carries the same
names.  Also: the oracle and generator libraries build and load."""
import ctypes
import os
import re

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _build_mod():
    """build.py loaded by path: the package itself refuses to import before the
    library exists, which is exactly the fresh-checkout state build() must handle."""
    import importlib.util
    spec = importlib.util.spec_from_file_location(
        "_wd_build", os.path.join(ROOT, "paper_conf_ipps_junger0s18_b200", "build.py"))
    m = importlib.util.module_from_spec(spec)
    spec.loader.exec_module(m)
    return m


def _declared():
    src = open(os.path.join(ROOT, "include", "warpdrive.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(wd_[a-z_]+)\s*\(", src)) - {"wd_allreduce_fn"})


@pytest.fixture(scope="module")
def lib():
    build = _build_mod()
    build.build()
    return ctypes.CDLL(build.LIB)


def test_header_declares_the_north_star_calls():
    names = _declared()
    for n in ["wd_create", "wd_insert", "wd_retrieve", "wd_size", "wd_destroy"]:
        assert n in names


def test_library_exports_every_declared_symbol(lib):
    missing = [n for n in _declared() if not hasattr(lib, n)]
    assert not missing, missing


def test_binding_names_match_header(lib):
    import paper_conf_ipps_junger0s18_b200 as wd
    assert sorted(wd.EXPORTS) == _declared()
    for n in wd.EXPORTS:
        assert callable(getattr(wd, n))


def test_error_strings_without_gpu(lib):
    import paper_conf_ipps_junger0s18_b200 as wd
    assert wd.wd_error_string(wd.WD_ERR_TABLE_FULL) == b"WD_ERR_TABLE_FULL"
    assert wd.wd_error_string(0) == b"WD_OK"


def test_sm100a_only_and_no_cpu_fallback(lib):
    # the product library contains sm_100a SASS only
    import subprocess
    build = _build_mod()
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", build.LIB],
                         capture_output=True, text=True).stdout
    assert "sm_100a" in out
    assert all("sm_100a" in line for line in out.splitlines() if ".cubin" in line)


def test_oracle_and_generator_libraries_load():
    import oracle
    assert os.path.exists(oracle.build())
    build = _build_mod()
    build.build()
    g = ctypes.CDLL(build.GENLIB)
    assert hasattr(g, "wdgen_unique_keys")


def test_binding_checks_dtypes_and_lengths(lib):
    # the binding must refuse buffers the C-ABI would misread (int64 / 1-2-byte
    # keys, float values, short outputs) instead of passing their bytes through
    import numpy as np
    import torch
    import paper_conf_ipps_junger0s18_b200 as wd
    a = wd._addr
    assert a(np.zeros(8, np.uint32), 4, "keys")[1] == 8
    assert a(torch.zeros(8, dtype=torch.int32), 4, "keys")[1] == 8
    assert a(torch.zeros(8, dtype=torch.uint8), 1, "found_out", 8)[1] == 8
    for bad in (np.zeros(8, np.int64), np.zeros(8, np.uint16), np.zeros(8, np.float32),
                torch.arange(8), torch.zeros(8, dtype=torch.float32)):
        with pytest.raises(TypeError):
            a(bad, 4, "keys")
    with pytest.raises(TypeError):
        a(torch.zeros(8, dtype=torch.bool), 1, "found_out")
    with pytest.raises(ValueError):
        a(np.zeros(7, np.uint32), 4, "vals_out", 8)
    with pytest.raises(ValueError):
        a(np.zeros((4, 4), np.uint32)[:, 0], 4, "keys")
