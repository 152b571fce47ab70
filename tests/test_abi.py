"""The C-ABI library builds, loads and exports every symbol include/*.h declares.

CPU-only (no compute calls): the CUDA path is exercised by the -m gpu tests.
"""
from __future__ import annotations

import ctypes
import glob
import os
import re
import subprocess

import pytest

from conftest import ROOT, cuda_available
from paper_conf_cluster_ajipbf15_b200 import build as mbuild
from paper_conf_cluster_ajipbf15_b200 import mcl

HEADERS = sorted(glob.glob(os.path.join(ROOT, "include", "*.h")))


def declared_functions() -> list[str]:
    names = []
    for h in HEADERS:
        text = open(h).read()
        text = re.sub(r"/\*.*?\*/", "", text, flags=re.S)
        names += re.findall(r"^\s*(?:const\s+)?[a-z_0-9]+\s*\*?\s*(mcl_[a-z_0-9]+)\s*\(", text, flags=re.M)
    return sorted(set(names))


@pytest.fixture(scope="module")
def lib():
    mbuild.build()
    return mcl.load_library()


def test_headers_present():
    assert [os.path.basename(h) for h in HEADERS] == ["mcl.h", "mcl_ext.h"]


def test_every_declared_symbol_is_exported(lib):
    names = declared_functions()
    assert {"mcl_mapper_create", "mcl_map_queues", "mcl_mapper_destroy"} <= set(names)
    out = subprocess.run(["nm", "-D", "--defined-only", mcl.LIB_PATH], capture_output=True, text=True).stdout
    exported = set(re.findall(r"\b(mcl_[a-z_0-9]+)\b", out))
    missing = [n for n in names if n not in exported]
    assert not missing, missing
    assert sorted(mcl.EXPORTED) == names  # the binding covers the whole ABI
    for n in names:
        getattr(lib, n)


def test_library_is_sm100a_and_has_no_torch_dependency(lib):
    ldd = subprocess.run(["ldd", mcl.LIB_PATH], capture_output=True, text=True).stdout
    assert "libtorch" not in ldd and "libnccl" not in ldd  # NCCL is dlopen'ed at run time
    sass = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "-lelf", mcl.LIB_PATH], capture_output=True,
                          text=True).stdout
    assert "sm_100a" in sass


def test_status_strings(lib):
    for code in (0, -1, -2, -3, -4, -5):
        s = mcl.mcl_status_string(code)
        assert s.startswith("MCL_")
    assert "sm_100a" in mcl.mcl_version()


def test_null_and_argument_errors_without_gpu(lib):
    # NULL config / out pointer
    assert lib.mcl_mapper_create(None, None) == mcl.MCL_E_INVAL
    # destroy(NULL) is a no-op
    lib.mcl_mapper_destroy(None)
    # NULL handle
    assert lib.mcl_map_queues(None, 2, 2, 1, None, None, None, None, None) == mcl.MCL_E_INVAL
    assert lib.mcl_force_path(None, 1) == mcl.MCL_E_INVAL


@pytest.mark.skipif(cuda_available(), reason="checks the no-GPU failure mode")
def test_create_fails_loudly_without_gpu(lib):
    cfg = mcl.mcl_config_t(0, None, None, 0, 1)
    h = ctypes.c_void_p()
    st = lib.mcl_mapper_create(ctypes.byref(cfg), ctypes.byref(h))
    assert st in (mcl.MCL_E_CUDA, mcl.MCL_E_INVAL)
    assert h.value is None
    with pytest.raises(mcl.MclError):
        mcl.Mapper(0)


def test_product_never_imports_oracle():
    """The product package and the library sources hold no reference to oracle/."""
    pkg = os.path.join(ROOT, "paper_conf_cluster_ajipbf15_b200")
    for path in glob.glob(os.path.join(pkg, "**", "*"), recursive=True):
        if path.endswith((".py", ".cu", ".cuh", ".h", ".cpp")):
            text = open(path).read()
            assert "import oracle" not in text and "from oracle" not in text, path
            assert "oracle.c" not in text and "liboracle" not in text, path
    for path in glob.glob(os.path.join(ROOT, "oracle", "*")):
        if path.endswith((".py", ".c")):
            text = open(path).read()
            assert not re.search(r"^\s*(from|import)\s+paper_conf", text, flags=re.M), path
            assert "#include" not in text or "mcl" not in "".join(re.findall(r"#include.*", text)), path


def test_binding_rejects_mismatched_shapes_before_the_library():
    """Mapper methods check every array against (E, Q, D) (and M for the cost model) and
    raise ValueError before any pointer reaches libmcl.so (a mismatch would read
    or write out of bounds). A handle-less Mapper shows no library call is made."""
    import numpy as np

    m = object.__new__(mcl.Mapper)
    m.handle = None
    m.device = 0
    K = np.zeros((3, 5, 4), np.uint64)
    ok_i, ok_ms, ok_mp = np.zeros(3, np.uint64), np.zeros(3, np.uint64), np.zeros((3, 5), np.uint8)
    bad = [
        (np.zeros((3, 5, 3), np.uint64), ok_i, ok_mp, ok_ms),  # X
        (K, np.zeros(2, np.uint64), ok_mp, ok_ms),            # index
        (K, ok_i, np.zeros((3, 4), np.uint8), ok_ms),         # mapping
        (K, ok_i, ok_mp, np.zeros(4, np.uint64)),             # makespan
    ]
    for X, i, mp, ms in bad:
        with pytest.raises(ValueError):
            m.map_queues_into(K, X, i, mp, ms)
    with pytest.raises(ValueError):
        m.map_queues_into(K[0], K[0], ok_i, ok_mp, ok_ms)  # not [E, Q, D]
    with pytest.raises(ValueError):
        m.map_queues_constrained(K, K, base=np.zeros((3, 5), np.uint64))
    with pytest.raises(ValueError):
        m.map_queues_constrained(K, K, eligible=np.zeros((3, 4), np.uint16))
    with pytest.raises(ValueError):
        m.score_mappings(K, K, np.zeros((3, 4), np.uint8))
    from paper_conf_cluster_ajipbf15_b200 import workloads

    model = workloads.cost_model(1, 3, 5, 4)
    for key, val in (("offsets", model["offsets"][:-1]), ("source", model["source"][:, :4]),
                     ("h2d_bw", model["h2d_bw"][:, :-1]), ("profile", model["profile"][:, :3])):
        with pytest.raises(ValueError):
            m._cost_model(dict(model, **{key: val}), 4)
