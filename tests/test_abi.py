"""CPU-side checks of the boundary: the C-ABI library loads and exports every symbol include/sfs.h
declares; host-only entry points behave; the oracle and the CUDA path share no code."""
import os
import re
import subprocess

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
PKG = os.path.join(ROOT, "paper_conf_icppw_dhandhaniadpbl21_b200")


@pytest.fixture(scope="module")
def sfs():
    import build_native
    build_native.build_sfs()
    import paper_conf_icppw_dhandhaniadpbl21_b200 as m
    return m


def declared_functions():
    src = open(os.path.join(ROOT, "include", "sfs.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(sfs_[a-z_]+)\s*\(", src)))


def test_header_declares_the_boundary():
    names = declared_functions()
    for n in ["sfs_features", "sfs_convert", "sfs_spmv", "sfs_label_corpus"]:
        assert n in names


def test_library_exports_every_declared_symbol(sfs):
    out = subprocess.check_output(["nm", "-D", "--defined-only", sfs.LIB_PATH], text=True)
    exported = set(l.split()[-1] for l in out.splitlines() if " T " in l)
    missing = [n for n in declared_functions() if n not in exported]
    assert not missing, missing
    L = sfs.lib()
    for n in declared_functions():
        assert hasattr(L, n)


def test_library_is_sm100a(sfs):
    out = subprocess.check_output(["/usr/local/cuda/bin/cuobjdump", "--list-elf", sfs.LIB_PATH], text=True)
    assert "sm_100a" in out


def test_host_only_calls(sfs):
    o = sfs.default_opts()
    assert (o.reps, o.warmup, o.formats_mask, o.max_fill, o.fill_slack, o.hyb_breakeven) == (100, 5, 31, 3.0,
                                                                                           1 << 20, 4096)
    assert sfs.lib().sfs_status_string(sfs.ERR_INADMISSIBLE) == b"SFS_ERR_INADMISSIBLE"
    f = {k: 0 for k in sfs.FEATURE_INT_FIELDS}
    f.update({k: 0.0 for k in sfs.FEATURE_FLOAT_FIELDS})
    f.update(nrows=4, ncols=4, nnz=7, ell_size=16, hyb_ell_size=4, hyb_coo=4, dia_size=20, diagonals=5,
             admissible_mask=31)
    # a9-a13 byte models for the 4x4 example, fp64
    assert sfs.spmv_bytes(f, sfs.CSR, sfs.F64) == 4 * 5 + 12 * 7 + 8 * 8
    assert sfs.spmv_bytes(f, sfs.COO, sfs.F64) == 16 * 7 + 64
    assert sfs.spmv_bytes(f, sfs.ELL, sfs.F64) == 12 * 16 + 64
    assert sfs.spmv_bytes(f, sfs.HYB, sfs.F64) == 12 * 4 + 16 * 4 + 64
    assert sfs.spmv_bytes(f, sfs.DIA, sfs.F64) == 8 * 20 + 4 * 5 + 64


def test_no_shared_code_between_oracle_and_product():
    csrc = os.path.join(PKG, "csrc")
    for fn in os.listdir(os.path.join(ROOT, "oracle")):
        if fn.endswith((".c", ".h", ".py")):
            s = open(os.path.join(ROOT, "oracle", fn)).read()
            assert not re.search(r'#include\s+[<"][^>"]*(sfs\.h|csrc|common\.cuh|internal\.h)', s), fn
            assert not re.search(r"^\s*(import|from)\s+paper_conf", s, re.M), fn
    for dirpath, _, files in os.walk(PKG):
        for fn in files:
            if fn.endswith((".cu", ".cuh", ".cpp", ".h", ".py")):
                s = open(os.path.join(dirpath, fn)).read()
                assert not re.search(r"^\s*(import|from)\s+oracle", s, re.M), fn
                assert '#include "oracle' not in s, fn


def test_product_fails_loudly_without_gpu(sfs):
    """No CPU fallback: a compute call without a CUDA device raises (CPU box) rather than computing."""
    import numpy as np
    import torch
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    A = sfs.Csr(2, 2, torch.tensor([0, 1, 2], dtype=torch.int32), torch.tensor([0, 1], dtype=torch.int32),
                torch.tensor([1.0, 2.0], dtype=torch.float64))
    with pytest.raises(Exception):
        sfs.features(A)
