"""GPU parity of the TMA ELL kernel (k_spmv_ell_tma: slot slabs streamed by cp.async.bulk through an
mbarrier ring) at every size.

The library uses it for banded (DIA-admissible) ELL matrices, and HYB matrices without a COO part, of
slabs of >= SFS_ELL_TMA_MB megabytes (the full-size stencil and band cases of test_gpu_configs.py run it
at the default threshold).  Here a child process sets SFS_ELL_TMA_MB=0 and SFS_ELL_TMA_K=0 (read once per process), so every
such SpMV below goes through it -- the parity suite's matrices plus shapes with a partial last block and
rows exactly filling the slots, both dtypes -- while the other ELL / HYB matrices check that the
selection leaves them on k_spmv_ell; each element by element against the oracle at the north_star
tolerances (tests/gpu_util.check_spmv).
"""
import os
import subprocess
import sys

import numpy as np
import pytest

import sfsgen

pytestmark = pytest.mark.gpu

HERE = os.path.dirname(os.path.abspath(__file__))


def extra_cases():
    from helpers import random_csr
    rng = np.random.default_rng(77)
    return {
        "ragged_2049": random_csr(rng, 2049, 1500, 0.01, empty_rows=0.1, dense_rows=1),
        "full_slots_f32": sfsgen.generate(sfsgen.make_spec(sfsgen.BLOCKDIAG, seed=21, m=5000, ia=8, pa=1.0,
                                                           dtype=sfsgen.F32)),
        "band_3001_f64": sfsgen.generate(sfsgen.make_spec(sfsgen.BAND, seed=24, m=3001, ia=5, pa=0.6)),
        "st2d5_40_f32": sfsgen.generate(sfsgen.make_spec(sfsgen.ST2D5, ia=40, dtype=sfsgen.F32)),
        "uniform_f32": sfsgen.generate(sfsgen.make_spec(sfsgen.UNIFORM, seed=22, m=7001, n=6000, pa=9.0,
                                                        dtype=sfsgen.F32)),
        "powerlaw_f64": sfsgen.generate(sfsgen.make_spec(sfsgen.POWERLAW, seed=23, m=20000, pa=2.3)),
    }


def run_all():
    """Child-process body (SFS_ELL_TMA_MB=0): every case's ELL and HYB SpMV against the oracle."""
    sys.path.insert(0, HERE)
    import oracle
    import paper_conf_icppw_dhandhaniadpbl21_b200 as sfs
    from gpu_util import check_spmv, to_dev
    from test_gpu_parity import NAMES, cases
    allc = dict(cases())
    allc.update(extra_cases())
    n_ok, n_tma = 0, 0
    for name, A in allc.items():
        fo = oracle.features(A.m, A.n, A.rp, A.col)
        dA = to_dev(A)
        for fmt in (sfs.ELL, sfs.HYB):
            if not (fo["admissible_mask"] >> fmt) & 1:
                continue
            M = sfs.convert(dA, fmt)
            lay = M.layout()
            n_tma += bool((fo["admissible_mask"] >> sfs.DIA) & 1) and (fmt == sfs.ELL or lay.coo_nnz == 0)
            for seed in (11, 12):
                check_spmv(A, fmt, M, sfsgen.vector(seed, A.n, A.dtype), A.dtype,
                           ctx=f"ell_tma {name} {sfs.FORMAT_NAMES[fmt]}")
            M.free()
            n_ok += 1
    assert n_tma >= 12, n_tma  # SpMVs that ran the TMA kernel
    print(f"ELL_TMA_OK {n_ok} {n_tma}")


def test_ell_tma_every_size():
    env = dict(os.environ, SFS_ELL_TMA_MB="0", SFS_ELL_TMA_K="0")
    code = f"import sys; sys.path.insert(0, {HERE!r}); import test_gpu_ell_tma as t; t.run_all()"
    r = subprocess.run([sys.executable, "-c", code], env=env, capture_output=True, text=True, timeout=300,
                       cwd=os.path.dirname(HERE))
    assert r.returncode == 0 and "ELL_TMA_OK" in r.stdout, r.stdout[-3000:] + r.stderr[-3000:]
