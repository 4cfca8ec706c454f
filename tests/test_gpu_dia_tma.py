"""GPU parity of the TMA DIA kernel (k_spmv_dia_tma: slab streamed by cp.async.bulk through an
mbarrier ring, x staged in shared memory) at every size.

The library uses it for matrices of >= SFS_DIA_SX_MIN blocks of 1024 rows (the full-size configs[3] and
ragged bandwidth-bound cases of test_gpu_configs.py run it at the default threshold).  Here a child
process sets SFS_DIA_SX_MIN=0 and SFS_DIA_TMA_ND=0 (read once per process), so every DIA SpMV below goes through it: small
and ragged shapes (partial last block, m < 1024, n != m), offsets forming many
windows (more than the 32 staged ones), windows past the shared-memory budget (x read from global
memory), windows clipped at both ends of x, explicit zeros, both dtypes -- each element by element
against the oracle at the north_star tolerances (tests/gpu_util.check_spmv).
"""
import os
import subprocess
import sys

import numpy as np
import pytest

import sfsgen

pytestmark = pytest.mark.gpu

HERE = os.path.dirname(os.path.abspath(__file__))


def diag_csr(m, n, offsets, dtype, seed, fill=1.0, zeros=0.0):
    """CSR whose entries lie on the given diagonals (col = row + off), values in +-[0.5, 1)."""
    rng = np.random.default_rng(seed)
    rows, cols = [], []
    for off in sorted(set(offsets)):
        r = np.arange(max(0, -off), min(m, n - off))
        if fill < 1.0:
            r = r[rng.random(len(r)) < fill]
        rows.append(r)
        cols.append(r + off)
    rows = np.concatenate(rows) if rows else np.zeros(0, np.int64)
    cols = np.concatenate(cols) if cols else np.zeros(0, np.int64)
    order = np.lexsort((cols, rows))
    rows, cols = rows[order], cols[order]
    vals = rng.uniform(0.5, 1.0, len(rows)) * rng.choice([-1.0, 1.0], len(rows))
    if zeros:
        vals[rng.random(len(rows)) < zeros] = 0.0
    rp = np.zeros(m + 1, np.int64)
    np.add.at(rp, rows + 1, 1)
    rp = np.cumsum(rp)
    return sfsgen.CSR(m, n, rp.astype(np.int32), cols.astype(np.int32), vals.astype(dtype))


def cases():
    f32, f64 = np.float32, np.float64
    scattered = [int(v) for v in np.arange(-20, 21) * 700]  # 41 windows (gaps 700 > 256): 9 unstaged
    return {
        "st3d27_20_f64": sfsgen.generate(sfsgen.make_spec(sfsgen.ST3D27, ia=20)),
        "st3d27_13_f32": sfsgen.generate(sfsgen.make_spec(sfsgen.ST3D27, ia=13, dtype=sfsgen.F32)),
        "band_f64": sfsgen.generate(sfsgen.make_spec(sfsgen.BAND, seed=3, m=20011, ia=9, pa=0.7)),
        "blockdiag_f32": sfsgen.generate(sfsgen.make_spec(sfsgen.BLOCKDIAG, seed=4, m=9001, ia=37, pa=0.8,
                                                          dtype=sfsgen.F32)),
        "tiny_m_lt_block": diag_csr(37, 37, [-3, 0, 1, 5], f64, 1),
        "rect_wide": diag_csr(3000, 5123, [-7, 0, 2, 900, 2000, 4000], f32, 2, zeros=0.1),
        "rect_tall": diag_csr(5123, 3000, [-4000, -2100, -1, 0, 3], f64, 3),
        "scattered_41_windows_f32": diag_csr(30011, 30011, scattered, f32, 4, fill=0.9),
        "scattered_41_windows_f64": diag_csr(30011, 30011, scattered, f64, 5, fill=0.9),
        # one window of 4096 + 1024 values: past the fp64 budget (4096), inside the fp32 one (8192)
        "wide_window_f64": diag_csr(8192, 8192, list(range(-2048, 2049, 200)), f64, 6),
        "wide_window_f32": diag_csr(8192, 8192, list(range(-2048, 2049, 200)), f32, 7),
        "two_budget_windows_f64": diag_csr(12000, 12000, list(range(-3000, -1000, 250)) + list(range(1000, 3001, 250)),
                                           f64, 8),
        "edge_offsets": diag_csr(4099, 4099, [-4098, -1, 0, 1, 4098], f64, 9),
    }


def run_all():
    """Child-process body (SFS_DIA_SX_MIN=0): every case's DIA SpMV against the oracle."""
    sys.path.insert(0, HERE)
    import oracle
    import paper_conf_icppw_dhandhaniadpbl21_b200 as sfs
    from gpu_util import check_spmv, to_dev
    n_ok = 0
    for name, A in cases().items():
        fo = oracle.features(A.m, A.n, A.rp, A.col)
        assert (fo["admissible_mask"] >> sfs.DIA) & 1, f"{name}: DIA inadmissible"
        M = sfs.convert(to_dev(A), sfs.DIA)
        for seed in (11, 12):
            check_spmv(A, sfs.DIA, M, sfsgen.vector(seed, A.n, A.dtype), A.dtype, ctx=f"dia_sx {name}")
        M.free()
        n_ok += 1
    print(f"DIA_TMA_OK {n_ok}")


def test_dia_tma_every_size():
    env = dict(os.environ, SFS_DIA_SX_MIN="0", SFS_DIA_TMA_ND="0")
    code = f"import sys; sys.path.insert(0, {HERE!r}); import test_gpu_dia_tma as t; t.run_all()"
    r = subprocess.run([sys.executable, "-c", code], env=env, capture_output=True, text=True, timeout=240,
                       cwd=os.path.dirname(HERE))
    assert r.returncode == 0 and f"DIA_TMA_OK {len(cases())}" in r.stdout, r.stdout[-3000:] + r.stderr[-3000:]
