"""The GPU generators (sfsgen/gen_device.cu) emit the host generators' CSR bit for bit (SURVEY App. B:
"host and device must emit bit-identical CSR"): every class, both value types, sampled rows with
duplicates, power-law rows in the Bernoulli mode, R-MAT, corpus specs of configs[1] and configs[4]."""
import numpy as np
import pytest

import sfsgen

pytestmark = pytest.mark.gpu


def _same(spec):
    A = sfsgen.generate(spec)
    m, n, rp, col, val = sfsgen.generate_device(spec)
    assert (m, n) == (A.m, A.n)
    assert np.array_equal(rp.cpu().numpy(), A.rp)
    assert np.array_equal(col.cpu().numpy(), A.col)
    v = val.cpu().numpy()
    assert v.dtype == A.val.dtype and v.tobytes() == A.val.tobytes()
    return A


CASES = {
    "band": sfsgen.make_spec(sfsgen.BAND, seed=3, m=20011, ia=9, pa=0.7),
    "band32": sfsgen.make_spec(sfsgen.BAND, seed=4, m=5000, ia=32, pa=0.55, dtype=sfsgen.F32),
    "blockdiag": sfsgen.make_spec(sfsgen.BLOCKDIAG, seed=5, m=9001, ia=37, pa=0.8, dtype=sfsgen.F32),
    "uniform": sfsgen.make_spec(sfsgen.UNIFORM, seed=6, m=12000, n=9000, pa=17.0),
    "uniform_dups": sfsgen.make_spec(sfsgen.UNIFORM, seed=7, m=3000, n=40, pa=60.0),  # many duplicate draws
    "powerlaw": sfsgen.make_spec(sfsgen.POWERLAW, seed=8, m=30000, pa=2.15, dtype=sfsgen.F32),
    "powerlaw_bern": sfsgen.make_spec(sfsgen.POWERLAW, seed=9, m=1500, pa=2.05),  # rows longer than n/8
    "rmat14": sfsgen.make_spec(sfsgen.RMAT, seed=7, ia=14, ib=16, dtype=sfsgen.F32),
    "rmat12_f64": sfsgen.make_spec(sfsgen.RMAT, seed=2, ia=12, ib=8, dtype=sfsgen.F64),
    "st2d5": sfsgen.make_spec(sfsgen.ST2D5, ia=64),
    "st3d7": sfsgen.make_spec(sfsgen.ST3D7, ia=33, dtype=sfsgen.F32),
    "st3d27": sfsgen.make_spec(sfsgen.ST3D27, ia=20),
}


@pytest.mark.parametrize("name", list(CASES))
def test_device_generator_bit_identical(name):
    A = _same(CASES[name])
    if name == "powerlaw_bern":
        lens = np.diff(A.rp)
        assert lens.max() > A.n // 8  # the Bernoulli mode was exercised


@pytest.mark.parametrize("corpus,i", [(200, 0), (200, 1), (200, 2), (200, 3), (200, 6), (200, 9), (2000, 0),
                                      (2000, 1), (2000, 5)])
def test_device_generator_corpus_specs(corpus, i):
    spec = sfsgen.corpus_spec(corpus, i)
    if corpus == 2000:
        m, _ = sfsgen.dims(spec)
        if m > 3_000_000:
            pytest.skip("large configs[4] matrix")
    _same(spec)


def test_device_vector_bit_identical():
    for dt in (sfsgen.F32, sfsgen.F64):
        x = sfsgen.vector(11, 100_003, dt)
        assert sfsgen.vector_device(11, 100_003, dt).cpu().numpy().tobytes() == x.tobytes()
