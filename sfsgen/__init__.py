"""sfsgen — seeded synthetic CSR generators (test / bench input only).

Thin ctypes wrapper over ``libsfsgen.so`` (``sfsgen/gen.c``).  This is the one module both the CPU
oracle and the CUDA path are fed from; it contains none of the method's arithmetic.  Recipe:
SURVEY.md Appendix B / DESIGN.md "Input recipe"; structure classes stand in for the SuiteSparse
classes of PAPER.md L194 (§5.1 "Benchmarks").
"""
from __future__ import annotations

import ctypes
import os
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libsfsgen.so")

BAND, BLOCKDIAG, UNIFORM, POWERLAW, RMAT, ST2D5, ST3D7, ST3D27 = range(8)
CLASS_NAMES = {BAND: "band", BLOCKDIAG: "blockdiag", UNIFORM: "uniform", POWERLAW: "powerlaw",
               RMAT: "rmat", ST2D5: "stencil2d5", ST3D7: "stencil3d7", ST3D27: "stencil3d27"}
F32, F64 = 0, 1


class Spec(ctypes.Structure):
    _fields_ = [("cls", ctypes.c_int32), ("dtype", ctypes.c_int32), ("seed", ctypes.c_uint64),
                ("m", ctypes.c_int64), ("n", ctypes.c_int64), ("ia", ctypes.c_int64),
                ("ib", ctypes.c_int64), ("pa", ctypes.c_double), ("pb", ctypes.c_double)]

    def describe(self) -> dict:
        return {"cls": CLASS_NAMES.get(self.cls, str(self.cls)), "dtype": "f64" if self.dtype else "f32",
                "seed": int(self.seed), "m": int(self.m), "n": int(self.n), "ia": int(self.ia),
                "ib": int(self.ib), "pa": float(self.pa)}


class _CSR(ctypes.Structure):
    _fields_ = [("m", ctypes.c_int64), ("n", ctypes.c_int64), ("nnz", ctypes.c_int64),
                ("rp", ctypes.POINTER(ctypes.c_int32)), ("col", ctypes.POINTER(ctypes.c_int32)),
                ("val", ctypes.c_void_p), ("dtype", ctypes.c_int32)]


_lib = None


def lib():
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise RuntimeError(f"{LIB_PATH} missing: run `python -c 'import __graft_entry__ as g; g.build()'`")
        L = ctypes.CDLL(LIB_PATH)
        L.sfsgen_generate.argtypes = [ctypes.POINTER(Spec), ctypes.POINTER(_CSR)]
        L.sfsgen_generate.restype = ctypes.c_int
        L.sfsgen_free.argtypes = [ctypes.POINTER(_CSR)]
        L.sfsgen_vector.argtypes = [ctypes.c_uint64, ctypes.c_int64, ctypes.c_int32, ctypes.c_void_p]
        L.sfsgen_corpus_spec.argtypes = [ctypes.c_int32, ctypes.c_int64, ctypes.POINTER(Spec)]
        L.sfsgen_corpus_spec.restype = ctypes.c_int
        L.sfsgen_dims.argtypes = [ctypes.POINTER(Spec), ctypes.POINTER(ctypes.c_int64), ctypes.POINTER(ctypes.c_int64)]
        L.sfsgen_hash.argtypes = [ctypes.c_uint64, ctypes.c_uint64, ctypes.c_uint64]
        L.sfsgen_hash.restype = ctypes.c_uint64
        L.sfsgen_threads.restype = ctypes.c_int
        _lib = L
    return _lib


@dataclass
class CSR:
    """Host CSR (numpy). rp int32[m+1], col int32[nnz], val float32/float64[nnz]."""
    m: int
    n: int
    rp: np.ndarray
    col: np.ndarray
    val: np.ndarray

    @property
    def nnz(self) -> int:
        return int(self.col.shape[0])

    @property
    def dtype(self) -> int:
        return F64 if self.val.dtype == np.float64 else F32

    def nbytes(self) -> int:
        return self.rp.nbytes + self.col.nbytes + self.val.nbytes


def make_spec(cls, *, seed=1, m=0, n=0, ia=0, ib=0, pa=0.0, pb=0.0, dtype=F64) -> Spec:
    return Spec(cls, dtype, seed & 0xFFFFFFFFFFFFFFFF, m, n or m, ia, ib, pa, pb)


def generate(spec: Spec) -> CSR:
    out = _CSR()
    rc = lib().sfsgen_generate(ctypes.byref(spec), ctypes.byref(out))
    if rc != 0:
        raise RuntimeError(f"sfsgen_generate failed for {spec.describe()}")
    try:
        m, nnz = out.m, out.nnz
        rp = np.ctypeslib.as_array(out.rp, shape=(m + 1,)).copy()
        col = np.ctypeslib.as_array(out.col, shape=(max(nnz, 1),))[:nnz].copy()
        vt = ctypes.c_double if out.dtype else ctypes.c_float
        vptr = ctypes.cast(out.val, ctypes.POINTER(vt))
        val = np.ctypeslib.as_array(vptr, shape=(max(nnz, 1),))[:nnz].copy()
        return CSR(int(out.m), int(out.n), rp, col, val)
    finally:
        lib().sfsgen_free(ctypes.byref(out))


def vector(seed: int, n: int, dtype: int = F64) -> np.ndarray:
    x = np.empty(n, dtype=np.float64 if dtype else np.float32)
    lib().sfsgen_vector(seed & 0xFFFFFFFFFFFFFFFF, n, dtype, x.ctypes.data)
    return x


def corpus_spec(corpus: int, i: int) -> Spec:
    s = Spec()
    if lib().sfsgen_corpus_spec(corpus, i, ctypes.byref(s)) != 0:
        raise ValueError(f"unknown corpus {corpus}")
    return s


def dims(spec: Spec):
    m, n = ctypes.c_int64(), ctypes.c_int64()
    lib().sfsgen_dims(ctypes.byref(spec), ctypes.byref(m), ctypes.byref(n))
    return m.value, n.value


def threads() -> int:
    return int(lib().sfsgen_threads())


# ---------------------------------------------------------------- named matrices of BASELINE configs
def laplace2d(N=64, dtype=F64) -> CSR:
    """configs[0]: 2D 5-point Laplacian on an N x N grid (Dirichlet, no wrap)."""
    return generate(make_spec(ST2D5, ia=N, dtype=dtype))


def stencil3d27(N=128, dtype=F64) -> CSR:
    """configs[3]: 3D 27-point stencil on an N^3 grid."""
    return generate(make_spec(ST3D27, ia=N, dtype=dtype))


def rmat(scale=22, seed=1, ef=16, dtype=F32) -> CSR:
    """configs[2]: R-MAT (Graph500 A/B/C/D = .57/.19/.19/.05), natural ordering, duplicates dropped."""
    return generate(make_spec(RMAT, seed=seed, ia=scale, ib=ef, dtype=dtype))


def from_dense(a: np.ndarray, dtype=None) -> CSR:
    """Tiny hand-written test matrices: CSR of the nonzero pattern of a dense array (zeros dropped)."""
    a = np.asarray(a)
    if dtype is None:
        dtype = np.float64
    m, n = a.shape
    rp = [0]
    cols, vals = [], []
    for r in range(m):
        for c in range(n):
            if a[r, c] != 0:
                cols.append(c)
                vals.append(a[r, c])
        rp.append(len(cols))
    return CSR(m, n, np.array(rp, np.int32), np.array(cols, np.int32), np.array(vals, dtype))


# ---------------------------------------------------------------- the same generators on the GPU
# libsfsgen_dev.so (gen_device.cu): bit-identical CSR built in device memory (§8(d) C5
# "Generated on device per rank").  Returned as torch tensors on the current CUDA device.
DEV_LIB_PATH = os.path.join(_HERE, "libsfsgen_dev.so")
_dlib = None


def dlib():
    global _dlib
    if _dlib is None:
        if not os.path.exists(DEV_LIB_PATH):
            raise RuntimeError(f"{DEV_LIB_PATH} missing: run build_native.build_gen_device()")
        L = ctypes.CDLL(DEV_LIB_PATH)
        L.sfsgen_generate_device.argtypes = [ctypes.POINTER(Spec), ctypes.POINTER(_CSR), ctypes.c_void_p]
        L.sfsgen_generate_device.restype = ctypes.c_int
        L.sfsgen_free_device.argtypes = [ctypes.POINTER(_CSR)]
        L.sfsgen_vector_device.argtypes = [ctypes.c_uint64, ctypes.c_int64, ctypes.c_int32, ctypes.c_void_p,
                                           ctypes.c_void_p]
        L.sfsgen_vector_device.restype = ctypes.c_int
        _dlib = L
    return _dlib


class _DevBuf:
    def __init__(self, ptr, n, typestr):
        self.__cuda_array_interface__ = {"shape": (n,), "typestr": typestr, "data": (ptr, False), "version": 3,
                                         "strides": None}


def generate_device(spec: Spec):
    """(m, n, rp, col, val) with rp/col/val torch tensors on the current CUDA device (copies of the library's
    buffers, which are freed before returning)."""
    import torch
    out = _CSR()
    st = torch.cuda.current_stream()
    rc = dlib().sfsgen_generate_device(ctypes.byref(spec), ctypes.byref(out), st.cuda_stream)
    if rc != 0:
        raise RuntimeError(f"sfsgen_generate_device failed for {spec.describe()}")
    try:
        m, nnz = int(out.m), int(out.nnz)
        dev = torch.device("cuda", torch.cuda.current_device())
        view = lambda p, k, t: torch.as_tensor(_DevBuf(ctypes.cast(p, ctypes.c_void_p).value, k, t), device=dev)
        rp = view(out.rp, m + 1, "<i4").clone()
        col = view(out.col, max(nnz, 1), "<i4")[:nnz].clone()
        val = view(out.val, max(nnz, 1), "<f8" if out.dtype else "<f4")[:nnz].clone()
        torch.cuda.synchronize()
        return m, int(out.n), rp, col, val
    finally:
        dlib().sfsgen_free_device(ctypes.byref(out))


def vector_device(seed: int, n: int, dtype: int = F64):
    import torch
    x = torch.empty(n, dtype=torch.float64 if dtype else torch.float32, device="cuda")
    if dlib().sfsgen_vector_device(seed & 0xFFFFFFFFFFFFFFFF, n, dtype, x.data_ptr(),
                                   torch.cuda.current_stream().cuda_stream) != 0:
        raise RuntimeError("sfsgen_vector_device failed")
    return x
