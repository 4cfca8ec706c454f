"""B200-native sparse-format labelling path (Dhandhania et al., ICPP Workshops '21).

Thin Python binding over the C ABI of ``include/sfs.h`` (``libsfs.so``, CUDA for sm_100a).  This
module only marshals arguments: every step of the path (features, conversions, SpMV, the race)
runs in the library's kernels.  PyTorch is used for device memory and streams only.  There is no
CPU fallback: without the built library or a GPU every call raises.
"""
from __future__ import annotations

import ctypes
import os
from dataclasses import dataclass, field
from typing import List, Optional, Sequence

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("SFS_LIB") or os.path.join(_HERE, "libsfs.so")  # SFS_LIB: A/B builds

CSR, COO, ELL, HYB, DIA = range(5)
NFMT = 5
FORMAT_NAMES = ["CSR", "COO", "ELL", "HYB", "DIA"]
F32, F64 = 0, 1
MEM_DEVICE, MEM_HOST = 0, 1

OK, ERR_INVALID_ARG, ERR_INVALID_CSR, ERR_INADMISSIBLE, ERR_OOM, ERR_CUDA, ERR_UNSUPPORTED, ERR_NOT_RUN = (
    0, -1, -2, -3, -4, -5, -6, -7)

_I64, _I32, _U32, _D, _P = ctypes.c_int64, ctypes.c_int32, ctypes.c_uint32, ctypes.c_double, ctypes.c_void_p


class SfsError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"{msg} (status {status})")
        self.status = status


class CsrStruct(ctypes.Structure):
    _fields_ = [("nrows", _I64), ("ncols", _I64), ("nnz", _I64), ("row_ptr", _P), ("col_idx", _P),
                ("values", _P), ("dtype", _I32), ("mem", _I32), ("x", _P)]


FEATURE_INT_FIELDS = ["nrows", "ncols", "nnz", "nnz_min", "nnz_max", "csr_max", "ell_size", "hyb_k",
                      "hyb_ell_size", "hyb_coo", "hyb_ell_nnz", "diagonals", "dia_size"]
FEATURE_FLOAT_FIELDS = ["nnz_frac", "nnz_mu", "nnz_sig", "max_mu", "mu_min", "sig_lower", "sig_higher",
                        "hyb_ell_frac", "dia_frac", "ell_frac"]


class FeaturesStruct(ctypes.Structure):
    _fields_ = ([(f, _I64) for f in FEATURE_INT_FIELDS] + [(f, _D) for f in FEATURE_FLOAT_FIELDS]
                + [("admissible_mask", _U32), ("csr_variant", _I32)])

    def as_dict(self) -> dict:
        d = {f: int(getattr(self, f)) for f in FEATURE_INT_FIELDS}
        d.update({f: float(getattr(self, f)) for f in FEATURE_FLOAT_FIELDS})
        d["admissible_mask"] = int(self.admissible_mask)
        d["csr_variant"] = int(self.csr_variant)
        return d


class LayoutStruct(ctypes.Structure):
    _fields_ = [("fmt", _I32), ("dtype", _I32), ("nrows", _I64), ("ncols", _I64), ("nnz", _I64), ("pitch", _I64),
                ("width", _I64), ("ndiag", _I64), ("coo_nnz", _I64), ("ptr", _P * 6), ("bytes", _I64),
                ("variant", _I32)]


class RaceOpts(ctypes.Structure):
    _fields_ = [("reps", _I32), ("warmup", _I32), ("formats_mask", _U32), ("cold", _I32), ("max_fill", _D),
                ("fill_slack", _I64), ("hyb_rel_speed", _D), ("hyb_breakeven", _I64), ("csr_variant", _I32),
                ("use_graphs", _I32), ("race_mask", _P)]


class LabelStruct(ctypes.Structure):
    _fields_ = [("label", _I32), ("admissible_mask", _U32), ("matrix_status", _I32), ("csr_variant", _I32),
                ("t_spmv_us", ctypes.c_float * NFMT), ("t_convert_us", ctypes.c_float * NFMT),
                ("status", _I32 * NFMT), ("bytes", _I64 * NFMT), ("t_features_us", ctypes.c_float)]

    def as_dict(self) -> dict:
        return {"label": int(self.label), "admissible_mask": int(self.admissible_mask),
                "matrix_status": int(self.matrix_status), "csr_variant": int(self.csr_variant),
                "t_spmv_us": list(self.t_spmv_us), "t_convert_us": list(self.t_convert_us),
                "status": list(self.status), "bytes": list(self.bytes), "t_features_us": float(self.t_features_us)}


_lib = None


def lib():
    """Load libsfs.so (fails loudly: there is no fallback)."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise RuntimeError(f"{LIB_PATH} is missing: build it with __graft_entry__.build()")
        L = ctypes.CDLL(LIB_PATH)
        L.sfs_default_opts.argtypes = [ctypes.POINTER(RaceOpts)]
        L.sfs_features.argtypes = [ctypes.POINTER(CsrStruct), ctypes.POINTER(RaceOpts), ctypes.POINTER(FeaturesStruct), _P]
        L.sfs_convert.argtypes = [ctypes.POINTER(CsrStruct), _I32, ctypes.POINTER(RaceOpts), ctypes.POINTER(_P), _P]
        L.sfs_spmv.argtypes = [_I32, _P, _P, _P, _P]
        L.sfs_gather.argtypes = [_I32, _P, _P, _I64, _P, _P]
        L.sfs_spmv_push.argtypes = [_I32, _P, _P, _P, ctypes.POINTER(PushStruct), _P]
        L.sfs_halo_push.argtypes = [_I32, _P, _I64, ctypes.POINTER(PushStruct), _P]
        L.sfs_ipc_alloc.argtypes = [ctypes.c_size_t, ctypes.POINTER(_P), ctypes.c_char_p]
        L.sfs_ipc_open.argtypes = [ctypes.c_char_p, ctypes.POINTER(_P)]
        L.sfs_ipc_close.argtypes = [_P]
        L.sfs_ipc_free.argtypes = [_P]
        L.sfs_label_corpus.argtypes = [ctypes.POINTER(CsrStruct), _I64, ctypes.POINTER(RaceOpts),
                                       ctypes.POINTER(FeaturesStruct), ctypes.POINTER(LabelStruct), _P]
        L.sfs_matrix_free.argtypes = [_P]
        L.sfs_matrix_describe.argtypes = [_P, ctypes.POINTER(LayoutStruct)]
        L.sfs_spmv_bytes.argtypes = [ctypes.POINTER(FeaturesStruct), _I32, _I32]
        L.sfs_spmv_bytes.restype = _I64
        L.sfs_status_string.argtypes = [_I32]
        L.sfs_status_string.restype = ctypes.c_char_p
        L.sfs_last_error.restype = ctypes.c_char_p
        L.sfs_launch_count.restype = _I64
        L.sfs_version.restype = ctypes.c_char_p
        L.sfs_set_allocator.argtypes = [_ALLOC_T, _FREE_T]
        L.sfs_set_allocator.restype = None
        for fn in ("sfs_features", "sfs_convert", "sfs_spmv", "sfs_label_corpus", "sfs_matrix_free",
                   "sfs_matrix_describe"):
            getattr(L, fn).restype = _I32
        _lib = L
        if os.environ.get("SFS_TORCH_ALLOC", "0") == "1":
            use_torch_allocator(True)
    return _lib


EXPORTED = ["sfs_features", "sfs_convert", "sfs_spmv", "sfs_label_corpus", "sfs_matrix_free",
            "sfs_matrix_describe", "sfs_status_string", "sfs_last_error", "sfs_set_allocator",
            "sfs_default_opts", "sfs_spmv_bytes", "sfs_launch_count", "sfs_version"]


# ------------------------------------------------------------------ allocator hook (§8(b) ownership)
# Library-owned buffers (converted matrices, race temporaries, staged inputs) come from torch's caching
# allocator, so they share one pool with the caller's tensors.  The library frees stream-ordered on the
# stream it names.  torch's allocator reuses a block on the stream it was allocated on, so a block freed
# on ANOTHER stream (host inputs are staged on the copy stream and released on the compute stream) is
# handed back only once an event recorded on the freeing stream has completed (the deferred-free
# discipline of torch's record_stream; nothing waits, so the copy / race overlap is kept).
# Opt-in (use_torch_allocator() or SFS_TORCH_ALLOC=1): every library allocation becomes a Python call
# under the GIL, which the device-resident race hides (bench 162.9 vs 162.7 matrices/s) but the
# chunk-synchronised host-input path does not (e2e 127 vs 161 matrices/s, profiles/r02/micro_ab.txt);
# by default the library keeps its own CUDA stream-ordered pool.
_ALLOC_T = ctypes.CFUNCTYPE(_P, ctypes.c_size_t, _P)
_FREE_T = ctypes.CFUNCTYPE(None, _P, _P)
_alloc_state = {"on": False, "blocks": {}, "pending": [], "cbs": None}


def _drain_pending(force=False):
    import torch
    pend = _alloc_state["pending"]
    keep = []
    for ev, ptr in pend:
        if force or ev.query():
            torch.cuda.caching_allocator_delete(ptr)
        else:
            keep.append((ev, ptr))
    _alloc_state["pending"] = keep


def _torch_alloc(nbytes, stream):
    try:
        import torch
        if _alloc_state["pending"]:
            _drain_pending()
        dev = torch.cuda.current_device()
        p = torch.cuda.caching_allocator_alloc(int(nbytes), dev, stream or 0)
        _alloc_state["blocks"][p] = (stream or 0, dev)
        return p
    except Exception:  # OOM or torch torn down: the library reports SFS_ERR_OOM
        return None


def _torch_free(ptr, stream):
    try:
        import torch
        a_stream, dev = _alloc_state["blocks"].pop(ptr, (stream or 0, None))
        if (stream or 0) != a_stream:
            sf = torch.cuda.ExternalStream(stream, device=dev) if stream else torch.cuda.default_stream(dev)
            ev = torch.cuda.Event()
            ev.record(sf)
            _alloc_state["pending"].append((ev, ptr))
        else:
            torch.cuda.caching_allocator_delete(ptr)
        if _alloc_state["pending"]:
            _drain_pending()
    except Exception:
        pass


def use_torch_allocator(enable: bool = True):
    """Route the library's device allocations through torch's caching allocator (sfs_set_allocator)."""
    L = lib()
    if enable and not _alloc_state["on"]:
        if _alloc_state["cbs"] is None:  # created once: handles built under the hook keep calling its free
            _alloc_state["cbs"] = (_ALLOC_T(_torch_alloc), _FREE_T(_torch_free))
        cbs = _alloc_state["cbs"]
        L.sfs_set_allocator(cbs[0], cbs[1])
        _alloc_state["on"] = True
    elif not enable and _alloc_state["on"]:
        L.sfs_set_allocator(_ALLOC_T(), _FREE_T())  # NULL pointers: back to the library pool
        _alloc_state["on"] = False


def torch_allocator_enabled() -> bool:
    return _alloc_state["on"]


def _check(st: int, what: str):
    if st != OK:
        err = lib().sfs_last_error().decode(errors="replace")
        raise SfsError(st, f"{what}: {lib().sfs_status_string(st).decode()} — {err}")


def default_opts(**kw) -> RaceOpts:
    o = RaceOpts()
    lib().sfs_default_opts(ctypes.byref(o))
    for k, v in kw.items():
        if not hasattr(o, k):
            raise AttributeError(k)
        setattr(o, k, v)
    return o


def launch_count() -> int:
    return int(lib().sfs_launch_count())


def _stream_ptr(stream) -> Optional[int]:
    import torch
    if stream is None:
        stream = torch.cuda.current_stream()
    return stream.cuda_stream


@dataclass
class Csr:
    """A CSR matrix held in torch tensors (device, or pinned host memory for the end-to-end path).
    rp int32[m+1], col int32[nnz], val float32/float64[nnz]; x optional race input (ncols)."""
    m: int
    n: int
    rp: "object"
    col: "object"
    val: "object"
    x: "object" = None

    @property
    def nnz(self) -> int:
        return int(self.col.numel())

    @property
    def dtype(self) -> int:
        import torch
        return F64 if self.val.dtype == torch.float64 else F32

    def struct(self) -> CsrStruct:
        """The sfs_csr view.  The library stages all four arrays from one `mem` flag, so they must
        share a placement: all on one CUDA device, or all in PINNED host memory (pageable host memory
        would silently serialise the copy-stream pipeline of sfs_label_corpus)."""
        import torch
        for t in (self.rp, self.col):
            if t.dtype != torch.int32 or not t.is_contiguous():
                raise SfsError(ERR_INVALID_ARG, "rp / col must be contiguous int32")
        if self.val.dtype not in (torch.float32, torch.float64) or not self.val.is_contiguous():
            raise SfsError(ERR_INVALID_ARG, "val must be contiguous float32 / float64")
        ts = [self.rp, self.col, self.val] + ([self.x] if self.x is not None else [])
        if self.x is not None and (self.x.dtype != self.val.dtype or not self.x.is_contiguous()):
            raise SfsError(ERR_INVALID_ARG, "x must be contiguous with the dtype of val")
        if self.rp.is_cuda:
            if any((not t.is_cuda) or t.device != self.rp.device for t in ts):
                raise SfsError(ERR_INVALID_ARG, "mixed placement: rp is on a device, another array is not (or on another device)")
            mem = MEM_DEVICE
        else:
            if any(t.is_cuda for t in ts):
                raise SfsError(ERR_INVALID_ARG, "mixed placement: rp is in host memory, another array is on a device")
            if any(t.numel() and not t.is_pinned() for t in ts):
                raise SfsError(ERR_INVALID_ARG, "host-memory CSR must be pinned (torch.Tensor.pin_memory())")
            mem = MEM_HOST
        return CsrStruct(self.m, self.n, self.nnz, self.rp.data_ptr(), self.col.data_ptr(), self.val.data_ptr(),
                         self.dtype, mem, self.x.data_ptr() if self.x is not None else None)

    def nbytes(self) -> int:
        return sum(t.numel() * t.element_size() for t in (self.rp, self.col, self.val))


def csr_from_host(A, device="cuda", pin=False, with_x: Optional[int] = None) -> Csr:
    """Move a host (numpy) CSR onto the device (or into pinned host memory)."""
    import torch
    if device == "host":
        t = lambda a: torch.from_numpy(a).pin_memory() if pin else torch.from_numpy(a)
    else:
        t = lambda a: torch.from_numpy(a).to(device)
    x = None
    if with_x is not None:
        import numpy as np
        x = t(with_x) if isinstance(with_x, np.ndarray) else None
    return Csr(A.m, A.n, t(A.rp), t(A.col), t(A.val), x)


def features(A: Csr, opts: Optional[RaceOpts] = None, stream=None) -> dict:
    """Table-1 features computed on the GPU (sfs_features)."""
    f = FeaturesStruct()
    s = A.struct()
    _check(lib().sfs_features(ctypes.byref(s), ctypes.byref(opts) if opts else None, ctypes.byref(f),
                              _stream_ptr(stream)), "sfs_features")
    return f.as_dict()


class Matrix:
    """Library-owned converted matrix (sfs_matrix)."""

    def __init__(self, handle, fmt, keepalive=None):
        self.handle = handle
        self.fmt = fmt
        self._keep = keepalive

    def layout(self) -> LayoutStruct:
        L = LayoutStruct()
        _check(lib().sfs_matrix_describe(self.handle, ctypes.byref(L)), "sfs_matrix_describe")
        return L

    def free(self):
        if self.handle:
            lib().sfs_matrix_free(self.handle)
            self.handle = None

    def __del__(self):
        try:
            self.free()
        except Exception:
            pass


def convert(A: Csr, fmt: int, opts: Optional[RaceOpts] = None, stream=None) -> Matrix:
    """CSR -> fmt on the GPU (sfs_convert)."""
    h = ctypes.c_void_p()
    s = A.struct()
    _check(lib().sfs_convert(ctypes.byref(s), fmt, ctypes.byref(opts) if opts else None, ctypes.byref(h),
                             _stream_ptr(stream)), f"sfs_convert({FORMAT_NAMES[fmt]})")
    return Matrix(h.value, fmt, keepalive=A if fmt == CSR else None)


def spmv(fmt: int, A: Matrix, x, y, stream=None):
    """y = A x on the GPU (sfs_spmv); asynchronous on `stream`."""
    _check(lib().sfs_spmv(fmt, A.handle, x.data_ptr(), y.data_ptr(), _stream_ptr(stream)), "sfs_spmv")
    return y


def gather(src, idx, dst, stream=None):
    """dst[i] = src[idx[i]] on the GPU (sfs_gather): the halo send buffer of the row partition."""
    dt = F64 if src.element_size() == 8 else F32
    _check(lib().sfs_gather(dt, src.data_ptr(), idx.data_ptr(), idx.numel(), dst.data_ptr(), _stream_ptr(stream)),
           "sfs_gather")
    return dst


MAX_PUSH = 8
MAX_PEERS = 16


class PushStruct(ctypes.Structure):
    """sfs_push_t (include/sfs.h): runs of y rows also stored into peer memory, wait / signal flags."""
    _fields_ = [("nseg", _I32), ("seg_begin", _I64 * MAX_PUSH), ("seg_end", _I64 * MAX_PUSH),
                ("seg_dst", _P * MAX_PUSH), ("nwait", _I32), ("wait_flag", _P * MAX_PEERS), ("wait_value", _U32),
                ("nsig", _I32), ("sig_flag", _P * MAX_PEERS), ("sig_value", _U32), ("counter", _P)]


def push_struct(runs, wait_flags, wait_value, sig_flags, sig_value, counter) -> PushStruct:
    """runs: [(begin, end, dst_address)]; flags / counter: device addresses (ints)."""
    if len(runs) > MAX_PUSH or len(wait_flags) > MAX_PEERS or len(sig_flags) > MAX_PEERS:
        raise SfsError(ERR_INVALID_ARG, "push plan too large")
    p = PushStruct()
    p.nseg = len(runs)
    for i, (b, e, d) in enumerate(runs):
        p.seg_begin[i], p.seg_end[i], p.seg_dst[i] = int(b), int(e), int(d)
    p.nwait = len(wait_flags)
    for i, f in enumerate(wait_flags):
        p.wait_flag[i] = int(f)
    p.wait_value = int(wait_value) & 0xFFFFFFFF
    p.nsig = len(sig_flags)
    for i, f in enumerate(sig_flags):
        p.sig_flag[i] = int(f)
    p.sig_value = int(sig_value) & 0xFFFFFFFF
    p.counter = int(counter)
    return p


def spmv_push(fmt: int, A: Matrix, x, y, push: PushStruct, stream=None):
    """y = A x with the halo push fused in (sfs_spmv_push); asynchronous on `stream`."""
    _check(lib().sfs_spmv_push(fmt, A.handle, x.data_ptr(), y.data_ptr(), ctypes.byref(push), _stream_ptr(stream)),
           "sfs_spmv_push")
    return y


def halo_push(src, push: PushStruct, stream=None):
    """The push alone (sfs_halo_push): initial ghost exchange of a row-partitioned iteration."""
    dt = F64 if src.element_size() == 8 else F32
    _check(lib().sfs_halo_push(dt, src.data_ptr(), src.numel(), ctypes.byref(push), _stream_ptr(stream)),
           "sfs_halo_push")


def ipc_alloc(nbytes: int):
    """Zeroed device memory shareable with other processes on the node: (address, 64-byte handle)."""
    p, h = _P(), ctypes.create_string_buffer(64)
    _check(lib().sfs_ipc_alloc(nbytes, ctypes.byref(p), h), "sfs_ipc_alloc")
    return int(p.value), h.raw


def ipc_open(handle: bytes) -> int:
    """Map another process's ipc_alloc buffer (peer access over NVLink when it lives on another GPU)."""
    p = _P()
    _check(lib().sfs_ipc_open(ctypes.create_string_buffer(handle, 64), ctypes.byref(p)), "sfs_ipc_open")
    return int(p.value)


def ipc_close(addr: int):
    _check(lib().sfs_ipc_close(addr), "sfs_ipc_close")


def ipc_free(addr: int):
    _check(lib().sfs_ipc_free(addr), "sfs_ipc_free")


def label_corpus(mats: Sequence[Csr], opts: Optional[RaceOpts] = None, stream=None, race_mask=None):
    """Features + format race + labels for a batch (sfs_label_corpus).  Returns (features, labels)
    as lists of dicts.  race_mask: optional per-matrix format masks (0 = features only; SURVEY §8(f)
    f2), passed as opts.race_mask."""
    n = len(mats)
    arr = (CsrStruct * max(n, 1))(*[m.struct() for m in mats])
    feats = (FeaturesStruct * max(n, 1))()
    labs = (LabelStruct * max(n, 1))()
    keep = None
    if race_mask is not None:
        if len(race_mask) != n:
            raise SfsError(ERR_INVALID_ARG, "race_mask needs one entry per matrix")
        o = RaceOpts()
        if opts is not None:
            ctypes.pointer(o)[0] = opts
        else:
            lib().sfs_default_opts(ctypes.byref(o))
        keep = (_U32 * max(n, 1))(*[int(v) & 0xFFFFFFFF for v in race_mask])
        o.race_mask = ctypes.cast(keep, _P)
        opts = o
    _check(lib().sfs_label_corpus(arr, n, ctypes.byref(opts) if opts else None, feats, labs, _stream_ptr(stream)),
           "sfs_label_corpus")
    del keep
    return [feats[i].as_dict() for i in range(n)], [labs[i].as_dict() for i in range(n)]


def spmv_bytes(feat: dict, fmt: int, dtype: int) -> int:
    f = FeaturesStruct(*[feat[k] for k in FEATURE_INT_FIELDS], *[feat[k] for k in FEATURE_FLOAT_FIELDS],
                       feat["admissible_mask"], feat.get("csr_variant", 0))
    return int(lib().sfs_spmv_bytes(ctypes.byref(f), fmt, dtype))


def decode(M: Matrix):
    """Copy a converted matrix's arrays to the host (numpy), following the documented layout of
    sfs_layout_t.  Test / inspection helper only (no arithmetic)."""
    import numpy as np
    import torch
    L = M.layout()
    vt = torch.float64 if L.dtype == F64 else torch.float32
    ne = int

    def fetch(ptr, n, dtype):
        np_t = {torch.int32: np.int32, torch.float32: np.float32, torch.float64: np.float64}[dtype]
        if n == 0:
            return np.zeros(0, dtype=np_t)
        torch.cuda.synchronize()
        return torch.as_tensor(_DevView(ptr, n, np.dtype(np_t).str), device="cuda").cpu().numpy().copy()

    P, K, m = L.pitch, L.width, L.nrows
    r = {"pitch": P, "width": K, "ndiag": L.ndiag, "coo_nnz": L.coo_nnz, "variant": L.variant, "bytes": L.bytes}
    if L.fmt == CSR:
        r.update(rp=fetch(L.ptr[0], m + 1, torch.int32), col=fetch(L.ptr[1], ne(L.nnz), torch.int32),
                 val=fetch(L.ptr[2], ne(L.nnz), vt))
    elif L.fmt == COO:
        r.update(row=fetch(L.ptr[0], ne(L.nnz), torch.int32), col=fetch(L.ptr[1], ne(L.nnz), torch.int32),
                 val=fetch(L.ptr[2], ne(L.nnz), vt))
    elif L.fmt in (ELL, HYB):
        r.update(ecol=fetch(L.ptr[0], K * P, torch.int32).reshape(K, P) if K else np.zeros((0, P), np.int32),
                 eval=fetch(L.ptr[1], K * P, vt).reshape(K, P) if K else np.zeros((0, P)))
        if L.fmt == HYB:
            c = ne(L.coo_nnz)
            r.update(crow=fetch(L.ptr[2], c, torch.int32), ccol=fetch(L.ptr[3], c, torch.int32),
                     cval=fetch(L.ptr[4], c, vt))
    elif L.fmt == DIA:
        nd = ne(L.ndiag)
        r.update(offs=fetch(L.ptr[0], nd, torch.int32),
                 dval=fetch(L.ptr[1], nd * P, vt).reshape(nd, P) if nd else np.zeros((0, P)))
    return r


class _DevView:
    """Zero-copy view of library-owned device memory (__cuda_array_interface__) for decode()."""

    def __init__(self, ptr: int, n: int, typestr: str):
        self.__cuda_array_interface__ = {"shape": (n,), "typestr": typestr, "data": (ptr, False), "version": 3,
                                         "strides": None}


# ------------------------------------------------------------------ semi-supervised predictor (f1)
NFEAT = 21


class ClusterOpts(ctypes.Structure):
    _fields_ = [("nc", _I32), ("pcs", _I32), ("max_iter", _I32)]


class ClusterInfo(ctypes.Structure):
    _fields_ = [("n", _I64), ("nc", _I32), ("pcs", _I32), ("iters", _I32), ("assign", _P), ("centroids", _P),
                ("basis", _P), ("eigval", _P), ("mins", _P), ("maxs", _P), ("mean", _P)]


_cl_ready = False


def _cl():
    global _cl_ready
    L = lib()
    if not _cl_ready:
        L.sfs_features_table1.argtypes = [ctypes.POINTER(FeaturesStruct), _I64, _P]
        L.sfs_cluster_fit.argtypes = [_P, _I64, _P, ctypes.POINTER(ClusterOpts), ctypes.POINTER(_P), _P]
        L.sfs_cluster_vote.argtypes = [_P, _P, _P, _P]
        L.sfs_cluster_predict.argtypes = [_P, _P, _I64, _P, _P]
        L.sfs_cluster_describe.argtypes = [_P, ctypes.POINTER(ClusterInfo)]
        L.sfs_cluster_free.argtypes = [_P]
        for fn in ("sfs_features_table1", "sfs_cluster_fit", "sfs_cluster_vote", "sfs_cluster_predict",
                   "sfs_cluster_describe", "sfs_cluster_free"):
            getattr(L, fn).restype = _I32
        _cl_ready = True
    return L


def features_table1(feats):
    """n x 21 Table-1 matrix (P:L79–102 order) from feature dicts (sfs_features_table1)."""
    import numpy as np
    n = len(feats)
    arr = (FeaturesStruct * max(n, 1))()
    for i, f in enumerate(feats):
        arr[i] = FeaturesStruct(*[f[k] for k in FEATURE_INT_FIELDS], *[f[k] for k in FEATURE_FLOAT_FIELDS],
                                f["admissible_mask"], f.get("csr_variant", 0))
    out = np.empty((n, NFEAT), np.float64)
    _check(_cl().sfs_features_table1(arr, n, out.ctypes.data), "sfs_features_table1")
    return out


class ClusterModel:
    """Fitted semi-supervised predictor (sfs_cluster_model): transform, min-max, PCA, K-Means."""

    def __init__(self, table1, init_idx, nc=None, pcs=8, max_iter=100, stream=None):
        import numpy as np
        self._np = np
        t = np.ascontiguousarray(table1, dtype=np.float64).reshape(-1, NFEAT)
        init = np.ascontiguousarray(init_idx, dtype=np.int32)
        opts = ClusterOpts(len(init) if nc is None else nc, pcs, max_iter)
        h = ctypes.c_void_p()
        _check(_cl().sfs_cluster_fit(t.ctypes.data, len(t), init.ctypes.data, ctypes.byref(opts), ctypes.byref(h),
                                     _stream_ptr(stream)), "sfs_cluster_fit")
        self.handle = h.value
        self.info = self._describe()

    def _describe(self):
        np = self._np
        I = ClusterInfo()
        _check(_cl().sfs_cluster_describe(self.handle, ctypes.byref(I)), "sfs_cluster_describe")
        arr = lambda p, n, t: np.ctypeslib.as_array(ctypes.cast(p, ctypes.POINTER(t)), shape=(n,)).copy()
        d = ctypes.c_double
        return {"n": I.n, "nc": I.nc, "pcs": I.pcs, "iters": I.iters,
                "assign": arr(I.assign, I.n, ctypes.c_int32),
                "centroids": arr(I.centroids, I.nc * I.pcs, d).reshape(I.nc, I.pcs),
                "basis": arr(I.basis, I.pcs * NFEAT, d).reshape(I.pcs, NFEAT), "eigval": arr(I.eigval, I.pcs, d),
                "mins": arr(I.mins, NFEAT, d), "maxs": arr(I.maxs, NFEAT, d), "mean": arr(I.mean, NFEAT, d)}

    def vote(self, labels, stream=None):
        np = self._np
        lab = np.ascontiguousarray(labels, dtype=np.int32)
        out = np.empty(self.info["nc"], np.int32)
        _check(_cl().sfs_cluster_vote(self.handle, lab.ctypes.data, out.ctypes.data, _stream_ptr(stream)),
               "sfs_cluster_vote")
        return out

    def predict(self, table1, stream=None):
        np = self._np
        t = np.ascontiguousarray(table1, dtype=np.float64).reshape(-1, NFEAT)
        out = np.empty(len(t), np.int32)
        _check(_cl().sfs_cluster_predict(self.handle, t.ctypes.data, len(t), out.ctypes.data, _stream_ptr(stream)),
               "sfs_cluster_predict")
        return out

    def free(self):
        if self.handle:
            _cl().sfs_cluster_free(self.handle)
            self.handle = None

    def __del__(self):
        try:
            self.free()
        except Exception:
            pass
