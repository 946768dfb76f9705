"""ctypes binding of libgmpsvm.so (include/gmpsvm.h) -- argument marshalling only.

Every step of the hot path runs in the library's sm_100a kernels; nothing here computes.
Inputs may be numpy arrays (host pointers; the library does H2D/D2H) or torch CUDA tensors
(device pointers on their device, launched on torch's current stream).  There is no CPU
fallback: if the shared library is missing, every call raises.
"""
from __future__ import annotations

import ctypes as ct
import os
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libgmpsvm.so")

OK, WARN_MAXITER, EINVAL, ENOMEM, ECUDA, ENOTIMPL, EFORMAT = 0, 1, -1, -2, -3, -4, -5


class GmpsvmError(RuntimeError):
    def __init__(self, code, msg):
        super().__init__(f"gmpsvm error {code}: {msg}")
        self.code = code


class Options(ct.Structure):
    _fields_ = [("struct_size", ct.c_int32), ("ws_size", ct.c_int32), ("q", ct.c_int32), ("device", ct.c_int32),
                ("cache_bytes", ct.c_int64), ("stream", ct.c_void_p), ("pair_ids", ct.POINTER(ct.c_int32)),
                ("n_pair_ids", ct.c_int32), ("inputs_on_device", ct.c_int32), ("max_outer_iter", ct.c_int64),
                ("inner_iter_cap", ct.c_int32), ("kernel", ct.c_int32), ("coef0", ct.c_double), ("degree", ct.c_int32),
                ("prob_folds", ct.c_int32), ("reserved", ct.c_int32 * 2)]


KERNELS = {"rbf": 0, "linear": 1, "poly": 2, "sigmoid": 3}  # GMPSVM_KERNEL_*


class TrainStats(ct.Structure):
    _fields_ = [("t_total_ms", ct.c_double), ("t_stage_ms", ct.c_double), ("t_kernel_ms", ct.c_double),
                ("t_select_ms", ct.c_double), ("t_subproblem_ms", ct.c_double), ("t_fupdate_ms", ct.c_double),
                ("t_finalize_ms", ct.c_double), ("kernel_flops", ct.c_double), ("kernel_values", ct.c_double),
                ("krow_launches", ct.c_int64), ("outer_iters_max", ct.c_int64), ("outer_iters_sum", ct.c_int64),
                ("inner_iters_sum", ct.c_int64), ("n_sv", ct.c_int64), ("cache_regime", ct.c_int32),
                ("n_pairs_trained", ct.c_int32), ("launches", ct.c_int64), ("smo_cycles_sum", ct.c_int64),
                ("t_solver_ms", ct.c_double), ("n_streams", ct.c_int32), ("kernel_path", ct.c_int32)]


class PredictStats(ct.Structure):
    _fields_ = [("t_total_ms", ct.c_double), ("t_stage_ms", ct.c_double), ("t_decision_ms", ct.c_double),
                ("t_couple_ms", ct.c_double), ("t_d2h_ms", ct.c_double), ("dec_flops", ct.c_double),
                ("dec_launches", ct.c_int64), ("launches", ct.c_int64), ("dec_path", ct.c_int32),
                ("pad0", ct.c_int32)]


def _struct_dict(s):
    return {name: getattr(s, name) for name, _ in s._fields_}


_lock = threading.Lock()
_lib = None

_P = ct.c_void_p
_SIGS = {
    "gmpsvm_options_init": (None, [_P]),
    "gmpsvm_train": (ct.c_int, [_P, _P, ct.c_int64, ct.c_int32, ct.c_int32, ct.c_double, ct.c_double, ct.c_double, _P]),
    "gmpsvm_train_ex": (ct.c_int, [_P, _P, ct.c_int64, ct.c_int32, ct.c_int32, ct.c_double, ct.c_double, ct.c_double,
                                   _P, _P]),
    "gmpsvm_predict_proba": (ct.c_int, [_P, _P, ct.c_int64, _P]),
    "gmpsvm_predict_proba_ex": (ct.c_int, [_P, _P, ct.c_int64, _P, _P]),
    "gmpsvm_predict_decision": (ct.c_int, [_P, _P, ct.c_int64, _P, _P]),
    "gmpsvm_model_free": (None, [_P]),
    "gmpsvm_last_error": (ct.c_char_p, []),
    "gmpsvm_model_dims": (ct.c_int, [_P, _P, _P, _P, _P]),
    "gmpsvm_model_pair": (ct.c_int, [_P, ct.c_int32, ct.c_int32, _P, _P, _P, _P]),
    "gmpsvm_model_sv_index": (ct.c_int, [_P, _P]),
    "gmpsvm_model_pair_iters": (ct.c_int, [_P, ct.c_int32, ct.c_int32, _P, _P, _P]),
    "gmpsvm_model_train_stats": (ct.c_int, [_P, _P]),
    "gmpsvm_last_predict_stats": (None, [_P]),
    "gmpsvm_model_serialize": (ct.c_int, [_P, _P, _P]),
    "gmpsvm_model_deserialize": (ct.c_int, [_P, ct.c_size_t, _P]),
    "gmpsvm_model_merge": (ct.c_int, [_P, ct.c_int32, _P]),
    "gmpsvm_train_csr": (ct.c_int, [_P, _P, _P, _P, ct.c_int64, ct.c_int32, ct.c_int32, ct.c_double, ct.c_double,
                                    ct.c_double, _P, _P]),
    "gmpsvm_predict_proba_csr": (ct.c_int, [_P, _P, _P, _P, ct.c_int64, _P, _P]),
    "gmpsvm_model_from_alpha": (ct.c_int, [_P, _P, ct.c_int64, ct.c_int32, ct.c_int32, ct.c_double, ct.c_double, _P, _P,
                                           _P, _P, _P, _P, _P]),
    "gmpsvm_rbf_kernel": (ct.c_int, [_P, ct.c_int64, _P, ct.c_int64, ct.c_int32, ct.c_double, _P, _P]),
    "gmpsvm_couple": (ct.c_int, [_P, ct.c_int64, ct.c_int32, _P, _P, _P, _P]),
    "gmpsvm_shard_create": (ct.c_int, [_P, _P, ct.c_int64, ct.c_int32, ct.c_int32, ct.c_int32, ct.c_int32, ct.c_double,
                                       ct.c_double, ct.c_double, ct.c_int32, ct.c_int32, _P, _P]),
    "gmpsvm_shard_cand_doubles": (ct.c_int32, [_P]),
    "gmpsvm_shard_slice": (ct.c_int, [_P, _P, _P, _P, _P]),
    "gmpsvm_shard_candidates": (ct.c_int, [_P, _P]),
    "gmpsvm_shard_select": (ct.c_int, [_P, _P, _P, _P]),
    "gmpsvm_shard_fws": (ct.c_int, [_P, _P]),
    "gmpsvm_shard_step": (ct.c_int, [_P, _P, _P]),
    "gmpsvm_shard_f": (ct.c_int, [_P, _P]),
    "gmpsvm_shard_finish": (ct.c_int, [_P, _P, _P, _P, _P, _P, _P, _P, _P]),
    "gmpsvm_shard_free": (None, [_P]),
    "gmpsvm_shard_merge": (ct.c_int, [_P, ct.c_int32, ct.c_int32, ct.c_int32, ct.c_int32, _P, _P, _P]),
    "gmpsvm_launch_count": (ct.c_uint64, []),
    "gmpsvm_abi_version": (ct.c_int32, []),
}


def lib():
    """The loaded libgmpsvm.so (raises if it has not been built -- no fallback)."""
    global _lib
    with _lock:
        if _lib is None:
            if not os.path.exists(LIB_PATH):
                raise ImportError(f"{LIB_PATH} is missing: build it with "
                                  "`python -m paper_conf_icde_wenshcc19_b200.build` (there is no CPU fallback)")
            L = ct.CDLL(LIB_PATH)
            for name, (res, args) in _SIGS.items():
                fn = getattr(L, name)
                fn.restype = res
                fn.argtypes = args
            _lib = L
        return _lib


def _check(rc):
    if rc < 0:
        raise GmpsvmError(rc, lib().gmpsvm_last_error().decode())
    return rc


# ------------------------------------------------------------------------------ marshalling
def _is_torch(x):
    return type(x).__module__.startswith("torch")


class _Arg:
    """A pointer to the data of a numpy array or torch tensor (keeps the object alive)."""

    def __init__(self, x, dtype, name, ndim=None):
        self.on_device = False
        self.device = 0
        if _is_torch(x):
            import torch
            tdt = {np.float32: torch.float32, np.float64: torch.float64, np.int32: torch.int32,
                   np.int64: torch.int64}[dtype]
            if x.dtype != tdt:
                raise TypeError(f"{name}: expected {tdt}, got {x.dtype}")
            if not x.is_contiguous():
                raise ValueError(f"{name}: must be contiguous")
            if x.is_cuda:
                self.on_device = True
                self.device = x.device.index
                self.obj = x
                self.ptr = x.data_ptr()
                self.shape = tuple(x.shape)
                return
            x = x.numpy()
        a = np.ascontiguousarray(x, dtype=dtype)
        self.obj = a
        self.ptr = a.ctypes.data
        self.shape = a.shape
        if ndim is not None and a.ndim != ndim:
            raise ValueError(f"{name}: expected {ndim}-d array, got shape {a.shape}")


def _options(args, ws_size=0, q=0, pair_ids=None, stream=None, max_outer_iter=0, inner_iter_cap=0, cache_bytes=0,
             device=None, kernel="rbf", coef0=0.0, degree=3, prob_folds=0):
    o = Options()
    lib().gmpsvm_options_init(ct.byref(o))
    dev_flags = {a.on_device for a in args if a is not None}
    if len(dev_flags) > 1:
        raise ValueError("mix of host and device buffers; pass all numpy or all CUDA tensors")
    on_dev = dev_flags.pop() if dev_flags else False
    o.inputs_on_device = 1 if on_dev else 0
    if on_dev:
        devs = {a.device for a in args if a is not None}
        if len(devs) > 1:
            raise ValueError("buffers on different devices")
        o.device = devs.pop()
        if stream is None:
            import torch
            stream = torch.cuda.current_stream(o.device).cuda_stream
    elif device is not None:
        o.device = int(device)
    o.stream = stream
    o.ws_size, o.q = int(ws_size), int(q)
    o.max_outer_iter, o.inner_iter_cap, o.cache_bytes = int(max_outer_iter), int(inner_iter_cap), int(cache_bytes)
    o.kernel, o.coef0, o.degree = KERNELS[kernel], float(coef0), int(degree)
    o.prob_folds = int(prob_folds)
    keep = None
    if pair_ids is not None:
        keep = (ct.c_int32 * len(pair_ids))(*[int(p) for p in pair_ids])
        o.pair_ids = ct.cast(keep, ct.POINTER(ct.c_int32))
        o.n_pair_ids = len(pair_ids)
    return o, keep


def _empty(shape, dtype, like: _Arg):
    if like.on_device:
        import torch
        tdt = {np.float32: torch.float32, np.float64: torch.float64}[dtype]
        return torch.empty(shape, dtype=tdt, device=f"cuda:{like.device}")
    return np.empty(shape, dtype=dtype)


def _data_ptr(x):
    return x.data_ptr() if _is_torch(x) else x.ctypes.data


# ------------------------------------------------------------------------------ public API
class Model:
    """Handle of a library-owned model (gmpsvm_model)."""

    def __init__(self, handle, status=OK):
        self._h = ct.c_void_p(handle)
        self.status = status
        k, d, nsv, npt = ct.c_int32(), ct.c_int32(), ct.c_int64(), ct.c_int32()
        _check(lib().gmpsvm_model_dims(self._h, ct.byref(k), ct.byref(d), ct.byref(nsv), ct.byref(npt)))
        self.k, self.d, self.n_sv, self.n_pairs_trained = k.value, d.value, nsv.value, npt.value

    def __del__(self):
        h = getattr(self, "_h", None)
        if h is not None and h.value and _lib is not None:
            _lib.gmpsvm_model_free(h)
            self._h = None

    @property
    def n_pairs(self):
        return self.k * (self.k - 1) // 2

    def predict_proba(self, Xt, out=None, **opts):
        """m x k FP64 probabilities (Eq 11, 12, 14/15)."""
        a = _Arg(Xt, np.float32, "Xtest", None)
        m = a.shape[0] if len(a.shape) else 0
        if len(a.shape) != 2 or (m and a.shape[1] != self.d):
            raise ValueError(f"Xtest must be m x {self.d}")
        if out is None:
            out = _empty((m, self.k), np.float64, a)
        o, keep = _options([a], **opts)
        _check(lib().gmpsvm_predict_proba_ex(self._h, a.ptr, m, _data_ptr(out), ct.byref(o)))
        return out

    def predict_proba_csr(self, csr, out=None, **opts):
        """predict_proba for CSR rows (gmpsvm_predict_proba_csr): a scipy.sparse CSR matrix, or
        (indptr int64, indices int32, values float32, (m, d)) as numpy arrays / CUDA tensors."""
        ip, ix, vv, (m, d) = _csr_args(csr)
        if d != self.d:
            raise ValueError(f"CSR rows must have {self.d} columns")
        if out is None:
            out = _empty((m, self.k), np.float64, ip)
        o, keep = _options([ip, ix, vv], **opts)
        _check(lib().gmpsvm_predict_proba_csr(self._h, ip.ptr, ix.ptr, vv.ptr, m, _data_ptr(out), ct.byref(o)))
        return out

    def decision_function(self, Xt, out=None, **opts):
        """m x P FP64 decision values (Eq 11, b included), pair order p = s*k - s(s+1)/2 + t-s-1."""
        a = _Arg(Xt, np.float32, "Xtest", 2)
        m = a.shape[0]
        if out is None:
            out = _empty((m, self.n_pairs), np.float64, a)
        o, keep = _options([a], **opts)
        _check(lib().gmpsvm_predict_decision(self._h, a.ptr, m, _data_ptr(out), ct.byref(o)))
        return out

    def pair(self, s, t, n_s=None, n_t=None, with_alpha=True):
        b, A, B = ct.c_double(), ct.c_double(), ct.c_double()
        alpha = None
        if with_alpha:
            if n_s is None or n_t is None:
                raise ValueError("pass n_s, n_t (class sizes) to receive alpha")
            alpha = np.empty(n_s + n_t)
        rc = _check(lib().gmpsvm_model_pair(self._h, s, t, ct.byref(b), ct.byref(A), ct.byref(B),
                                            alpha.ctypes.data if alpha is not None else None))
        return dict(b=b.value, A=A.value, B=B.value, alpha=alpha, status=rc)

    def pair_iters(self, s, t):
        """(outer iterations, inner SMO steps, kernel rows computed) of pair (s, t)'s training."""
        o, i, r = ct.c_int64(), ct.c_int64(), ct.c_int64()
        _check(lib().gmpsvm_model_pair_iters(self._h, int(s), int(t), ct.byref(o), ct.byref(i), ct.byref(r)))
        return o.value, i.value, r.value

    def trained_pairs(self):
        """Indices of the pairs this model holds (all of them unless trained with pair_ids)."""
        out = []
        for p, (s, t) in enumerate((s, t) for s in range(self.k) for t in range(s + 1, self.k)):
            if lib().gmpsvm_model_pair(self._h, s, t, None, None, None, None) >= 0:
                out.append(p)
        return out

    def sv_index(self):
        idx = np.empty(self.n_sv, dtype=np.int64)
        _check(lib().gmpsvm_model_sv_index(self._h, idx.ctypes.data))
        return idx

    def train_stats(self):
        s = TrainStats()
        _check(lib().gmpsvm_model_train_stats(self._h, ct.byref(s)))
        return _struct_dict(s)

    def serialize(self) -> np.ndarray:
        n = ct.c_size_t(0)
        _check(lib().gmpsvm_model_serialize(self._h, None, ct.byref(n)))
        buf = np.empty(n.value, dtype=np.uint8)
        _check(lib().gmpsvm_model_serialize(self._h, buf.ctypes.data, ct.byref(n)))
        return buf

    @staticmethod
    def deserialize(buf) -> "Model":
        b = np.ascontiguousarray(np.frombuffer(bytes(buf), dtype=np.uint8) if isinstance(buf, (bytes, bytearray))
                                 else buf, dtype=np.uint8)
        h = ct.c_void_p()
        _check(lib().gmpsvm_model_deserialize(b.ctypes.data, b.nbytes, ct.byref(h)))
        return Model(h.value)

    @staticmethod
    def merge(parts) -> "Model":
        arr = (ct.c_void_p * len(parts))(*[p._h.value for p in parts])
        h = ct.c_void_p()
        _check(lib().gmpsvm_model_merge(arr, len(parts), ct.byref(h)))
        return Model(h.value)


def train(X, y, k, C, gamma, eps, **opts) -> Model:
    """gmpsvm_train_ex: all k(k-1)/2 pairs (or opts['pair_ids']) of the RBF MP-SVM."""
    a = _Arg(X, np.float32, "X", 2)
    b = _Arg(y, np.int32, "y", 1)
    n, d = a.shape
    if b.shape[0] != n:
        raise ValueError("len(y) != len(X)")
    o, keep = _options([a, b], **opts)
    h = ct.c_void_p()
    rc = _check(lib().gmpsvm_train_ex(a.ptr, b.ptr, n, d, int(k), float(C), float(gamma), float(eps), ct.byref(o),
                                      ct.byref(h)))
    return Model(h.value, rc)


def _csr_args(csr):
    if isinstance(csr, tuple):
        ip, ix, vv, shape = csr
    else:  # scipy.sparse
        c = csr.tocsr()
        ip, ix, vv, shape = c.indptr.astype(np.int64), c.indices.astype(np.int32), c.data.astype(np.float32), c.shape
    return (_Arg(ip, np.int64, "indptr", 1), _Arg(ix, np.int32, "indices", 1), _Arg(vv, np.float32, "values", 1),
            (int(shape[0]), int(shape[1])))


def train_csr(csr, y, k, C, gamma, eps, **opts) -> Model:
    """gmpsvm_train_csr: CSR rows (the paper's sparse format) densified on the device, then train."""
    ip, ix, vv, (n, d) = _csr_args(csr)
    b = _Arg(y, np.int32, "y", 1)
    o, keep = _options([ip, ix, vv, b], **opts)
    h = ct.c_void_p()
    rc = _check(lib().gmpsvm_train_csr(ip.ptr, ix.ptr, vv.ptr, b.ptr, n, d, int(k), float(C), float(gamma), float(eps),
                                       ct.byref(o), ct.byref(h)))
    return Model(h.value, rc)


def model_from_alpha(X, y, k, C, gamma, alpha, b, A, B, status=None, **opts) -> Model:
    """gmpsvm_model_from_alpha: the complete model from every pair's (alpha, b, A, B) -- alpha
    concatenated over pairs in index order, each pair in pair-local order (Model.pair layout)."""
    a = _Arg(X, np.float32, "X", 2)
    yy = _Arg(y, np.int32, "y", 1)
    n, d = a.shape
    P = int(k) * (int(k) - 1) // 2
    al = np.ascontiguousarray(alpha, dtype=np.float64)
    bb, AA, BB = (np.ascontiguousarray(v, dtype=np.float64) for v in (b, A, B))
    if bb.size != P or AA.size != P or BB.size != P:
        raise ValueError("b, A, B need k(k-1)/2 entries")
    st = None if status is None else np.ascontiguousarray(status, dtype=np.int32)
    o, keep = _options([a, yy], **opts)
    h = ct.c_void_p()
    rc = _check(lib().gmpsvm_model_from_alpha(a.ptr, yy.ptr, n, d, int(k), float(C), float(gamma), al.ctypes.data,
                                              bb.ctypes.data, AA.ctypes.data, BB.ctypes.data,
                                              st.ctypes.data if st is not None else None, ct.byref(o), ct.byref(h)))
    return Model(h.value, rc)


def rbf_kernel(X, Y, gamma, out=None, **opts):
    """K1 alone: K[i, j] = exp(-gamma ||X_i - Y_j||^2), FP32 (norm expansion, clamped)."""
    a = _Arg(X, np.float32, "X", 2)
    b = _Arg(Y, np.float32, "Y", 2)
    if a.shape[1] != b.shape[1]:
        raise ValueError("feature dimensions differ")
    if out is None:
        out = _empty((a.shape[0], b.shape[0]), np.float32, a)
    o, keep = _options([a, b], **opts)
    _check(lib().gmpsvm_rbf_kernel(a.ptr, a.shape[0], b.ptr, b.shape[0], a.shape[1], float(gamma), _data_ptr(out),
                                   ct.byref(o)))
    return out


def couple(dec, k, A, B, out=None, **opts):
    """a11 + a12 alone: probabilities from decision values (m x P) and per-pair sigmoids."""
    a = _Arg(dec, np.float64, "dec", 2)
    aA = _Arg(A, np.float64, "A", 1)
    aB = _Arg(B, np.float64, "B", 1)
    if out is None:
        out = _empty((a.shape[0], int(k)), np.float64, a)
    o, keep = _options([a, aA, aB], **opts)
    _check(lib().gmpsvm_couple(a.ptr, a.shape[0], int(k), aA.ptr, aB.ptr, _data_ptr(out), ct.byref(o)))
    return out


class Shard:
    """NEXT-1: this rank's part of one pair's solver, the pair's instances sharded over `world`
    ranks (gmpsvm_shard_*; the collectives between the calls are the caller's, see
    dist.train_pair_sharded).  Host numpy buffers throughout."""

    def __init__(self, X, y, k, s, t, C, gamma, eps, rank=0, world=1, **opts):
        a = _Arg(X, np.float32, "X", 2)
        b = _Arg(y, np.int32, "y", 1)
        n, d = a.shape
        o, keep = _options([a, b], **opts)
        h = ct.c_void_p()
        _check(lib().gmpsvm_shard_create(a.ptr, b.ptr, n, d, int(k), int(s), int(t), float(C), float(gamma), float(eps),
                                         int(rank), int(world), ct.byref(o), ct.byref(h)))
        self.h = h.value
        self.cand_doubles = int(lib().gmpsvm_shard_cand_doubles(self.h))
        lo, hi, npp, wsz = ct.c_int64(), ct.c_int64(), ct.c_int64(), ct.c_int32()
        _check(lib().gmpsvm_shard_slice(self.h, ct.byref(lo), ct.byref(hi), ct.byref(npp), ct.byref(wsz)))
        self.lo, self.hi, self.n_p, self.ws_size = lo.value, hi.value, npp.value, wsz.value

    def __del__(self):
        if getattr(self, "h", None):
            lib().gmpsvm_shard_free(self.h)
            self.h = None

    def candidates(self):
        out = np.zeros(self.cand_doubles)
        _check(lib().gmpsvm_shard_candidates(self.h, out.ctypes.data))
        return out

    def select(self, all_cands, want_fws=False):
        """The merge; returns stop, or (stop, this rank's f of the new working set) with want_fws."""
        a = np.ascontiguousarray(all_cands, dtype=np.float64)
        stop = ct.c_int32()
        fw = np.zeros(self.ws_size) if want_fws else None
        _check(lib().gmpsvm_shard_select(self.h, a.ctypes.data, ct.byref(stop), fw.ctypes.data if want_fws else None))
        return (bool(stop.value), fw) if want_fws else bool(stop.value)

    def fws(self):
        out = np.zeros(self.ws_size)
        _check(lib().gmpsvm_shard_fws(self.h, out.ctypes.data))
        return out

    def step(self, fws_sum, want_cands=False):
        """Local SMO + f update; with want_cands the next iteration's candidate block."""
        a = np.ascontiguousarray(fws_sum, dtype=np.float64)
        c = np.zeros(self.cand_doubles) if want_cands else None
        _check(lib().gmpsvm_shard_step(self.h, a.ctypes.data, c.ctypes.data if want_cands else None))
        return c

    def f_slice(self):
        out = np.zeros(self.hi - self.lo)
        if out.size:
            _check(lib().gmpsvm_shard_f(self.h, out.ctypes.data))
        return out

    def finish(self, f_full):
        f = np.ascontiguousarray(f_full, dtype=np.float64)
        alpha = np.zeros(self.n_p)
        b, A, B = ct.c_double(), ct.c_double(), ct.c_double()
        st, outer, inner = ct.c_int32(), ct.c_int64(), ct.c_int64()
        rc = _check(lib().gmpsvm_shard_finish(self.h, f.ctypes.data, alpha.ctypes.data, ct.byref(b), ct.byref(A),
                                              ct.byref(B), ct.byref(st), ct.byref(outer), ct.byref(inner)))
        return dict(alpha=alpha, b=b.value, A=A.value, B=B.value, status=st.value, outer_iters=outer.value,
                    inner_iters=inner.value, rc=rc)


def shard_merge(all_cands, world, cand_doubles, need, need_u):
    """gmpsvm_shard_merge: the exact candidate merge of the sharded solver (host arithmetic)."""
    a = np.ascontiguousarray(all_cands, dtype=np.float64)
    picks = np.zeros(max(int(need), 1), dtype=np.int32)
    n, gap = ct.c_int32(), ct.c_double()
    _check(lib().gmpsvm_shard_merge(a.ctypes.data, int(world), int(cand_doubles), int(need), int(need_u),
                                    picks.ctypes.data, ct.byref(n), ct.byref(gap)))
    return picks[: n.value], gap.value


def launch_count() -> int:
    return int(lib().gmpsvm_launch_count())


def last_predict_stats():
    s = PredictStats()
    lib().gmpsvm_last_predict_stats(ct.byref(s))
    return _struct_dict(s)
