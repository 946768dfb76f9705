"""CPU FP64 oracle for the GMP-SVM hot path -- TEST INFRASTRUCTURE ONLY.

Only tests/, __graft_entry__.smoke() and bench.py (cpu_baseline / --impl reference)
may import this package.  The product path (paper_conf_icde_wenshcc19_b200) never
imports it, and it never imports the product path.  The arithmetic lives in
gmpsvm_oracle.cpp (plain C++17, FP64, std::thread); this file is ctypes marshalling.

Paper: /root/reference/PAPER.md ("Efficient Multi-Class Probabilistic SVMs on GPUs").
Readings of silent/garbled passages: SURVEY.md §8(c), repeated in DESIGN.md.
"""
from __future__ import annotations

import contextlib
import ctypes as ct
import os
import subprocess
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "gmpsvm_oracle.cpp")
_LIB = os.path.join(_HERE, "liboracle.so")
_lock = threading.Lock()
_lib = None

_f32p = np.ctypeslib.ndpointer(dtype=np.float32, flags="C_CONTIGUOUS")
_f64p = np.ctypeslib.ndpointer(dtype=np.float64, flags="C_CONTIGUOUS")
_i32p = np.ctypeslib.ndpointer(dtype=np.int32, flags="C_CONTIGUOUS")
_i64p = np.ctypeslib.ndpointer(dtype=np.int64, flags="C_CONTIGUOUS")


def build(force: bool = False) -> str:
    """Compile liboracle.so with g++ (-O3, no -ffast-math: IEEE FP64)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".{os.getpid()}.tmp"
        subprocess.check_call(["g++", "-O3", "-march=native", "-std=c++17", "-fPIC", "-shared",
                               "-o", tmp, _SRC, "-lpthread"])
        os.replace(tmp, _LIB)
    return _LIB


def _load():
    global _lib
    with _lock:
        if _lib is not None:
            return _lib
        lib = ct.CDLL(build())
        lib.oracle_rbf_matrix.argtypes = [_f32p, ct.c_int64, _f32p, ct.c_int64, ct.c_int, ct.c_double, _f64p, ct.c_int]
        lib.oracle_rbf_matrix.restype = None
        lib.oracle_smo.argtypes = [_f32p, _i32p, ct.c_int64, ct.c_int, ct.c_double, ct.c_double, ct.c_double,
                                   ct.c_int64, _f64p, _f64p, ct.POINTER(ct.c_int64), ct.c_void_p, ct.c_int64]
        lib.oracle_smo.restype = ct.c_int
        lib.oracle_exact_f.argtypes = [_f32p, _i32p, ct.c_int64, ct.c_int, ct.c_double, _f64p, _f64p, ct.c_int]
        lib.oracle_exact_f.restype = None
        lib.oracle_rho.argtypes = [_f64p, _f64p, _i32p, ct.c_int64, ct.c_double]
        lib.oracle_rho.restype = ct.c_double
        lib.oracle_sigmoid_fit.argtypes = [_f64p, _i32p, ct.c_int64, ct.POINTER(ct.c_double),
                                           ct.POINTER(ct.c_double), ct.POINTER(ct.c_int)]
        lib.oracle_sigmoid_fit.restype = ct.c_int
        lib.oracle_couple.argtypes = [_f64p, ct.c_int, _f64p]
        lib.oracle_couple.restype = ct.c_int
        lib.oracle_train.argtypes = [_f32p, _i32p, ct.c_int64, ct.c_int, ct.c_int, ct.c_double, ct.c_double,
                                     ct.c_double, ct.c_int, _f64p, _f64p, _f64p, _f64p, _f64p, _i64p, _i32p]
        lib.oracle_train.restype = ct.c_int
        lib.oracle_predict.argtypes = [_f32p, _i32p, ct.c_int64, ct.c_int, ct.c_int, ct.c_double, _f64p, _f64p,
                                       _f64p, _f64p, _f32p, ct.c_int64, ct.c_void_p, ct.c_void_p, ct.c_int]
        lib.oracle_predict.restype = ct.c_int
        lib.oracle_set_kernel.argtypes = [ct.c_int, ct.c_double, ct.c_int]
        lib.oracle_set_kernel.restype = ct.c_int
        _lib = lib
        return lib


KERNELS = {"rbf": 0, "linear": 1, "poly": 2, "sigmoid": 3}


@contextlib.contextmanager
def kernel(kind="rbf", coef0=0.0, degree=3):
    """Every oracle call inside uses this kernel (LibSVM definitions):
    rbf exp(-gamma |x-y|^2), linear x.y, poly (gamma x.y + coef0)^degree, sigmoid
    tanh(gamma x.y + coef0).  Process-wide; restored to rbf on exit."""
    if _load().oracle_set_kernel(KERNELS[kind], float(coef0), int(degree)) != 0:
        raise ValueError("bad kernel parameters")
    try:
        yield
    finally:
        _load().oracle_set_kernel(0, 0.0, 3)


def default_threads() -> int:
    return max(1, len(os.sched_getaffinity(0)))


def _f32(a):
    return np.ascontiguousarray(a, dtype=np.float32)


def _f64(a):
    return np.ascontiguousarray(a, dtype=np.float64)


def _i32(a):
    return np.ascontiguousarray(a, dtype=np.int32)


# ---------------------------------------------------------------------------------------------
def rbf_matrix(X, Y, gamma, nthreads=None):
    """K[i, j] = exp(-gamma ||X_i - Y_j||^2) in FP64, direct differences."""
    X, Y = _f32(X), _f32(Y)
    n, d = X.shape
    m = Y.shape[0]
    out = np.empty((n, m), dtype=np.float64)
    _load().oracle_rbf_matrix(X, n, Y, m, d, float(gamma), out, nthreads or default_threads())
    return out


def smo(X, y, C, gamma, eps, max_iter=0, trace=0):
    """Binary SMO, Algorithm 1 + WSS2 (Eq 3-10).  y in {+1,-1}.

    Returns dict(alpha, f, iters, status[, dual]).  status 0 = converged, 1 = cap reached.
    """
    X, y = _f32(X), _i32(y)
    n, d = X.shape
    alpha = np.zeros(n)
    f = np.zeros(n)
    it = ct.c_int64(0)
    tr = np.zeros(max(trace, 1))
    st = _load().oracle_smo(X, y, n, d, float(C), float(gamma), float(eps), int(max_iter), alpha, f,
                            ct.byref(it), tr.ctypes.data if trace else None, int(trace))
    out = dict(alpha=alpha, f=f, iters=int(it.value), status=int(st))
    if trace:
        out["dual"] = tr[: min(trace, it.value + 1)]
    return out


def exact_f(X, y, alpha, gamma, nthreads=None):
    """f_i = sum_j alpha_j y_j K(x_i, x_j) - y_i (Eq 3) recomputed from scratch in FP64."""
    X, y, alpha = _f32(X), _i32(y), _f64(alpha)
    n, d = X.shape
    f = np.empty(n)
    _load().oracle_exact_f(X, y, n, d, float(gamma), alpha, f, nthreads or default_threads())
    return f


def rho(alpha, f, y, C):
    """LibSVM bias rule in f terms (b = -rho); f must be exact for alpha."""
    return float(_load().oracle_rho(_f64(alpha), _f64(f), _i32(y), len(alpha), float(C)))


def sigmoid_fit(v, y):
    """(A, B, iters, status) minimising Eq 13 (L179-L185) by Newton + backtracking [15]."""
    A, B, it = ct.c_double(0), ct.c_double(0), ct.c_int(0)
    st = _load().oracle_sigmoid_fit(_f64(v), _i32(y), len(v), ct.byref(A), ct.byref(B), ct.byref(it))
    return A.value, B.value, it.value, st


def couple(r):
    """p solving Eq 14 via the bordered KKT system (Eq 15).  r is k x k, r[s, t] = r_st."""
    r = _f64(r)
    k = r.shape[0]
    p = np.empty(k)
    st = _load().oracle_couple(r, k, p)
    if st != 0:
        raise FloatingPointError("coupling system singular")
    return p


def pair_list(k):
    """[(s, t)] in pair-index order p = s*k - s(s+1)/2 + (t-s-1)."""
    return [(s, t) for s in range(k) for t in range(s + 1, k)]


def train(X, labels, k, C, gamma, eps, nthreads=None):
    """Algorithm 2 (L333-L361) on all k(k-1)/2 pairs, FP64.

    Returns dict with per-pair lists: alpha[p] (pair-local order: class s then t, original
    order within class), f[p] (exact Eq 3), b, A, B, iters, status arrays.
    """
    X, labels = _f32(X), _i32(labels)
    n, d = X.shape
    counts = np.bincount(labels, minlength=k)
    pairs = pair_list(k)
    sizes = np.array([counts[s] + counts[t] for s, t in pairs], dtype=np.int64)
    tot = int(sizes.sum())
    P = len(pairs)
    alpha = np.zeros(tot)
    f = np.zeros(tot)
    b, A, B = np.zeros(P), np.zeros(P), np.zeros(P)
    iters = np.zeros(P, dtype=np.int64)
    status = np.zeros(P, dtype=np.int32)
    rc = _load().oracle_train(X, labels, n, d, k, float(C), float(gamma), float(eps),
                              nthreads or default_threads(), alpha, f, b, A, B, iters, status)
    if rc != 0:
        raise ValueError("oracle_train: invalid labels")
    off = np.concatenate([[0], np.cumsum(sizes)])
    return dict(alpha=[alpha[off[p]:off[p + 1]] for p in range(P)], f=[f[off[p]:off[p + 1]] for p in range(P)],
                alpha_flat=alpha, b=b, A=A, B=B, iters=iters, status=status, pairs=pairs, k=k,
                gamma=float(gamma), C=float(C))


def fold_of(labels, k, folds):
    """Fold of each instance for cross-validated sigmoids (NEXT-2; R30): its rank
    within its class (original order) mod folds.  Returns (fold, rank, class counts)."""
    labels = np.asarray(labels)
    rank = np.zeros(len(labels), dtype=np.int64)
    cnt = np.zeros(k, dtype=np.int64)
    for i, c in enumerate(labels):
        rank[i] = cnt[c]
        cnt[c] += 1
    return rank % folds, rank, cnt


def train_cv(X, labels, k, C, gamma, eps, folds=5, nthreads=None):
    """LibSVM's probability training (ref [15]) with deterministic folds: for each fold, train
    (Alg 2) on the other folds and evaluate Eq 11 on the held-out rows; each pair's sigmoid
    (Eq 12-13) is fitted on its out-of-fold decision values; the final model is trained on all
    rows and carries those A, B.  Also returns the out-of-fold values v[p] (pair-local order)."""
    X, labels = _f32(X), _i32(labels)
    fold, rank, cnt = fold_of(labels, k, folds)
    pairs = pair_list(k)
    v = [np.full(cnt[s] + cnt[t], np.nan) for s, t in pairs]
    for f in range(folds):
        tr, ho = fold != f, fold == f
        mf = train(X[tr], labels[tr], k, C, gamma, eps, nthreads)
        dec, _ = predict(mf, X[tr], labels[tr], X[ho], nthreads)
        for h, i in enumerate(np.flatnonzero(ho)):
            c, r = labels[i], rank[i]
            for p, (s, t) in enumerate(pairs):
                if c == s:
                    v[p][r] = dec[h, p]
                elif c == t:
                    v[p][cnt[s] + r] = dec[h, p]
    A, B = np.zeros(len(pairs)), np.zeros(len(pairs))
    for p, (s, t) in enumerate(pairs):
        ypm = np.concatenate([np.ones(cnt[s], np.int32), -np.ones(cnt[t], np.int32)])
        A[p], B[p], _, _ = sigmoid_fit(v[p], ypm)
    model = train(X, labels, k, C, gamma, eps, nthreads)
    model["A"], model["B"], model["v_cv"] = A, B, v
    return model


def predict(model, X, labels, Xt, nthreads=None, want_dec=True):
    """(dec [m, P], prob [m, k]) by Eq 11, 12, 14/15 from an oracle-format model."""
    X, labels, Xt = _f32(X), _i32(labels), _f32(Xt)
    n, d = X.shape
    m = Xt.shape[0]
    k = model["k"]
    P = k * (k - 1) // 2
    alpha = np.concatenate(model["alpha"]) if "alpha_flat" not in model else model["alpha_flat"]
    dec = np.empty((m, P)) if want_dec else None
    prob = np.empty((m, k))
    rc = _load().oracle_predict(X, labels, n, d, k, float(model["gamma"]), _f64(alpha), _f64(model["b"]),
                                _f64(model["A"]), _f64(model["B"]), Xt, m,
                                dec.ctypes.data if want_dec else None, prob.ctypes.data, nthreads or default_threads())
    if rc != 0:
        raise FloatingPointError("oracle_predict: coupling failed")
    return dec, prob


def pair_members(labels, k, s, t):
    """Original indices of pair (s,t) in pair-local order and their +-1 labels."""
    labels = np.asarray(labels)
    ms = np.flatnonzero(labels == s)
    mt = np.flatnonzero(labels == t)
    idx = np.concatenate([ms, mt])
    y = np.concatenate([np.ones(len(ms), np.int32), -np.ones(len(mt), np.int32)])
    return idx, y
