"""Pins for the oracle's kernel values and SMO (runs on CPU, -m "not gpu").

Each pin is something other than the oracle itself: a library routine (scipy cdist),
a closed form, brute-force enumeration of the QP's active sets, a third-party solver
(scikit-learn's LibSVM), or an invariant the paper's equations fix.
"""
import itertools

import numpy as np
import pytest
from scipy.spatial.distance import cdist

import datagen
import oracle


def _rbf_ref(X, Y, gamma):
    # library routine (scipy) for ||x - y||^2, then exp: PAPER.md L75
    return np.exp(-gamma * cdist(X.astype(np.float64), Y.astype(np.float64), "sqeuclidean"))


def test_rbf_matches_cdist_and_diagonal():
    rng = np.random.default_rng(3)
    X = rng.normal(size=(37, 11)).astype(np.float32)
    Y = rng.normal(size=(23, 11)).astype(np.float32)
    K = oracle.rbf_matrix(X, Y, 0.3)
    np.testing.assert_allclose(K, _rbf_ref(X, Y, 0.3), rtol=1e-13, atol=0)
    Kxx = oracle.rbf_matrix(X, X, 0.3)
    assert np.all(np.diag(Kxx) == 1.0)
    np.testing.assert_array_equal(Kxx, Kxx.T)


# --------------------------------------------------------------------------------------------
def _brute_force_qp(K, y, C):
    """Exact optimum of Eq 2 by enumerating (alpha=0 / alpha=C / free) for every variable and
    solving the KKT system of each status pattern.  Returns (alpha, b_interval)."""
    n = len(y)
    Q = (y[:, None] * y[None, :]) * K
    best = None
    for st in itertools.product((0, 1, 2), repeat=n):
        st = np.array(st)
        F = np.flatnonzero(st == 2)
        Cs = np.flatnonzero(st == 1)
        a = np.zeros(n)
        a[Cs] = C
        if len(F):
            m = len(F)
            M = np.zeros((m + 1, m + 1))
            M[:m, :m] = Q[np.ix_(F, F)]
            M[:m, m] = y[F]
            M[m, :m] = y[F]
            rhs = np.concatenate([1.0 - Q[np.ix_(F, Cs)] @ a[Cs], [-(y[Cs] * C).sum()]])
            try:
                sol = np.linalg.solve(M, rhs)
            except np.linalg.LinAlgError:
                continue
            a[F] = sol[:m]
            b = sol[m]
            if np.any(a[F] <= 1e-12) or np.any(a[F] >= C - 1e-12):
                continue
            g = Q @ a + y * b - 1.0  # = y_i v_i - 1
            ok = np.all(g[st == 0] >= -1e-9) and np.all(g[st == 1] <= 1e-9)
            if not ok:
                continue
            lo = hi = b
        else:
            if abs((y * a).sum()) > 1e-12:
                continue
            g0 = Q @ a - 1.0  # need g0_i + y_i b >= 0 (alpha=0), <= 0 (alpha=C)
            lo, hi = -np.inf, np.inf
            for i in range(n):
                # alpha=0: y_i b >= -g0_i ; alpha=C: y_i b <= -g0_i
                bound = -g0[i] * y[i]
                if (st[i] == 0) == (y[i] > 0):
                    lo = max(lo, bound)
                else:
                    hi = min(hi, bound)
            if lo > hi + 1e-9:
                continue
        W = a.sum() - 0.5 * a @ Q @ a
        if best is None or W > best[0] + 1e-12:
            best = (W, a.copy(), (lo, hi))
    return best[1], best[2]


@pytest.mark.parametrize("seed,C", [(0, 0.5), (1, 1.0), (2, 5.0), (3, 1.0), (4, 100.0)])
def test_smo_matches_brute_force_qp(seed, C):
    rng = np.random.default_rng(seed)
    n = 8
    X = rng.normal(size=(n, 2)).astype(np.float32)
    y = np.where(rng.random(n) < 0.5, 1, -1).astype(np.int32)
    y[0], y[1] = 1, -1
    gamma = 0.7
    K = _rbf_ref(X, X, gamma)
    a_bf, (blo, bhi) = _brute_force_qp(K, y.astype(np.float64), C)
    r = oracle.smo(X, y, C, gamma, 1e-12)
    assert r["status"] == 0
    np.testing.assert_allclose(r["alpha"], a_bf, atol=1e-7 * max(1.0, C))
    f = oracle.exact_f(X, y, r["alpha"], gamma)
    b = -oracle.rho(r["alpha"], f, y, C)
    assert blo - 1e-7 <= b <= bhi + 1e-7


@pytest.mark.parametrize("C", [0.5, 10.0])
def test_smo_two_point_closed_form(C):
    # n=2, y=(+1,-1): alpha_1 = alpha_2 = min(C, 1/(1-K12)), b = 0 (SURVEY §8(c) pins, A.7)
    X = np.array([[0.0, 0.0], [0.5, 1.0]], dtype=np.float32)
    gamma = 0.7
    y = np.array([1, -1], dtype=np.int32)
    r = oracle.smo(X, y, C, gamma, 1e-12)
    K12 = np.exp(-gamma * 1.25)
    a = min(C, 1.0 / (1.0 - K12))
    np.testing.assert_allclose(r["alpha"], [a, a], rtol=1e-12)
    f = oracle.exact_f(X, y, r["alpha"], gamma)
    assert abs(oracle.rho(r["alpha"], f, y, C)) < 1e-12
    if C == 10.0:
        np.testing.assert_allclose(a, 1.714860, atol=1e-6)  # value quoted in SURVEY Appendix A.7


def _pair(name, s, t, n=None):
    spec, X, y, _, _ = datagen.make_config(name, n_train=n)
    idx, ypm = oracle.pair_members(y, spec.k, s, t)
    return spec, X[idx], ypm


@pytest.mark.parametrize("eps", [1e-3, 1e-5])
def test_smo_kkt_invariants_and_dual_monotone(eps):
    spec, X, y = _pair("blobs", 0, 1)
    r = oracle.smo(X, y, spec.C, spec.gamma, eps, trace=100000)
    assert r["status"] == 0
    a = r["alpha"]
    C = spec.C
    assert np.all(a >= 0) and np.all(a <= C)
    assert abs((y * a).sum()) <= 1e-10 * C * len(a)
    f = oracle.exact_f(X, y, a, spec.gamma)
    np.testing.assert_allclose(r["f"], f, atol=1e-9)  # maintained f (Eq 8) == Eq 3
    iu = ((y > 0) & (a < C)) | ((y < 0) & (a > 0))
    il = ((y > 0) & (a > 0)) | ((y < 0) & (a < C))
    gap = f[il].max() - f[iu].min()
    assert gap < eps + 1e-9
    dual = r["dual"]
    assert np.all(np.diff(dual) >= -1e-12 * np.abs(dual[1:]).max())
    assert dual[-1] > 0


def test_smo_matches_sklearn_libsvm():
    sk = pytest.importorskip("sklearn.svm")
    for s, t in [(0, 1), (0, 2), (1, 2)]:
        spec, X, y = _pair("blobs", s, t)
        clf = sk.SVC(C=spec.C, kernel="rbf", gamma=spec.gamma, tol=1e-10, shrinking=False, cache_size=200)
        clf.fit(X.astype(np.float64), y)
        r = oracle.smo(X, y, spec.C, spec.gamma, 1e-10)
        a = r["alpha"]
        a_sk = np.zeros(len(y))
        a_sk[clf.support_] = np.abs(clf.dual_coef_[0])
        np.testing.assert_allclose(a, a_sk, atol=1e-6 * spec.C)
        assert set(np.flatnonzero(a > 1e-8 * spec.C)) == set(clf.support_[np.abs(clf.dual_coef_[0]) > 1e-8 * spec.C])
        # orientation: sklearn's positive class may be ours (+1 = class s) or the other one
        sign = np.sign(clf.dual_coef_[0][0] * y[clf.support_[0]])
        f = oracle.exact_f(X, y, a, spec.gamma)
        b = -oracle.rho(a, f, y, spec.C)
        np.testing.assert_allclose(sign * clf.intercept_[0], b, atol=1e-6)


# ------------------------------------------------------------------------------------ NEXT-4
@pytest.mark.parametrize("kind,gamma,coef0,degree", [("linear", 1.0, 0.0, 3), ("poly", 0.5, 1.0, 3),
                                                     ("poly", 0.3, 0.5, 2), ("sigmoid", 0.05, -0.5, 3)])
def test_other_kernels_match_closed_forms_and_sklearn(kind, gamma, coef0, degree):
    """The paper's other kernels (L76-L78, LibSVM definitions): the kernel matrix equals the
    closed form computed with numpy, and the SMO fixed point (alpha, SV set, intercept) equals
    scikit-learn's LibSVM with the same kernel at tight tolerance."""
    sk = pytest.importorskip("sklearn.svm")
    spec, X, y = _pair("blobs", 0, 1)
    X64 = X.astype(np.float64)
    dot = X64 @ X64.T
    closed = {"linear": dot, "poly": (gamma * dot + coef0) ** degree, "sigmoid": np.tanh(gamma * dot + coef0)}[kind]
    C = 0.5 if kind == "sigmoid" else spec.C
    with oracle.kernel(kind, coef0, degree):
        K = oracle.rbf_matrix(X, X, gamma)
        np.testing.assert_allclose(K, closed, rtol=1e-12, atol=1e-12)
        r = oracle.smo(X, y, C, gamma, 1e-10)
        a = r["alpha"]
        f = oracle.exact_f(X, y, a, gamma)
        b = -oracle.rho(a, f, y, C)
    clf = sk.SVC(C=C, kernel=kind, gamma=gamma, coef0=coef0, degree=degree, tol=1e-10, shrinking=False,
                 cache_size=200)
    clf.fit(X64, y)
    a_sk = np.zeros(len(y))
    a_sk[clf.support_] = np.abs(clf.dual_coef_[0])
    np.testing.assert_allclose(a, a_sk, atol=1e-5 * C)
    sign = np.sign(clf.dual_coef_[0][0] * y[clf.support_[0]])
    np.testing.assert_allclose(sign * clf.intercept_[0], b, atol=1e-5)
    # and the default is restored
    np.testing.assert_allclose(np.diag(oracle.rbf_matrix(X[:5], X[:5], gamma)), 1.0)
