"""Pins for the oracle's sigmoid fit, coupling and whole pipeline (CPU, -m "not gpu")."""
import json
import os

import numpy as np
import pytest
from scipy.optimize import minimize

import datagen
import oracle

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


# ----------------------------------------------------------------------------- sigmoid (Eq 12-13)
def _F(ab, v, t):
    # Eq 13 written as a minimisation of the negative log likelihood, P = 1/(1+exp(Av+B)).
    z = ab[0] * v + ab[1]
    logP = -np.logaddexp(0.0, z)       # log 1/(1+e^z)
    log1mP = z - np.logaddexp(0.0, z)  # log e^z/(1+e^z)
    return -(t * logP + (1 - t) * log1mP).sum()


def _targets(y):
    Np, Nm = (y > 0).sum(), (y < 0).sum()
    return np.where(y > 0, (Np + 1.0) / (Np + 2.0), 1.0 / (Nm + 2.0))


@pytest.mark.parametrize("seed", [0, 1, 2])
def test_sigmoid_fit_matches_bfgs_and_zero_gradient(seed):
    rng = np.random.default_rng(seed)
    n = 500
    y = np.where(rng.random(n) < 0.4, 1, -1).astype(np.int32)
    v = y * rng.gamma(2.0, 0.7, size=n) + rng.normal(0, 0.8, size=n)
    A, B, it, st = oracle.sigmoid_fit(v, y)
    assert st == 0
    t = _targets(y)
    res = minimize(_F, x0=np.array([0.0, 0.0]), args=(v, t), method="BFGS", options=dict(gtol=1e-11))
    np.testing.assert_allclose([A, B], res.x, atol=1e-6)
    # gradient of Eq 13 (L254-L255): sum v (t - P), sum (t - P) vanish at the optimum
    P = 1.0 / (1.0 + np.exp(A * v + B))
    assert abs((v * (t - P)).sum()) < 1e-5 and abs((t - P).sum()) < 1e-5


def test_sigmoid_constant_decision_values_closed_form():
    # v = 0 for all instances: only B matters, optimum P = mean(t) => B = log((1 - tbar)/tbar)
    y = np.array([1] * 30 + [-1] * 70, dtype=np.int32)
    v = np.zeros(100)
    A, B, _, st = oracle.sigmoid_fit(v, y)
    tbar = _targets(y).mean()
    assert A == 0.0
    np.testing.assert_allclose(B, np.log((1 - tbar) / tbar), atol=1e-9)


# ----------------------------------------------------------------------------- coupling (Eq 14-15)
def _rmat(k, rng, lo=0.05, hi=0.95):
    r = np.zeros((k, k))
    for s in range(k):
        for t in range(s + 1, k):
            r[s, t] = rng.uniform(lo, hi)
            r[t, s] = 1.0 - r[s, t]
    return r


def _Q(r):
    k = r.shape[0]
    Q = -r * r.T
    for s in range(k):
        Q[s, s] = sum(r[u, s] ** 2 for u in range(k) if u != s)
    return Q


def test_couple_k2_closed_form():
    for r12 in [0.01, 0.3, 0.5, 0.77, 0.999]:
        r = np.array([[0.0, r12], [1 - r12, 0.0]])
        np.testing.assert_allclose(oracle.couple(r), [r12, 1 - r12], atol=1e-14)


@pytest.mark.parametrize("k", [3, 5, 10, 26])
def test_couple_bradley_terry_consistent(k):
    rng = np.random.default_rng(k)
    p_star = rng.dirichlet(np.ones(k))
    r = p_star[:, None] / (p_star[:, None] + p_star[None, :])
    np.fill_diagonal(r, 0.0)
    np.testing.assert_allclose(oracle.couple(r), p_star, atol=1e-12)


@pytest.mark.parametrize("k", [3, 4, 10, 26])
def test_couple_eq15_inverse_and_direct_minimisation(k):
    rng = np.random.default_rng(100 + k)
    for _ in range(5):
        r = _rmat(k, rng)
        p = oracle.couple(r)
        assert abs(p.sum() - 1.0) < 1e-12 and np.all(p >= 0)
        Q = _Q(r)
        qe = np.linalg.solve(Q, np.ones(k))  # Eq 15: p = Q^-1 e / (e^T Q^-1 e)
        np.testing.assert_allclose(p, qe / qe.sum(), atol=1e-10)
        # Eq 14 objective as printed (double sum), minimised under sum p = 1
        def obj(q):
            return sum((r[t, s] * q[s] - r[s, t] * q[t]) ** 2 for s in range(k) for t in range(k) if t != s)
        res = minimize(obj, np.full(k, 1.0 / k), method="SLSQP",
                       constraints=[dict(type="eq", fun=lambda q: q.sum() - 1.0)],
                       options=dict(ftol=1e-15, maxiter=500))
        np.testing.assert_allclose(p, res.x, atol=2e-5)
        assert obj(p) <= obj(res.x) + 1e-12


def test_couple_example1_ordering():
    g = json.load(open(os.path.join(GOLDEN, "example1_coupling.json")))
    r = np.zeros((3, 3))
    r[0, 1], r[0, 2], r[1, 2] = g["r12"], g["r13"], g["r23"]
    r[1, 0], r[2, 0], r[2, 1] = 1 - g["r12"], 1 - g["r13"], 1 - g["r23"]
    p = oracle.couple(r)
    printed = np.array(g["printed_p"])
    # only the ordering of the printed result is reproducible
    assert list(np.argsort(-p)) == list(np.argsort(-printed))
    assert np.argmax(p) == 0


# ----------------------------------------------------------------------------- pipeline
def test_pipeline_in_sample_identity_and_sklearn():
    spec, X, y, Xt, yt = datagen.make_config("blobs")
    m = oracle.train(X, y, spec.k, spec.C, spec.gamma, 1e-10)
    assert np.all(m["status"] == 0)
    # Eq 11 on the training instances == f + y - rho from Eq 3 (two different code paths)
    dec, prob = oracle.predict(m, X, y, X)
    for p, (s, t) in enumerate(m["pairs"]):
        idx, ypm = oracle.pair_members(y, spec.k, s, t)
        v = m["f"][p] + ypm + m["b"][p]
        np.testing.assert_allclose(dec[idx, p], v, atol=1e-10)
    np.testing.assert_allclose(prob.sum(1), 1.0, atol=1e-12)
    assert np.all(prob >= 0)
    sk = pytest.importorskip("sklearn.svm")
    for p, (s, t) in enumerate(m["pairs"]):
        idx, ypm = oracle.pair_members(y, spec.k, s, t)
        clf = sk.SVC(C=spec.C, kernel="rbf", gamma=spec.gamma, tol=1e-10, shrinking=False).fit(
            X[idx].astype(np.float64), ypm)
        a_sk = np.zeros(len(idx))
        a_sk[clf.support_] = np.abs(clf.dual_coef_[0])
        np.testing.assert_allclose(m["alpha"][p], a_sk, atol=1e-6 * spec.C)
        sign = np.sign(clf.dual_coef_[0][0] * ypm[clf.support_[0]])
        np.testing.assert_allclose(sign * clf.intercept_[0], m["b"][p], atol=1e-6)
    # Table-4 pattern (L423-L436): errors of the probabilistic classifier are sane
    test_err = (prob_t := oracle.predict(m, X, y, Xt, want_dec=False)[1]).argmax(1) != yt
    assert test_err.mean() < 0.2


# ------------------------------------------------------------------------------------ NEXT-2
def test_cross_validated_sigmoids_oracle():
    """oracle.train_cv (LibSVM's F-fold probability training, deterministic folds R30): every
    pair's out-of-fold decision value of an instance equals Eq 11 evaluated independently (numpy,
    direct-difference RBF) with the model trained without that instance's fold; the sigmoid is
    the unique minimiser on those values (zero gradient); every value is filled exactly once."""
    import datagen

    spec, X, y, _, _ = datagen.make_config("blobs")
    folds = 3
    m = oracle.train_cv(X, y, spec.k, spec.C, spec.gamma, 1e-6, folds=folds)
    fold, rank, cnt = oracle.fold_of(y, spec.k, folds)
    pairs = oracle.pair_list(spec.k)
    assert all(np.isfinite(v).all() for v in m["v_cv"])
    rng = np.random.default_rng(3)
    for i in rng.choice(len(y), size=6, replace=False):
        f = fold[i]
        tr = fold != f
        mf = oracle.train(X[tr], y[tr], spec.k, spec.C, spec.gamma, 1e-6)
        Xtr, ytr = X[tr].astype(np.float64), y[tr]
        for p, (s, t) in enumerate(pairs):
            if y[i] not in (s, t):
                continue
            idx = np.concatenate([np.flatnonzero(ytr == s), np.flatnonzero(ytr == t)])
            ypm = np.where(ytr[idx] == s, 1.0, -1.0)
            Kx = np.exp(-spec.gamma * ((Xtr[idx] - X[i].astype(np.float64)) ** 2).sum(1))
            dec = (mf["alpha"][p] * ypm * Kx).sum() + mf["b"][p]
            j = rank[i] if y[i] == s else cnt[s] + rank[i]
            np.testing.assert_allclose(m["v_cv"][p][j], dec, rtol=1e-9, atol=1e-9)
    for p, (s, t) in enumerate(pairs):
        ypm = np.concatenate([np.ones(cnt[s]), -np.ones(cnt[t])])
        tgt = np.where(ypm > 0, (cnt[s] + 1) / (cnt[s] + 2), 1 / (cnt[t] + 2))
        z = m["A"][p] * m["v_cv"][p] + m["B"][p]
        P1 = 1 / (1 + np.exp(z))
        gA, gB = ((tgt - P1) * m["v_cv"][p]).sum(), (tgt - P1).sum()
        assert abs(gA) < 1e-4 and abs(gB) < 1e-4


# ----------------------------------------------------------------------------- predict (Eq 11, 12, 14-15)
@pytest.mark.parametrize("name,C,gamma", [("blobs", 1.0, 0.5), ("blobs", 100.0, 0.03), ("letter", 10.0, 0.5)])
def test_predict_pinned_by_independent_numpy(name, C, gamma):
    """oracle.predict re-derived independently: Eq 11 by a direct-difference numpy RBF, the pair
    sigmoid of Eq 12 with r_st = P(class s | pair) = 1/(1 + exp(A dec + B)) for s the +1 class,
    clamped to [1e-7, 1 - 1e-7] (reading R15) and r_ts = 1 - r_st (L208), then Eq 14-15 as the
    bordered linear system [Q e; e^T 0][p; mu] = [0; 1] solved by scipy.linalg.solve.  A swapped
    orientation (r_st <-> r_ts), a different clamp or a wrong Q entry fails here."""
    from scipy.linalg import solve

    n = None if name == "blobs" else 1300
    spec, X, y, Xt, yt = datagen.make_config(name, n_train=n, n_test=None if name == "blobs" else 60)
    m = oracle.train(X, y, spec.k, C, gamma, 1e-6)
    dec, prob = oracle.predict(m, X, y, Xt)
    k, pairs = spec.k, m["pairs"]
    X64, Xt64 = X.astype(np.float64), Xt.astype(np.float64)
    dec_np = np.zeros((len(Xt), len(pairs)))
    for p, (s, t) in enumerate(pairs):
        idx, ypm = oracle.pair_members(y, k, s, t)
        Kt = np.exp(-gamma * ((Xt64[:, None, :] - X64[idx][None, :, :]) ** 2).sum(-1))
        dec_np[:, p] = Kt @ (m["alpha"][p] * ypm) + m["b"][p]
    np.testing.assert_allclose(dec, dec_np, rtol=1e-10, atol=1e-10)
    clamped = 0
    for i in range(len(Xt)):
        r = np.zeros((k, k))
        for p, (s, t) in enumerate(pairs):
            rst = 1.0 / (1.0 + np.exp(m["A"][p] * dec_np[i, p] + m["B"][p]))
            clamped += int(rst < 1e-7 or rst > 1 - 1e-7)
            rst = min(max(rst, 1e-7), 1 - 1e-7)
            r[s, t], r[t, s] = rst, 1.0 - rst
        Q = np.zeros((k, k))
        for s in range(k):
            for t in range(k):
                Q[s, t] = sum(r[u, s] ** 2 for u in range(k) if u != s) if s == t else -r[t, s] * r[s, t]
        M = np.zeros((k + 1, k + 1))
        M[:k, :k], M[:k, k], M[k, :k] = Q, 1.0, 1.0
        rhs = np.zeros(k + 1)
        rhs[k] = 1.0
        p_np = solve(M, rhs)[:k]
        np.testing.assert_allclose(prob[i], p_np, atol=1e-12)
    if name == "blobs" and C == 1.0:
        # the argmax of p agrees with the pair votes' winner for confidently classified rows
        votes = np.zeros((len(Xt), k))
        for p, (s, t) in enumerate(pairs):
            votes[:, s] += dec_np[:, p] > 0
            votes[:, t] += dec_np[:, p] <= 0
        sure = np.sort(prob, 1)[:, -1] > 0.9
        assert np.all(prob.argmax(1)[sure] == votes.argmax(1)[sure])
