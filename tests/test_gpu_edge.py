"""Edge cases of the CUDA path through the C ABI: degenerate sizes, duplicates (eta = 0),
every alpha at a bound, k = 2, invalid inputs, iteration caps, partial (multi-GPU style)
training + merge, serialization round trips.  Reference: the FP64 oracle."""
import numpy as np
import pytest

import datagen
import oracle

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu
EPS = 1e-5


@pytest.fixture(scope="module")
def gm():
    import __graft_entry__

    __graft_entry__.build()
    import paper_conf_icde_wenshcc19_b200 as m

    return m


def _pairs_close(model, ref, y, C, tol_a=1e-3, tol_b=1e-3):
    for p, (s, t) in enumerate(ref["pairs"]):
        info = model.pair(s, t, int((y == s).sum()), int((y == t).sum()))
        assert np.abs(info["alpha"] - ref["alpha"][p]).max() <= tol_a * C
        assert abs(info["b"] - ref["b"][p]) <= tol_b * max(1.0, abs(ref["b"][p]))


def test_two_points_closed_form(gm):
    X = np.array([[0.0, 0.0], [0.5, 1.0]], np.float32)
    y = np.array([0, 1], np.int32)
    for C in (0.5, 10.0):
        m = gm.train(X, y, 2, C, 0.7, 1e-8)
        info = m.pair(0, 1, 1, 1)
        a = min(C, 1.0 / (1.0 - np.exp(-0.7 * 1.25)))
        np.testing.assert_allclose(info["alpha"], [a, a], rtol=1e-5)
        assert abs(info["b"]) < 1e-6


def test_binary_k2_probabilities(gm):
    spec, X, y, Xt, yt = datagen.make_config("blobs")
    keep = y < 2
    X2, y2 = X[keep], y[keep]
    ref = oracle.train(X2, y2, 2, spec.C, spec.gamma, EPS)
    m = gm.train(X2, y2, 2, spec.C, spec.gamma, EPS)
    _pairs_close(m, ref, y2, spec.C)
    _, p_o = oracle.predict(ref, X2, y2, Xt, want_dec=False)
    p = m.predict_proba(Xt)
    assert np.abs(p - p_o).max() <= 1e-4
    dec = m.decision_function(Xt)[:, 0]
    r = 1.0 / (1.0 + np.exp(dec * m.pair(0, 1, with_alpha=False)["A"] + m.pair(0, 1, with_alpha=False)["B"]))
    np.testing.assert_allclose(p[:, 0], np.clip(r, 1e-7, 1 - 1e-7), atol=1e-12)  # k = 2: p = (r12, r21)


@pytest.mark.parametrize("n", [3, 129, 255, 257, 385])
def test_ragged_sizes(gm, n):
    rng = np.random.default_rng(n)
    X = rng.normal(0, 1, size=(n, 5)).astype(np.float32)
    y = (np.arange(n) % 3).astype(np.int32)
    ref = oracle.train(X, y, 3, 1.0, 0.5, EPS)
    m = gm.train(X, y, 3, 1.0, 0.5, EPS, ws_size=64)
    _pairs_close(m, ref, y, 1.0)
    Xt = rng.normal(0, 1, size=(n + 3, 5)).astype(np.float32)
    _, p_o = oracle.predict(ref, X, y, Xt, want_dec=False)
    assert np.abs(m.predict_proba(Xt) - p_o).max() <= 1e-4


def test_d_equals_one(gm):
    rng = np.random.default_rng(1)
    X = rng.normal(0, 1, size=(300, 1)).astype(np.float32)
    y = (X[:, 0] > 0).astype(np.int32) + (X[:, 0] > 1).astype(np.int32)
    ref = oracle.train(X, y, 3, 1.0, 1.0, EPS)
    m = gm.train(X, y, 3, 1.0, 1.0, EPS)
    _pairs_close(m, ref, y, 1.0)


def test_exact_duplicates_eta_zero(gm):
    # duplicated rows make K singular (eta = 0 for a duplicate pair, reading R3); alpha is then
    # unique only as sums over duplicate groups, probabilities are unique
    spec, X, y, Xt, yt = datagen.make_config("blobs")
    X = np.concatenate([X, X[:40]]).astype(np.float32)
    y = np.concatenate([y, y[:40]]).astype(np.int32)
    ref = oracle.train(X, y, 3, spec.C, spec.gamma, EPS)
    m = gm.train(X, y, 3, spec.C, spec.gamma, EPS)
    assert m.status == 0
    _, p_o = oracle.predict(ref, X, y, Xt, want_dec=False)
    assert np.abs(m.predict_proba(Xt) - p_o).max() <= 1e-4
    for p, (s, t) in enumerate(ref["pairs"]):
        info = m.pair(s, t, int((y == s).sum()), int((y == t).sum()))
        a = info["alpha"]
        assert np.all(a >= 0) and np.all(a <= spec.C)
        assert abs(info["b"] - ref["b"][p]) <= 1e-3 * max(1, abs(ref["b"][p]))


def test_all_alpha_at_bound_midpoint_bias(gm):
    # tiny C: every SV at the upper bound, no free SV -> b from the midpoint rule (reading R7/#28)
    spec, X, y, Xt, yt = datagen.make_config("blobs")
    C = 1e-3
    ref = oracle.train(X, y, 3, C, spec.gamma, EPS)
    m = gm.train(X, y, 3, C, spec.gamma, EPS)
    for p, (s, t) in enumerate(ref["pairs"]):
        a = ref["alpha"][p]
        assert not np.any((a > 0) & (a < C))  # the oracle agrees there is no free SV
    _pairs_close(m, ref, y, C)


def test_predict_empty_and_invalid_inputs(gm):
    spec, X, y, Xt, yt = datagen.make_config("blobs")
    m = gm.train(X, y, 3, spec.C, spec.gamma, 1e-3)
    assert m.predict_proba(np.zeros((0, 8), np.float32)).shape == (0, 3)
    bad = Xt.copy()
    bad[3, 2] = np.nan
    with pytest.raises(gm.GmpsvmError) as e:
        m.predict_proba(bad)
    assert e.value.code == gm.EINVAL
    for lab in (np.where(y == 2, 3, y), np.where(y == 2, -1, y), np.where(y == 2, 1, y)):
        with pytest.raises(gm.GmpsvmError) as e:
            gm.train(X, lab.astype(np.int32), 3, 1.0, 0.5, 1e-3)
        assert e.value.code == gm.EINVAL
    Xn = X.copy()
    Xn[5, 0] = np.inf
    with pytest.raises(gm.GmpsvmError) as e:
        gm.train(Xn, y, 3, 1.0, 0.5, 1e-3)
    assert e.value.code == gm.EINVAL


def test_outer_iteration_cap_warns(gm):
    spec, X, y, Xt, yt = datagen.make_config("blobs")
    m = gm.train(X, y, 3, spec.C, spec.gamma, 1e-8, ws_size=16, max_outer_iter=2)
    assert m.status == gm.WARN_MAXITER
    assert m.predict_proba(Xt).shape == (200, 3)


def test_partial_training_merge_and_serialization_bitwise(gm):
    # multi-GPU plumbing on one GPU: shards of pairs trained separately, merged == full model
    spec, X, y, Xt, yt = datagen.make_config("letter", n_train=2000, n_test=100)
    full = gm.train(X, y, spec.k, spec.C, spec.gamma, 1e-3, ws_size=128)
    from paper_conf_icde_wenshcc19_b200 import dist as gdist

    shards = gdist.plan_pairs(np.bincount(y, minlength=spec.k), 3)
    parts = [gm.train(X, y, spec.k, spec.C, spec.gamma, 1e-3, ws_size=128, pair_ids=sh) for sh in shards]
    with pytest.raises(gm.GmpsvmError):
        parts[0].predict_proba(Xt)  # a partial model cannot predict
    merged = gm.Model.merge([gm.Model.deserialize(p.serialize()) for p in parts])
    assert merged.n_sv == full.n_sv and merged.n_pairs_trained == full.n_pairs
    np.testing.assert_array_equal(merged.sv_index(), full.sv_index())
    p_full = full.predict_proba(Xt)
    np.testing.assert_array_equal(merged.predict_proba(Xt), p_full)
    rt = gm.Model.deserialize(full.serialize())
    np.testing.assert_array_equal(rt.predict_proba(Xt), p_full)
    counts = np.bincount(y, minlength=spec.k)
    for s, t in [(0, 1), (4, 17), (24, 25)]:
        a1 = full.pair(s, t, counts[s], counts[t])
        a2 = merged.pair(s, t, counts[s], counts[t])
        np.testing.assert_array_equal(a1["alpha"], a2["alpha"])
        assert a1["b"] == a2["b"] and a1["A"] == a2["A"]


def test_model_from_alpha_and_sharded_gather_bitwise(gm):
    """The multi-GPU gather path (dist.gather_solutions -> gmpsvm_model_from_alpha): shards of
    pairs trained separately, their disjoint per-pair solutions summed (gloo, world size 1 here;
    NCCL across ranks), the complete model rebuilt from X -- predicts bitwise like the full model;
    a vector that misses a pair or an alpha outside [0, C] is rejected."""
    import torch.distributed as dist

    from paper_conf_icde_wenshcc19_b200 import dist as gdist

    spec, X, y, Xt, yt = datagen.make_config("letter", n_train=2000, n_test=100)
    full = gm.train(X, y, spec.k, spec.C, spec.gamma, 1e-3, ws_size=128)
    counts = np.bincount(y, minlength=spec.k)
    shards = gdist.plan_pairs(counts, 3)
    parts = [gm.train(X, y, spec.k, spec.C, spec.gamma, 1e-3, ws_size=128, pair_ids=sh) for sh in shards]
    v = sum(gdist.pack_solutions(p, counts) for p in parts)
    pairs, off = gdist.pair_layout(counts)
    P, tot = len(pairs), int(off[-1])
    assert np.all(v[tot + 4 * P:] == 1.0)
    m = gm.model_from_alpha(X, y, spec.k, spec.C, spec.gamma, v[:tot], v[tot:tot + P], v[tot + P:tot + 2 * P],
                            v[tot + 2 * P:tot + 3 * P])
    assert m.n_sv == full.n_sv
    np.testing.assert_array_equal(m.sv_index(), full.sv_index())
    np.testing.assert_array_equal(m.predict_proba(Xt), full.predict_proba(Xt))
    np.testing.assert_array_equal(m.decision_function(Xt), full.decision_function(Xt))
    bad = v[:tot].copy()
    bad[3] = spec.C * 2
    with pytest.raises(gm.GmpsvmError):
        gm.model_from_alpha(X, y, spec.k, spec.C, spec.gamma, bad, v[tot:tot + P], v[tot + P:tot + 2 * P],
                            v[tot + 2 * P:tot + 3 * P])
    # the dist driver end to end on a single-process gloo group
    import os
    os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
    os.environ.setdefault("MASTER_PORT", "29611")
    dist.init_process_group("gloo", rank=0, world_size=1)
    try:
        model, prob = gdist.train_predict(X, y, Xt, spec.k, spec.C, spec.gamma, 1e-3, ws_size=128)
        np.testing.assert_array_equal(np.asarray(prob), full.predict_proba(Xt))
        # the rebuilt model keeps a non-Gaussian kernel (L76-L78)
        kw = dict(ws_size=128, kernel="poly", coef0=1.0, degree=2)
        fp = gm.train(X, y, spec.k, 1.0, 0.3, 1e-3, **kw)
        _, pp = gdist.train_predict(X, y, Xt, spec.k, 1.0, 0.3, 1e-3, **kw)
        np.testing.assert_array_equal(np.asarray(pp), fp.predict_proba(Xt))
    finally:
        dist.destroy_process_group()


def test_sv_index_matches_alpha(gm):
    spec, X, y, Xt, yt = datagen.make_config("blobs")
    m = gm.train(X, y, 3, spec.C, spec.gamma, 1e-3)
    sv = set(m.sv_index().tolist())
    expect = set()
    for s, t in oracle.pair_list(3):
        idx, _ = oracle.pair_members(y, 3, s, t)
        a = m.pair(s, t, int((y == s).sum()), int((y == t).sum()))["alpha"]
        expect |= set(idx[a > 0].tolist())
    assert sv == expect


def test_csr_input_matches_dense_bitwise(gm):
    """CSR rows (NEXT-3: the paper's sparse format; MNIST-shaped data is ~68 % zeros) are densified
    on the device and take the dense path: the same model and probabilities, bitwise, from host
    scipy CSR and from CUDA tensors; a column index outside [0, d) is rejected."""
    sp = pytest.importorskip("scipy.sparse")
    spec, X, y, Xt, yt = datagen.make_config("mnist", n_train=1500, n_test=150)
    dense = gm.train(X, y, spec.k, spec.C, spec.gamma, 1e-3)
    p_dense = dense.predict_proba(Xt)
    A, At = sp.csr_matrix(X), sp.csr_matrix(Xt)
    assert A.nnz < 0.5 * X.size
    m = gm.train_csr(A, y, spec.k, spec.C, spec.gamma, 1e-3)
    np.testing.assert_array_equal(m.sv_index(), dense.sv_index())
    np.testing.assert_array_equal(m.predict_proba_csr(At), p_dense)
    np.testing.assert_array_equal(m.predict_proba(Xt), p_dense)
    dev = torch.device("cuda:0")
    tup = (torch.from_numpy(A.indptr.astype(np.int64)).to(dev), torch.from_numpy(A.indices.astype(np.int32)).to(dev),
           torch.from_numpy(A.data.astype(np.float32)).to(dev), A.shape)
    md = gm.train_csr(tup, torch.from_numpy(y).to(dev), spec.k, spec.C, spec.gamma, 1e-3)
    tupt = (torch.from_numpy(At.indptr.astype(np.int64)).to(dev), torch.from_numpy(At.indices.astype(np.int32)).to(dev),
            torch.from_numpy(At.data.astype(np.float32)).to(dev), At.shape)
    np.testing.assert_array_equal(md.predict_proba_csr(tupt).cpu().numpy(), p_dense)
    bad = A.copy()
    bad.indices = bad.indices.copy()
    bad.indices[0] = spec.d + 5
    with pytest.raises(gm.GmpsvmError):
        gm.train_csr((bad.indptr.astype(np.int64), bad.indices.astype(np.int32), bad.data.astype(np.float32), bad.shape),
                     y, spec.k, spec.C, spec.gamma, 1e-3)
