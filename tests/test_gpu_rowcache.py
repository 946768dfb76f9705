"""GPU parity of the ROW_CACHE regime (a2/a3 when the n x n kernel matrix does not fit the
cache budget: per outer iteration only the rows of the q new working-set
entries are computed, into a B-row buffer per pair; the B - q retained rows are reused).

The regime is forced on small problems with cache_bytes=1 so the oracle can check every
output; tolerances are the same as test_gpu_parity.py.
"""
import numpy as np
import pytest

import datagen
import oracle
from test_gpu_parity import EPS, _compare_models

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def gm():
    import __graft_entry__

    __graft_entry__.build()
    import paper_conf_icde_wenshcc19_b200 as m

    assert torch.cuda.is_available()
    return m


def _check(gm, name, n_train, n_test, audit=True, **opts):
    spec, X, y, Xt, yt = datagen.make_config(name, n_train=n_train, n_test=n_test)
    ref = oracle.train(X, y, spec.k, spec.C, spec.gamma, EPS)
    model = gm.train(X, y, spec.k, spec.C, spec.gamma, EPS, cache_bytes=1, **opts)
    st = model.train_stats()
    assert st["cache_regime"] == 1
    assert st["krow_launches"] >= 1
    _compare_models(model, ref, X, y, spec.C, audit=audit)
    _, prob_o = oracle.predict(ref, X, y, Xt, want_dec=False)
    prob = model.predict_proba(Xt)
    assert np.abs(prob - prob_o).max() <= 1e-4
    top = np.sort(prob_o, 1)
    sure = top[:, -1] - top[:, -2] >= 2e-4
    assert np.all(prob.argmax(1)[sure] == prob_o.argmax(1)[sure])
    return model, st


@pytest.mark.parametrize("ws,q", [(64, 32), (128, 64), (224, 112), (64, 16), (1024, 512)])
def test_row_cache_blobs_vs_oracle(gm, ws, q):
    # n_p = 400: B < n_p exercises slot reuse over many outer iterations; B = 1024 >= n_p
    # computes every row once (ws_keep = n_p afterwards)
    model, st = _check(gm, "blobs", None, None, ws_size=ws, q=q)
    counts = np.bincount(datagen.make_config("blobs")[2], minlength=3)
    n_p = [counts[s] + counts[t] for s, t in oracle.pair_list(3)]
    if ws >= max(n_p):
        assert st["kernel_values"] == sum(x * x for x in n_p)
    else:
        assert st["outer_iters_max"] > 1
        # each outer iteration computes at most B rows of n_p values per pair (first: B, then <= q)
        assert st["kernel_values"] <= sum(x * (ws + q * (st["outer_iters_max"] - 1)) for x in n_p)


def test_row_cache_covtype_shaped_subset(gm):
    # covtype is the config whose kernel matrix does not fit at full size (581k^2 x 4 B)
    _check(gm, "covtype", 3000, 400, audit=False, ws_size=128)


def test_row_cache_mnist_shaped_subset(gm):
    _check(gm, "mnist", 2000, 300, audit=False)


def test_row_cache_letter_shaped_subset(gm):
    # 325 pairs with ragged n_p around B: mixes whole-pair and multi-iteration pairs
    _check(gm, "letter", 3000, 300, audit=False, ws_size=128)


def test_row_cache_matches_full_k_model(gm):
    # same seeded input, both regimes: same classifier up to the shared tolerances
    spec, X, y, Xt, yt = datagen.make_config("mnist", n_train=1500, n_test=200)
    m_full = gm.train(X, y, spec.k, spec.C, spec.gamma, EPS)
    m_rc = gm.train(X, y, spec.k, spec.C, spec.gamma, EPS, cache_bytes=1)
    assert m_full.train_stats()["cache_regime"] == 0 and m_rc.train_stats()["cache_regime"] == 1
    counts = np.bincount(y, minlength=spec.k)
    for s, t in oracle.pair_list(spec.k):
        a1 = m_full.pair(s, t, int(counts[s]), int(counts[t]))["alpha"]
        a2 = m_rc.pair(s, t, int(counts[s]), int(counts[t]))["alpha"]
        assert np.abs(a1 - a2).max() <= 2e-3 * spec.C
    assert np.abs(m_full.predict_proba(Xt) - m_rc.predict_proba(Xt)).max() <= 2e-4


def test_row_cache_device_inputs_deterministic(gm):
    spec, X, y, Xt, yt = datagen.make_config("blobs")
    m1 = gm.train(X, y, spec.k, spec.C, spec.gamma, EPS, cache_bytes=1)
    m2 = gm.train(torch.from_numpy(X).cuda(), torch.from_numpy(y).cuda(), spec.k, spec.C, spec.gamma, EPS,
                  cache_bytes=1)
    np.testing.assert_array_equal(m1.predict_proba(Xt), m2.predict_proba(torch.from_numpy(Xt).cuda()).cpu().numpy())
