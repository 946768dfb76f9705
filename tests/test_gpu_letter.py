"""Full-size parity of BASELINE.json configs[1] -- letter-shaped 20,000 x 16, 26 classes (325 binary
SVMs, more than the solver graph's concurrent branches, so several pairs share a branch), C = 10,
gamma = 0.5 -- in the default launch configuration, against tests/golden/letter_eps1e-05.npz
(oracle only: every alpha, b, A, B, and the probabilities of all 5,000 test instances)."""
import os

import numpy as np
import pytest

import datagen
import oracle
from test_gpu_full import compare_pairs, kkt_audit, load_golden

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

GOLDEN = os.path.join(os.path.dirname(__file__), "golden", "letter_eps1e-05.npz")


@pytest.fixture(scope="module")
def setup():
    import __graft_entry__

    __graft_entry__.build()
    import paper_conf_icde_wenshcc19_b200 as gm

    g = load_golden(GOLDEN)
    spec, X, y, Xt, yt = datagen.make_config("letter")
    model = gm.train(X, y, spec.k, spec.C, spec.gamma, g["meta"]["eps"])
    return gm, g, spec, X, y, Xt, yt, model


def test_letter_full_every_alpha_vs_golden(setup):
    gm, g, spec, X, y, Xt, yt, model = setup
    assert model.n_pairs_trained == 325
    compare_pairs(model, g, y, spec.k, spec.C)
    st = model.train_stats()
    assert st["n_streams"] > 0


def test_letter_full_every_probability_vs_golden(setup):
    gm, g, spec, X, y, Xt, yt, model = setup
    prob = model.predict_proba(Xt)
    prob_o = g["prob"]
    assert prob.shape == prob_o.shape == (5_000, 26)
    assert np.abs(prob - prob_o).max() <= 1e-4
    top = np.sort(prob_o, 1)
    sure = top[:, -1] - top[:, -2] >= 2e-4
    assert np.all(prob.argmax(1)[sure] == prob_o.argmax(1)[sure])
    assert np.abs(model.decision_function(Xt) - g["dec"].astype(np.float64)).max() <= 1e-3


@pytest.mark.parametrize("s,t", [(0, 1), (7, 19), (24, 25)])
def test_letter_full_kkt_audit(setup, s, t):
    gm, g, spec, X, y, Xt, yt, model = setup
    kkt_audit(X, y, spec.k, spec.C, spec.gamma, g["meta"]["eps"], model, s, t)
