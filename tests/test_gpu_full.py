"""Full-size parity (BASELINE.json configs[2], MNIST-shaped 60k x 784, k=10) in the launch
configuration bench.py times (device-resident inputs, default working set) and at the paper's
B = 1024, against tests/golden/mnist_eps1e-05.npz -- written by tests/golden/make_full_golden.py
from the oracle only (every alpha of every pair, b, A, B, and the decision values and
probabilities of all 10,000 test instances) -- plus properties the oracle checks one by one:
sampled kernel rows and a per-pair FP64 KKT audit.
"""
import json
import os

import numpy as np
import pytest

import datagen
import oracle

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

GOLDEN = os.path.join(os.path.dirname(__file__), "golden", "mnist_eps1e-05.npz")


def load_golden(path):
    z = np.load(path)
    g = {key: z[key] for key in z.files}
    g["meta"] = json.loads(str(g["meta"]))
    return g


def compare_pairs(model, g, y, k, C):
    """Every alpha within 1e-3 C, SV sets equal except documented ties (alpha < 1e-4 C on the side
    that has it), b within 1e-3 max(1, |b|) (SURVEY §8(c) parity contract).  Returns the ties."""
    counts = np.bincount(y, minlength=k)
    off = g["pair_off"]
    ties = 0
    for p, (s, t) in enumerate(oracle.pair_list(k)):
        info = model.pair(s, t, int(counts[s]), int(counts[t]))
        a, a_o = info["alpha"], g["alpha"][off[p]:off[p + 1]]
        assert len(a) == len(a_o)
        assert np.abs(a - a_o).max() <= 1e-3 * C, (s, t, np.abs(a - a_o).max())
        diff = (a > 0) != (a_o > 0)
        assert np.all(np.maximum(a, a_o)[diff] < 1e-4 * C), (s, t, np.flatnonzero(diff))
        ties += int(diff.sum())
        assert abs(info["b"] - g["b"][p]) <= 1e-3 * max(1.0, abs(g["b"][p])), (s, t, info["b"], g["b"][p])
    return ties


def kkt_audit(X, y, k, C, gamma, eps, model, s, t):
    """The oracle recomputes f (Eq 3) in FP64 from the GPU's alpha of pair (s, t)."""
    counts = np.bincount(y, minlength=k)
    a = model.pair(s, t, int(counts[s]), int(counts[t]))["alpha"]
    idx, ypm = oracle.pair_members(y, k, s, t)
    f = oracle.exact_f(X[idx], ypm, a, gamma)
    iu = ((ypm > 0) & (a < C)) | ((ypm < 0) & (a > 0))
    il = ((ypm > 0) & (a > 0)) | ((ypm < 0) & (a < C))
    gap = f[il].max() - f[iu].min()
    # slack: FP32 kernel values of the training path (relative error <= 1e-4, the T1 tolerance)
    # applied to sum_j alpha_j K_ij <= sum_j alpha_j
    slack = 2 * 1e-4 * a.sum()
    assert gap <= eps + slack, (s, t, gap, slack)
    assert abs((ypm * a).sum()) <= 1e-9 * C * len(a)
    assert np.all(a >= 0) and np.all(a <= C)


@pytest.fixture(scope="module", params=[None, 1024], ids=["bench-config", "ws1024"])
def setup(request):
    import __graft_entry__

    __graft_entry__.build()
    import paper_conf_icde_wenshcc19_b200 as gm

    g = load_golden(GOLDEN)
    spec, X, y, Xt, yt = datagen.make_config("mnist")
    dev = torch.device("cuda:0")
    Xd, yd = torch.from_numpy(X).to(dev), torch.from_numpy(y).to(dev)
    opts = {} if request.param is None else {"ws_size": request.param}  # None: bench.py's defaults
    model = gm.train(Xd, yd, spec.k, spec.C, spec.gamma, g["meta"]["eps"], **opts)
    return gm, g, spec, X, y, Xt, yt, model


def test_full_size_every_alpha_vs_golden(setup):
    gm, g, spec, X, y, Xt, yt, model = setup
    ties = compare_pairs(model, g, y, spec.k, spec.C)
    st = model.train_stats()
    assert st["n_sv"] > 0 and st["krow_launches"] == 1
    print(f"documented SV ties: {ties}")


def test_full_size_every_probability_vs_golden(setup):
    gm, g, spec, X, y, Xt, yt, model = setup
    prob = model.predict_proba(torch.from_numpy(Xt).cuda()).cpu().numpy()
    assert gm.last_predict_stats()["dec_path"] == 1  # the int8-digit tensor-core path (routing bound)
    prob_o = g["prob"]
    assert prob.shape == prob_o.shape == (10_000, spec.k)
    assert np.abs(prob - prob_o).max() <= 1e-4
    top = np.sort(prob_o, 1)
    sure = top[:, -1] - top[:, -2] >= 2e-4
    assert np.all(prob.argmax(1)[sure] == prob_o.argmax(1)[sure])
    dec = model.decision_function(Xt)
    assert np.abs(dec - g["dec"].astype(np.float64)).max() <= 1e-3


def test_full_size_sampled_kernel_rows(setup):
    gm, g, spec, X, y, Xt, yt, model = setup
    rows = np.random.default_rng(5).choice(X.shape[0], size=24, replace=False)
    K = gm.rbf_kernel(X[rows], X, spec.gamma)
    K64 = oracle.rbf_matrix(X[rows], X, spec.gamma)
    assert np.all(np.abs(K.astype(np.float64) - K64) <= 1e-4 * K64 + 1e-30)


@pytest.mark.parametrize("s,t", [(3, 5), (0, 8)])
def test_full_size_kkt_audit(setup, s, t):
    gm, g, spec, X, y, Xt, yt, model = setup
    kkt_audit(X, y, spec.k, spec.C, spec.gamma, g["meta"]["eps"], model, s, t)
