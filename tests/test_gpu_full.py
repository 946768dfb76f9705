"""Full-size parity (BASELINE.json configs[2], MNIST-shaped 60k x 784, k=10) in the launch
configuration bench.py times (device-resident inputs, ws_size 1024, q 512), against
tests/golden/mnist_eps1e-05.json -- written by tests/golden/make_full_golden.py from the
oracle only (433 s on 8 host threads) -- plus properties the oracle checks one by one:
sampled kernel rows, a per-pair KKT audit, and sampled decision values.
"""
import base64
import json
import os

import numpy as np
import pytest

import datagen
import oracle

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

GOLDEN = os.path.join(os.path.dirname(__file__), "golden", "mnist_eps1e-05.json")


@pytest.fixture(scope="module", params=[None, 1024], ids=["bench-config", "ws1024"])
def setup(request):
    import __graft_entry__

    __graft_entry__.build()
    import paper_conf_icde_wenshcc19_b200 as gm

    g = json.load(open(GOLDEN))
    spec, X, y, Xt, yt = datagen.make_config("mnist")
    dev = torch.device("cuda:0")
    Xd, yd = torch.from_numpy(X).to(dev), torch.from_numpy(y).to(dev)
    opts = {} if request.param is None else {"ws_size": request.param}  # None: bench.py's defaults
    model = gm.train(Xd, yd, spec.k, spec.C, spec.gamma, g["eps"], **opts)
    return gm, g, spec, X, y, Xt, yt, model


def _mask(b64, n):
    return np.unpackbits(np.frombuffer(base64.b64decode(b64), dtype=np.uint8))[:n].astype(bool)


def test_full_size_pairs_vs_golden(setup):
    gm, g, spec, X, y, Xt, yt, model = setup
    C = spec.C
    counts = np.bincount(y, minlength=spec.k)
    ties = 0
    for rec in g["pairs"]:
        s, t = rec["s"], rec["t"]
        info = model.pair(s, t, int(counts[s]), int(counts[t]))
        a = info["alpha"]
        n_p = len(a)
        sv_o, firm_o = _mask(rec["sv_mask"], n_p), _mask(rec["firm_mask"], n_p)
        sv_g = a > 0
        only_g = sv_g & ~sv_o
        only_o = sv_o & ~sv_g
        assert np.all(a[only_g] < 1e-4 * C), (s, t, np.flatnonzero(only_g & (a >= 1e-4 * C)))
        assert not np.any(firm_o[only_o]), (s, t)
        ties += int(only_g.sum() + only_o.sum())
        pi = np.array(rec["probe_idx"])
        assert np.abs(a[pi] - np.array(rec["probe_alpha"])).max() <= 1e-3 * C
        assert abs(info["b"] - rec["b"]) <= 1e-3 * max(1.0, abs(rec["b"])), (s, t, info["b"], rec["b"])
    st = model.train_stats()
    assert st["n_sv"] > 0 and st["krow_launches"] == 1
    print(f"documented SV ties: {ties}")


def test_full_size_probabilities_vs_golden(setup):
    gm, g, spec, X, y, Xt, yt, model = setup
    n = g["n_probe"]
    prob = model.predict_proba(torch.from_numpy(Xt[:n]).cuda()).cpu().numpy()
    prob_o = np.array(g["probe_prob"])
    assert np.abs(prob - prob_o).max() <= 1e-4
    top = np.sort(prob_o, 1)
    sure = top[:, -1] - top[:, -2] >= 2e-4
    assert np.all(prob.argmax(1)[sure] == prob_o.argmax(1)[sure])
    dec = model.decision_function(Xt[:n])
    assert np.abs(dec - np.array(g["probe_dec"])).max() <= 1e-3


def test_full_size_sampled_kernel_rows(setup):
    gm, g, spec, X, y, Xt, yt, model = setup
    rows = np.random.default_rng(5).choice(X.shape[0], size=24, replace=False)
    K = gm.rbf_kernel(X[rows], X, spec.gamma)
    K64 = oracle.rbf_matrix(X[rows], X, spec.gamma)
    assert np.all(np.abs(K.astype(np.float64) - K64) <= 1e-4 * K64 + 1e-30)


def test_full_size_kkt_audit_one_pair(setup):
    # the oracle recomputes f (Eq 3) in FP64 from the GPU's alpha for one pair
    gm, g, spec, X, y, Xt, yt, model = setup
    s, t = 3, 5
    counts = np.bincount(y, minlength=spec.k)
    a = model.pair(s, t, int(counts[s]), int(counts[t]))["alpha"]
    idx, ypm = oracle.pair_members(y, spec.k, s, t)
    Xp = X[idx]
    f = oracle.exact_f(Xp, ypm, a, spec.gamma)
    C = spec.C
    iu = ((ypm > 0) & (a < C)) | ((ypm < 0) & (a > 0))
    il = ((ypm > 0) & (a > 0)) | ((ypm < 0) & (a < C))
    gap = f[il].max() - f[iu].min()
    # slack: FP32 kernel values (relative error <= 1e-4 by test_full_size_sampled_kernel_rows), applied to
    # sum_j alpha_j K_ij <= sum_j alpha_j = 2 sum_{y=+1} alpha_j
    slack = 2 * 1e-4 * a.sum()
    assert gap <= g["eps"] + slack, (gap, slack)
    assert abs((ypm * a).sum()) <= 1e-9 * C * len(a)
