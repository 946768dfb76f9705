"""GPU parity of the CUDA path (through the C ABI) against the FP64 oracle.

Tolerances (SURVEY.md §8(c) "Parity contract"):
  kernel values      |K32 - K64| <= 1e-4 K64 + 1e-30            (FP32 norm expansion, reading R27)
  alpha              |da| <= 1e-3 C ; SV sets equal except alpha < 1e-4 C in either solution
  b                  |db| <= 1e-3 max(1, |b|)
  probabilities      |dp| <= 1e-4 ; labels equal except top-2 ties (< 2e-4)
  KKT audit          exact-K gap of the GPU alpha <= eps + 2 max_i |sum_j a_j y_j (K32_ij - K64_ij)|
All at eps = 1e-5 (at 1e-3 even LibSVM sits 1.7e-3 C from the optimum).
"""
import os

import numpy as np
import pytest

import datagen
import oracle

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

EPS = 1e-5
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def gm():
    import __graft_entry__

    __graft_entry__.build()
    import paper_conf_icde_wenshcc19_b200 as m

    assert torch.cuda.is_available()
    return m


def _rel_ok(K32, K64, rtol=1e-4):
    return np.all(np.abs(K32.astype(np.float64) - K64) <= rtol * K64 + 1e-30)


# ------------------------------------------------------------------------------------ a2
@pytest.mark.parametrize("n,m,d,gamma", [(37, 23, 11, 0.3), (300, 517, 8, 0.5), (1000, 260, 16, 0.5),
                                         (129, 385, 784, 0.125)])
def test_rbf_kernel_rect_vs_oracle(gm, n, m, d, gamma):
    rng = np.random.default_rng(n + m)
    if d == 784:
        _, X, _, Y, _ = datagen.make_config("mnist", n_train=n, n_test=m)
    else:
        X = rng.normal(0, 0.5, size=(n, d)).astype(np.float32)
        Y = rng.normal(0, 0.5, size=(m, d)).astype(np.float32)
    K = gm.rbf_kernel(X, Y, gamma)
    K64 = oracle.rbf_matrix(X, Y, gamma)
    assert K.shape == (n, m)
    assert _rel_ok(K, K64)


@pytest.mark.parametrize("n,d,gamma", [(600, 8, 0.5), (1000, 784, 0.125), (257, 16, 0.5), (2, 1, 1.0)])
def test_rbf_kernel_symmetric_full_k_vs_oracle(gm, n, d, gamma):
    if d == 784:
        _, X, _, _, _ = datagen.make_config("mnist", n_train=n, n_test=1)
    else:
        X = np.random.default_rng(n).normal(0, 0.5, size=(n, d)).astype(np.float32)
    K = gm.rbf_kernel(X, X, gamma)
    assert np.all(np.diag(K) == 1.0)
    np.testing.assert_array_equal(K, K.T)
    assert _rel_ok(K, oracle.rbf_matrix(X, X, gamma))


@pytest.mark.parametrize("n,d,gamma", [(1000, 784, 0.125), (513, 16, 0.5), (300, 8, 0.5)])
def test_rbf_kernel_cta_pair_variant(gm, tmp_path, n, d, gamma):
    """The opt-in CTA-pair (cta_group::2) kernel-value launch (GMPSVM_KROW_CTA=2, read once per
    process, hence the subprocess): same tolerance, exact symmetry and K_ii = 1."""
    import os
    import subprocess
    import sys

    if d == 784:
        _, X, _, _, _ = datagen.make_config("mnist", n_train=n, n_test=1)
    else:
        X = np.random.default_rng(n).normal(0, 0.5, size=(n, d)).astype(np.float32)
    np.save(tmp_path / "x.npy", X)
    code = (f"import sys, numpy as np; sys.path.insert(0, {ROOT!r}); import paper_conf_icde_wenshcc19_b200 as gm; "
            f"X = np.load({str(tmp_path / 'x.npy')!r}); np.save({str(tmp_path / 'k.npy')!r}, gm.rbf_kernel(X, X, {gamma}))")
    subprocess.run([sys.executable, "-c", code], check=True, env=dict(os.environ, GMPSVM_KROW_CTA="2"), timeout=300)
    K = np.load(tmp_path / "k.npy")
    assert np.all(np.diag(K) == 1.0)
    np.testing.assert_array_equal(K, K.T)
    assert _rel_ok(K, oracle.rbf_matrix(X, X, gamma))


def test_rbf_kernel_device_pointers(gm):
    X = np.random.default_rng(0).normal(size=(200, 30)).astype(np.float32)
    Xd = torch.from_numpy(X).cuda()
    K = gm.rbf_kernel(Xd, Xd, 0.2)
    assert K.is_cuda
    assert _rel_ok(K.cpu().numpy(), oracle.rbf_matrix(X, X, 0.2))


# ------------------------------------------------------------------------------------ a11-a12
@pytest.mark.parametrize("k", [2, 3, 10, 26])
def test_couple_vs_oracle(gm, k):
    rng = np.random.default_rng(k)
    m, P = 300, k * (k - 1) // 2
    dec = rng.normal(0, 2, size=(m, P))
    A = -rng.uniform(0.5, 3, size=P)
    B = rng.normal(0, 0.3, size=P)
    prob = gm.couple(dec, k, A, B)
    pairs = oracle.pair_list(k)
    for i in range(0, m, 7):
        r = np.zeros((k, k))
        for p, (s, t) in enumerate(pairs):
            z = dec[i, p] * A[p] + B[p]
            rst = np.exp(-z) / (1 + np.exp(-z)) if z >= 0 else 1 / (1 + np.exp(z))
            rst = min(max(rst, 1e-7), 1 - 1e-7)
            r[s, t], r[t, s] = rst, 1 - rst
        np.testing.assert_allclose(prob[i], oracle.couple(r), atol=1e-12)
    np.testing.assert_allclose(prob.sum(1), 1.0, atol=1e-12)


# ------------------------------------------------------------------------------------ a1-a12
def _compare_models(gm_model, ref, X, y, spec_C, eps=EPS, audit=True):
    k = ref["k"]
    C = spec_C
    ties = 0
    for p, (s, t) in enumerate(ref["pairs"]):
        ns, nt = int((y == s).sum()), int((y == t).sum())
        info = gm_model.pair(s, t, ns, nt)
        a_g, a_o = info["alpha"], ref["alpha"][p]
        assert np.abs(a_g - a_o).max() <= 1e-3 * C, (p, np.abs(a_g - a_o).max())
        sv_g, sv_o = a_g > 0, a_o > 0
        diff = sv_g != sv_o
        tie = np.maximum(a_g, a_o) < 1e-4 * C  # SV in one solution only: its alpha must be tiny
        assert np.all(tie[diff]), (p, np.flatnonzero(diff & ~tie))
        ties += int(diff.sum())
        assert abs(info["b"] - ref["b"][p]) <= 1e-3 * max(1.0, abs(ref["b"][p])), (p, info["b"], ref["b"][p])
        if audit:
            idx, ypm = oracle.pair_members(y, k, s, t)
            Xp = X[idx]
            f64 = oracle.exact_f(Xp, ypm, a_g, ref["gamma"])
            K64 = oracle.rbf_matrix(Xp, Xp, ref["gamma"])
            iu = ((ypm > 0) & (a_g < C)) | ((ypm < 0) & (a_g > 0))
            il = ((ypm > 0) & (a_g > 0)) | ((ypm < 0) & (a_g < C))
            gap = f64[il].max() - f64[iu].min()
            # bound on |f(K32) - f(K64)| from the FP32 kernel-value error (<= 1e-4 relative)
            slack = 2 * 1e-4 * np.abs(K64 @ a_g).max()
            assert gap <= eps + slack + 1e-12, (p, gap, slack)
            assert abs((ypm * a_g).sum()) <= 1e-9 * C * len(a_g)
            assert np.all(a_g >= 0) and np.all(a_g <= C)
    return ties


def _gpu_model(gm, X, y, spec, eps=EPS, **opts):
    return gm.train(X, y, spec.k, spec.C, spec.gamma, eps, **opts)


def test_train_predict_blobs_vs_oracle(gm):
    spec, X, y, Xt, yt = datagen.make_config("blobs")
    ref = oracle.train(X, y, spec.k, spec.C, spec.gamma, EPS)
    model = _gpu_model(gm, X, y, spec)
    assert model.status == 0
    _compare_models(model, ref, X, y, spec.C)
    dec_o, prob_o = oracle.predict(ref, X, y, Xt)
    prob = model.predict_proba(Xt)
    assert np.abs(prob - prob_o).max() <= 1e-4
    top = np.sort(prob_o, 1)
    sure = top[:, -1] - top[:, -2] >= 2e-4
    assert np.all(prob.argmax(1)[sure] == prob_o.argmax(1)[sure])
    st = model.train_stats()
    assert st["krow_launches"] == 1 and st["launches"] > 0


def test_decision_values_vs_oracle_from_gpu_model(gm):
    # the oracle evaluates Eq 11 in FP64 with the GPU's own alpha and b
    spec, X, y, Xt, yt = datagen.make_config("blobs")
    model = _gpu_model(gm, X, y, spec)
    ref = dict(k=spec.k, gamma=spec.gamma, alpha=[], b=np.zeros(3), A=np.zeros(3), B=np.zeros(3))
    for p, (s, t) in enumerate(oracle.pair_list(spec.k)):
        info = model.pair(s, t, int((y == s).sum()), int((y == t).sum()))
        ref["alpha"].append(info["alpha"])
        ref["b"][p], ref["A"][p], ref["B"][p] = info["b"], info["A"], info["B"]
    dec_o, prob_o = oracle.predict(ref, X, y, Xt)
    dec = model.decision_function(Xt)
    scale = 1.0 + np.abs(dec_o)
    assert np.all(np.abs(dec - dec_o) <= 1e-4 * scale)
    prob = model.predict_proba(Xt)
    assert np.abs(prob - prob_o).max() <= 1e-5


@pytest.mark.parametrize("C,gamma", [(0.01, 0.03), (0.1, 0.3), (1.0, 3.0), (10.0, 10.0), (100.0, 0.3),
                                     (0.01, 10.0), (100.0, 0.03), (10.0, 0.3)])
def test_hyperparameter_grid_blobs(gm, C, gamma):
    # E6: C in [0.01, 100], gamma in [0.03, 10] give identical classifiers
    spec, X, y, Xt, yt = datagen.make_config("blobs")
    ref = oracle.train(X, y, spec.k, C, gamma, EPS)
    model = gm.train(X, y, spec.k, C, gamma, EPS)
    _compare_models(model, ref, X, y, C)
    _, prob_o = oracle.predict(ref, X, y, Xt, want_dec=False)
    assert np.abs(model.predict_proba(Xt) - prob_o).max() <= 1e-4


@pytest.mark.parametrize("ws,q", [(64, 32), (128, 64), (256, 128), (64, 16), (100, 50), (224, 112), (224, 56)])
def test_batched_working_set_multi_outer_iterations(gm, ws, q):
    # n_p = 400 > B: exercises the radix selection, retention of the newest B-q rows and
    # many outer iterations (L289-L305); the fixed point must not depend on B, q.
    spec, X, y, Xt, yt = datagen.make_config("blobs")
    ref = oracle.train(X, y, spec.k, spec.C, spec.gamma, EPS)
    model = gm.train(X, y, spec.k, spec.C, spec.gamma, EPS, ws_size=ws, q=q)
    assert model.train_stats()["outer_iters_max"] > 1
    _compare_models(model, ref, X, y, spec.C)
    _, prob_o = oracle.predict(ref, X, y, Xt, want_dec=False)
    assert np.abs(model.predict_proba(Xt) - prob_o).max() <= 1e-4


def test_mnist_shaped_subset(gm):
    spec, X, y, Xt, yt = datagen.make_config("mnist", n_train=2000, n_test=300)
    ref = oracle.train(X, y, spec.k, spec.C, spec.gamma, EPS)
    model = gm.train(X, y, spec.k, spec.C, spec.gamma, EPS, ws_size=128)
    _compare_models(model, ref, X, y, spec.C, audit=False)
    _, prob_o = oracle.predict(ref, X, y, Xt, want_dec=False)
    prob = model.predict_proba(Xt)
    assert np.abs(prob - prob_o).max() <= 1e-4


def test_letter_shaped_subset(gm):
    spec, X, y, Xt, yt = datagen.make_config("letter", n_train=3000, n_test=400)
    ref = oracle.train(X, y, spec.k, spec.C, spec.gamma, EPS)
    model = gm.train(X, y, spec.k, spec.C, spec.gamma, EPS, ws_size=64)
    _compare_models(model, ref, X, y, spec.C, audit=False)
    _, prob_o = oracle.predict(ref, X, y, Xt, want_dec=False)
    assert np.abs(model.predict_proba(Xt) - prob_o).max() <= 1e-4


def test_device_inputs_match_host_inputs(gm):
    spec, X, y, Xt, yt = datagen.make_config("blobs")
    m1 = gm.train(X, y, spec.k, spec.C, spec.gamma, EPS)
    m2 = gm.train(torch.from_numpy(X).cuda(), torch.from_numpy(y).cuda(), spec.k, spec.C, spec.gamma, EPS)
    p1 = m1.predict_proba(Xt)
    p2 = m2.predict_proba(torch.from_numpy(Xt).cuda()).cpu().numpy()
    np.testing.assert_array_equal(p1, p2)  # deterministic kernels: bitwise identical


def test_fused_and_split_solver_paths_agree(gm, tmp_path):
    """The fused selection + gather + local-SMO kernel (wsolve.cu, default for B <= 224) and the
    split select_ws / gather_kws / local_smo kernels (GMPSVM_WSOLVE=0) implement the same
    readings (R19, R20); both must reach the same fixed point (Eq 9) on a multi-pair
    MNIST-shaped problem with many outer iterations."""
    import subprocess
    import sys

    spec, X, y, Xt, yt = datagen.make_config("mnist", n_train=3000, n_test=200)
    m1 = gm.train(X, y, spec.k, spec.C, spec.gamma, EPS, ws_size=96)
    assert m1.train_stats()["outer_iters_max"] > 3
    p1 = m1.predict_proba(Xt)
    code = (
        "import sys, json, numpy as np; sys.path.insert(0, %r); import datagen, paper_conf_icde_wenshcc19_b200 as gm;"
        "spec, X, y, Xt, yt = datagen.make_config('mnist', n_train=3000, n_test=200);"
        "m = gm.train(X, y, spec.k, spec.C, spec.gamma, %r, ws_size=96);"
        "np.save(%r, m.predict_proba(Xt))" % (ROOT, EPS, str(tmp_path / "p2.npy"))
    )
    env = dict(os.environ, GMPSVM_WSOLVE="0")
    subprocess.run([sys.executable, "-c", code], check=True, env=env, timeout=600)
    p2 = np.load(tmp_path / "p2.npy")
    assert np.abs(p1 - p2).max() <= 1e-4


def test_mixed_solver_paths_in_one_graph(gm, tmp_path):
    """Pairs above the wsolve.cu size limit run the solver.cu kernels in the same device-driven
    graph as the others (covtype-shaped data: one 17k-instance pair next to small ones).  The
    limit is lowered (GMPSVM_WS_MAXNP, read once per process: subprocess) so a small problem
    mixes both paths; both must share the per-pair K_ws,ws slot stride (regression: mixed
    strides overlapped slots and corrupted the working-set state) and reach the oracle's fixed
    point (Eq 9)."""
    import subprocess
    import sys

    spec, X, y, Xt, yt = datagen.make_config("mnist", n_train=2000, n_test=200)
    ref = oracle.train(X, y, spec.k, spec.C, spec.gamma, EPS)
    _, prob_o = oracle.predict(ref, X, y, Xt, want_dec=False)
    sizes = sorted(int((y == s).sum() + (y == t).sum()) for s, t in oracle.pair_list(spec.k))
    limit = sizes[len(sizes) // 2]  # about half of the pairs on each path
    code = (
        "import sys, numpy as np; sys.path.insert(0, %r); import datagen, paper_conf_icde_wenshcc19_b200 as gm;"
        "spec, X, y, Xt, yt = datagen.make_config('mnist', n_train=2000, n_test=200);"
        "m = gm.train(X, y, spec.k, spec.C, spec.gamma, %r, ws_size=96);"
        "np.save(%r, m.predict_proba(Xt))" % (ROOT, EPS, str(tmp_path / "p.npy"))
    )
    env = dict(os.environ, GMPSVM_WS_MAXNP=str(limit))
    subprocess.run([sys.executable, "-c", code], check=True, env=env, timeout=600)
    p = np.load(tmp_path / "p.npy")
    assert np.abs(p - prob_o).max() <= 1e-4


def test_fp64_decision_path_vs_oracle(gm, tmp_path):
    """The FP64 decision-value path (taken automatically for ill-conditioned models; forced here
    with GMPSVM_DEC=f64, read once per process: subprocess) evaluates Eq 11 with FP64 kernel
    values: against the oracle's FP64 evaluation of the same model it agrees to rounding."""
    import subprocess
    import sys

    spec, X, y, Xt, yt = datagen.make_config("mnist", n_train=1500, n_test=300)
    code = (
        "import sys, numpy as np; sys.path.insert(0, %r); import datagen, paper_conf_icde_wenshcc19_b200 as gm;"
        "spec, X, y, Xt, yt = datagen.make_config('mnist', n_train=1500, n_test=300);"
        "m = gm.train(X, y, spec.k, spec.C, spec.gamma, %r);"
        "al = [m.pair(s, t, int((y == s).sum()), int((y == t).sum())) for s in range(spec.k) for t in range(s + 1, spec.k)];"
        "np.savez(%r, dec=m.decision_function(Xt), prob=m.predict_proba(Xt), alpha=np.concatenate([a['alpha'] for a in al]),"
        " b=[a['b'] for a in al], A=[a['A'] for a in al], B=[a['B'] for a in al])" % (ROOT, EPS, str(tmp_path / "r.npz"))
    )
    subprocess.run([sys.executable, "-c", code], check=True, env=dict(os.environ, GMPSVM_DEC="f64"), timeout=600)
    r = np.load(tmp_path / "r.npz")
    ref = dict(k=spec.k, gamma=spec.gamma, alpha_flat=r["alpha"], b=r["b"], A=r["A"], B=r["B"])
    dec_o, prob_o = oracle.predict(ref, X, y, Xt)
    assert np.abs(r["dec"] - dec_o).max() <= 1e-9 * max(1.0, np.abs(dec_o).max())
    assert np.abs(r["prob"] - prob_o).max() <= 1e-9


def _gpu_model_as_oracle(model, y, k, gamma):
    al, b, A, B = [], [], [], []
    for s_, t_ in oracle.pair_list(k):
        info = model.pair(s_, t_, int((y == s_).sum()), int((y == t_).sum()))
        al.append(info["alpha"])
        b.append(info["b"]), A.append(info["A"]), B.append(info["B"])
    return dict(k=k, gamma=gamma, alpha_flat=np.concatenate(al), b=np.array(b), A=np.array(A), B=np.array(B))


@pytest.mark.parametrize("name,n,m,C,gamma", [("mnist", 1500, 300, 10.0, 0.125), ("blobs", None, None, 100.0, 0.03),
                                             ("letter", 2000, 300, 10.0, 0.5), ("mnist", 800, 200, 1000.0, 0.006)])
def test_int8_decision_path_vs_oracle(gm, name, n, m, C, gamma):
    """The default RBF decision path (dec_i8.cu, DESIGN.md §3/§6.4): exact int8-digit dot products
    on tcgen05 and FP64 kernel values -- Eq 11 against the oracle's FP64 evaluation of the SAME
    model (the GPU's alpha, b, A, B) to ~1e-9, so the probabilities carry no FP32 kernel error;
    the model's routing bound selects it (predict stats dec_path == 1)."""
    spec, X, y, Xt, yt = datagen.make_config(name, n_train=n, n_test=m)
    model = gm.train(X, y, spec.k, C, gamma, EPS)
    dec = model.decision_function(Xt)
    assert gm.last_predict_stats()["dec_path"] == 1
    prob = model.predict_proba(Xt)
    ref = _gpu_model_as_oracle(model, y, spec.k, gamma)
    dec_o, prob_o = oracle.predict(ref, X, y, Xt)
    assert np.abs(dec - dec_o).max() <= 1e-9 * max(1.0, np.abs(dec_o).max())
    assert np.abs(prob - prob_o).max() <= 1e-9


def test_forced_fp16_decision_path(gm, tmp_path):
    """The FP16-split tensor-core decision path (dec_tc, FP32 kernel values) is never chosen by the
    routing bound for these models; forced (GMPSVM_DEC=f16, read once per process: subprocess) on
    a well-conditioned model it still meets the contract."""
    import subprocess
    import sys

    spec, X, y, Xt, yt = datagen.make_config("blobs")
    code = (
        "import sys, numpy as np; sys.path.insert(0, %r); import datagen, paper_conf_icde_wenshcc19_b200 as gm;"
        "spec, X, y, Xt, yt = datagen.make_config('blobs');"
        "m = gm.train(X, y, spec.k, 0.1, 0.3, %r); p = m.predict_proba(Xt);"
        "assert gm.last_predict_stats()['dec_path'] == 2;"
        "np.save(%r, p)" % (ROOT, EPS, str(tmp_path / "p.npy"))
    )
    subprocess.run([sys.executable, "-c", code], check=True, env=dict(os.environ, GMPSVM_DEC="f16"), timeout=600)
    ref = oracle.train(X, y, spec.k, 0.1, 0.3, EPS)
    _, prob_o = oracle.predict(ref, X, y, Xt, want_dec=False)
    assert np.abs(np.load(tmp_path / "p.npy") - prob_o).max() <= 1e-4


# ------------------------------------------------------------------------------------ NEXT-4
@pytest.mark.parametrize("name,kind,gamma,coef0,degree,C", [
    ("blobs", "linear", 1.0, 0.0, 3, 1.0), ("blobs", "poly", 0.5, 1.0, 3, 1.0), ("blobs", "sigmoid", 0.02, 0.0, 3, 1.0),
    ("letter", "poly", 0.3, 1.0, 2, 1.0), ("letter", "linear", 1.0, 0.0, 3, 0.5)])
def test_other_kernels_vs_oracle(gm, name, kind, gamma, coef0, degree, C):
    """The paper's other kernels (L76-L78; NEXT-4) through the same FULL_K tensor-core
    contraction (uncentred rows; K = f(x.y)) and the FP64 decision path: the same fixed point
    (alpha, SV sets, b, probabilities, KKT audit) as the oracle with that kernel.  The sigmoid
    kernel is not positive semi-definite in general (the dual then has several KKT points, SURVEY
    §8(c) #28); it is checked where it is close to the linear one (coef0 = 0, small gamma)."""
    n = None if name == "blobs" else 1200
    spec, X, y, Xt, yt = datagen.make_config(name, n_train=n, n_test=None if name == "blobs" else 200)
    with oracle.kernel(kind, coef0, degree):
        ref = oracle.train(X, y, spec.k, C, gamma, EPS)
        model = gm.train(X, y, spec.k, C, gamma, EPS, kernel=kind, coef0=coef0, degree=degree)
        _compare_models(model, ref, X, y, C)
        _, prob_o = oracle.predict(ref, X, y, Xt, want_dec=False)
    prob = model.predict_proba(Xt)
    assert np.abs(prob - prob_o).max() <= 1e-4
    # round trip keeps the kernel
    rt = gm.Model.deserialize(model.serialize())
    np.testing.assert_array_equal(rt.predict_proba(Xt), prob)


def test_other_kernels_need_full_k(gm):
    spec, X, y, Xt, yt = datagen.make_config("blobs")
    with pytest.raises(gm.GmpsvmError):
        gm.train(X, y, spec.k, 1.0, 1.0, 1e-3, kernel="linear", cache_bytes=1)  # ROW_CACHE: not built


# ------------------------------------------------------------------------------------ NEXT-2
@pytest.mark.parametrize("name,folds", [("blobs", 5), ("mnist", 3)])
def test_cross_validated_sigmoids_vs_oracle(gm, name, folds):
    """prob_folds = F (LibSVM's probability training, NEXT-2): F extra trainings on the other
    folds, each pair's sigmoid fitted on its out-of-fold decision values -- the same A, B and
    probabilities as oracle.train_cv on the same deterministic folds (R30)."""
    n, m = (None, None) if name == "blobs" else (1500, 200)
    spec, X, y, Xt, yt = datagen.make_config(name, n_train=n, n_test=m)
    ref = oracle.train_cv(X, y, spec.k, spec.C, spec.gamma, EPS, folds=folds)
    model = gm.train(X, y, spec.k, spec.C, spec.gamma, EPS, prob_folds=folds)
    counts = np.bincount(y, minlength=spec.k)
    for p, (s, t) in enumerate(oracle.pair_list(spec.k)):
        info = model.pair(s, t, counts[s], counts[t])
        assert abs(info["A"] - ref["A"][p]) <= 1e-3 * max(1.0, abs(ref["A"][p])), (p, info["A"], ref["A"][p])
        assert abs(info["B"] - ref["B"][p]) <= 1e-3 * max(1.0, abs(ref["B"][p])), (p, info["B"], ref["B"][p])
    _, prob_o = oracle.predict(ref, X, y, Xt, want_dec=False)
    assert np.abs(model.predict_proba(Xt) - prob_o).max() <= 1e-4
