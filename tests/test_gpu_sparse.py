"""NEXT-3 compute side: kernel values from CSR rows (csr.cu, sparse x dense -- the paper's format
and design, PAPER.md L299 / L513) against the FP64 oracle on the same rows, densified for it.

GMPSVM_CSR=sparse forces the sparse path (by default CSR rows are densified unless the dense copy
would not fit comfortably: on these shapes the dense tcgen05 contraction is faster);
`train_stats()["kernel_path"] == 2` says it ran.  Same parity contract as
test_gpu_parity.py (alpha, SV sets, b, FP64 KKT audit at eps = 1e-5, probabilities 1e-4).
"""
import os
import subprocess
import sys

import numpy as np
import pytest

import datagen
import oracle
from test_gpu_parity import EPS, ROOT, _compare_models, gm  # noqa: F401  (gm: the module fixture)

torch = pytest.importorskip("torch")
sp = pytest.importorskip("scipy.sparse")
pytestmark = pytest.mark.gpu


@pytest.fixture
def sparse_env(monkeypatch):
    monkeypatch.setenv("GMPSVM_CSR", "sparse")


def test_sparse_kernel_values_vs_oracle(gm, sparse_env):  # noqa: F811
    spec, X, y, Xt, yt = datagen.make_config("news20")
    A, At = sp.csr_matrix(X), sp.csr_matrix(Xt)
    assert A.nnz < 0.02 * X.size
    model = gm.train_csr(A, y, spec.k, spec.C, spec.gamma, EPS)
    assert model.train_stats()["kernel_path"] == 2
    ref = oracle.train(X, y, spec.k, spec.C, spec.gamma, EPS)
    _compare_models(model, ref, X, y, spec.C)
    _, prob_o = oracle.predict(ref, X, y, Xt, want_dec=False)
    assert np.abs(model.predict_proba_csr(At) - prob_o).max() <= 1e-4
    assert np.abs(model.predict_proba(Xt) - prob_o).max() <= 1e-4


def test_sparse_edge_rows_vs_oracle(gm, sparse_env):  # noqa: F811
    """Empty rows, single-entry rows, several row blocks with a ragged tail, device CSR input."""
    spec, X, y, Xt, yt = datagen.make_config("news20", n_train=700, n_test=100)
    X = X.copy()
    X[3] = 0.0      # an empty document
    X[10] = 0.0
    X[10, 17] = 1.0  # one word
    X[11] = 0.0
    X[11, 18] = 1.0  # another one-word document
    A = sp.csr_matrix(X)
    dev = torch.device("cuda:0")
    tup = (torch.from_numpy(A.indptr.astype(np.int64)).to(dev), torch.from_numpy(A.indices.astype(np.int32)).to(dev),
           torch.from_numpy(A.data.astype(np.float32)).to(dev), A.shape)
    model = gm.train_csr(tup, torch.from_numpy(y).to(dev), spec.k, spec.C, spec.gamma, EPS)
    assert model.train_stats()["kernel_path"] == 2
    ref = oracle.train(X, y, spec.k, spec.C, spec.gamma, EPS)
    _, prob_o = oracle.predict(ref, X, y, Xt, want_dec=False)
    assert np.abs(model.predict_proba(Xt) - prob_o).max() <= 1e-4
    for p, (s, t) in enumerate(ref["pairs"]):
        info = model.pair(s, t, int((y == s).sum()), int((y == t).sum()))
        assert np.abs(info["alpha"] - ref["alpha"][p]).max() <= 1e-3 * spec.C
        assert abs(info["b"] - ref["b"][p]) <= 1e-3 * max(1.0, abs(ref["b"][p]))


def test_sparse_and_dense_paths_agree(gm, sparse_env, tmp_path):  # noqa: F811
    """The same CSR rows through the densified tensor-core path (GMPSVM_CSR=dense, another
    process: the choice is read once) reach the same fixed point."""
    spec, X, y, Xt, yt = datagen.make_config("news20", n_train=1500, n_test=200)
    A = sp.csr_matrix(X)
    m1 = gm.train_csr(A, y, spec.k, spec.C, spec.gamma, EPS)
    assert m1.train_stats()["kernel_path"] == 2
    p1 = m1.predict_proba(Xt)
    code = (
        "import sys, numpy as np, scipy.sparse as sp; sys.path.insert(0, %r); import datagen, "
        "paper_conf_icde_wenshcc19_b200 as gm;"
        "spec, X, y, Xt, yt = datagen.make_config('news20', n_train=1500, n_test=200);"
        "m = gm.train_csr(sp.csr_matrix(X), y, spec.k, spec.C, spec.gamma, %r);"
        "assert m.train_stats()['kernel_path'] == 0;"
        "np.save(%r, m.predict_proba(Xt))" % (ROOT, EPS, str(tmp_path / "p2.npy"))
    )
    subprocess.run([sys.executable, "-c", code], check=True, env=dict(os.environ, GMPSVM_CSR="dense"), timeout=600)
    assert np.abs(np.load(tmp_path / "p2.npy") - p1).max() <= 1e-4
