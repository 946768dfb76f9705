"""Small T1-shaped workload for compute-sanitizer (memcheck / racecheck / synccheck):
blobs and MNIST-shaped subsets through train (multi outer iterations), predict (int8 and FP64
decision paths) and the rectangular / symmetric kernel-value launches.

    compute-sanitizer --tool memcheck python tools/sanitize.py
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

import datagen  # noqa: E402
import paper_conf_icde_wenshcc19_b200 as gm  # noqa: E402

spec, X, y, Xt, yt = datagen.make_config("blobs")
m = gm.train(X, y, spec.k, spec.C, spec.gamma, 1e-5, ws_size=64)
p = m.predict_proba(Xt)
assert np.allclose(p.sum(1), 1.0)
spec, X, y, Xt, yt = datagen.make_config("mnist", n_train=1200, n_test=150)
m = gm.train(X, y, spec.k, spec.C, spec.gamma, 1e-3, ws_size=96)
p = m.predict_proba(Xt)
K = gm.rbf_kernel(X[:300], X[:200], spec.gamma)
K2 = gm.rbf_kernel(X[:257], X[:257], spec.gamma)
if os.environ.get("SANITIZE_SPARSE", "1") == "1":  # NEXT-3: sparse kernel values from CSR rows (csr.cu)
    import scipy.sparse as sps
    os.environ["GMPSVM_CSR"] = "sparse"
    specn, Xn, yn, Xnt, ynt = datagen.make_config("news20", n_train=400, n_test=50)
    ms = gm.train_csr(sps.csr_matrix(Xn), yn, specn.k, specn.C, specn.gamma, 1e-3)
    assert ms.train_stats()["kernel_path"] == 2
    ps = ms.predict_proba(Xnt)
    del os.environ["GMPSVM_CSR"]
    print("sparse ok", ms.n_sv, float(ps.sum()))
print("sanitize workload ok", m.n_sv, float(p.sum()), float(K.sum()), float(K2.sum()))
