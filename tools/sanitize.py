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
print("sanitize workload ok", m.n_sv, float(p.sum()), float(K.sum()), float(K2.sum()))
