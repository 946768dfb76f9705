"""Write tests/golden/<config>_eps<eps>.npz from the ORACLE ONLY (no CUDA path involved).

    python tests/golden/make_full_golden.py mnist 1e-5
    python tests/golden/make_full_golden.py letter 1e-5

Stores, for the full-size config (datagen recipe) and every pair: alpha of
every instance (pair-local order: class s then t, original order within class; Alg 2),
b, A, B, oracle iterations and status; and, for EVERY test instance, the decision values
(Eq 11, stored as FP32: compared at 1e-3) and probabilities (Eq 12, 14-15, FP64).  The GPU parity tests (tests/test_gpu_full.py,
tests/test_gpu_letter.py) compare the CUDA path element by element against it.
"""
import json
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)

import datagen  # noqa: E402
import oracle  # noqa: E402


def main():
    name = sys.argv[1]
    eps = float(sys.argv[2])
    spec, X, y, Xt, yt = datagen.make_config(name)
    t0 = time.time()
    m = oracle.train(X, y, spec.k, spec.C, spec.gamma, eps)
    t_train = time.time() - t0
    t0 = time.time()
    dec, prob = oracle.predict(m, X, y, Xt)
    t_pred = time.time() - t0
    counts = np.bincount(y, minlength=spec.k)
    sizes = np.array([counts[s] + counts[t] for s, t in m["pairs"]], dtype=np.int64)
    meta = dict(config=name, eps=eps, C=spec.C, gamma=spec.gamma, k=spec.k, n_train=int(X.shape[0]),
                n_test=int(Xt.shape[0]), generator="datagen.make_config(%r)" % name,
                written_by="tests/golden/make_full_golden.py (oracle only)",
                oracle_threads=oracle.default_threads(), oracle_train_s=t_train, oracle_predict_s=t_pred)
    path = os.path.join(os.path.dirname(os.path.abspath(__file__)), f"{name}_eps{eps:g}.npz")
    np.savez_compressed(path, meta=np.array(json.dumps(meta)), alpha=m["alpha_flat"],
                        pair_off=np.concatenate([[0], np.cumsum(sizes)]), b=m["b"], A=m["A"], B=m["B"],
                        iters=m["iters"], status=m["status"], dec=dec.astype(np.float32), prob=prob, label=yt.astype(np.int32))
    print("wrote", path, "train %.1fs predict %.1fs" % (t_train, t_pred))


if __name__ == "__main__":
    main()
