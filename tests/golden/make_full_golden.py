"""Write tests/golden/<config>_eps<eps>.json from the ORACLE ONLY (no CUDA path involved).

    python tests/golden/make_full_golden.py mnist 1e-5 [n_probe]

Stores, for the full-size config (datagen recipe): per-pair b, A, B,
n_sv, n_bound, sum(alpha), oracle iterations; and dec values / probabilities of the first
n_probe test instances.  The GPU parity test (tests/test_gpu_full.py) compares against it.
"""
import base64
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
    n_probe = int(sys.argv[3]) if len(sys.argv) > 3 else 200
    spec, X, y, Xt, yt = datagen.make_config(name)
    t0 = time.time()
    m = oracle.train(X, y, spec.k, spec.C, spec.gamma, eps)
    t_train = time.time() - t0
    t0 = time.time()
    dec, prob = oracle.predict(m, X, y, Xt[:n_probe])
    t_pred = time.time() - t0
    pairs = []
    rng = np.random.default_rng(7)
    for p, (s, t) in enumerate(m["pairs"]):
        a = m["alpha"][p]
        probe = np.sort(rng.choice(len(a), size=min(64, len(a)), replace=False))
        pairs.append(dict(s=s, t=t, b=float(m["b"][p]), A=float(m["A"][p]), B=float(m["B"][p]),
                          n_sv=int((a > 0).sum()), n_bound=int((a >= spec.C).sum()),
                          sum_alpha=float(a.sum()), iters=int(m["iters"][p]), status=int(m["status"][p]),
                          sv_mask=base64.b64encode(np.packbits(a > 0).tobytes()).decode(),
                          firm_mask=base64.b64encode(np.packbits(a >= 1e-4 * spec.C).tobytes()).decode(),
                          probe_idx=probe.tolist(), probe_alpha=a[probe].tolist()))
    out = dict(config=name, eps=eps, C=spec.C, gamma=spec.gamma, k=spec.k, n_train=int(X.shape[0]),
               n_probe=n_probe, generator="datagen.make_config(%r)" % name,
               written_by="tests/golden/make_full_golden.py (oracle only)",
               oracle_threads=oracle.default_threads(), oracle_train_s=t_train, oracle_predict_s=t_pred,
               pairs=pairs, probe_dec=dec.tolist(), probe_prob=prob.tolist(),
               probe_label=[int(v) for v in yt[:n_probe]])
    path = os.path.join(os.path.dirname(os.path.abspath(__file__)), f"{name}_eps{eps:g}.json")
    with open(path, "w") as fh:
        json.dump(out, fh)
    print("wrote", path, "train %.1fs predict %.1fs" % (t_train, t_pred))


if __name__ == "__main__":
    main()
