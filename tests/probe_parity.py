"""Diagnostic (not collected by pytest): where do GPU-vs-oracle probability differences come
from?  For each case: total max|dp|, the part from training (oracle FP64 evaluation of the GPU
model vs the oracle model) and the part from the decision path (GPU prediction vs the oracle's
FP64 evaluation of the same GPU model).  Run once plainly and once with GMPSVM_DEC=f64.

    python tests/probe_parity.py [json-out]
"""
import json
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import datagen  # noqa: E402
import oracle  # noqa: E402

EPS = 1e-5


def gpu_as_oracle_model(model, y, k, gamma):
    pairs = oracle.pair_list(k)
    counts = np.bincount(y, minlength=k)
    al, b, A, B = [], np.zeros(len(pairs)), np.zeros(len(pairs)), np.zeros(len(pairs))
    for p, (s, t) in enumerate(pairs):
        info = model.pair(s, t, int(counts[s]), int(counts[t]))
        al.append(info["alpha"])
        b[p], A[p], B[p] = info["b"], info["A"], info["B"]
    return dict(k=k, gamma=gamma, alpha=al, alpha_flat=np.concatenate(al), b=b, A=A, B=B)


def main():
    import paper_conf_icde_wenshcc19_b200 as gm

    cases = [("blobs", None, C, g) for C, g in [(0.01, 0.03), (0.1, 0.3), (1.0, 3.0), (10.0, 10.0), (100.0, 0.3),
                                                 (0.01, 10.0), (100.0, 0.03), (10.0, 0.3), (1.0, 0.5)]]
    cases += [("mnist", (2000, 300), None, None), ("mnist", (6000, 1000), None, None),
              ("letter", (3000, 400), None, None)]
    rows = []
    for name, sz, C, g in cases:
        n, m = sz if sz else (None, None)
        spec, X, y, Xt, yt = datagen.make_config(name, n_train=n, n_test=m)
        C = spec.C if C is None else C
        g = spec.gamma if g is None else g
        t0 = time.time()
        ref = oracle.train(X, y, spec.k, C, g, EPS)
        _, p_o = oracle.predict(ref, X, y, Xt, want_dec=False)
        model = gm.train(X, y, spec.k, C, g, EPS)
        p_g = model.predict_proba(Xt)
        gref = gpu_as_oracle_model(model, y, spec.k, g)
        dec_og, p_og = oracle.predict(gref, X, y, Xt)
        dec_g = model.decision_function(Xt)
        abs_sum = [np.abs(a).sum() for a in gref["alpha"]]
        cond22 = max(abs(gref["A"][p]) / 4 * 2.0 ** -22 * abs_sum[p] for p in range(len(abs_sum)))
        da = max(np.abs(a - b).max() for a, b in zip(gref["alpha"], ref["alpha"])) / C
        r = dict(case=name, n=int(X.shape[0]), C=C, gamma=g, dp_total=float(np.abs(p_g - p_o).max()),
                 dp_train=float(np.abs(p_og - p_o).max()), dp_dec=float(np.abs(p_g - p_og).max()),
                 ddec_dec=float(np.abs(dec_g - dec_og).max()), dalpha_over_C=float(da),
                 db=float(np.abs(gref["b"] - ref["b"]).max()), dA=float(np.abs(gref["A"] - ref["A"]).max()),
                 dB=float(np.abs(gref["B"] - ref["B"]).max()), cond22=float(cond22),
                 maxA=float(np.abs(gref["A"]).max()), max_abs_alpha=float(max(abs_sum)),
                 dec_env=os.environ.get("GMPSVM_DEC", ""), secs=time.time() - t0)
        print(json.dumps(r), flush=True)
        rows.append(r)
    if len(sys.argv) > 1:
        json.dump(rows, open(sys.argv[1], "w"), indent=1)


if __name__ == "__main__":
    main()
