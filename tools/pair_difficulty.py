"""Which pair bounds the solver, and can a cheap pre-solve statistic predict it?  Per pair of a
config: outer / inner SMO iterations (gmpsvm_model_pair_iters) next to candidate predictors
computed on a subsample: Fisher ratio of the class means, kernel MMD^2, and the fraction of
subsampled rows whose nearest other-class kernel value exceeds their mean same-class one.

    python tools/pair_difficulty.py [config] [n_train] [sub]
"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402

import datagen  # noqa: E402
import paper_conf_icde_wenshcc19_b200 as gm  # noqa: E402
from paper_conf_icde_wenshcc19_b200 import dist as gdist  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else "mnist"
n = int(sys.argv[2]) if len(sys.argv) > 2 and sys.argv[2] != "-" else None
sub = int(sys.argv[3]) if len(sys.argv) > 3 else 512
spec, X, y, Xt, yt = datagen.make_config(name, n_train=n, n_test=100)
dev = torch.device("cuda:0")
m = gm.train(torch.from_numpy(X).to(dev), torch.from_numpy(y).to(dev), spec.k, spec.C, spec.gamma, 1e-3)
rng = np.random.default_rng(0)
S = {c: X[rng.choice(np.flatnonzero(y == c), size=min(sub, int((y == c).sum())), replace=False)].astype(np.float64)
     for c in range(spec.k)}
mu = {c: X[y == c].mean(0) for c in range(spec.k)}
var = {c: X[y == c].var(0).sum() for c in range(spec.k)}


def kern(A, B):
    d2 = (A * A).sum(1)[:, None] + (B * B).sum(1)[None, :] - 2 * A @ B.T
    return np.exp(-spec.gamma * np.maximum(d2, 0))


Kc = {(a, b): kern(S[a], S[b]) for a in range(spec.k) for b in range(a, spec.k)}
rows = []
for p, (s, t) in enumerate(gdist.pair_list(spec.k)):
    o, i, r = m.pair_iters(s, t)
    fisher = float(((mu[s] - mu[t]) ** 2).sum() / (var[s] + var[t]))
    kss, ktt, kst = Kc[(s, s)], Kc[(t, t)], Kc[(s, t)]
    mmd = float(kss.mean() + ktt.mean() - 2 * kst.mean())
    # overlap: rows of s whose largest kernel value to t beats their mean to s (and vice versa)
    ov = float(((kst.max(1) > kss.mean(1)).mean() + (kst.max(0) > ktt.mean(1)).mean()) / 2)
    nn = float(((kst.max(1) > np.sort(kss, 1)[:, -2]).mean() + (kst.max(0) > np.sort(ktt, 1)[:, -2]).mean()) / 2)
    rows.append({"pair": [s, t], "outer": o, "inner": i, "fisher": fisher, "mmd2": mmd, "overlap": ov, "nn_cross": nn})
rows.sort(key=lambda r: -r["inner"])
for r in rows:
    print(json.dumps(r))
def rank_corr(a, b):
    ra, rb = np.argsort(np.argsort(a)), np.argsort(np.argsort(b))
    return float(np.corrcoef(ra, rb)[0, 1])
inner = [r["inner"] for r in rows]
for key, sgn in (("fisher", -1), ("mmd2", -1), ("overlap", 1), ("nn_cross", 1)):
    print(key, "spearman vs inner:", round(rank_corr(inner, [sgn * r[key] for r in rows]), 3),
          "top-by-proxy:", max(rows, key=lambda r: sgn * r[key])["pair"])
