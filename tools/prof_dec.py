"""Prediction only (MNIST-shaped model trained once): CUDA-event time of predict_proba on the
device-resident 10k test rows, per decision-value path, for ncu / A-B timing.

    python tools/prof_dec.py [--reps 10] [--config mnist]
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import datagen  # noqa: E402
import paper_conf_icde_wenshcc19_b200 as gm  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="mnist")
ap.add_argument("--eps", type=float, default=1e-3)
ap.add_argument("--reps", type=int, default=10)
a = ap.parse_args()
spec, X, y, Xt, yt = datagen.make_config(a.config)
dev = torch.device("cuda:0")
Xd, yd, Xtd = torch.from_numpy(X).to(dev), torch.from_numpy(y).to(dev), torch.from_numpy(Xt).to(dev)
m = gm.train(Xd, yd, spec.k, spec.C, spec.gamma, a.eps)
p = m.predict_proba(Xtd)
ts = []
for _ in range(a.reps):
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    e0.record()
    p = m.predict_proba(Xtd)
    e1.record()
    torch.cuda.synchronize()
    ts.append(e0.elapsed_time(e1))
st = gm.last_predict_stats()
print(json.dumps(dict(env={k: v for k, v in os.environ.items() if k.startswith("GMPSVM_")}, predict_ms=sorted(ts),
                      dec_ms=st["t_decision_ms"], path=st["dec_path"], n_sv=m.n_sv)))
