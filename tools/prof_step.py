"""One MNIST-shaped train + predict through the C ABI (device-resident inputs) for ncu.

    ncu ... python tools/prof_step.py [--config mnist] [--eps 1e-3] [--reps 1]
"""
import argparse
import os
import sys

os.environ.setdefault("CUDA_DEVICE_MAX_CONNECTIONS", "32")

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import datagen  # noqa: E402
import paper_conf_icde_wenshcc19_b200 as gm  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="mnist")
ap.add_argument("--eps", type=float, default=1e-3)
ap.add_argument("--reps", type=int, default=1)
ap.add_argument("--ws-size", type=int, default=224)
a = ap.parse_args()
spec, X, y, Xt, yt = datagen.make_config(a.config)
dev = torch.device("cuda:0")
Xd, yd, Xtd = torch.from_numpy(X).to(dev), torch.from_numpy(y).to(dev), torch.from_numpy(Xt).to(dev)
for _ in range(a.reps):
    m = gm.train(Xd, yd, spec.k, spec.C, spec.gamma, a.eps, ws_size=a.ws_size)
    p = m.predict_proba(Xtd)
torch.cuda.synchronize()
s = m.train_stats()
print({k: round(v, 3) if isinstance(v, float) else v for k, v in s.items()})
print(gm.last_predict_stats())
