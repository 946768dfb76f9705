"""The oracle (the CPU baseline, as it stands) on a FULL workload on this host: train and
predict timed separately, with the host's thread count and CPU model.

    python tools/cpu_full.py [config] [eps] [out.json]
"""
import json
import os
import subprocess
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

import datagen  # noqa: E402
import oracle  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else "mnist"
eps = float(sys.argv[2]) if len(sys.argv) > 2 else 1e-3
out = sys.argv[3] if len(sys.argv) > 3 else None
spec, X, y, Xt, yt = datagen.make_config(name)
model_str = ""
try:
    model_str = [ln.split(":", 1)[1].strip() for ln in subprocess.run(["lscpu"], capture_output=True, text=True).stdout.splitlines()
                 if ln.startswith("Model name")][0]
except Exception:
    pass
t0 = time.perf_counter()
m = oracle.train(X, y, spec.k, spec.C, spec.gamma, eps)
t1 = time.perf_counter()
_, prob = oracle.predict(m, X, y, Xt, want_dec=False)
t2 = time.perf_counter()
res = {"config": name, "n_train": int(X.shape[0]), "n_test": int(Xt.shape[0]), "eps": eps, "kind": "oracle",
       "threads": oracle.default_threads(), "cpu_model": model_str, "train_s": t1 - t0, "predict_s": t2 - t1,
       "total_s": t2 - t0, "test_accuracy": float((prob.argmax(1) == yt).mean()),
       "n_sv": int(sum(int((a > 0).sum()) for a in m["alpha"]))}
print(json.dumps(res), flush=True)
if out:
    json.dump(res, open(out, "w"), indent=1)
