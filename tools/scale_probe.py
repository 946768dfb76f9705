"""Timing probe of the large-n configs (ROW_CACHE regime): one train + predict on 1 GPU.

    python tools/scale_probe.py <config> <n_train> <n_test> [ws_size]
"""
import json
import os
import sys
import time

os.environ.setdefault("CUDA_DEVICE_MAX_CONNECTIONS", "32")
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import datagen  # noqa: E402
import paper_conf_icde_wenshcc19_b200 as gm  # noqa: E402

name, n, m = sys.argv[1], int(sys.argv[2]), int(sys.argv[3])
ws = int(sys.argv[4]) if len(sys.argv) > 4 else 0
t0 = time.perf_counter()
spec, X, y, Xt, yt = datagen.make_config(name, n_train=n, n_test=m)
print(f"generated {name} {X.shape} in {time.perf_counter() - t0:.1f} s; classes {np.bincount(y).tolist()}", flush=True)
dev = torch.device("cuda:0")
Xd, yd, Xtd = torch.from_numpy(X).to(dev), torch.from_numpy(y).to(dev), torch.from_numpy(Xt).to(dev)
torch.cuda.synchronize()
t0 = time.perf_counter()
model = gm.train(Xd, yd, spec.k, spec.C, spec.gamma, 1e-3, ws_size=ws)
torch.cuda.synchronize()
t1 = time.perf_counter()
prob = model.predict_proba(Xtd)
torch.cuda.synchronize()
t2 = time.perf_counter()
acc = float((prob.argmax(1).cpu().numpy() == yt).mean())
st = model.train_stats()
out = {"config": name, "n_train": n, "n_test": m, "d": spec.d, "k": spec.k, "C": spec.C, "gamma": spec.gamma,
       "train_s": t1 - t0, "predict_s": t2 - t1, "test_acc": acc,
       "stats": {k: (round(v, 3) if isinstance(v, float) else v) for k, v in st.items()},
       # FULL_K only: ROW_CACHE rows run inside the solver graph, t_kernel_ms does not time them
       # (their time comes from the ncu launch list, profiles/r02)
       "kernel_tflops": (st["kernel_flops"] / (st["t_kernel_ms"] * 1e-3) / 1e12
                         if st["cache_regime"] == 0 and st["t_kernel_ms"] > 0 else None)}
print(json.dumps(out), flush=True)
