"""Where the bench step's time goes on the host side: Python-timed train / predict calls vs the
library's own host clocks, per step (device-resident inputs, as bench.py's `value`)."""
import os
import sys
import time

os.environ.setdefault("CUDA_DEVICE_MAX_CONNECTIONS", "32")
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import datagen  # noqa: E402
import paper_conf_icde_wenshcc19_b200 as gm  # noqa: E402

spec, X, y, Xt, yt = datagen.make_config("mnist")
dev = torch.device("cuda:0")
Xd, yd, Xtd = torch.from_numpy(X).to(dev), torch.from_numpy(y).to(dev), torch.from_numpy(Xt).to(dev)
model = None
for it in range(8):
    torch.cuda.synchronize()
    td = time.perf_counter()
    del model
    model = None
    t0 = time.perf_counter()
    model = gm.train(Xd, yd, spec.k, spec.C, spec.gamma, 1e-3)
    t1 = time.perf_counter()
    prob = model.predict_proba(Xtd)
    t2 = time.perf_counter()
    torch.cuda.synchronize()
    t3 = time.perf_counter()
    s, ps = model.train_stats(), gm.last_predict_stats()
    print(f"step {it}: train call {1e3*(t1-t0):.2f} (lib {s['t_total_ms']:.2f}) predict call {1e3*(t2-t1):.2f} "
          f"(lib {ps['t_total_ms']:.2f}) tail sync {1e3*(t3-t2):.2f} total {1e3*(t3-t0):.2f} ms; "
          f"free of the previous model {1e3*(t0-td):.2f} ms", flush=True)
