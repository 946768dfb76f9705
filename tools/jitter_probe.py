"""Repeated device-resident train+predict: wall time per call, to find host-side outliers."""
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
m = None
for i in range(int(sys.argv[1]) if len(sys.argv) > 1 else 12):
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    m2 = gm.train(Xd, yd, spec.k, spec.C, spec.gamma, 1e-3)
    t1 = time.perf_counter()
    p = m2.predict_proba(Xtd)
    torch.cuda.synchronize()
    t2 = time.perf_counter()
    m = m2
    s = m.train_stats()
    print(f"{i}: train {1e3*(t1-t0):6.1f} predict {1e3*(t2-t1):5.1f} | krow {s['t_kernel_ms']:5.1f} solver "
          f"{s['t_solver_ms']:5.1f} fin {s['t_finalize_ms']:5.1f} stage {s['t_stage_ms']:5.1f}", flush=True)
