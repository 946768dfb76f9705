"""Tuning sweep of the solver options on the MNIST-shaped workload (E7/E8 of the paper:
buffer size and number of new violators).  Prints phase times per setting.

    python tools/sweep.py "ws_size=1024,q=512,inner_iter_cap=0" "ws_size=512" ...
"""
import os
import sys
import time

os.environ.setdefault("CUDA_DEVICE_MAX_CONNECTIONS", "32")

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import datagen  # noqa: E402
import paper_conf_icde_wenshcc19_b200 as gm  # noqa: E402

spec, X, y, Xt, yt = datagen.make_config(os.environ.get("CFG", "mnist"))
eps = float(os.environ.get("EPS", "1e-3"))
dev = torch.device("cuda:0")
Xd, yd, Xtd = torch.from_numpy(X).to(dev), torch.from_numpy(y).to(dev), torch.from_numpy(Xt).to(dev)
m = gm.train(Xd, yd, spec.k, spec.C, spec.gamma, eps)  # warm-up
for arg in sys.argv[1:]:
    opts = {kv.split("=")[0]: int(kv.split("=")[1]) for kv in arg.split(",") if kv}
    best = None
    for rep in range(2):
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        m = gm.train(Xd, yd, spec.k, spec.C, spec.gamma, eps, **opts)
        p = m.predict_proba(Xtd)
        torch.cuda.synchronize()
        t = time.perf_counter() - t0
        if best is None or t < best[0]:
            best = (t, m.train_stats())
    t, s = best
    print(f"{arg:40s} total {t*1e3:7.1f} ms | kern {s["t_kernel_ms"]:5.1f} solver {s["t_solver_ms"]:5.1f} sel {s['t_select_ms']:5.1f} "
          f"sub {s['t_subproblem_ms']:5.1f} fup {s['t_fupdate_ms']:5.1f} fin {s['t_finalize_ms']:5.1f} | "
          f"outer {s['outer_iters_max']} inner {s['inner_iters_sum']} cyc/step "
          f"{s['smo_cycles_sum']/max(1,s['inner_iters_sum']):.0f} nsv {s['n_sv']}", flush=True)
