"""MNIST-shaped train + predict with each kernel of PAPER.md L75-L78 (device-resident inputs,
eps 1e-3): host-timed best of 3 after a warm-up, with the kernel-value launch time."""
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
for kind, gamma, coef0, degree, C in [("rbf", 0.125, 0.0, 3, 10.0), ("linear", 1.0, 0.0, 3, 0.01),
                                      ("poly", 0.01, 1.0, 3, 1.0), ("sigmoid", 0.002, 0.0, 3, 1.0)]:
    best = None
    for r in range(4):
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        m = gm.train(Xd, yd, spec.k, C, gamma, 1e-3, kernel=kind, coef0=coef0, degree=degree)
        p = m.predict_proba(Xtd)
        torch.cuda.synchronize()
        t = time.perf_counter() - t0
        if r and (best is None or t < best[0]):
            best = (t, m.train_stats(), gm.last_predict_stats(), float((p.argmax(1).cpu().numpy() == yt).mean()))
    t, s, ps, acc = best
    print(f"{kind:8s} C={C:g} gamma={gamma:g}: train+predict {t*1e3:.1f} ms (kernel values {s['t_kernel_ms']:.2f} ms, "
          f"predict {ps['t_total_ms']:.2f} ms), outer {s['outer_iters_max']}, n_sv {s['n_sv']}, test acc {acc:.4f}",
          flush=True)
