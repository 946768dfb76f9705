"""Wall-clock probe of the host-pointer (e2e) path: train / predict / free separately."""
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
Xp, yp, Xtp = torch.from_numpy(X).pin_memory(), torch.from_numpy(y).pin_memory(), torch.from_numpy(Xt).pin_memory()
Xh, yh, Xth = Xp.numpy(), yp.numpy(), Xtp.numpy()
for mode in ["pinned", "pageable"]:
    A, B_, C_ = (Xh, yh, Xth) if mode == "pinned" else (X, y, Xt)
    m = None
    for i in range(5):
        t0 = time.perf_counter()
        m2 = gm.train(A, B_, spec.k, spec.C, spec.gamma, 1e-3)
        t1 = time.perf_counter()
        p = m2.predict_proba(C_)
        t2 = time.perf_counter()
        del m
        t3 = time.perf_counter()
        m = m2
        s = m.train_stats()
        print(f"{mode} {i}: train {1e3*(t1-t0):7.1f} (lib {s['t_total_ms']:6.1f} stage {s['t_stage_ms']:5.1f} "
              f"krow {s['t_kernel_ms']:5.1f} solver {s['t_solver_ms']:5.1f} fin {s['t_finalize_ms']:5.1f}) "
              f"predict {1e3*(t2-t1):6.1f} free {1e3*(t3-t2):6.1f}", flush=True)
