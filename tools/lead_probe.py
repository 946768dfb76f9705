"""Lead mode vs not: train_stats phases and device time of gm.train on the bench workload."""
import os, sys, json, time
os.environ.setdefault("CUDA_DEVICE_MAX_CONNECTIONS", "32")
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np, torch
import datagen
import paper_conf_icde_wenshcc19_b200 as gm
spec, X, y, Xt, yt = datagen.make_config("mnist")
dev = torch.device("cuda:0")
Xd, yd = torch.from_numpy(X).to(dev), torch.from_numpy(y).to(dev)
for it in range(8):
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    t0 = time.perf_counter()
    e0.record()
    m = gm.train(Xd, yd, spec.k, spec.C, spec.gamma, 1e-3)
    t1 = time.perf_counter()
    e1.record()
    torch.cuda.synchronize()
    t2 = time.perf_counter()
    st = m.train_stats()
    if it >= 3:
        print(os.environ.get("GMPSVM_LEAD"), "dev_ms", round(e0.elapsed_time(e1), 2), "host_call_ms", round((t1 - t0) * 1e3, 2),
              {k: round(v, 2) for k, v in st.items() if isinstance(v, float) and k.startswith("t_")})
