import sys, time, os
sys.path.insert(0, os.environ.get("GRAFT_REPO_ROOT", "/root/repo"))
import torch, numpy as np, datagen, paper_conf_icde_wenshcc19_b200 as gm
spec, X, y, Xt, yt = datagen.make_config("letter")
dev = torch.device("cuda:0")
Xd, yd, Xtd = torch.from_numpy(X).to(dev), torch.from_numpy(y).to(dev), torch.from_numpy(Xt).to(dev)
for r in range(4):
    torch.cuda.synchronize(); t0 = time.perf_counter()
    m = gm.train(Xd, yd, spec.k, spec.C, spec.gamma, 1e-3)
    p = m.predict_proba(Xtd); torch.cuda.synchronize()
    s = m.train_stats()
    print(r, round((time.perf_counter() - t0) * 1e3, 2), "ms; stage", round(s["t_stage_ms"], 2), "kv", round(s["t_kernel_ms"], 2), "solver", round(s["t_solver_ms"], 2), "fin", round(s["t_finalize_ms"], 2), "acc", float((p.argmax(1).cpu().numpy() == yt).mean()))
