"""Per-rank work of the pair-sharded multi-GPU path, measured one rank at a time on one GPU.

For world = 1, 2, 4, 8 every rank's share (LPT pair subset for training, its test-row shard for
prediction; dist.plan_pairs / dist.row_range) is run through the C ABI on cuda:0 and timed on the
device; the estimate for N GPUs is the slowest rank (the NCCL model / probability gathers are not
included).  An estimate, not a multi-GPU measurement.

    python tools/shard_probe.py [config] [reps]
"""
import json
import os
import sys

os.environ.setdefault("CUDA_DEVICE_MAX_CONNECTIONS", "32")
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import datagen  # noqa: E402
import paper_conf_icde_wenshcc19_b200 as gm  # noqa: E402
from paper_conf_icde_wenshcc19_b200 import dist as gdist  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else "mnist"
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 3
spec, X, y, Xt, yt = datagen.make_config(name)
dev = torch.device("cuda:0")
Xd, yd, Xtd = torch.from_numpy(X).to(dev), torch.from_numpy(y).to(dev), torch.from_numpy(Xt).to(dev)
counts = np.bincount(y, minlength=spec.k)
gm.train(Xd, yd, spec.k, spec.C, spec.gamma, 1e-3)  # warm-up
out = {"config": name, "note": "per-rank device time measured one rank at a time on one B200; N-GPU estimate = slowest rank; gathers excluded"}
for world in (1, 2, 4, 8):
    shards = gdist.plan_pairs(counts, world)
    ranks = []
    for r in range(world):
        best = None
        for _ in range(reps):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            torch.cuda.synchronize()
            e0.record()
            m = gm.train(Xd, yd, spec.k, spec.C, spec.gamma, 1e-3, pair_ids=shards[r] if world > 1 else None)
            e1.record()
            torch.cuda.synchronize()
            t_train = e0.elapsed_time(e1)
            best = t_train if best is None else min(best, t_train)
        st = m.train_stats()
        ranks.append({"pairs": len(shards[r]), "train_ms": round(best, 2), "kernel_ms": round(st["t_kernel_ms"], 2),
                      "outer_max": st["outer_iters_max"]})
    # prediction: the full model on each rank's row shard
    full = gm.train(Xd, yd, spec.k, spec.C, spec.gamma, 1e-3)
    pm = []
    for r in range(world):
        lo, hi = gdist.row_range(Xt.shape[0], world, r)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize()
        e0.record()
        full.predict_proba(Xtd[lo:hi])
        e1.record()
        torch.cuda.synchronize()
        pm.append(e0.elapsed_time(e1))
    est = max(x["train_ms"] for x in ranks) + max(pm)
    out[f"world{world}"] = {"ranks": ranks, "predict_ms_max": round(max(pm), 2), "est_step_ms": round(est, 2)}
    print(world, round(est, 2), [x["train_ms"] for x in ranks], flush=True)
print(json.dumps(out))
