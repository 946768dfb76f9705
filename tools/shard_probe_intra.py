"""NEXT-1 estimate on one GPU: the N-GPU training time of a job whose hardest pair is trained by
every rank at once (intra-pair sharding, gmpsvm_shard_*) and whose other pairs are pair-sharded
(LPT), against the measured 1-GPU time.  An estimate, not a multi-GPU measurement:

  1. main solver, all pairs, 1 GPU: T1 (device events); per pair (outer, inner) from pair_iters
  2. hardest pair (most inner SMO steps): the sharded solver with world = 1 gives its outer
     iteration count O (world > 1 gives bitwise the same iterates, so the same O); rank 0 of an
     N-rank shard (the other ranks' candidate blocks empty) is timed for a few dozen iterations:
     t_N per iteration (host round trips included) -> T_pair(N) = O (t_N + 2 c), c = an assumed
     small-message NCCL latency per collective (all_gather + all_reduce per iteration)
  3. the other pairs: LPT over N ranks, each rank's subset trained by the main solver one rank at
     a time -> slowest rank
  4. estimate(N) = T_pair(N) + slowest rank; the whole job at N = 1 is T1

    python tools/shard_probe_intra.py <config> <n_train> [ws_size] [coll_us]
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
from paper_conf_icde_wenshcc19_b200 import dist as gdist  # noqa: E402

name, n = sys.argv[1], int(sys.argv[2])
ws = int(sys.argv[3]) if len(sys.argv) > 3 else 192
coll_us = float(sys.argv[4]) if len(sys.argv) > 4 else 20.0
eps = 1e-3
t0 = time.perf_counter()
spec, X, y, Xt, yt = datagen.make_config(name, n_train=n, n_test=1000)
print(f"generated {X.shape} in {time.perf_counter() - t0:.1f} s", flush=True)
dev = torch.device("cuda:0")
Xd, yd = torch.from_numpy(X).to(dev), torch.from_numpy(y).to(dev)
counts = np.bincount(y, minlength=spec.k)
pairs = gdist.pair_list(spec.k)


def timed_train(**opts):
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    e0.record()
    m = gm.train(Xd, yd, spec.k, spec.C, spec.gamma, eps, **opts)
    e1.record()
    torch.cuda.synchronize()
    return m, e0.elapsed_time(e1) / 1e3


full, T1 = timed_train()
iters = {p: full.pair_iters(s, t) for p, (s, t) in enumerate(pairs)}
hard = max(iters, key=lambda p: iters[p][1])
s, t = pairs[hard]
print(f"1 GPU: {T1:.3f} s; hardest pair {pairs[hard]} outer/inner/rows {iters[hard]}", flush=True)


def shard_run(world, max_iters=None):
    sh = gm.Shard(X, y, spec.k, s, t, spec.C, spec.gamma, eps, 0, world, ws_size=ws)
    blk = sh.cand_doubles
    empty = np.zeros(blk)
    sub = 4 + 4 * sh.ws_size
    for c in range(blk // sub):  # a peer sub-block without candidates whose I_l keeps the gap open
        empty[c * sub], empty[c * sub + 1] = np.finfo(np.float64).max, 1e300
    it, t_iter = 0, []
    c = sh.candidates()
    while max_iters is None or it < max_iters:
        ta = time.perf_counter()
        stop, fw = sh.select(np.concatenate([c] + [empty] * (world - 1)), want_fws=True)
        if stop:
            break
        c = sh.step(fw, want_cands=True)
        t_iter.append(time.perf_counter() - ta)
        it += 1
    return sh, it, t_iter


sh1, O, t1 = shard_run(1)
res1 = sh1.finish(sh1.f_slice())
# the same pair's kernel rows on their own: q rows x the pair's n_p columns (rectangular SIMT
# contraction, as rows_contract / the sharded solver run it), timed on the device
idx = np.concatenate([np.flatnonzero(y == s), np.flatnonzero(y == t)])
Xp = torch.from_numpy(X[idx]).to(dev)
rows = Xp[:ws // 2].contiguous()
gm.rbf_kernel(rows, Xp, spec.gamma)
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record()
for _ in range(5):
    gm.rbf_kernel(rows, Xp, spec.gamma)
e1.record()
torch.cuda.synchronize()
rows_ms = e0.elapsed_time(e1) / 5
rows_tflops = (ws // 2) * len(idx) * (2 * spec.d + 3) / (rows_ms * 1e-3) / 1e12
out = {"config": name, "n_train": n, "ws_size": ws, "coll_us_assumed": coll_us, "T1_s": T1,
       "hard_pair": list(pairs[hard]), "hard_pair_main_solver": iters[hard],
       "hard_pair_sharded_world1": {"outer": O, "inner": res1["inner_iters"], "s": sum(t1),
                                    "per_iter_ms": 1e3 * float(np.median(t1))},
       "rows_contract_isolated": {"rows": ws // 2, "cols": int(len(idx)), "ms": rows_ms, "tflops": rows_tflops},
       "estimates": {}}
print(f"sharded solver world 1: {O} outer iterations, {sum(t1):.3f} s", flush=True)
for N in (2, 4, 8):
    _, _, tN = shard_run(N, max_iters=min(O, 60))
    t_pair = O * (float(np.median(tN)) + 2 * coll_us * 1e-6)
    rest = [p for p in range(len(pairs)) if p != hard]
    shards = gdist.plan_pairs(counts, N, only=rest)
    ranks = []
    for r in range(N):
        if not shards[r]:
            ranks.append(0.0)
            continue
        _, tr = timed_train(pair_ids=shards[r])
        ranks.append(tr)
    est = t_pair + max(ranks)
    out["estimates"][N] = {"hard_pair_s": t_pair, "per_iter_ms": 1e3 * float(np.median(tN)), "rest_ranks_s": ranks,
                           "est_s": est, "speedup_vs_1gpu": T1 / est}
    print(N, json.dumps(out["estimates"][N]), flush=True)
print(json.dumps(out))
