"""Time one training run (+ prediction) of a named config in a forced cache regime.

  python tools/rc_probe.py --config covtype --n 100000 --rc      # ROW_CACHE
  python tools/rc_probe.py --config mnist                         # FULL_K (if it fits)
"""
import argparse
import os
import sys
import time

os.environ.setdefault("CUDA_DEVICE_MAX_CONNECTIONS", "32")
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import numpy as np  # noqa: E402
import torch  # noqa: E402

import datagen  # noqa: E402
import paper_conf_icde_wenshcc19_b200 as gm  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="covtype")
    ap.add_argument("--n", type=int, default=None)
    ap.add_argument("--m", type=int, default=None)
    ap.add_argument("--eps", type=float, default=1e-3)
    ap.add_argument("--rc", action="store_true")
    ap.add_argument("--ws", type=int, default=0)
    ap.add_argument("--q", type=int, default=0)
    ap.add_argument("--reps", type=int, default=2)
    args = ap.parse_args()
    t0 = time.time()
    spec, X, y, Xt, yt = datagen.make_config(args.config, n_train=args.n, n_test=args.m)
    print(f"data {args.config} n={len(y)} m={len(yt)} gen {time.time() - t0:.1f}s", flush=True)
    dev = torch.device("cuda:0")
    Xd, yd, Xtd = (torch.from_numpy(a).to(dev) for a in (X, y, Xt))
    opts = dict(cache_bytes=1 if args.rc else 0, ws_size=args.ws, q=args.q)
    for r in range(args.reps):
        torch.cuda.synchronize()
        t = time.time()
        model = gm.train(Xd, yd, spec.k, spec.C, spec.gamma, args.eps, **opts)
        torch.cuda.synchronize()
        t_train = time.time() - t
        t = time.time()
        prob = model.predict_proba(Xtd)
        torch.cuda.synchronize()
        t_pred = time.time() - t
        st = model.train_stats()
        acc = float((prob.argmax(1).cpu().numpy() == yt).mean())
        print(f"rep {r}: train {t_train:.3f}s predict {t_pred:.3f}s acc {acc:.4f} regime {st['cache_regime']} "
              f"solver {st['t_solver_ms']:.1f}ms kernel {st['t_kernel_ms']:.1f}ms outer_max {st['outer_iters_max']} "
              f"outer_sum {st['outer_iters_sum']} inner_sum {st['inner_iters_sum']} n_sv {st['n_sv']} "
              f"kvalues {st['kernel_values']:.3e} krow_launches {st['krow_launches']} launches {st['launches']}",
              flush=True)


if __name__ == "__main__":
    main()
