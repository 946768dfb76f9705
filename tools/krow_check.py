"""Quick check of the symmetric kernel-value launch (tensor-core or SIMT by GMPSVM_KROW)."""
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402

import datagen  # noqa: E402
import oracle  # noqa: E402
import paper_conf_icde_wenshcc19_b200 as gm  # noqa: E402

for n, d, g in [(300, 8, 0.5), (1000, 784, 0.125), (777, 16, 0.5)]:
    if d == 784:
        _, X, _, _, _ = datagen.make_config("mnist", n_train=n, n_test=1)
    else:
        X = np.random.default_rng(n).normal(0, 0.5, size=(n, d)).astype(np.float32)
    K = gm.rbf_kernel(X, X, g)
    K64 = oracle.rbf_matrix(X, X, g)
    rel = np.abs(K.astype(np.float64) - K64) / np.maximum(K64, 1e-30)
    i, j = np.unravel_index(np.argmax(rel), rel.shape)
    d2 = -np.log(K64[i, j]) / g
    nx = (X.astype(np.float64) ** 2).sum(1)
    print(f"n={n} d={d}: max rel err {rel.max():.3e} median {np.median(rel):.3e} p99.9 {np.quantile(rel, 0.999):.3e} "
          f"sym {np.abs(K-K.T).max():.1e} diag {np.abs(np.diag(K)-1).max()} | at max: K64 {K64[i,j]:.3e} d2 {d2:.1f} "
          f"|x|2 {nx[i]:.1f} |y|2 {nx[j]:.1f}", flush=True)
spec, X, y, _, _ = datagen.make_config("mnist")
Xd = torch.from_numpy(X).cuda()
for rep in range(3):
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    m = gm.train(Xd, torch.from_numpy(y).cuda(), 10, spec.C, spec.gamma, 1e-3)
    torch.cuda.synchronize()
    s = m.train_stats()
    print(f"train {1e3*(time.perf_counter()-t0):.1f} ms, krow {s['t_kernel_ms']:.2f} ms = "
          f"{s['kernel_flops']/s['t_kernel_ms']/1e9:.1f} TFLOP/s, nsv {s['n_sv']}", flush=True)
