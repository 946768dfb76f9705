"""NEXT-3 measurement: the same CSR rows through the sparse kernel-value path (csr.cu) and through
the densified tensor-core path, news20-shaped (4 classes, d = 5000, ~1 % non-zero).

    python tools/sparse_probe.py [--n 3000 20000] [--reps 3]
Prints one JSON line per (n, path): kernel-value ms, train ms, predict ms, test accuracy.
"""
import argparse
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

CODE = r"""
import sys, json, time, numpy as np, scipy.sparse as sp, torch
sys.path.insert(0, {root!r})
import datagen, paper_conf_icde_wenshcc19_b200 as gm
spec, X, y, Xt, yt = datagen.make_config('news20', n_train={n}, n_test=1000)
A, At = sp.csr_matrix(X), sp.csr_matrix(Xt)
dev = torch.device('cuda:0')
def t(M):
    return (torch.from_numpy(M.indptr.astype(np.int64)).to(dev), torch.from_numpy(M.indices.astype(np.int32)).to(dev),
            torch.from_numpy(M.data.astype(np.float32)).to(dev), M.shape)
Ad, Atd, yd = t(A), t(At), torch.from_numpy(y).to(dev)
rows = []
for r in range({reps} + 1):
    torch.cuda.synchronize(); t0 = time.perf_counter()
    m = gm.train_csr(Ad, yd, spec.k, spec.C, spec.gamma, 1e-3)
    p = m.predict_proba_csr(Atd); torch.cuda.synchronize(); t1 = time.perf_counter()
    s = m.train_stats()
    rows.append(dict(kv_ms=s['t_kernel_ms'], train_ms=s['t_total_ms'], wall_ms=(t1 - t0) * 1e3, path=s['kernel_path'],
                     n_sv=s['n_sv'], acc=float((p.argmax(1).cpu().numpy() == yt).mean())))
best = min(rows[1:], key=lambda x: x['wall_ms'])
print(json.dumps(dict(n={n}, d=spec.d, nnz=int(A.nnz), density=A.nnz / X.size, **best)))
"""

ap = argparse.ArgumentParser()
ap.add_argument("--n", type=int, nargs="+", default=[3000, 20000])
ap.add_argument("--reps", type=int, default=3)
a = ap.parse_args()
for n in a.n:
    for mode in ("sparse", "dense"):
        r = subprocess.run([sys.executable, "-c", CODE.format(root=ROOT, n=n, reps=a.reps)], capture_output=True,
                           text=True, env=dict(os.environ, GMPSVM_CSR=mode), timeout=1800)
        line = r.stdout.strip().splitlines()[-1] if r.returncode == 0 else json.dumps({"error": r.stderr[-400:]})
        print(json.dumps({"mode": mode, **json.loads(line)}), flush=True)
