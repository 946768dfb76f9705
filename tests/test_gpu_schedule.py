"""Scheduling of the training call must not change its result (engine.cu lead mode, cached solver
graphs / arena / tile list).  Every pair's solve is a deterministic chain of kernels whatever the
order the pairs run in, so the model is bitwise the same with lead mode off, with more lead pairs
and groups, with the graph cache disabled, when the cached graphs are reused or rebuilt after
a call of another shape, on the per-kernel graphs (default) or the persistent solver (opt-in), and
with the kernel values from 2-CTA clusters (default) or single CTAs.  The default configuration itself is parity-tested against the oracle
(test_gpu_parity.py, test_gpu_full.py).
"""
import os
import subprocess
import sys

import numpy as np
import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

SCRIPT = r"""
import os, sys
sys.path.insert(0, {root!r})
import numpy as np
import datagen
import paper_conf_icde_wenshcc19_b200 as gm
spec, X, y, Xt, yt = datagen.make_config("mnist", n_train=3000, n_test=200)
spec2, X2, y2, _, _ = datagen.make_config("letter", n_train=1500, n_test=10)
out = []
m1 = gm.train(X, y, spec.k, spec.C, spec.gamma, 1e-3)           # builds (or uses) the cached graphs
m2 = gm.train(X, y, spec.k, spec.C, spec.gamma, 1e-3)           # same shape: cached graphs relaunched
gm.train(X2, y2, spec2.k, spec2.C, spec2.gamma, 1e-3)           # another shape: cache rebuilt
m3 = gm.train(X, y, spec.k, spec.C, spec.gamma, 1e-3)           # and back
counts = np.bincount(y, minlength=spec.k)
for m in (m1, m2, m3):
    parts = []
    for s in range(spec.k):
        for t in range(s + 1, spec.k):
            info = m.pair(s, t, counts[s], counts[t])
            parts += [info["alpha"], np.array([info["b"], info["A"], info["B"]])]
    out.append(np.concatenate(parts))
    out.append(np.asarray(m.sv_index(), dtype=np.int64))
    out.append(np.asarray(m.predict_proba(Xt)))
np.savez({path!r}, *out)
"""


def _run(tmp_path, tag, env):
    path = str(tmp_path / f"{tag}.npz")
    e = dict(os.environ)
    e.update(env)
    r = subprocess.run([sys.executable, "-c", SCRIPT.format(root=ROOT, path=path)], env=e, capture_output=True,
                       text=True, timeout=600)
    assert r.returncode == 0, r.stderr[-2000:]
    z = np.load(path)
    return [z[f"arr_{i}"] for i in range(len(z.files))]


def test_schedule_does_not_change_the_model(tmp_path):
    base = _run(tmp_path, "default", {})
    for i in (3, 6):  # repeated calls and a rebuilt cache: bitwise the first call's model
        for j in range(3):
            np.testing.assert_array_equal(base[i + j], base[j])
    for tag, env in [("nolead", {"GMPSVM_LEAD": "0"}),
                     ("lead2_groups2", {"GMPSVM_LEAD": "2", "GMPSVM_GROUPS": "2", "GMPSVM_LEAD_RESERVE": "16"}),
                     ("noreuse", {"GMPSVM_GRAPH_REUSE": "0"}),
                     ("krow_no_cluster", {"GMPSVM_KROW_MC": "0"}),
                     ("persistent", {"GMPSVM_PERSIST": "1"}),
                     ("persistent_nolead", {"GMPSVM_PERSIST": "1", "GMPSVM_LEAD": "0"}),
                     ("persistent_lead_only", {"GMPSVM_PERSIST": "lead"})]:
        other = _run(tmp_path, tag, env)
        for a, b in zip(other, base):
            np.testing.assert_array_equal(a, b, err_msg=tag)
