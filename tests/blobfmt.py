"""Test helper: write a gmpsvm model blob (the little-endian format of gmpsvm_model_serialize,
csrc/api.cpp) from Python, so the multi-process model plumbing can be exercised on CPU
without training on a GPU."""
import ctypes as ct
import struct

import numpy as np


def pair_list(k):
    return [(s, t) for s in range(k) for t in range(s + 1, k)]


def make_blob(X, y, k, C, gamma, eps, alphas, b, A, B, stats_size):
    """alphas: dict pair_index -> alpha array (pair-local order) for the trained pairs."""
    n, d = X.shape
    P = k * (k - 1) // 2
    counts = np.bincount(y, minlength=k).astype(np.int64)
    perm = np.argsort(y, kind="stable").astype(np.int64)  # sorted position -> original index
    off = np.concatenate([[0], np.cumsum(counts)])
    pairs = pair_list(k)
    sizes = [counts[s] + counts[t] for s, t in pairs]
    po = np.concatenate([[0], np.cumsum(sizes)]).astype(np.int64)
    trained = np.zeros(P, np.uint8)
    alpha = np.zeros(po[-1])
    sv = set()
    for p, a in alphas.items():
        s, t = pairs[p]
        trained[p] = 1
        alpha[po[p]:po[p + 1]] = a
        for j in np.flatnonzero(a > 0):
            g = off[s] + j if j < counts[s] else off[t] + (j - counts[s])
            sv.add(int(g))
    sv_pos = np.array(sorted(sv), dtype=np.int64)
    sv_X = X[perm[sv_pos]].astype(np.float32) if len(sv_pos) else np.zeros((0, d), np.float32)
    out = bytearray(b"GMPSVM01")
    out += struct.pack("<iiii", 1, k, d, 0)
    out += struct.pack("<ddd", C, gamma, eps)
    out += struct.pack("<q", n)
    out += counts.tobytes() + perm.tobytes() + trained.tobytes()
    out += np.asarray(b, np.float64).tobytes() + np.asarray(A, np.float64).tobytes()
    out += np.asarray(B, np.float64).tobytes() + np.zeros(P, np.int32).tobytes()
    out += alpha.tobytes()
    out += struct.pack("<q", len(sv_pos)) + sv_pos.tobytes() + sv_X.tobytes()
    out += bytes(stats_size)
    out += struct.pack("<di", 0.0, 3)  # kernel coef0, degree (the kernel type is the header's 4th int: 0 = RBF)
    return np.frombuffer(bytes(out), dtype=np.uint8), perm, sv_pos
