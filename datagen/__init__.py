"""Seeded synthetic workloads shaped like the paper's datasets.

This module is shared by the CUDA path's tests/bench and by the oracle's
tests.  It holds NO arithmetic of the method (no kernel values, no SMO, no
sigmoid, no coupling) -- only random-number recipes that produce inputs.

Recipes follow SURVEY.md §8(d) "Synthetic inputs"; hyper-parameters follow
PAPER.md Table 2 (L381-L387) and BASELINE.json `configs`:

  blobs    3 classes, n=600, d=8, gamma=0.5,  C=1   (config 1)
  letter   26 classes, 20k x 16, gamma=0.5, C=10    (config 2)
  mnist    10 classes, 60k/10k x 784, gamma=0.125, C=10 (config 3, Table 2)
  covtype  7 classes, 581,012 x 54, gamma=1, C=3    (config 4)
  mnist8m  10 classes, 8.1M x 784, gamma=0.006, C=1000 (config 5, Table 2)
  news20   4 classes, 3k/600 x 5000 sparse text-like rows (~1.2 % non-zero), gamma=0.5, C=10
           (NEXT-3: the CSR path; shaped like the paper's News20 / RCV1 sparse inputs, L479, L513)

Every array is float32 features (row-major n x d) and int32 labels in [0, k).
"""
from __future__ import annotations

from dataclasses import dataclass

import numpy as np

__all__ = ["ConfigSpec", "CONFIGS", "make_config", "make_split", "subsample"]


@dataclass(frozen=True)
class ConfigSpec:
    name: str
    k: int
    d: int
    n_train: int
    n_test: int
    gamma: float
    C: float
    structure_seed: int
    train_seed: int
    test_seed: int


CONFIGS = {
    "blobs": ConfigSpec("blobs", 3, 8, 600, 200, 0.5, 1.0, 0, 0, 1),
    "letter": ConfigSpec("letter", 26, 16, 20_000, 5_000, 0.5, 10.0, 77, 1, 2),
    "mnist": ConfigSpec("mnist", 10, 784, 60_000, 10_000, 0.125, 10.0, 1234, 1, 2),
    "covtype": ConfigSpec("covtype", 7, 54, 581_012, 58_101, 1.0, 3.0, 4242, 1, 2),
    "mnist8m": ConfigSpec("mnist8m", 10, 784, 8_100_000, 10_000, 0.006, 1000.0, 1234, 3, 2),
    "news20": ConfigSpec("news20", 4, 5000, 3_000, 600, 0.5, 10.0, 2020, 1, 2),
}

_CHUNK = 100_000  # rows generated per child stream for the big configs


# ----------------------------------------------------------------------------------------
# blobs: centres ~ N(0, 0.5^2 I_8); train 200/class, x = centre + N(0, 0.5^2 I_8);
# test 200 points with uniform labels.  (SURVEY.md §8(d) row "1 blobs", Appendix A.2)
# ----------------------------------------------------------------------------------------
def _blobs_structure(spec: ConfigSpec):
    rng = np.random.default_rng(spec.structure_seed)
    return rng.normal(0.0, 0.5, size=(spec.k, spec.d))


def _blobs(spec: ConfigSpec, split: str, n: int):
    centres = _blobs_structure(spec)
    if split == "train":
        # structure and train share seed 0 (the recipe's "structure+train 0"): continue the stream
        rng = np.random.default_rng(spec.structure_seed)
        rng.normal(0.0, 0.5, size=(spec.k, spec.d))
        per = n // spec.k
        y = np.repeat(np.arange(spec.k), per)
        y = np.concatenate([y, np.arange(n - per * spec.k)])
    else:
        rng = np.random.default_rng(spec.test_seed)
        y = rng.integers(0, spec.k, size=n)
    X = centres[y] + rng.normal(0.0, 0.5, size=(n, spec.d))
    return X.astype(np.float32), y.astype(np.int32)


# ----------------------------------------------------------------------------------------
# letter: 26 classes x 3 sub-modes, mu ~ U(-0.6,0.6)^16, x = clip(mu + N(0,0.25^2), -1, 1),
# uniform labels, continuous (no quantisation -> no exact duplicates).
# ----------------------------------------------------------------------------------------
def _letter(spec: ConfigSpec, split: str, n: int):
    srng = np.random.default_rng(spec.structure_seed)
    modes = srng.uniform(-0.6, 0.6, size=(spec.k, 3, spec.d))
    rng = np.random.default_rng(spec.train_seed if split == "train" else spec.test_seed)
    y = rng.integers(0, spec.k, size=n)
    sub = rng.integers(0, 3, size=n)
    X = np.clip(modes[y, sub] + rng.normal(0.0, 0.25, size=(n, spec.d)), -1.0, 1.0)
    return X.astype(np.float32), y.astype(np.int32)


# ----------------------------------------------------------------------------------------
# mnist / mnist8m: 28x28 grid, 48 Gaussian bumps (sigma 2.2 px, centres U(5,23)^2) form a
# basis B (784 x 48).  Per class 10 active bumps: 5 shared by all classes + 5 of its own;
# base amplitudes U(0.6,1.1).  30 styles/class = base + N(0,0.6^2) on the active bumps;
# instance = style + N(0,0.5^2) on the active bumps; x = clip(B a - 0.3, 0, 1).
# Dense storage, most pixels exactly zero (like MNIST).
# ----------------------------------------------------------------------------------------
def _mnist_structure(spec: ConfigSpec):
    srng = np.random.default_rng(spec.structure_seed)
    n_bumps, side = 48, 28
    centres = srng.uniform(5.0, 23.0, size=(n_bumps, 2))
    yy, xx = np.meshgrid(np.arange(side), np.arange(side), indexing="ij")
    grid = np.stack([yy.ravel(), xx.ravel()], axis=1).astype(np.float64)  # 784 x 2
    d2 = ((grid[:, None, :] - centres[None, :, :]) ** 2).sum(-1)  # 784 x 48
    basis = np.exp(-d2 / (2.0 * 2.2 ** 2))
    shared = srng.choice(n_bumps, size=5, replace=False)
    rest = np.setdiff1d(np.arange(n_bumps), shared)
    active = np.zeros((spec.k, n_bumps), dtype=bool)
    base = np.zeros((spec.k, n_bumps))
    for c in range(spec.k):
        own = srng.choice(rest, size=5, replace=False)
        idx = np.concatenate([shared, own])
        active[c, idx] = True
        base[c, idx] = srng.uniform(0.6, 1.1, size=10)
    n_styles = 30
    styles = base[:, None, :] + srng.normal(0.0, 0.6, size=(spec.k, n_styles, n_bumps)) * active[:, None, :]
    return basis, active, styles


def _mnist_rows(spec, basis, active, styles, rng, n):
    y = rng.integers(0, spec.k, size=n)
    st = rng.integers(0, styles.shape[1], size=n)
    amp = styles[y, st] + rng.normal(0.0, 0.5, size=(n, basis.shape[1])) * active[y]
    X = np.clip(amp @ basis.T - 0.3, 0.0, 1.0)
    return X.astype(np.float32), y.astype(np.int32)


def _mnist(spec: ConfigSpec, split: str, n: int):
    basis, active, styles = _mnist_structure(spec)
    seed = spec.train_seed if split == "train" else spec.test_seed
    if n <= _CHUNK:
        return _mnist_rows(spec, basis, active, styles, np.random.default_rng(seed), n)
    X = np.empty((n, spec.d), dtype=np.float32)
    y = np.empty(n, dtype=np.int32)
    children = np.random.SeedSequence(seed).spawn((n + _CHUNK - 1) // _CHUNK)
    for c, ss in enumerate(children):
        lo, hi = c * _CHUNK, min(n, (c + 1) * _CHUNK)
        X[lo:hi], y[lo:hi] = _mnist_rows(spec, basis, active, styles, np.random.default_rng(ss), hi - lo)
    return X, y


# ----------------------------------------------------------------------------------------
# covtype: 10 continuous features with class-dependent means U(0.2,0.8), sigma 0.12,
# clipped to [0,1]; one-hot 4-way and 40-way categorical blocks with per-class
# Dirichlet(0.3) probabilities; class proportions of UCI covtype.
# ----------------------------------------------------------------------------------------
_COVTYPE_COUNTS = np.array([211_840, 283_301, 35_754, 2_747, 9_493, 17_367, 20_510], dtype=np.float64)


def _covtype(spec: ConfigSpec, split: str, n: int):
    srng = np.random.default_rng(spec.structure_seed)
    means = srng.uniform(0.2, 0.8, size=(spec.k, 10))
    p4 = srng.dirichlet(np.full(4, 0.3), size=spec.k)
    p40 = srng.dirichlet(np.full(40, 0.3), size=spec.k)
    rng = np.random.default_rng(spec.train_seed if split == "train" else spec.test_seed)
    y = rng.choice(spec.k, size=n, p=_COVTYPE_COUNTS / _COVTYPE_COUNTS.sum())
    X = np.zeros((n, 54), dtype=np.float32)
    X[:, :10] = np.clip(means[y] + rng.normal(0.0, 0.12, size=(n, 10)), 0.0, 1.0)
    u4 = rng.random(n)[:, None]
    c4 = (u4 > np.cumsum(p4[y], axis=1)).sum(1).clip(0, 3)
    u40 = rng.random(n)[:, None]
    c40 = (u40 > np.cumsum(p40[y], axis=1)).sum(1).clip(0, 39)
    X[np.arange(n), 10 + c4] = 1.0
    X[np.arange(n), 14 + c40] = 1.0
    return X, y.astype(np.int32)


# ----------------------------------------------------------------------------------------
# news20 (sparse, text-like): a Zipf word distribution over d words; each class prefers its own
# 250 topic words.  A document has 30 + Poisson(30) word draws, half from its class's topic words,
# half from the Zipf distribution; value = log(1 + count), rows scaled to unit L2 norm.
# ----------------------------------------------------------------------------------------
def _news20(spec: ConfigSpec, split: str, n: int):
    srng = np.random.default_rng(spec.structure_seed)
    zipf = 1.0 / np.arange(1, spec.d + 1) ** 1.1
    zipf /= zipf.sum()
    topics = np.stack([srng.choice(spec.d, size=250, replace=False) for _ in range(spec.k)])
    rng = np.random.default_rng(spec.train_seed if split == "train" else spec.test_seed)
    y = rng.integers(0, spec.k, size=n)
    X = np.zeros((n, spec.d), dtype=np.float32)
    for i in range(n):
        m = 30 + rng.poisson(30)
        h = m // 2
        words = np.concatenate([topics[y[i]][rng.integers(0, 250, size=h)], rng.choice(spec.d, size=m - h, p=zipf)])
        idx, cnt = np.unique(words, return_counts=True)
        v = np.log1p(cnt.astype(np.float64))
        X[i, idx] = (v / np.linalg.norm(v)).astype(np.float32)
    return X, y.astype(np.int32)


_GEN = {"blobs": _blobs, "letter": _letter, "mnist": _mnist, "mnist8m": _mnist, "covtype": _covtype,
        "news20": _news20}


def make_split(name: str, split: str, n: int | None = None):
    """Return (X float32 [n,d], y int32 [n]) for `split` in {"train","test"}.

    `n` overrides the config's size (used for parity-sized subsets); rows are a
    prefix-stable function of the seed only for n <= 100k.
    """
    spec = CONFIGS[name]
    if n is None:
        n = spec.n_train if split == "train" else spec.n_test
    X, y = _GEN[name](spec, split, int(n))
    return np.ascontiguousarray(X), np.ascontiguousarray(y)


def make_config(name: str, n_train: int | None = None, n_test: int | None = None):
    """(spec, Xtr, ytr, Xte, yte) for a named config."""
    spec = CONFIGS[name]
    Xtr, ytr = make_split(name, "train", n_train)
    Xte, yte = make_split(name, "test", n_test)
    return spec, Xtr, ytr, Xte, yte


def subsample(X, y, n: int, seed: int = 0):
    """Deterministic class-covering subsample of n rows (keeps original order)."""
    rng = np.random.default_rng(seed)
    idx = np.sort(rng.choice(X.shape[0], size=n, replace=False))
    return np.ascontiguousarray(X[idx]), np.ascontiguousarray(y[idx])
