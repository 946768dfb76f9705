"""The seeded input recipes: shapes, determinism and the structure each recipe
promises -- no method arithmetic is involved (datagen/ holds none)."""
import numpy as np

import datagen


def test_recipes_are_deterministic_and_shaped():
    for name, n, m in [("blobs", None, None), ("letter", 500, 50), ("mnist", 300, 30), ("news20", 200, 20)]:
        spec, X, y, Xt, yt = datagen.make_config(name, n_train=n, n_test=m)
        spec2, X2, y2, _, _ = datagen.make_config(name, n_train=n, n_test=m)
        assert X.dtype == np.float32 and y.dtype == np.int32
        assert X.shape[1] == spec.d and Xt.shape[1] == spec.d
        assert y.min() >= 0 and y.max() < spec.k
        np.testing.assert_array_equal(X, X2)
        np.testing.assert_array_equal(y, y2)


def test_news20_is_sparse_text_like():
    """NEXT-3's workload: ~1 % non-zero, non-negative, unit-norm rows, every class present."""
    spec, X, y, Xt, yt = datagen.make_config("news20", n_train=600, n_test=60)
    density = (X != 0).mean()
    assert 0.005 < density < 0.02
    assert (X >= 0).all()
    np.testing.assert_allclose(np.linalg.norm(X, axis=1), 1.0, rtol=1e-5)
    assert np.bincount(y, minlength=spec.k).min() > 0


def test_mnist_recipe_zero_fraction():
    """The calibration DESIGN.md §4 quotes: about two thirds of the pixels are exact zeros."""
    _, X, _, _, _ = datagen.make_config("mnist", n_train=1000, n_test=10)
    assert 0.6 < (X == 0).mean() < 0.75
