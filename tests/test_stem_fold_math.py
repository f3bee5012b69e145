"""D16 (stem fold) as a mathematical identity, on CPU against the oracle conv:
a conv over few channels equals the R2 x 1, stride-1, unpadded conv of the
folded input with the regrouped weights (D16), for the geometries the
runtime folds (ResNet-50's 7x7 s2 p3 stem, R not a multiple of the stride,
stride 3) -- exact up to fp64 rounding, since the two sums hold the same
products plus zeros."""
import numpy as np
import pytest

from oracle import ops

from .stem_fold_ref import fold_input, fold_weights

CASES = [  # (C, K, H, W, R, stride, pad)
    (3, 8, 37, 36, 7, 2, 3),
    (3, 5, 29, 44, 7, 2, 3),
    (4, 6, 20, 20, 5, 2, 2),
    (2, 4, 40, 32, 5, 3, 2),
    (1, 3, 12, 16, 3, 1, 1),
]


@pytest.mark.parametrize("case", CASES, ids=[str(c) for c in CASES])
def test_fold_identity(case):
    c, k, h, w, r, st, pd = case
    rng = np.random.default_rng(7)
    x = rng.standard_normal((2, c, h, w))
    wt = rng.standard_normal((k, c, r, r))
    ref = ops.conv2d(x, wt, None, (st, st), (pd, pd))
    got = ops.conv2d(fold_input(x, r, r, (st, st), (pd, pd)), fold_weights(wt, (st, st)), None)
    assert got.shape == ref.shape
    np.testing.assert_allclose(got, ref, rtol=0, atol=1e-12 * np.abs(ref).max())


def test_fold_catches_a_wrong_index():
    """The identity is sharp: regrouping the weights with j and the tap swapped
    (a plausible indexing slip) breaks it."""
    c, k, h, w, r, st, pd = CASES[0]
    rng = np.random.default_rng(8)
    x = rng.standard_normal((1, c, h, w))
    wt = rng.standard_normal((k, c, r, r))
    ref = ops.conv2d(x, wt, None, (st, st), (pd, pd))
    bad = fold_weights(np.flip(wt, axis=3).copy(), (st, st))
    got = ops.conv2d(fold_input(x, r, r, (st, st), (pd, pd)), bad, None)
    assert np.abs(got - ref).max() > 1e-3 * np.abs(ref).max()
