"""Pins of oracle.extend_add (§III-A: the child's Schur complement is
"added into the parent frontal matrix ... this requires a scatter operation").

The pins do not retype the oracle's loop: they use the selection-matrix form
Fp + R^T F22 R (R[i, rel_i] = 1, an n2 x np matrix) by a numpy matmul on
integer-valued data (exact), the identity-map special case (a plain matrix
sum), invariants (total sum, untouched entries) and argument errors.
"""
import numpy as np
import pytest

import irrgen
import oracle


def _ints(rng, m, n):
    return np.asfortranarray(rng.integers(-50, 50, size=(m, n)).astype(np.float64))


@pytest.mark.parametrize("np_,n2", [(1, 1), (7, 3), (40, 17), (64, 64), (33, 1)])
def test_selection_matrix_form(np_, n2):
    rng = np.random.default_rng(np_ * 100 + n2)
    Fp, F22 = _ints(rng, np_, np_), _ints(rng, n2, n2)
    rel = np.sort(rng.choice(np_, size=n2, replace=False))
    R = np.zeros((n2, np_))
    R[np.arange(n2), rel] = 1.0
    want = Fp + R.T @ F22 @ R
    got = oracle.extend_add(Fp, F22, rel)
    assert np.array_equal(got, want)


def test_identity_map_is_matrix_sum():
    rng = np.random.default_rng(5)
    Fp, F22 = _ints(rng, 20, 20), _ints(rng, 20, 20)
    assert np.array_equal(oracle.extend_add(Fp, F22, np.arange(20)), Fp + F22)


def test_unsorted_map_and_invariants():
    rng = np.random.default_rng(9)
    Fp, F22 = _ints(rng, 30, 30), _ints(rng, 12, 12)
    rel = rng.choice(30, size=12, replace=False)          # any order, not only sorted
    got = oracle.extend_add(Fp, F22, rel)
    assert got.sum() == Fp.sum() + F22.sum()
    mask = np.ones((30, 30), bool)
    mask[np.ix_(rel, rel)] = False
    assert np.array_equal(got[mask], Fp[mask])            # outside rel x rel untouched
    assert np.array_equal(got[np.ix_(rel, rel)], Fp[np.ix_(rel, rel)] + F22)


def test_two_children_commute_on_integers():
    lvl = irrgen.extend_add_level(3, 4, 40)
    nps, parent, n2, rel, F22, Fp = lvl
    for p in range(len(nps)):
        kids = np.nonzero(parent == p)[0]
        a = np.asfortranarray(np.round(Fp[p] * 64))
        x = [np.asfortranarray(np.round(F22[c] * 64)) for c in kids]
        r1 = oracle.extend_add(oracle.extend_add(a, x[0], rel[kids[0]]), x[1], rel[kids[1]])
        r2 = oracle.extend_add(oracle.extend_add(a, x[1], rel[kids[1]]), x[0], rel[kids[0]])
        assert np.array_equal(r1, r2)


def test_empty_child_and_errors():
    Fp = np.ones((4, 4), order="F")
    assert np.array_equal(oracle.extend_add(Fp, np.zeros((0, 0)), np.zeros(0, np.int32)), Fp)
    with pytest.raises(ValueError):
        oracle.extend_add(Fp, np.ones((2, 2)), np.array([0, 4]))
    with pytest.raises(ValueError):
        oracle.extend_add(Fp, np.ones((2, 2)), np.array([-1, 0]))


def test_level_generator_shapes():
    nps, parent, n2, rel, F22, Fp = irrgen.extend_add_level(1, 10, 100)
    assert len(parent) == 20 and len(rel) == 20
    for c in range(20):
        s = nps[parent[c]]
        assert 1 <= n2[c] <= s and F22[c].shape == (n2[c], n2[c])
        assert np.all(np.diff(rel[c]) > 0) and rel[c][0] >= 0 and rel[c][-1] < s
