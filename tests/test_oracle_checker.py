"""Pins for the parity checker itself: ``oracle.normalised_error`` (the
north_star comparison rule, BASELINE.json: elementwise |C_gpu - C_ref| / S
with S = sum_l |a_il||b_lj|, max over elements; S = 0 requires C_gpu = 0)
and ``oracle.to_row_major`` (how every column-major GPU output is read; the
layout convention of SURVEY.md 8(b): element (i, j) of a col-major R x C
matrix sits at j R + i).

Each case is hand-computed, and each is chosen so that a plausible mistake
turns it red: mean instead of max, a dropped S = 0 branch, a signed instead
of absolute difference, division by |C_ref| instead of S, an identity (or
plain reshape) view for column-major storage, a transpose that mixes batch
entries.  CPU only."""
import math

import numpy as np

import oracle


def arr(*x):
    return np.asarray(x, dtype=np.float64)


# ------------------------------------------------------------ normalised_error


def test_hand_value():
    # |1.5 - 1.0| / 2.0 = 0.25
    assert oracle.normalised_error(arr(1.5), arr(1.0), arr(2.0)) == 0.25


def test_absolute_difference():
    # |0.5 - 1.0| / 2.0 = 0.25 (a signed difference would give -0.25 or 0)
    assert oracle.normalised_error(arr(0.5), arr(1.0), arr(2.0)) == 0.25
    assert oracle.normalised_error(arr(0.5, 1.0), arr(1.0, 1.0), arr(2.0, 2.0)) == 0.25


def test_max_not_mean():
    # errors 0.25, 0, 0, 0 -> max 0.25 (mean 0.0625, median 0)
    got = oracle.normalised_error(arr(1.5, 3.0, -2.0, 7.0), arr(1.0, 3.0, -2.0, 7.0), arr(2.0, 4.0, 4.0, 8.0))
    assert got == 0.25


def test_normalised_by_scale_not_by_reference():
    # C_ref = 0 but S = 4 (cancellation: a b = +2 and -2): error |1 - 0| / 4
    assert oracle.normalised_error(arr(1.0), arr(0.0), arr(4.0)) == 0.25
    # large reference, small scale would be impossible; S >= |C_ref| always --
    # here S = 10, C_ref = 1, error |3 - 1| / 10 = 0.2 (|C_ref| would give 2)
    assert oracle.normalised_error(arr(3.0), arr(1.0), arr(10.0)) == 0.2


def test_zero_scale_requires_exact_zero():
    # S = 0 means every product a_il b_lj is 0: the GPU value must be exactly 0
    assert oracle.normalised_error(arr(0.0), arr(0.0), arr(0.0)) == 0.0
    assert oracle.normalised_error(arr(-0.0), arr(0.0), arr(0.0)) == 0.0  # -0 == 0
    assert math.isinf(oracle.normalised_error(arr(1e-300), arr(0.0), arr(0.0)))
    # one bad S = 0 element among good ones still fails
    assert math.isinf(oracle.normalised_error(arr(1.0, 2.0, 5e-8), arr(1.0, 2.0, 0.0), arr(1.0, 2.0, 0.0)))
    # and S = 0 elements with exact zeros do not mask a real error elsewhere
    assert oracle.normalised_error(arr(0.0, 1.5), arr(0.0, 1.0), arr(0.0, 2.0)) == 0.25


def test_nan_and_inf_outputs_fail():
    e = oracle.normalised_error(arr(np.nan, 1.0), arr(1.0, 1.0), arr(1.0, 1.0))
    assert math.isinf(e)  # a NaN output is never within tolerance
    assert math.isinf(oracle.normalised_error(arr(np.inf), arr(1.0), arr(1.0)))


def test_shapes_batched():
    c_ref = np.zeros((2, 2, 3))
    s = np.ones((2, 2, 3))
    c = c_ref.copy()
    c[1, 1, 2] = 0.125  # the worst element is the last one of the second entry
    assert oracle.normalised_error(c, c_ref, s) == 0.125
    assert oracle.normalised_error(np.zeros(0), np.zeros(0), np.zeros(0)) == 0.0


# ----------------------------------------------------------------- to_row_major


def test_row_major_is_reshape():
    X = np.arange(12)
    got = oracle.to_row_major(X, 2, 2, 3, "row")
    np.testing.assert_array_equal(got, [[[0, 1, 2], [3, 4, 5]], [[6, 7, 8], [9, 10, 11]]])


def test_col_major_hand_transposed():
    # M = [[1, 2, 3], [4, 5, 6]] (2 x 3) stored column-major: 1 4 2 5 3 6
    got = oracle.to_row_major(np.array([1, 4, 2, 5, 3, 6]), 1, 2, 3, "col")
    np.testing.assert_array_equal(got, [[[1, 2, 3], [4, 5, 6]]])
    # a plain reshape (the identity view) would read [[1, 4, 2], [5, 3, 6]]
    assert not np.array_equal(got[0], np.array([1, 4, 2, 5, 3, 6]).reshape(2, 3))


def test_col_major_batched_entries_stay_separate():
    # entry 0: [[1, 2], [3, 4], [5, 6]] (3 x 2), entry 1: 10x that; col-major packs
    # each entry's columns: 1 3 5 2 4 6 | 10 30 50 20 40 60
    X = np.array([1, 3, 5, 2, 4, 6, 10, 30, 50, 20, 40, 60])
    got = oracle.to_row_major(X, 2, 3, 2, "col")
    np.testing.assert_array_equal(got[0], [[1, 2], [3, 4], [5, 6]])
    np.testing.assert_array_equal(got[1], [[10, 20], [30, 40], [50, 60]])


def test_col_major_element_address():
    # element (i, j) of entry b of an R x C col-major batch is at b R C + j R + i
    R, C, batch = 5, 3, 4
    X = np.arange(batch * R * C)
    got = oracle.to_row_major(X, batch, R, C, "col")
    for b in range(batch):
        for i in range(R):
            for j in range(C):
                assert got[b, i, j] == b * R * C + j * R + i
