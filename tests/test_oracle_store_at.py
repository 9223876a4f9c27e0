"""Pins for oracle O8 (store_at / decouple_at, reading A26).

Each pin checks the oracle against something other than itself: a pure-Python
element loop, numpy's concatenate (the library routine the definition reduces
to), the inverse round trip, and — for the GEMM with the attached bias — the
textbook augmented-matrix identity  A W + 1 b^T = [A | 1] [W ; b^T].
"""
import itertools

import numpy as np
import pytest

from oracle.store_at import decouple_at, gemm_store_at_f64, store_at


def _rng(seed):
    return np.random.default_rng(seed)


@pytest.mark.parametrize("shape,dim", [((3, 4), 0), ((3, 4), 1), ((2, 3, 5), 1), ((2, 1, 3, 2), 3)])
def test_store_at_elementwise_loop(shape, dim):
    g = _rng(1)
    A = g.standard_normal(shape)
    b = g.standard_normal(shape[:dim] + shape[dim + 1:])
    Z = store_at(A, b, dim)
    E = shape[dim]
    assert Z.shape == shape[:dim] + (E + 1,) + shape[dim + 1:]
    for i in itertools.product(*[range(e) for e in Z.shape]):
        rest = i[:dim] + i[dim + 1:]
        want = A[i] if i[dim] < E else b[rest]
        assert Z[i] == want


@pytest.mark.parametrize("dim", [0, 1, 2])
def test_store_at_is_concatenate(dim):
    g = _rng(2)
    A = g.standard_normal((4, 5, 6))
    b = g.standard_normal(A.shape[:dim] + A.shape[dim + 1:])
    Z = store_at(A, b, dim)
    np.testing.assert_array_equal(Z, np.concatenate([A, np.expand_dims(b, dim)], axis=dim))


def test_decouple_inverts_store():
    g = _rng(3)
    A = g.standard_normal((7, 3))
    b = g.standard_normal(3)
    A2, b2 = decouple_at(store_at(A, b, 0), 0)
    np.testing.assert_array_equal(A2, A)
    np.testing.assert_array_equal(b2, b)
    Z = g.standard_normal((5, 4))
    np.testing.assert_array_equal(store_at(*decouple_at(Z, 1), 1), Z)


def test_store_at_rejects_bad_shapes():
    with pytest.raises(ValueError):
        store_at(np.zeros((3, 4)), np.zeros(3), 0)   # b must be [4]
    with pytest.raises(ValueError):
        decouple_at(np.zeros((1, 4)), 0)             # nothing attached


def test_gemm_attached_equals_augmented_matmul():
    g = _rng(4)
    M, K, N = 9, 13, 6
    A = g.standard_normal((M, K))
    W = g.standard_normal((K, N))
    bias = g.standard_normal(N)
    Z = store_at(W, bias, 0)
    Aaug = np.concatenate([A, np.ones((M, 1))], axis=1)
    np.testing.assert_allclose(gemm_store_at_f64(A, Z), Aaug @ Z, rtol=1e-13, atol=1e-13)


def test_gemm_attached_brute_force_epilogue():
    g = _rng(5)
    M, K, N = 3, 4, 5
    A, W = g.standard_normal((M, K)), g.standard_normal((K, N))
    bias, scale, res = g.standard_normal(N), g.standard_normal(N), g.standard_normal((M, N))
    Z = store_at(W, bias, 0)
    y = gemm_store_at_f64(A, Z, scale=scale, residual=res, act="relu")
    for m in range(M):
        for n in range(N):
            acc = 0.0
            for k in range(K):
                acc += A[m, k] * W[k, n]
            assert y[m, n] == pytest.approx(max(scale[n] * acc + bias[n] + res[m, n], 0.0), abs=1e-12)


def test_gemm_attached_zero_bias_is_plain_gemm():
    g = _rng(6)
    A, W = g.standard_normal((4, 8)), g.standard_normal((8, 3))
    np.testing.assert_allclose(gemm_store_at_f64(A, store_at(W, np.zeros(3), 0)), A @ W, rtol=1e-14)
