"""The seeded input generators (rgsqr_inputs, shared by the oracle tests and the GPU tests;
no method arithmetic): chunked / storage-typed variants equal the reference constructions."""
import numpy as np
import pytest

import rgsqr_inputs as gi


@pytest.mark.parametrize("st", ["fp16", "bf16", "fp32"])
def test_dyadic_storage_equals_reference(st):
    A, R0 = gi.dyadic_mixed(4096, 300, seed=3)
    B, R1 = gi.dyadic_mixed_storage(4096, 300, seed=3, dtype=st, chunk=64)
    np.testing.assert_array_equal(gi.to_storage(A, st), B)
    np.testing.assert_array_equal(R0, R1)


def test_hadamard_cols_equals_hadamard():
    np.testing.assert_array_equal(gi.hadamard_cols(4096, 17, 99), gi.hadamard(4096, 99)[:, 17:])
    H = gi.hadamard_cols(1024, 0, 64)
    np.testing.assert_array_equal(H.T @ H, np.eye(64))
