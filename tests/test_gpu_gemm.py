"""Dense-transform kernels in isolation (mars_debug_gemm) vs fp64 numpy:
tcgen05 3xFP16 ('auto' rows) and 3xTF32 ('3xtf32', and 'auto' dW) and FFMA
paths, ragged row counts, both operand majors, wide dynamic ranges."""
import numpy as np
import pytest

import paper_conf_icpp_lancl21_b200 as mars
from tests.util import scaled_err

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("impl", ["auto", "3xtf32", "simt"])
@pytest.mark.parametrize("M,N,K", [(128, 256, 64), (1000, 256, 256), (4133, 256, 64),
                                   (777, 64, 256), (300, 128, 256)])
def test_rows(impl, M, N, K):
    rng = np.random.default_rng(M + N + K)
    A = rng.standard_normal((M, K)).astype(np.float32)
    B = rng.standard_normal((N, K)).astype(np.float32)
    C, _ = mars.debug_gemm("rows", A, B, impl)
    ref = A.astype(np.float64) @ B.astype(np.float64).T
    e = scaled_err(C, ref)
    print(impl, M, N, K, e)
    assert e < 5e-6


@pytest.mark.parametrize("impl", ["auto", "simt"])
@pytest.mark.parametrize("H", [256, 128])
@pytest.mark.parametrize("M,K", [(16, 64), (5000, 256), (40001, 64), (123457, 256), (3001, 128)])
def test_dw(impl, H, M, K):
    rng = np.random.default_rng(M + K + H)
    A = rng.standard_normal((M, K)).astype(np.float32)
    B = rng.standard_normal((M, H)).astype(np.float32)
    C, _ = mars.debug_gemm("dw", A, B, impl)
    ref = A.astype(np.float64).T @ B.astype(np.float64)
    e = scaled_err(C, ref)
    print(impl, M, K, e)
    assert e < 5e-6


def _row_err(C, ref):
    """max over rows of the row-scaled error max_n |C - ref| / max_n |ref|."""
    num = np.max(np.abs(C - ref), axis=1)
    den = np.maximum(np.max(np.abs(ref), axis=1), 1e-300)
    return float(np.max(num / den))


@pytest.mark.parametrize("impl", ["auto", "3xtf32"])
@pytest.mark.parametrize("N,K", [(256, 256), (64, 256), (256, 64)])
def test_rows_dynamic_range(impl, N, K):
    """Rows spanning 1e-30 .. 1e30 (far outside fp16's range; the 3xFP16 kernel
    scales every row by a power of two), zero rows, and weights of magnitude
    1e4 and 1e-6: every row accurate relative to its own scale."""
    rng = np.random.default_rng(N + K)
    M = 1031
    A = rng.standard_normal((M, K))
    A *= 10.0 ** rng.uniform(-30, 30, (M, 1))
    A[rng.integers(0, M, 7)] = 0.0
    A = A.astype(np.float32)
    for wscale in (1e4, 1e-6):
        B = (rng.standard_normal((N, K)) * wscale).astype(np.float32)
        C, _ = mars.debug_gemm("rows", A, B, impl)
        ref = A.astype(np.float64) @ B.astype(np.float64).T
        e = _row_err(C, ref)
        print(impl, N, K, wscale, e)
        assert np.all(np.isfinite(C)) and e < 5e-6


def test_timing_report():
    rng = np.random.default_rng(0)
    R = 419232
    for K in (64, 256):
        A = rng.standard_normal((R, K)).astype(np.float32)
        W = rng.standard_normal((256, K)).astype(np.float32)
        D = rng.standard_normal((R, 256)).astype(np.float32)
        for impl in ("auto", "3xtf32", "simt"):
            _, t1 = mars.debug_gemm("rows", A, W, impl, iters=5)
            _, t2 = mars.debug_gemm("dw", A, D, impl, iters=5)
            print(f"TIMING K={K} {impl}: rows {t1:.3f} ms  dw {t2:.3f} ms")
