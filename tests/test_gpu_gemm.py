"""Dense-transform kernels in isolation (mars_debug_gemm) vs fp64 numpy:
tcgen05 3xFP16 ('auto') and FFMA ('simt') paths, ragged row counts, both
operand majors, wide dynamic ranges."""
import numpy as np
import pytest

import paper_conf_icpp_lancl21_b200 as mars
from tests.util import scaled_err

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("impl", ["auto", "simt"])
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
@pytest.mark.parametrize("M,K", [(16, 64), (16, 256), (33, 256), (5000, 256), (40001, 64), (123457, 256), (3001, 128)])
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


@pytest.mark.parametrize("N,K", [(256, 256), (64, 256), (256, 64)])
def test_rows_dynamic_range(N, K):
    """Rows spanning 1e-30 .. 1e30 and rows near the top of fp32's range
    (max |x| up to 2^126: the 3xFP16 kernel scales every row by a power of two,
    unclamped for large rows), zero rows, and weights of magnitude 1e4 and 1e-6:
    every row accurate relative to its own scale."""
    rng = np.random.default_rng(N + K)
    M = 1031
    A = rng.standard_normal((M, K))
    A *= 10.0 ** rng.uniform(-30, 30, (M, 1))
    A[rng.integers(0, M, 7)] = 0.0
    big = rng.integers(0, M, 9)
    A[big] = rng.standard_normal((9, K)) * 2.0 ** rng.uniform(110, 122, (9, 1))
    A = A.astype(np.float32)
    for wscale in (1e-4, 1e-6):
        B = (rng.standard_normal((N, K)) * wscale).astype(np.float32)
        C, _ = mars.debug_gemm("rows", A, B, "auto")
        ref = A.astype(np.float64) @ B.astype(np.float64).T
        e = _row_err(C, ref)
        print(N, K, wscale, e)
        assert np.all(np.isfinite(C)) and e < 5e-6


@pytest.mark.parametrize("H,K", [(256, 64), (256, 256), (128, 128)])
def test_dw_mixed_magnitude_columns(H, K):
    """The weight gradient scales each operand by ONE power of two per row chunk
    (the chunk's largest value), so its error bound is normwise
    per chunk, not per element.  Columns whose magnitudes span 8 decades
    (shape features normalised to ~1e-6 next to one-hot features) must still
    meet the componentwise GEMM bound |err_ij| <= tol · Σ_r |A_ri| |B_rj|."""
    rng = np.random.default_rng(H + K)
    M = 20011
    A = rng.standard_normal((M, K)) * 10.0 ** rng.uniform(-8, 0, (1, K))
    B = rng.standard_normal((M, H)) * 10.0 ** rng.uniform(-4, 0, (1, H))
    A = A.astype(np.float32)
    B = B.astype(np.float32)
    C, _ = mars.debug_gemm("dw", A, B, "auto")
    A64, B64 = A.astype(np.float64), B.astype(np.float64)
    ref = A64.T @ B64
    bound = np.abs(A64).T @ np.abs(B64)
    comp = float(np.max(np.abs(C - ref) / bound))
    print("componentwise", H, K, comp, "normwise", scaled_err(C, ref))
    assert comp < 2e-5


# The tiny configuration's widths (H in {32, 64}, C_in in {16, 32}) on the
# tcgen05 kernels: wider tiles whose missing rows / columns TMA zero-fills.
@pytest.mark.parametrize("M,N,K", [(1000, 32, 16), (777, 64, 32), (300, 32, 64), (4133, 64, 16),
                                   (129, 32, 256), (5001, 32, 32)])
def test_rows_narrow(M, N, K):
    rng = np.random.default_rng(M + 3 * N + K)
    A = rng.standard_normal((M, K)).astype(np.float32)
    B = rng.standard_normal((N, K)).astype(np.float32)
    C, _ = mars.debug_gemm("rows", A, B, "auto")
    e = scaled_err(C, A.astype(np.float64) @ B.astype(np.float64).T)
    print("rows narrow", M, N, K, e)
    assert e < 5e-6


@pytest.mark.parametrize("M,K,H", [(5000, 16, 32), (3001, 32, 64), (40001, 16, 64), (777, 64, 32),
                                   (12345, 32, 32), (1000, 256, 32), (2048, 128, 64)])
def test_dw_narrow(M, K, H):
    rng = np.random.default_rng(M + K + 7 * H)
    A = rng.standard_normal((M, K)).astype(np.float32)
    B = rng.standard_normal((M, H)).astype(np.float32)
    C, _ = mars.debug_gemm("dw", A, B, "auto")
    e = scaled_err(C, A.astype(np.float64).T @ B.astype(np.float64))
    print("dw narrow", M, K, H, e)
    assert e < 5e-6


# Large launches (M >= 2 x 128 x SMs) run the CTA-pair row kernel
# (k_tc3h_rows_pair: half the weight operand per CTA, cta_group::2 MMAs),
# including an odd tile count (the odd CTA's last tile is empty).
@pytest.mark.parametrize("M,K", [(100003, 256), (419232, 256), (77777, 64), (38144, 128)])
def test_rows_pair(M, K):
    rng = np.random.default_rng(M + K)
    A = rng.standard_normal((M, K)).astype(np.float32)
    A[::7] *= 1e-20                                  # rows of very different magnitude
    B = rng.standard_normal((256, K)).astype(np.float32)
    C, _ = mars.debug_gemm("rows", A, B, "auto")
    ref = A.astype(np.float64) @ B.astype(np.float64).T
    e = _row_err(C, ref)
    print("rows pair", M, K, e)
    assert e < 5e-6
