"""Pins the tcgen05 conventions of csrc/tc.cuh (descriptors, canonical layouts,
TMEM lane mapping, 3xTF32 split) against a plain fp64 product."""
import numpy as np
import pytest
import torch

import gen
from helpers import to_gpu

pytestmark = pytest.mark.gpu


def _cond(A, B):
    return np.abs(A) @ np.abs(B)


@pytest.mark.parametrize("M,K,N", [(128, 8, 16), (128, 64, 96), (256, 96, 64), (128, 32, 256), (384, 128, 32),
                                   (128, 64, 128), (128, 128, 48)])
def test_tc_gemm_kmajor(stg, M, K, N):
    A = gen.uniform_pm1(1, M + K, M * K).reshape(M, K).astype(np.float64)
    B = gen.uniform_pm1(2, K + N, K * N).reshape(K, N).astype(np.float64)
    C = stg.stg_debug_tc_gemm(0, to_gpu(A), to_gpu(B)).cpu().numpy()
    err = np.max(np.abs(C - A @ B) / _cond(A, B))
    assert err < 2e-6, err      # 3xTF32: ~fp32-class (plain TF32 would be ~1e-3)


@pytest.mark.parametrize("R,N", [(128, 32), (512, 96), (1024, 64), (256, 128)])
def test_tc_gemm_mn_major_reduction(stg, R, N):
    X = gen.uniform_pm1(3, R, R * 128).reshape(R, 128).astype(np.float64)
    Y = gen.uniform_pm1(4, N, R * N).reshape(R, N).astype(np.float64)
    C = stg.stg_debug_tc_gemm(1, to_gpu(X), to_gpu(Y)).cpu().numpy()
    err = np.max(np.abs(C - X.T @ Y) / _cond(X.T, Y))
    assert err < 2e-6, err


@pytest.mark.parametrize("M,K,N", [(128, 8, 16), (128, 64, 96), (256, 96, 64), (128, 128, 32), (128, 32, 256)])
def test_tc_gemm_a_in_tmem(stg, M, K, N):
    """A operand written to tensor memory by the threads (tcgen05.st, lane = row,
    column = k) and read by tcgen05.mma.kind::tf32 [d], [a_tmem], b_desc."""
    A = gen.uniform_pm1(5, M + K, M * K).reshape(M, K).astype(np.float64)
    B = gen.uniform_pm1(6, K + N, K * N).reshape(K, N).astype(np.float64)
    C = stg.stg_debug_tc_gemm(2, to_gpu(A), to_gpu(B)).cpu().numpy()
    err = np.max(np.abs(C - A @ B) / _cond(A, B))
    assert err < 2e-6, err


def _tf32_trunc(x):
    u = np.asarray(x, np.float32).view(np.uint32) & np.uint32(0xFFFFE000)
    return u.view(np.float32).astype(np.float64)


def _tf32_rna(x):
    u = np.asarray(x, np.float32).view(np.uint32).astype(np.uint64)
    u = ((u + np.uint64(0x1000)) & np.uint64(0xFFFFE000)).astype(np.uint32)
    return u.view(np.float32).astype(np.float64)


def test_tf32_input_conversion(stg):
    """Pins how kind::tf32 reads fp32 operands: one unsplit pass equals the
    product of the TRUNCATED (low 13 mantissa bits dropped) operands, which is
    why 3xTF32 takes hi = a & 0xFFFFE000 and lo = a - hi."""
    M, K, N = 128, 64, 64
    A = gen.uniform_pm1(7, 1, M * K).reshape(M, K).astype(np.float64)
    B = gen.uniform_pm1(8, 1, K * N).reshape(K, N).astype(np.float64)
    C = stg.stg_debug_tc_gemm(3, to_gpu(A), to_gpu(B)).cpu().numpy()
    cond = _cond(A, B)
    e_trunc = np.max(np.abs(C - _tf32_trunc(A) @ _tf32_trunc(B)) / cond)
    e_rna = np.max(np.abs(C - _tf32_rna(A) @ _tf32_rna(B)) / cond)
    print("tf32 conversion: err vs truncation %.3g, vs round-nearest %.3g" % (e_trunc, e_rna))
    assert e_trunc < 1e-6 and e_rna > 1e-5, (e_trunc, e_rna)


@pytest.mark.parametrize("R,N", [(128, 32), (512, 96), (1024, 64), (256, 32)])
def test_tc_gemm_mn_major_tma(stg, R, N):
    """Xᵀ·Y with both operands loaded by 2-D TMA boxes in the MN-major
    SWIZZLE_128B_BASE32B layout (the reduction GEMMs dW / dL): no thread
    transposition, hi = raw (truncation), lo computed in place."""
    X = gen.uniform_pm1(9, R, R * 128).reshape(R, 128).astype(np.float64)
    Y = gen.uniform_pm1(10, N, R * N).reshape(R, N).astype(np.float64)
    C = stg.stg_debug_tc_gemm(4, to_gpu(X), to_gpu(Y)).cpu().numpy()
    err = np.max(np.abs(C - X.T @ Y) / _cond(X.T, Y))
    assert err < 2e-6, err


@pytest.mark.parametrize("nb", [1, 15, 17, 148, 296, 1024])
@pytest.mark.parametrize("n", [1, 100, 4103])
def test_sum_parts_parallel_is_bit_identical(stg, nb, n):
    """k_tc_sum_parts2 (parallel over 16-partial groups) == k_tc_sum_parts (serial)
    bit for bit, and both == the fp32 sum in the documented order (blocks of 16 in
    order, then the block sums in order)."""
    rng = np.random.default_rng(nb * 7919 + n)
    part = (rng.standard_normal((nb, n)) * 1e3 ** rng.integers(-1, 2, (nb, n))).astype(np.float32)
    pg = to_gpu(part)
    a = stg.stg_debug_sum_parts(pg, 0).cpu().numpy()
    b = stg.stg_debug_sum_parts(pg, 1).cpu().numpy()
    assert np.array_equal(a.view(np.uint32), b.view(np.uint32))
    want = np.zeros(n, np.float32)
    for b0 in range(0, nb, 16):
        blk = np.zeros(n, np.float32)
        for k in range(b0, min(b0 + 16, nb)):
            blk = (blk + part[k]).astype(np.float32)
        want = (want + blk).astype(np.float32)
    assert np.array_equal(a.view(np.uint32), want.view(np.uint32))
