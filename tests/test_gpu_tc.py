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
