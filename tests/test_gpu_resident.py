"""The fully asynchronous single-launch kernel (k_block_resident) when it cannot have all its
blocks resident at once (R12).

k_block_resident gives each thread block one subdomain for the whole solve and lets a block lead
the last completed global iteration by at most `lead` sweeps (P:109's bounded delay). If other
work holds most of the SMs, some blocks cannot start until others exit: a waiting block then
times out (~2 ms), the launch stops, and the host continues the solve from the current iterate
with per-launch kernels. Before that fix the waiting blocks went on "unpaced" without publishing
residuals, no global iteration ever completed, and the solve ran to max_global_iters (VERDICT
r01). A test-only helper kernel (tests/helpers/spin.cu) holds all but two SMs.
"""
import ctypes
import os
import time

import numpy as np
import pytest

import oracle as O
import workloads as W
from conftest import ROOT

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def spin():
    from tools.build import build_test_helpers

    lib = ctypes.CDLL(build_test_helpers())
    lib.spin_launch.restype = ctypes.c_int
    lib.spin_launch.argtypes = [ctypes.c_int, ctypes.c_int, ctypes.c_int, ctypes.c_ulonglong, ctypes.c_void_p]
    lib.spin_sm_count.restype = ctypes.c_int
    lib.spin_sm_count.argtypes = [ctypes.c_int]
    return lib


@pytest.mark.parametrize("n,envelope", [(2000, (15, 35)), (20000, (15, 35))])
@pytest.mark.parametrize("graph", [0, -1])
def test_single_launch_with_device_held(bar, spin, n, envelope, graph):
    """Trefethen_2000 / _20000 (C1 / C3, R = 128), async-(5): with all but two SMs held by another
    stream's kernel, the solve still converges, with an iteration count inside the P5 envelope
    (not max_global_iters), and the exact residual holds."""
    import torch

    A = W.trefethen(n)
    b = np.ones(n)
    M = bar.Matrix.from_csr(A, 128, tuning={"graph": graph})
    bd = torch.from_numpy(b).cuda()
    x = torch.empty_like(bd)
    _, info0 = M.solve(bd, None, x, k=5, tol=1e-10, mode="async")  # normal: captured / resident
    assert "resident" in M.info()["last_sweep_kernel"] and info0["converged"]
    s_spin, s_solve = torch.cuda.Stream(), torch.cuda.Stream()
    sms = spin.spin_sm_count(0)
    for rep in range(2):  # the first pass also loads the fallback kernels (lazy module loading)
        assert spin.spin_launch(sms - 2, 1024, 200 * 1024, 400_000_000, ctypes.c_void_p(s_spin.cuda_stream)) == 0
        time.sleep(0.05)  # the spinner now holds sms - 2 SMs for ~0.35 s more
        t0 = time.perf_counter()
        _, info = M.solve(bd, None, x, k=5, tol=1e-10, mode="async", stream=s_solve, max_global_iters=20000)
        s_solve.synchronize()
        dt = time.perf_counter() - t0
        torch.cuda.synchronize()
    assert info["converged"] and info["rel_res"] <= 1e-10, info
    assert O.rel_res(A, b, x.cpu().numpy()) <= 1e-10 * (1 + 1e-6)
    assert envelope[0] <= info["iters"] <= envelope[1], info
    # the fallback ran per-launch kernels (the single launch alone is 3 launches)
    assert info["kernel_launches"] > 4, info
    assert dt < 0.3, dt  # finished while the spinner still held the device
    M.close()
