"""Small solves that exercise every default kernel path once, for compute-sanitizer
(memcheck / racecheck / synccheck). Not a test of results — the GPU test suite
checks those; here every launch must run clean under the sanitizer.

    compute-sanitizer --tool memcheck python tools/sanitize_cases.py
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    import numpy as np
    import torch

    import workloads as W
    from paper_conf_ipps_anzttdh12_b200 import bar
    from paper_conf_ipps_anzttdh12_b200 import dist as D

    cases = [
        ("tref500 resident (single launch)", W.trefethen(500), 128, {}),
        ("tref500 work-queue single launch", W.trefethen(500), 128, {"resident": -1}),
        ("tref500 per-launch stage", W.trefethen(500), 128, {"single_launch": -1}),
        ("s7_m32 duo (default, b_J/x_J staged)", W.stencil7_3d(32), 256, {"single_launch": -1}),
        ("s7_m32 duo coded, b/x direct", W.stencil7_3d(32), 256, {"single_launch": -1, "stage_bx": -1}),
        ("s7_m32 duo staged gathers", W.stencil7_3d(32), 256, {"single_launch": -1, "coded": 2}),
        ("s7_m32 duo int32", W.stencil7_3d(32), 256, {"single_launch": -1, "coded": -1}),
        ("s7_m24 pipe", W.stencil7_3d(24), 288, {"duo": -1, "pipe": 1}),
        ("s9_m40 k_block", W.stencil9_2d(40), 100, {"kernel": "block"}),
        ("s9_m40 k_reg_tma", W.stencil9_2d(40), 128, {"kernel": "reg_tma"}),
        ("s9_m40 k_block_pers", W.stencil9_2d(40), 128, {"kernel": "pers"}),
        ("s9_m40 rowwise jacobi", W.stencil9_2d(40), 128, {"jacobi_rowwise": 1}),
    ]
    for name, A, R, tune in cases:
        M = bar.Matrix.from_csr(A, R, tuning=tune)
        b = torch.ones(A.n, dtype=torch.float64, device="cuda")
        x0 = torch.from_numpy(np.random.default_rng(1).uniform(-1, 1, A.n)).cuda()
        kernels = []
        for mode, k in (("async", 5), ("sync-block", 5), ("jacobi", 1), ("async", 2)):
            M.solve(b, x0, None, k=k, max_global_iters=6, tol=0.0, mode=mode)
            kernels.append(M.info()["last_sweep_kernel"])
        M.solve(b, None, None, k=5, tol=1e-8, mode="async")
        kernels.append(M.info()["last_sweep_kernel"])
        r = M.residual(b, x0)
        print(f"{name}: ok ({', '.join(dict.fromkeys(kernels))}; residual {r[0]:.3e})", flush=True)
        M.close()
    # the partitioned path: loopback ranks, collective exchange and peer memory
    A = W.stencil7_3d(16)
    blocks = [W.stencil7_3d(16, row_lo=a, row_hi=c) for a, c in D.partition(A.n, 128, 3)]
    G = D.LoopbackGroup(blocks, A.n, 128)
    bs = [torch.ones(c - a, dtype=torch.float64, device="cuda") for a, c in G.ranges]
    G.solve(bs, None, None, k=5, max_global_iters=6, tol=0.0, mode="sync-block")
    G.enable_p2p()
    G.solve(bs, None, None, k=5, tol=1e-8, mode="async")
    G.close()
    print("loopback dist (collective + peer memory): ok", flush=True)
    torch.cuda.synchronize()


if __name__ == "__main__":
    main()
