"""Fixed-cost breakdown of a small single-launch async solve (C1 / C3): wall and device time of
bar_solve through the binding and through ctypes directly, for max_global_iters = 0 / 1 / to tol,
and the graph-replayed kernel's own duration (tuning aid; not a bench value).

    python tools/latency_probe.py --workload c1
"""
import argparse
import ctypes
import os
import statistics
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--workload", default="c1")
    ap.add_argument("--reps", type=int, default=200)
    a = ap.parse_args()
    import torch

    import bench
    from paper_conf_ipps_anzttdh12_b200 import bar

    A = bench.make_matrix(a.workload)
    R = bench.WORKLOADS[a.workload][2]
    M = bar.Matrix.from_csr(A, R)
    b = torch.ones(A.n, dtype=torch.float64, device="cuda")
    x = torch.empty_like(b)
    st = torch.cuda.current_stream()
    info = bar.SolveInfo()
    h = M.handle

    def direct(maxit, tol):
        return bar._lib.bar_solve(h, b.data_ptr(), None, x.data_ptr(), 5, maxit, tol, 0, st.cuda_stream,
                                  ctypes.byref(info))

    for label, fn in (("binding, to 1e-10", lambda: M.solve(b, None, x, k=5, tol=1e-10, mode="async")),
                      ("ctypes, to 1e-10", lambda: direct(20000, 1e-10)),
                      ("ctypes, 1 iteration", lambda: direct(1, 0.0)),
                      ("ctypes, 0 iterations", lambda: direct(0, 0.0))):
        for _ in range(20):
            fn()
        torch.cuda.synchronize()
        walls, devs = [], []
        for _ in range(a.reps):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            t0 = time.perf_counter()
            e0.record(st)
            fn()
            e1.record(st)
            torch.cuda.synchronize()
            walls.append((time.perf_counter() - t0) * 1e6)
            devs.append(e0.elapsed_time(e1) * 1e3)
        print(f"{label:24s} wall {statistics.median(walls):7.1f} us  device span {statistics.median(devs):7.1f} us  "
              f"iters {info.iters}  kernel {info.sweep_kernel_ms * 1e3:.1f} us", flush=True)


if __name__ == "__main__":
    main()
