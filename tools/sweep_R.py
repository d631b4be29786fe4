"""Convergence / speed survey over the subdomain size R (tuning aid; numbers go to DESIGN.md)."""
import argparse
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--workload", default="c4")
    ap.add_argument("--R", default="1024,2048,4000,8000")
    ap.add_argument("--modes", default="async,sync-block")
    ap.add_argument("--k", default="5")
    a = ap.parse_args()
    import torch

    import bench
    from paper_conf_ipps_anzttdh12_b200 import bar

    A = bench.make_matrix(a.workload)
    n = A.n
    b = torch.ones(n, dtype=torch.float64, device="cuda")
    x = torch.empty_like(b)
    for R in [int(r) for r in a.R.split(",")]:
        M = bar.Matrix.from_csr(A, rows_per_block=R)
        for k in [int(v) for v in a.k.split(",")]:
            for mode in a.modes.split(","):
                M.solve(b, None, x, k=k, mode=mode)  # warm-up
                ts, its = [], []
                for _ in range(5):
                    torch.cuda.synchronize()
                    t0 = time.perf_counter()
                    _, info = M.solve(b, None, x, k=k, mode=mode)
                    torch.cuda.synchronize()
                    ts.append(time.perf_counter() - t0)
                    its.append(info["iters"])
                dt = sorted(ts)[2]
                print(json.dumps({"workload": a.workload, "R": R, "k": k, "mode": mode, "iters": info["iters"],
                                  "s": round(dt, 5), "ms_per_iter": round(dt / max(1, info["iters"]) * 1e3, 4),
                                  "rel_res": info["rel_res"], "iters_all": its,
                                  "kernel": M.info()["last_sweep_kernel"]}), flush=True)
        M.close()


if __name__ == "__main__":
    main()
