"""Launch a few sweeps of one workload for ncu (no timing here — ncu numbers are never bench values).

    ncu --set full -k regex:k_block -s 2 -c 2 -o gpurun_out/prof python tools/profile_sweep.py --workload c4
"""
import argparse
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--workload", default="c5")
    ap.add_argument("--mode", default="async")
    ap.add_argument("--k", type=int, default=5)
    ap.add_argument("--R", type=int, default=None)
    ap.add_argument("--sweeps", type=int, default=6)
    ap.add_argument("--tune", default="", help="bar_tuning fields, e.g. async_order=3")
    a = ap.parse_args()
    import torch

    import bench
    from paper_conf_ipps_anzttdh12_b200 import bar

    R = a.R or bench.WORKLOADS[a.workload][2]
    A = bench.make_matrix(a.workload)
    tune = {}
    for kv in filter(None, a.tune.split(",")):
        k, v = kv.split("=")
        tune[k] = int(v) if v.lstrip("-").isdigit() else v
    M = bar.Matrix.from_csr(A, rows_per_block=R, tuning=tune or None)
    del A
    b = torch.ones(M.n, dtype=torch.float64, device="cuda")
    x = torch.zeros(M.n, dtype=torch.float64, device="cuda")
    M.sweep(b, x, k=a.k, nsweeps=a.sweeps, mode=a.mode)
    torch.cuda.synchronize()
    print("done", M.info())


if __name__ == "__main__":
    main()
