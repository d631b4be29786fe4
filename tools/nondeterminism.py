"""N2: run-to-run variation of async-(k) on B200, in the format of the paper's
Tables 2-3: for each checkpoint m, N independent async solves of exactly m
global iterations (tol = 0) and the EXACT relative residual of each, then avg / max / min / abs
and rel variation / variance / std dev / std error, next to the paper's 1000-run averages.

    python tools/nondeterminism.py --workload c1 --runs 200 > profiles/r01_n2_c1.txt
"""
import argparse
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--workload", default="c1", choices=["c1", "c2"])
    ap.add_argument("--runs", type=int, default=200)
    ap.add_argument("--k", type=int, default=5)
    ap.add_argument("--R", type=int, default=128)
    ap.add_argument("--single-launch", type=int, default=-1, help="-1 auto, 0 per-launch, 1 single launch")
    a = ap.parse_args()
    import torch

    import bench
    from conftest import load_golden
    from paper_conf_ipps_anzttdh12_b200 import bar

    A = bench.make_matrix(a.workload)
    M = bar.Matrix.from_csr(A, a.R)
    b = torch.ones(A.n, dtype=torch.float64, device="cuda")
    x = torch.empty_like(b)
    table, checkpoints = ("table3_trefethen2000.txt", list(range(5, 55, 5))) if a.workload == "c1" else \
        ("table2_fv1.txt", list(range(10, 160, 10)))
    paper = {int(r[0]): float(r[1]) for r in load_golden(table)}
    print(f"# N2: async-({a.k}), R={a.R}, {A.name}, b=1, x0=0, {a.runs} runs per checkpoint, exact residuals;")
    print(f"# paper column: the 1000-run average of {table} (C2070; fv1 there is the real fv1, here the "
          f"pattern-exact synthetic)")
    print(f"{'iters':>5} {'avg':>11} {'max':>11} {'min':>11} {'abs.var':>10} {'rel.var':>10} {'variance':>10} "
          f"{'std.dev':>10} {'std.err':>10} {'paper.avg':>11}")
    for m in checkpoints:
        res = []
        for _ in range(a.runs):
            _, info = M.solve(b, None, x, k=a.k, max_global_iters=m, tol=0.0, mode="async",
                              async_single_launch=a.single_launch)
            res.append(info["rel_res"])
        r = np.array(res)
        avg, mx, mn = r.mean(), r.max(), r.min()
        var = r.var(ddof=1) if len(r) > 1 else 0.0
        print(f"{m:5d} {avg:11.4e} {mx:11.4e} {mn:11.4e} {mx - mn:10.3e} {(mx - mn) / avg:10.3e} {var:10.3e} "
              f"{np.sqrt(var):10.3e} {np.sqrt(var / len(r)):10.3e} {paper.get(m, float('nan')):11.4e}")


if __name__ == "__main__":
    main()
