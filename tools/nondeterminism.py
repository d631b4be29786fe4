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


def table(workload="c1", runs=200, k=5, R=128, single_launch=-1, checkpoints=None, tuning=None):
    """[(m, residuals of `runs` independent async solves of exactly m global iterations)]."""
    import torch

    import bench
    from paper_conf_ipps_anzttdh12_b200 import bar

    A = bench.make_matrix(workload)
    M = bar.Matrix.from_csr(A, R, tuning=tuning)
    b = torch.ones(A.n, dtype=torch.float64, device="cuda")
    x = torch.empty_like(b)
    if checkpoints is None:
        checkpoints = list(range(5, 55, 5)) if workload == "c1" else list(range(10, 160, 10))
    out = []
    for m in checkpoints:
        res = []
        for _ in range(runs):
            _, info = M.solve(b, None, x, k=k, max_global_iters=m, tol=0.0, mode="async",
                              async_single_launch=single_launch)
            res.append(info["rel_res"])
        out.append((m, np.array(res)))
    M.close()
    return A.name, out


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--workload", default="c1", choices=["c1", "c2"])
    ap.add_argument("--runs", type=int, default=200)
    ap.add_argument("--k", type=int, default=5)
    ap.add_argument("--R", type=int, default=128)
    ap.add_argument("--single-launch", type=int, default=-1, help="-1 auto, 0 per-launch, 1 single launch")
    ap.add_argument("--lead", type=int, default=0, help="single-launch kernel's lead bound (0 = default 48)")
    a = ap.parse_args()
    from conftest import load_golden

    tab = "table3_trefethen2000.txt" if a.workload == "c1" else "table2_fv1.txt"
    paper = {int(r[0]): float(r[1]) for r in load_golden(tab)}
    name, rows = table(a.workload, a.runs, a.k, a.R, a.single_launch, tuning={"lead": a.lead} if a.lead else None)
    clk = os.popen("nvidia-smi --query-gpu=clocks.sm,clocks.max.sm,clocks_event_reasons.active --format=csv,noheader")
    print(f"# N2: async-({a.k}), R={a.R}, {name}, b=1, x0=0, {a.runs} runs per checkpoint, exact residuals;"
          f" lead {a.lead or 48}; clocks after the run: {clk.read().strip()}")
    print(f"# paper column: the 1000-run average of {tab} (C2070; fv1 there is the real fv1, here the "
          f"pattern-exact synthetic)")
    print(f"{'iters':>5} {'avg':>11} {'max':>11} {'min':>11} {'abs.var':>10} {'rel.var':>10} {'variance':>10} "
          f"{'std.dev':>10} {'std.err':>10} {'paper.avg':>11}")
    for m, r in rows:
        avg, mx, mn = r.mean(), r.max(), r.min()
        var = r.var(ddof=1) if len(r) > 1 else 0.0
        print(f"{m:5d} {avg:11.4e} {mx:11.4e} {mn:11.4e} {mx - mn:10.3e} {(mx - mn) / avg:10.3e} {var:10.3e} "
              f"{np.sqrt(var):10.3e} {np.sqrt(var / len(r)):10.3e} {paper.get(m, float('nan')):11.4e}")


if __name__ == "__main__":
    main()
