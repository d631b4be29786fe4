"""Outlier study for the resident single-launch kernel: iteration count, max sweeps per block and
exact residual of repeated C1 solves, with and without a concurrent NVML-polling thread."""
import collections, os, sys, threading, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import bench
from paper_conf_ipps_anzttdh12_b200 import bar
A = bench.make_matrix("c1"); M = bar.Matrix.from_csr(A, 128)
b = torch.ones(A.n, dtype=torch.float64, device="cuda"); x = torch.empty_like(b)
def run(tag):
    c = collections.Counter()
    for _ in range(100):
        _, info = M.solve(b, None, x, k=5, tol=1e-10, mode="async")
        c[(info["iters"], info["cta_iters_max"])] += 1
    print(tag, sorted(c.items()), flush=True)
run("plain")
clk = bench.ClockSampler(0)
with clk:
    run("with NVML sampler")
run("plain again")
