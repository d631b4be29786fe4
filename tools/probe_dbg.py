import os, sys
sys.path.insert(0, os.getcwd())
import torch, bench
from paper_conf_ipps_anzttdh12_b200 import bar
A = bench.make_matrix("c1"); M = bar.Matrix.from_csr(A, 128)
b = torch.ones(A.n, dtype=torch.float64, device="cuda"); x = torch.empty_like(b)
for i in range(8):
    _, info = M.solve(b, None, x, k=5, tol=1e-10, mode="async")
    torch.cuda.synchronize()
    print("SOLVE", i, info["iters"], info["cta_iters_max"], flush=True)
