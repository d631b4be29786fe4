"""Distribution of iteration counts and kernel launches (resumes) of repeated small async solves."""
import collections, sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import bench
from paper_conf_ipps_anzttdh12_b200 import bar
w = sys.argv[1] if len(sys.argv) > 1 else "c1"
A = bench.make_matrix(w); M = bar.Matrix.from_csr(A, bench.WORKLOADS[w][2])
b = torch.ones(A.n, dtype=torch.float64, device="cuda"); x = torch.empty_like(b)
c = collections.Counter()
for _ in range(200):
    _, info = M.solve(b, None, x, k=5, tol=1e-10, mode="async")
    c[(info["iters"], info["kernel_launches"])] += 1
print(os.environ.get("BAR_LIB", "libbar.so"), w, sorted(c.items()))
# the same after back-to-back bar_sweep launches (as tools/kernel_ab.py does first)
for n in (4, 8, 40, 8, 40):
    M.sweep(b, x, k=5, nsweeps=n, mode="async")
torch.cuda.synchronize()
c = collections.Counter()
for _ in range(200):
    _, info = M.solve(b, None, x, k=5, tol=1e-10, mode="async")
    c[(info["iters"], info["kernel_launches"])] += 1
print("after sweeps", w, sorted(c.items()))
