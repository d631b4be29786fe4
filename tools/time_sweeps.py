"""Per-launch time of the async-(k) sweep (slope of 8 vs 40 launches) for the library BAR_LIB points
at — for A/B of experimental builds whose iterates need not be meaningful."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import bench
from paper_conf_ipps_anzttdh12_b200 import bar
w = sys.argv[1] if len(sys.argv) > 1 else "c4"
A = bench.make_matrix(w); M = bar.Matrix.from_csr(A, bench.WORKLOADS[w][2]); del A
b = torch.ones(M.n, dtype=torch.float64, device="cuda"); x = torch.zeros_like(b)
st = torch.cuda.current_stream()
def timed(n):
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(st); M.sweep(b, x, k=5, nsweeps=n, mode="async"); e1.record(st); torch.cuda.synchronize()
    return e0.elapsed_time(e1)
timed(4)
t = (min(timed(40) for _ in range(3)) - min(timed(8) for _ in range(3))) / 32
print(os.environ.get("BAR_LIB", "libbar.so"), w, round(t, 4), "ms/launch", M.info()["last_sweep_kernel"])
