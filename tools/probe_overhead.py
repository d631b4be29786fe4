import time, torch, sys
sys.path.insert(0, '.')
import bench
from paper_conf_ipps_anzttdh12_b200 import bar
A = bench.make_matrix('c1'); M = bar.Matrix.from_csr(A, 128)
b = torch.ones(A.n, dtype=torch.float64, device='cuda'); x = torch.empty_like(b)
st = torch.cuda.current_stream()
def t(fn, reps=50):
    fn(); torch.cuda.synchronize()
    ts = []
    for _ in range(reps):
        t0 = time.perf_counter(); fn(); torch.cuda.synchronize(); ts.append(time.perf_counter() - t0)
    ts.sort(); return ts[len(ts)//2] * 1e6
print("solve max_iters=0  us", t(lambda: M.solve(b, None, x, k=5, max_global_iters=0, tol=1e-10, mode='async', stream=st)))
print("solve max_iters=1  us", t(lambda: M.solve(b, None, x, k=5, max_global_iters=1, tol=0.0, mode='async', stream=st)))
print("solve max_iters=10 us", t(lambda: M.solve(b, None, x, k=5, max_global_iters=10, tol=0.0, mode='async', stream=st)))
print("solve to 1e-10     us", t(lambda: M.solve(b, None, x, k=5, max_global_iters=20000, tol=1e-10, mode='async', stream=st)))
print("residual           us", t(lambda: M.residual(b, x, stream=st)))
e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
def ev():
    e0.record(st); M.solve(b, None, x, k=5, max_global_iters=20000, tol=1e-10, mode='async', stream=st); e1.record(st); torch.cuda.synchronize(); return e0.elapsed_time(e1)*1e3
print("solve events us", sorted(ev() for _ in range(20))[10])
