"""N4: cost of the local iterations on B200 — time per global iteration of
async-(k) for k = 1..9 (CUDA-event slope of back-to-back sweep launches, as bench.py), against
the paper's Table 4 (fv3 on a C2070: +19% at k=5, +39% at k=9 over async-(1); the
text claims "<5%" for k=2 and "<35%" for k=9).

    python tools/local_iters.py --workload c4 > profiles/r01_n4_c4.txt
"""
import argparse
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def table(workload="c4", R=None, mode="async", ks=range(1, 10), tuning=None):
    """[(k, ms per global iteration)] from the slope of 8 vs 40 back-to-back bar_sweep launches."""
    import torch

    import bench
    from paper_conf_ipps_anzttdh12_b200 import bar

    R = R or bench.WORKLOADS[workload][2]
    A = bench.make_matrix(workload)
    M = bar.Matrix.from_csr(A, R, tuning=tuning)
    del A
    info = M.info()
    b = torch.ones(M.n, dtype=torch.float64, device="cuda")
    x = torch.zeros_like(b)
    st = torch.cuda.current_stream()

    def timed(k, nsw):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(st)
        M.sweep(b, x, k=k, nsweeps=nsw, mode=mode)
        e1.record(st)
        torch.cuda.synchronize()
        return e0.elapsed_time(e1)

    out = []
    for k in ks:
        timed(k, 4)
        t = (min(timed(k, 40) for _ in range(3)) - min(timed(k, 8) for _ in range(3))) / 32
        out.append((k, t))
    kernel = M.info()["last_sweep_kernel"]
    M.close()
    return info, kernel, out


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--workload", default="c4")
    ap.add_argument("--R", type=int, default=None)
    ap.add_argument("--mode", default="async")
    a = ap.parse_args()
    import bench

    R = a.R or bench.WORKLOADS[a.workload][2]
    info, kernel, rows = table(a.workload, R, a.mode)
    clk = os.popen("nvidia-smi --query-gpu=clocks.sm,clocks.max.sm,clocks_event_reasons.active --format=csv,noheader")
    nb = info["model_bytes_per_iter"]
    print(f"# N4: {a.mode}-(k), {a.workload}, R={R}, kernel {kernel}; ms per global iteration (slope of 8 vs 40 "
          f"launches); clocks after the run (sm, max sm, reasons): {clk.read().strip()}")
    print(f"# paper Table 4 (fv3, C2070): async-(5) +19%, async-(9) +39% per global iteration over async-(1)")
    print(f"{'k':>3} {'ms/iter':>10} {'vs k=1':>8} {'GB/s':>8}")
    base = rows[0][1]
    for k, t in rows:
        print(f"{k:3d} {t:10.4f} {100 * (t / base - 1):+7.1f}% {nb / (t * 1e-3) / 1e9:8.1f}")


if __name__ == "__main__":
    main()
