"""Per-phase cycle counts of k_block_duo (profiling aid): build the instrumented library first
with `python tools/build.py --profile-duo` (-> libbar_duoprof.so), then run on a GPU box:

    python tools/duo_phase_probe.py --workload c5 [--tune unroll_off=-1]

Lane 0 of warp 0 (issues the slab's values), warp 3 (b_J / x_J or their L2 prefetch, the ghost
prefetch, the ring of bounds) and the last warp (rows only) sum clock64 deltas between the marks
of each subdomain; printed as cycles per subdomain."""
import argparse
import ctypes
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
os.environ["BAR_LIB"] = os.path.join(ROOT, "paper_conf_ipps_anzttdh12_b200", "libbar_duoprof.so")

PHASES = ["slab wait", "phase 1", "barrier 1", "issue", "sweep 1", "barrier 2", "sweeps 2..k", "write-back"]


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--workload", default="c5")
    ap.add_argument("--mode", default="async")
    ap.add_argument("--k", type=int, default=5)
    ap.add_argument("--sweeps", type=int, default=10)
    ap.add_argument("--tune", default="")
    a = ap.parse_args()
    import torch

    import bench
    from paper_conf_ipps_anzttdh12_b200 import bar

    tune = {}
    for kv in filter(None, a.tune.split(",")):
        k, v = kv.split("=")
        tune[k] = int(v)
    A = bench.make_matrix(a.workload)
    M = bar.Matrix.from_csr(A, rows_per_block=bench.WORKLOADS[a.workload][2], tuning=tune or None)
    del A
    b = torch.ones(M.n, dtype=torch.float64, device="cuda")
    x = torch.zeros(M.n, dtype=torch.float64, device="cuda")
    M.sweep(b, x, k=a.k, nsweeps=3, mode=a.mode)
    torch.cuda.synchronize()
    out = (ctypes.c_ulonglong * 32)()
    bar._lib.bar_debug_duo_profile(out, 1)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    M.sweep(b, x, k=a.k, nsweeps=a.sweeps, mode=a.mode)
    e1.record()
    torch.cuda.synchronize()
    bar._lib.bar_debug_duo_profile(out, 1)
    ms = e0.elapsed_time(e1) / a.sweeps
    nb = out[28]
    span_avg = out[24] / max(nb, 1) / 1e3  # us per block per launch (summed over launches)
    print(f"  launch {ms * 1e3:.1f} us (events); blocks {nb // a.sweeps} per launch; block span avg "
          f"{span_avg / a.sweeps * a.sweeps:.1f} us (entry to exit, per launch), max {out[25] / 1e3:.1f} us")
    q = M.info()["num_subdomains"]
    print(f"{a.workload} {a.mode} k={a.k} kernel={M.info()['last_sweep_kernel']} tune={tune}: cycles per subdomain")
    for w, name in enumerate(["warp 0", "warp 3", "last warp"]):
        per = [out[8 * w + i] / (a.sweeps * q) for i in range(8)]
        print(f"  {name:10s} " + " ".join(f"{p}={c:.0f}" for p, c in zip(PHASES, per)) + f" total={sum(per):.0f}")
    M.close()


if __name__ == "__main__":
    main()
