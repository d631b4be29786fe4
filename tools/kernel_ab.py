"""A/B timing of kernel variants selected by bar_tuning fields (tuning aid, not a bench value).

For one matrix, each variant (a set of bar_tuning fields, set on the handle with bar_set_tuning;
the library reads no environment variable) is timed two ways with CUDA events on the launching
stream:
  * per launch: slope of 8 vs 40 back-to-back bar_sweep launches (cancels fixed overheads);
  * whole solve: bar_solve to tol, median of --reps solves, with its global-iteration count.

    python tools/kernel_ab.py --workload c5 --modes async,sync-block \
        --variants 'base:;nopf:ghost_prefetch=-1;pipe:pipe=1,duo=-1;strided:async_order=3'
"""
import argparse
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def parse_variants(spec):
    out = []
    for item in spec.split(";"):
        if not item.strip():
            continue
        name, _, fields = item.partition(":")
        tune = {}
        for kv in fields.split(","):
            if kv.strip():
                k, _, v = kv.partition("=")
                v = v.strip()
                tune[k.strip()] = int(v) if v.lstrip("-").isdigit() else v
        out.append((name.strip(), tune))
    return out


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--workload", default="c5")
    ap.add_argument("--R", type=int, default=None)
    ap.add_argument("--modes", default="async")
    ap.add_argument("--k", type=int, default=5)
    ap.add_argument("--reps", type=int, default=3)
    ap.add_argument("--variants", default="base:")
    ap.add_argument("--rounds", type=int, default=1, help="repeat the variant list (A B A B ...); medians at the end")
    a = ap.parse_args()
    import torch

    import bench
    from paper_conf_ipps_anzttdh12_b200 import bar

    R = a.R or bench.WORKLOADS[a.workload][2]
    A = bench.make_matrix(a.workload)
    M = bar.Matrix.from_csr(A, rows_per_block=R)
    info = M.info()
    del A
    n = M.n
    b = torch.ones(n, dtype=torch.float64, device="cuda")
    x = torch.zeros(n, dtype=torch.float64, device="cuda")
    st = torch.cuda.current_stream()

    def ev_time(fn):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize()
        e0.record(st)
        out = fn()
        e1.record(st)
        torch.cuda.synchronize()
        return e0.elapsed_time(e1), out

    # box reference: device copy bandwidth (read + write bytes), as MEASURED_PEAKS.json measures it
    src = torch.empty(1 << 27, dtype=torch.float64, device="cuda")
    dst = torch.empty_like(src)
    dst.copy_(src)
    copy_ms = min(ev_time(lambda: dst.copy_(src))[0] for _ in range(10))
    copy_gbs = 2 * src.numel() * 8 / copy_ms / 1e6
    del src, dst
    clk = os.popen("nvidia-smi --query-gpu=clocks.sm,clocks.mem,power.draw --format=csv,noheader").read().strip()
    print(json.dumps({"box": {"copy_GBs": round(copy_gbs, 1), "clocks": clk}}), flush=True)
    summary = {}
    for mode, rnd, (name, tune) in [(m, r, v) for m in a.modes.split(",") for r in range(a.rounds)
                                     for v in parse_variants(a.variants)]:
            M.set_tuning(tune or None)
            M.sweep(b, x, k=a.k, nsweeps=4, mode=mode)
            lo, hi = 8, 40
            t_lo = min(ev_time(lambda: M.sweep(b, x, k=a.k, nsweeps=lo, mode=mode))[0] for _ in range(3))
            t_hi = min(ev_time(lambda: M.sweep(b, x, k=a.k, nsweeps=hi, mode=mode))[0] for _ in range(3))
            per_launch = (t_hi - t_lo) / (hi - lo)
            M.solve(b, None, x, k=a.k, mode=mode)
            solves = [ev_time(lambda: M.solve(b, None, x, k=a.k, mode=mode)) for _ in range(a.reps)]
            ms = statistics.median(s[0] for s in solves)
            iters = [s[1][1]["iters"] for s in solves]
            summary.setdefault((mode, name), []).append((per_launch, ms))
            print(json.dumps({"workload": a.workload, "R": R, "k": a.k, "mode": mode, "variant": name, "tuning": tune,
                              "launch_ms": round(per_launch, 4),
                              "contract_GBs": round(info["model_bytes_per_iter"] / per_launch / 1e6, 1),
                              "frac_of_copy": round(info["model_bytes_per_iter"] / per_launch / 1e6 / copy_gbs, 3),
                              "kernel": M.info()["last_sweep_kernel"],
                              "solve_ms": round(ms, 3), "iters": iters}), flush=True)
    if a.rounds > 1:
        for (mode, name), v in summary.items():
            print(json.dumps({"median_over_rounds": True, "mode": mode, "variant": name,
                              "launch_ms": round(statistics.median(t for t, _ in v), 4),
                              "solve_ms": round(statistics.median(s_ for _, s_ in v), 3), "rounds": len(v)}), flush=True)
    M.close()


if __name__ == "__main__":
    main()
