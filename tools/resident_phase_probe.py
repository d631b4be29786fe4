"""Per-phase cycle counts of k_block_resident (R17): build the instrumented library
first with `python tools/build.py --profile-resident` (-> libbar_prof.so), then run on a GPU box."""
import ctypes, os, sys
sys.path.insert(0, os.getcwd())
os.environ["BAR_LIB"] = "paper_conf_ipps_anzttdh12_b200/libbar_prof.so"
import torch, bench
from paper_conf_ipps_anzttdh12_b200 import bar
for wl in ("c1", "c3", "c2"):
    A = bench.make_matrix(wl); R = bench.WORKLOADS[wl][2]
    for lead in (3, 48):
        M = bar.Matrix.from_csr(A, R, tuning={"lead": lead})
        b = torch.ones(A.n, dtype=torch.float64, device="cuda")
        x = torch.empty_like(b)
        for _ in range(5): M.solve(b, None, x, k=5, tol=1e-10, mode="async")
        out = (ctypes.c_ulonglong * 8)()
        bar._lib.bar_debug_resident_profile(out, 1)
        reps = 50
        its = 0
        for _ in range(reps):
            _, info = M.solve(b, None, x, k=5, tol=1e-10, mode="async"); its += info["cta_iters_max"]
        torch.cuda.synchronize()
        bar._lib.bar_debug_resident_profile(out, 1)
        q = M.info()["num_subdomains"]
        per = [out[i] / (its * q) for i in range(6)]  # cycles per block-iteration
        names = ["lead+go", "gathers+sweep1", "sweeps2..k", "writeback+reduce", "publish", "(top)"]
        print(wl, "lead", lead, "q", q, "iters/solve", its / reps, " ".join(f"{n}={c:.0f}" for n, c in zip(["top->go","go->sw1","sw2..k","wb+red","publish"], [per[1], per[2], per[3], per[4], per[5]])), "total", sum(per[1:6]) + per[0])
        M.close()
