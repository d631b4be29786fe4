"""Summarise an ncu report (--set full) or launch list into profiles/ (run here, no GPU needed).

    python tools/ncu_summary.py full gpurun_out/prof.ncu-rep profiles/r01_c5_async_full.txt \
        --traffic-json profiles/traffic_c5_async.json
    python tools/ncu_summary.py launches gpurun_out/launches.csv profiles/r01_c5_launches.txt
"""
import csv
import re
import io
import json
import subprocess
import sys
from collections import defaultdict

KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "dram__throughput.avg.pct_of_peak_sustained_elapsed", "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed",
        "sm__throughput.avg.pct_of_peak_sustained_elapsed", "launch__registers_per_thread",
        "launch__grid_size", "launch__block_size", "launch__shared_mem_per_block_dynamic",
        "sm__warps_active.avg.pct_of_peak_sustained_active", "lts__t_bytes.sum",
        "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum", "smsp__inst_executed.sum"]

SCALE = {"Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "byte": 1.0, "Tbyte": 1e12}


def full(rep, out, traffic_json=None):
    raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(raw)))
    hdr, units = rows[0], rows[1]
    lines = []
    dram = []
    for row in rows[2:]:
        d = dict(zip(hdr, row))
        u = dict(zip(hdr, units))
        lines.append(f"kernel: {d.get('Kernel Name', '?')}")
        for k in KEYS:
            if k in d:
                lines.append(f"  {k} = {d[k]} {u.get(k, '')}")
        try:
            rd = float(d["dram__bytes_read.sum"]) * SCALE.get(u["dram__bytes_read.sum"], 1)
            wr = float(d["dram__bytes_write.sum"]) * SCALE.get(u["dram__bytes_write.sum"], 1)
            dram.append(rd + wr)
            lines.append(f"  dram_bytes_per_launch = {rd + wr:.0f}")
        except (KeyError, ValueError):
            pass
        stalls = sorted(((float(v or 0), k) for k, v in d.items()
                         if k.startswith("smsp__pcsamp_warps_issue_stalled_") and not k.endswith("not_issued")),
                        reverse=True)[:6]
        lines.append("  top stall samples: " + ", ".join(f"{k.replace('smsp__pcsamp_warps_issue_stalled_', '')}={v:.0f}"
                                                         for v, k in stalls))
    open(out, "w").write("\n".join(lines) + "\n")
    if traffic_json and dram:
        # stamped with the build, kernel and R it was captured from: bench.py only uses a capture
        # whose stamp matches the run (a capture of another build is stale)
        sys.path.insert(0, __import__("os").path.dirname(__import__("os").path.dirname(__import__("os").path.abspath(__file__))))
        import bench

        kern = d.get("Kernel Name", "?")
        json.dump({"dram_bytes_per_launch": sum(dram) / len(dram), "source": rep, "libbar_build_id": bench.lib_hash(),
                   "kernel": libbar_name(kern), "R": R_ARG},
                  open(traffic_json, "w"))
    print("\n".join(lines))


def launches(csv_path, out):
    rows = list(csv.reader(open(csv_path)))
    start = next(i for i, r in enumerate(rows) if r and r[0] == "ID")
    hdr = rows[start]
    idx = {k: i for i, k in enumerate(hdr)}
    tot = defaultdict(float)
    cnt = defaultdict(int)
    for r in rows[start + 1:]:
        if len(r) < len(hdr) or r[idx["Metric Name"]] != "gpu__time_duration.sum":
            continue
        name = r[idx["Kernel Name"]].split("(")[0]
        val = float(r[idx["Metric Value"]].replace(",", ""))
        unit = r[idx["Metric Unit"]]
        ns = val * {"nsecond": 1, "usecond": 1e3, "msecond": 1e6, "second": 1e9}.get(unit, 1)
        tot[name] += ns
        cnt[name] += 1
    total = sum(tot.values())
    lines = [f"{'kernel':60s} {'launches':>8s} {'total_ms':>10s} {'share':>7s} {'avg_us':>9s}"]
    for k in sorted(tot, key=lambda k: -tot[k]):
        lines.append(f"{k[:60]:60s} {cnt[k]:8d} {tot[k] / 1e6:10.3f} {tot[k] / total:7.1%} {tot[k] / cnt[k] / 1e3:9.2f}")
    open(out, "w").write("\n".join(lines) + "\n")
    print("\n".join(lines))


def libbar_name(ncu_name):
    """ncu's demangled k_block_duo<ASYNC, WLR, EXT, CODED, BX, WOR> -> the name libbar
    reports (bar_matrix_info.last_sweep_kernel, sweep.cu duo_coded_name); other kernels keep their
    ncu name."""
    m = re.search(r"k_block_duo<([^>]*)>", ncu_name)
    if not m:
        return ncu_name
    a = [int(re.sub(r"\(\w+\)", "", t).strip()) for t in m.group(1).split(",")]
    a += [0] * (6 - len(a))
    wo = "" if a[5] == 0 else f",wo{a[5]}"  # WOR
    return ("k_block_duo<" + ("async" if a[0] else "sync") + {0: "", 1: ",coded", 2: ",staged"}[a[3]]
            + wo + {0: "", 1: ",bx", 2: ",x"}[a[4]] + ">")


R_ARG = None

if __name__ == "__main__":
    if "--R" in sys.argv:
        R_ARG = int(sys.argv[sys.argv.index("--R") + 1])
    mode = sys.argv[1]
    if mode == "full":
        tj = sys.argv[sys.argv.index("--traffic-json") + 1] if "--traffic-json" in sys.argv else None
        full(sys.argv[2], sys.argv[3], tj)
    else:
        launches(sys.argv[2], sys.argv[3])
