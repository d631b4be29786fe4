"""bench.py's JSON line: the keys the driver and the judge read (the run contract in DESIGN.md §5).

The reference arm (the CPU oracle) runs here on CPU; our arm needs the B200.
"""
import json
import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _run(args, timeout=600):
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), *args], cwd=ROOT, capture_output=True,
                       text=True, timeout=timeout)
    assert r.returncode == 0, r.stderr[-2000:]
    lines = [ln for ln in r.stdout.splitlines() if ln.startswith("{")]
    assert len(lines) == 1, r.stdout
    return json.loads(lines[0])


def test_reference_arm_line():
    d = _run(["--impl", "reference", "--workload", "c1", "--steps", "1", "--warmup", "0"])
    assert d["impl"] == "reference" and d["unit"] == "s" and d["higher_is_better"] is False
    assert d["value"] > 0 and d["cpu_baseline"]["kind"] == "oracle" and d["cpu_baseline"]["cores"] == 1
    assert d["e2e"]["h2d_bytes_per_step"] == 0 and d["e2e"]["value"] == d["value"]
    assert d["config"]["workload"].startswith("c1")
    assert d["extrapolated"] is False and d["oracle_iters"] == 28  # a full oracle sync-block-(5) solve


@pytest.mark.gpu
def test_our_arm_line(bar):
    d = _run(["--workload", "c1", "--steps", "3", "--warmup", "3"])
    for k in ("metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better", "scaling",
              "vs_baseline", "dtype", "data", "config", "roofline", "cpu_baseline", "e2e", "clocks", "gpu_launches"):
        assert k in d, k
    assert d["n_gpus"] == 1 and d["steps"] == 3 and d["warmup"] == 3 and d["dtype"] == "f64"
    assert d["higher_is_better"] is False and d["value"] > 0 and d["gpu_launches"] > 0
    assert d["global_iters"] >= 15
    r = d["roofline"]
    for k in ("bound", "achieved", "peak", "unit", "frac", "traffic"):
        assert k in r, k
    assert r["bound"] == "hbm" and r["unit"] == "GB/s" and abs(r["frac"] - r["achieved"] / r["peak"]) < 1e-3
    c = d["cpu_baseline"]
    assert c["kind"] == "oracle" and c["cores"] == 1 and c["value"] > 0 and c["sample"]
    assert c["jacobi"]["iters"] == 137 and c["gauss_seidel"]["iters"] == 14  # SURVEY P12 counts
    assert c["sync_block_5"]["iters"] == 28 and d["oracle_iters"] == 28 and not c["extrapolated"]
    assert d["partitioned_1rank"]["converged"] and d["lead_3"]["global_iters"] > 0
    e = d["e2e"]
    assert e["h2d_bytes_per_step"] == 8 * 2000 and e["d2h_bytes_per_step"] == 8 * 2000 and e["value"] > 0
    assert d["clocks"]["sm_max_mhz"]


def test_ncu_kernel_names_map_to_libbar_names():
    """tools/ncu_summary.libbar_name: ncu's demangled k_block_duo template arguments -> the name
    libbar reports (bar_matrix_info.last_sweep_kernel), which bench.py matches against the kernel
    stamped into profiles/traffic_*.json (a capture of another kernel variant is never used)."""
    import sys

    sys.path.insert(0, os.path.join(ROOT, "tools"))
    from ncu_summary import libbar_name

    base = "void bar::<unnamed>::k_block_duo<{}>(bar::<unnamed>::KP)"
    assert libbar_name(base.format("(bool)1, (int)4, (bool)0, (int)1, (bool)1, (int)4")) == "k_block_duo<async,coded,wo4,bx>"
    assert libbar_name(base.format("(bool)1, (int)4, (bool)0, (int)1, (bool)0, (int)0")) == "k_block_duo<async,coded>"
    assert libbar_name(base.format("(bool)0, (int)4, (bool)0, (int)1, (bool)1")) == "k_block_duo<sync,coded,bx>"
    assert libbar_name(base.format("(bool)1, (int)4, (bool)1, (int)2")) == "k_block_duo<async,staged>"
    assert libbar_name("void bar::<unnamed>::k_block_resident<16, 2>(bar::<unnamed>::KP)").startswith("void bar")
    # the committed captures name a kernel variant libbar can report
    for wl in ("c4", "c5"):
        tj = json.load(open(os.path.join(ROOT, "profiles", f"traffic_{wl}_async.json")))
        assert tj["kernel"].startswith("k_block_duo<async,coded") and tj["dram_bytes_per_launch"] > 0
