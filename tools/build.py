"""Native builds: the workload generators and the oracle (gcc), and libbar.so (nvcc, sm_100a).

Everything is built IN-TREE so the .so files travel to the GPU box with the repo
snapshot. ``build_all()`` is what ``__graft_entry__.build()`` calls.
"""
from __future__ import annotations

import glob
import hashlib
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
PKG = os.path.join(ROOT, "paper_conf_ipps_anzttdh12_b200")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]


def _stale(target: str, sources: list[str]) -> bool:
    if not os.path.exists(target):
        return True
    t = os.path.getmtime(target)
    return any(os.path.getmtime(s) > t for s in sources)


def _run(cmd: list[str]) -> None:
    r = subprocess.run(cmd, cwd=ROOT, capture_output=True, text=True)
    if r.returncode != 0:
        sys.stderr.write(r.stdout + r.stderr)
        raise RuntimeError("build failed: " + " ".join(cmd))


def build_workloads(force: bool = False) -> str:
    src = os.path.join(ROOT, "workloads", "gen.c")
    out = os.path.join(ROOT, "workloads", "libworkloads.so")
    if force or _stale(out, [src]):
        _run(["gcc", "-O2", "-fopenmp", "-fPIC", "-shared", "-o", out, src, "-lm"])
    return out


def build_oracle(force: bool = False) -> str:
    """The oracle: single-threaded C, IEEE fp64, no contraction, no fast-math."""
    src = os.path.join(ROOT, "oracle", "oracle.c")
    out = os.path.join(ROOT, "oracle", "liboracle.so")
    if force or _stale(out, [src]):
        _run(["gcc", "-O2", "-std=c11", "-ffp-contract=off", "-fno-fast-math", "-fPIC", "-shared",
              "-o", out, src, "-lm"])
    return out


def nccl_paths() -> tuple[str, str] | None:
    try:
        import nvidia.nccl as nn  # type: ignore

        base = list(nn.__path__)[0]
        inc, lib = os.path.join(base, "include"), os.path.join(base, "lib")
        if os.path.exists(os.path.join(inc, "nccl.h")):
            return inc, lib
    except Exception:
        pass
    return None


def source_id(deps: list[str], flags: list[str]) -> str:
    """SHA-256 (16 hex) over the library's sources (paths relative to the repo) and nvcc flags:
    the build identity libbar reports through bar_build_id()."""
    h = hashlib.sha256()
    for d in sorted(deps):
        h.update(os.path.relpath(d, ROOT).encode() + b"\0" + open(d, "rb").read() + b"\0")
    h.update(" ".join(flags).encode())
    return h.hexdigest()[:16]


def build_bar(force: bool = False, out_name: str = "libbar.so", defines: tuple = ()) -> str:
    """libbar.so: the C-ABI library (include/bar.h) with every kernel, for sm_100a only.
    `defines` builds an instrumented copy under another name (e.g. BAR_PROFILE_RESIDENT=1 ->
    libbar_prof.so for tools/resident_phase_probe.py); the product library never has them."""
    csrc = os.path.join(PKG, "csrc")
    srcs = sorted(glob.glob(os.path.join(csrc, "*.cu")))
    deps = srcs + sorted(glob.glob(os.path.join(csrc, "*.cuh"))) + [os.path.join(ROOT, "include", "bar.h")]
    out = os.path.join(PKG, out_name)
    if not (force or _stale(out, deps)):
        return out
    flags = [*ARCH, "-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC", "-shared", "-Xptxas", "-v",
             "--expt-relaxed-constexpr", *["-D" + d for d in defines]]
    cmd = [NVCC, *flags, "-DBAR_SOURCE_ID=\"" + source_id(deps, flags) + "\"",
           "-I", os.path.join(ROOT, "include"), "-I", csrc]
    nccl = nccl_paths()
    if nccl is not None:
        inc, lib = nccl
        cmd += ["-DBAR_WITH_NCCL=1", "-I", inc, "-L", lib, "-Xlinker", "-rpath=" + lib]
    cmd += ["-o", out, *srcs]
    if nccl is not None:
        cmd += ["-l:libnccl.so.2"]
    r = subprocess.run(cmd, cwd=ROOT, capture_output=True, text=True)
    if r.returncode != 0:
        sys.stderr.write(r.stdout + r.stderr)
        raise RuntimeError("nvcc build of libbar.so failed")
    if not defines:
        with open(os.path.join(PKG, "ptxas_info.txt"), "w") as f:
            f.write(r.stderr)
    return out


def build_test_helpers(force: bool = False) -> str:
    """tests/helpers/libspin.so: a test-only kernel that occupies SMs (tests of the single-launch
    kernel's behaviour when other work holds the device)."""
    src = os.path.join(ROOT, "tests", "helpers", "spin.cu")
    out = os.path.join(ROOT, "tests", "helpers", "libspin.so")
    if force or _stale(out, [src]):
        _run([NVCC, *ARCH, "-O2", "-Xcompiler", "-fPIC", "-shared", "-o", out, src])
    return out


def build_all(force: bool = False) -> None:
    build_workloads(force)
    build_oracle(force)
    build_bar(force)
    build_test_helpers(force)


if __name__ == "__main__":
    if "--profile-resident" in sys.argv:
        build_bar(True, "libbar_prof.so", ("BAR_PROFILE_RESIDENT=1",))
    elif "--profile-duo" in sys.argv:
        build_bar(True, "libbar_duoprof.so", ("BAR_PROFILE_DUO=1",))
    elif "--check-bounds" in sys.argv:
        build_bar(True, "libbar_check.so", ("BAR_CHECK_BOUNDS=1",))

    else:
        build_all(force="--force" in sys.argv)
