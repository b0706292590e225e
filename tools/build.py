"""Native build: the CUDA library (sm_100a) and the C oracle.

    python tools/build.py            # both
    python tools/build.py oracle     # only the oracle
    python tools/build.py lib        # only libmicco.so

Called by __graft_entry__.build() and by tests/conftest.py (oracle only, so
the CPU suite never needs nvcc).  Outputs stay in-tree (git-ignored, shipped
to the GPU box by gpurun): oracle/liboracle.so and
paper_conf_ipps_wangr0e22_b200/libmicco.so.
"""
from __future__ import annotations

import os
import shutil
import subprocess
import sys
from pathlib import Path

ROOT = Path(__file__).resolve().parent.parent
PKG = ROOT / "paper_conf_ipps_wangr0e22_b200"
CSRC = PKG / "csrc"
ORACLE_SO = ROOT / "oracle" / "liboracle.so"
LIB_SO = PKG / "libmicco.so"

NVCC_ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]


def _run(cmd, cwd=ROOT):
    print("+", " ".join(str(c) for c in cmd), flush=True)
    subprocess.run([str(c) for c in cmd], cwd=cwd, check=True)


def _stale(out: Path, srcs) -> bool:
    if not out.exists():
        return True
    t = out.stat().st_mtime
    return any(Path(s).stat().st_mtime > t for s in srcs)


def build_oracle(force: bool = False) -> Path:
    srcs = [ROOT / "oracle" / "micco_oracle.c", ROOT / "oracle" / "micco_oracle.h",
            ROOT / "micco_inputs" / "synth.h"]
    if force or _stale(ORACLE_SO, srcs):
        tmp = ORACLE_SO.with_suffix(".so.tmp")
        _run(["gcc", "-std=c99", "-O2", "-ffp-contract=off", "-fno-fast-math", "-fPIC", "-shared",
              "-pthread", "-Wall", "-o", tmp, srcs[0]])
        os.replace(tmp, ORACLE_SO)
    return ORACLE_SO


def _nvcc() -> str:
    for c in (shutil.which("nvcc"), "/usr/local/cuda/bin/nvcc"):
        if c and Path(c).exists():
            return c
    raise RuntimeError("nvcc not found")


def lib_sources():
    return sorted(CSRC.glob("*.cu")) + sorted(CSRC.glob("*.cpp"))


def build_lib(force: bool = False, jobs: int = 8) -> Path:
    srcs = lib_sources()
    hdrs = list(CSRC.glob("*.h")) + list(CSRC.glob("*.cuh")) + [ROOT / "include" / "micco.h",
                                                                  ROOT / "micco_inputs" / "synth.h"]
    if not (force or _stale(LIB_SO, srcs + hdrs)):
        return LIB_SO
    nvcc = _nvcc()
    objdir = ROOT / "build" / "obj"
    objdir.mkdir(parents=True, exist_ok=True)
    common = ["-std=c++17", "-O3", "-Xcompiler", "-fPIC", "-Xcompiler", "-fvisibility=hidden",
              "-I", ROOT / "include", "-I", ROOT, "-I", CSRC]
    procs, objs = [], []
    for s in srcs:
        o = objdir / (s.name + ".o")
        objs.append(o)
        if not force and not _stale(o, [s] + hdrs):
            continue
        if s.suffix == ".cu":
            cmd = [nvcc] + NVCC_ARCH + ["-lineinfo", "-Xptxas", "-v", "--expt-relaxed-constexpr"] + common + [
                "-c", s, "-o", o]
        else:
            cmd = [nvcc] + NVCC_ARCH + common + ["-x", "cu", "-c", s, "-o", o]
        print("+", " ".join(str(c) for c in cmd), flush=True)
        procs.append((s, subprocess.Popen([str(c) for c in cmd], cwd=ROOT, stdout=subprocess.PIPE,
                                          stderr=subprocess.STDOUT, text=True)))
        if len(procs) >= jobs:
            _drain(procs)
    _drain(procs)
    tmp = LIB_SO.with_suffix(".so.tmp")
    # shared cudart: the library links the system libcudart.so instead of embedding a static copy
    _run([nvcc] + NVCC_ARCH + ["-shared", "-cudart", "shared", "-o", tmp] + objs + ["-lpthread", "-ldl"])
    os.replace(tmp, LIB_SO)
    return LIB_SO


def _drain(procs):
    while procs:
        s, p = procs.pop(0)
        out, _ = p.communicate()
        log = ROOT / "build" / (s.name + ".log")
        log.write_text(out)
        if p.returncode != 0:
            sys.stderr.write(out)
            raise RuntimeError(f"nvcc failed on {s}")


def main(argv):
    what = argv[1] if len(argv) > 1 else "all"
    force = "--force" in argv
    if what in ("all", "oracle"):
        build_oracle(force)
    if what in ("all", "lib"):
        build_lib(force)


if __name__ == "__main__":
    main(sys.argv)
