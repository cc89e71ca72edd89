"""Native build of every shared library in the repo (in-tree, so the .so files travel to the GPU box).

    liboracle.so      oracle/sat_oracle.c           gcc, strict IEEE (test infrastructure)
    libsatgen.so      satgen/satgen.c               gcc (seeded input generator, host)
    libsatgen_cuda.so satgen/satgen_cuda.cu         nvcc sm_100a (seeded input generator, device)
    libsat.so         paper_conf_ipps_emotofthni18_b200/csrc/*.cu   nvcc sm_100a (the product)

Each target is rebuilt only when one of its sources (or headers) is newer than the .so.
"""
from __future__ import annotations

import os
import shutil
import subprocess
import sys
from pathlib import Path

ROOT = Path(__file__).resolve().parent
PKG = ROOT / "paper_conf_ipps_emotofthni18_b200"
CSRC = PKG / "csrc"

NVCC = os.environ.get("NVCC", shutil.which("nvcc") or "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]


def _nccl_include() -> str | None:
    try:
        import nvidia.nccl  # type: ignore

        inc = Path(list(nvidia.nccl.__path__)[0]) / "include"
        if (inc / "nccl.h").exists():
            return str(inc)
    except Exception:
        pass
    return "/usr/include" if Path("/usr/include/nccl.h").exists() else None


def _stale(target: Path, sources: list[Path]) -> bool:
    if not target.exists():
        return True
    t = target.stat().st_mtime
    return any(s.stat().st_mtime > t for s in sources)


def _run(cmd: list[str]) -> None:
    print("[build]", " ".join(cmd), file=sys.stderr)
    subprocess.run(cmd, check=True)


def build_oracle(force: bool = False) -> Path:
    src = ROOT / "oracle" / "sat_oracle.c"
    out = ROOT / "oracle" / "liboracle.so"
    if force or _stale(out, [src]):
        _run(["gcc", "-O2", "-std=c11", "-ffp-contract=off", "-fno-fast-math", "-fPIC", "-shared",
              "-fvisibility=hidden", str(src), "-o", str(out), "-lm"])
    return out


def build_satgen(force: bool = False, cuda: bool = True) -> list[Path]:
    outs = []
    src = ROOT / "satgen" / "satgen.c"
    out = ROOT / "satgen" / "libsatgen.so"
    if force or _stale(out, [src]):
        _run(["gcc", "-O2", "-std=c11", "-ffp-contract=off", "-fPIC", "-shared", "-fvisibility=hidden",
              str(src), "-o", str(out)])
    outs.append(out)
    if cuda:
        csrc = ROOT / "satgen" / "satgen_cuda.cu"
        cout = ROOT / "satgen" / "libsatgen_cuda.so"
        if force or _stale(cout, [csrc]):
            _run([NVCC, *ARCH, "-O3", "-std=c++17", "-Xcompiler", "-fPIC,-fvisibility=hidden", "-shared",
                  "--cudart", "shared", str(csrc), "-o", str(cout)])
        outs.append(cout)
    return outs


def libsat_sources() -> list[Path]:
    return sorted(CSRC.glob("*.cu")) + sorted(CSRC.glob("*.cuh")) + sorted(CSRC.glob("*.h")) + \
        sorted((ROOT / "include").glob("*.h"))


def build_libsat(force: bool = False, extra: list[str] | None = None, out: Path | None = None) -> Path:
    out = out or (PKG / "libsat.so")
    srcs = libsat_sources()
    cu = [str(s) for s in sorted(CSRC.glob("*.cu"))]
    if force or extra or _stale(out, srcs):
        inc = ["-I", str(ROOT / "include"), "-I", str(CSRC)]
        nccl = _nccl_include()
        if nccl:
            inc += ["-I", nccl, "-DSAT_HAVE_NCCL_H=1"]
        _run([NVCC, *ARCH, "-O3", "-std=c++17", "-lineinfo", "-Xptxas", "-v,-warn-spills",
              "-Xcompiler", "-fPIC,-fvisibility=hidden,-Wall", "-shared", "--cudart", "shared",
              *inc, *(extra or []), *cu, "-o", str(out), "-ldl"])
    return out


def build_stats(force: bool = False) -> Path:
    """Instrumented libsat (per-CTA phase counters, sat_debug_stats) for tools/stats.py."""
    out = PKG / "libsat_stats.so"
    if force or _stale(out, libsat_sources()):
        build_libsat(extra=["-DSAT_STATS=1"], out=out)
    return out


def build_experimental(force: bool = False) -> Path:
    """Tuning build (-DSAT_EXPERIMENTAL=1): the shipped variants plus the unshipped configurations, for
    tools/sweep_variants.py via SAT_LIB=paper_conf_ipps_emotofthni18_b200/libsat_exp.so.  Not the product."""
    out = PKG / "libsat_exp.so"
    if force or _stale(out, libsat_sources()):
        build_libsat(extra=["-DSAT_EXPERIMENTAL=1"], out=out)
    return out


def build_stress(force: bool = False) -> Path:
    """Protocol-stress build: -DSAT_JITTER=1 (random __nanosleep before every status-word
    publication) and -DSAT_WATCHDOG=1 (bounded spins that trap).  For tests/test_gpu_stress.py via
    SAT_LIB=paper_conf_ipps_emotofthni18_b200/libsat_stress.so.  Not the product."""
    out = PKG / "libsat_stress.so"
    if force or _stale(out, libsat_sources()):
        build_libsat(extra=["-DSAT_JITTER=1", "-DSAT_WATCHDOG=1"], out=out)
    return out


def build_all(force: bool = False) -> None:
    """Oracle, generators, libsat.so and the protocol-stress build (the two nvcc runs in parallel)."""
    from concurrent.futures import ThreadPoolExecutor

    build_oracle(force)
    build_satgen(force)
    with ThreadPoolExecutor(2) as ex:
        jobs = [ex.submit(build_libsat, force), ex.submit(build_stress, force)]
        for j in jobs:
            j.result()


if __name__ == "__main__":
    build_all(force="--force" in sys.argv)
    if "--experimental" in sys.argv:
        build_experimental(force="--force" in sys.argv)
