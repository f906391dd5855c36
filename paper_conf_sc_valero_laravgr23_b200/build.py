"""Build libmrlbm.so in-tree with nvcc for sm_100a (no JIT, no torch extension)."""
from __future__ import annotations

import os
import subprocess
import sys
from pathlib import Path

PKG = Path(__file__).resolve().parent
ROOT = PKG.parent
CSRC = PKG / "csrc"
LIB = PKG / "libmrlbm.so"
# one translation unit per lattice (compiled in parallel) + the host / ABI unit
SOURCES = [CSRC / "mrlbm.cu", CSRC / "var_d2q9.cu", CSRC / "var_d3q19.cu", CSRC / "var_d3q27.cu", CSRC / "var_st.cu"]
DEPS = SOURCES + sorted(CSRC.glob("*.cuh")) + [ROOT / "include" / "mrlbm.h", Path(__file__).resolve()]

ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
# Per-unit flags.  The D3Q19 unit (the rotated fp64 sweep) is compiled without
# implicit FMA contraction: its arithmetic spells every fused multiply-add as
# fma(), so the two halves of the unrolled sweep and the P2P push instance
# round identically and slab / P2P decompositions stay bitwise equal to one
# rank (with contraction the compiler fused differently in the two halves:
# 1-ulp differences; measured cost -0.5% on C5, profiles/r03/ab12.jsonl).
UNIT_FLAGS = {"var_d3q19.cu": ["-fmad=false"]}


def nccl_dirs():
    try:
        import nvidia.nccl as nn  # the NCCL torch is built against (2.28.x)
        base = Path(list(nn.__path__)[0])
        inc, lib = base / "include", base / "lib"
        if (inc / "nccl.h").exists():
            return inc, lib
    except Exception:
        pass
    return Path("/usr/include"), Path("/usr/lib/x86_64-linux-gnu")


def nvcc():
    for cand in (os.environ.get("NVCC"), "/usr/local/cuda/bin/nvcc", "nvcc"):
        if cand and (Path(cand).exists() or cand == "nvcc"):
            return cand
    return "nvcc"


def needs_build() -> bool:
    if not LIB.exists():
        return True
    t = LIB.stat().st_mtime
    return any(p.stat().st_mtime > t for p in DEPS)


def build(force: bool = False, verbose: bool = False, out: Path | None = None, defines=(), extra=()) -> Path:
    """out / defines: a variant build for A/B comparisons (e.g. ab/libmrlbm_X.so, -DNAME)."""
    from concurrent.futures import ThreadPoolExecutor
    import tempfile

    target = Path(out) if out else LIB
    if not force and not out and not needs_build():
        return LIB
    inc, lib = nccl_dirs()
    ncclso = "libnccl.so.2" if (lib / "libnccl.so.2").exists() else "libnccl.so"
    tmp = target.with_suffix(f".{os.getpid()}.tmp.so")
    common = [nvcc(), "-O3", "-std=c++17", *ARCH, "-lineinfo", "--expt-relaxed-constexpr", "-Xcompiler", "-fPIC",
              f"-I{ROOT / 'include'}", f"-I{inc}", *[f"-D{d}" for d in defines], *extra]
    if verbose:
        common += ["-Xptxas", "-v"]
    with tempfile.TemporaryDirectory(prefix="mrlbm_build_") as td:
        objs = [Path(td) / (src.stem + ".o") for src in SOURCES]

        def compile_one(i):
            flags = UNIT_FLAGS.get(SOURCES[i].name, [])
            return subprocess.run(common + flags + ["-c", "-o", str(objs[i]), str(SOURCES[i])], capture_output=True,
                                  text=True)

        with ThreadPoolExecutor(max_workers=len(SOURCES)) as ex:
            results = list(ex.map(compile_one, range(len(SOURCES))))
        for src, r in zip(SOURCES, results):
            if r.returncode != 0:
                sys.stderr.write(r.stdout + r.stderr)
                raise RuntimeError(f"nvcc failed compiling {src.name}")
            if verbose:
                sys.stderr.write(f"== {src.name}\n" + r.stderr)
        r = subprocess.run([nvcc(), *ARCH, "-shared", "-o", str(tmp), *map(str, objs), f"-L{lib}", f"-l:{ncclso}",
                            "-lcuda", "-Xlinker", f"-rpath,{lib}"], capture_output=True, text=True)
        if r.returncode != 0:
            sys.stderr.write(r.stdout + r.stderr)
            raise RuntimeError("nvcc failed linking libmrlbm.so")
    os.replace(tmp, target)
    return target


if __name__ == "__main__":
    a = sys.argv[1:]
    out = a[a.index("-o") + 1] if "-o" in a else None
    defs = [x[2:] for x in a if x.startswith("-D")]
    print(build(force="--force" in a, verbose="-v" in a, out=out, defines=defs))
