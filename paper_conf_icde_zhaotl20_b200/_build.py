"""Compile libsong.so (the C-ABI library of include/song.h) for sm_100a, in-tree.

The kernel variants are split over one translation unit per row width
(csrc/launch_nch{1,2,4,8}.cu) and compiled in parallel, then linked with the
C-ABI (csrc/song_api.cu) into one shared library.
"""
import concurrent.futures
import os
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
BUILD = os.path.join(PKG, "build")
LIB = os.path.join(PKG, "libsong.so")
SOURCES = ["song_api.cu", "launch_nch1.cu", "launch_nch2.cu", "launch_nch4.cu", "launch_nch8.cu",
           "graph_build.cu"]
DEPS = [os.path.join(CSRC, f) for f in os.listdir(CSRC)] + [os.path.join(ROOT, "include", "song.h")]

NVCC_FLAGS = [
    "-gencode", "arch=compute_100a,code=sm_100a",
    "-O3", "-lineinfo", "-std=c++17",
    "-Xcompiler", "-fPIC",
    "-Xptxas", "-v",
]


def _compile(src, defines=(), build_dir=BUILD):
    obj = os.path.join(build_dir, src.replace(".cu", ".o"))
    cmd = ["nvcc", *NVCC_FLAGS, *[f"-D{d}" for d in defines], "-I", os.path.join(ROOT, "include"),
           "-I", CSRC, "-c", "-o", obj, os.path.join(CSRC, src)]
    res = subprocess.run(cmd, capture_output=True, text=True)
    return src, obj, res


def build(force: bool = False, verbose: bool = False, defines=(), out: str = LIB) -> str:
    """Build libsong.so; ``defines``/``out`` build an experiment variant (A/B
    measurements, e.g. SONG_DIST_V1) next to it without touching the default."""
    newest = max(os.path.getmtime(p) for p in DEPS)
    if not force and os.path.exists(out) and os.path.getmtime(out) >= newest:
        return out
    build_dir = BUILD if not defines else BUILD + "_" + "_".join(d.replace("=", "") for d in defines)
    os.makedirs(build_dir, exist_ok=True)
    with concurrent.futures.ThreadPoolExecutor(max_workers=len(SOURCES)) as ex:
        results = list(ex.map(lambda src: _compile(src, defines, build_dir), SOURCES))
    report = []
    for src, obj, res in results:
        if res.returncode != 0:
            sys.stderr.write(res.stdout + res.stderr)
            raise RuntimeError(f"nvcc failed compiling {src}")
        report.append(res.stderr)
    link = ["nvcc", "-shared", "-gencode", "arch=compute_100a,code=sm_100a", "-o", out,
            *[obj for _, obj, _ in results]]
    res = subprocess.run(link, capture_output=True, text=True)
    if res.returncode != 0:
        sys.stderr.write(res.stdout + res.stderr)
        raise RuntimeError("nvcc failed linking libsong.so")
    if out == LIB:
        with open(os.path.join(PKG, "ptxas_report.txt"), "w") as f:
            f.write("\n".join(report))
    if verbose:
        sys.stderr.write("\n".join(report))
    return out


if __name__ == "__main__":
    import argparse
    ap = argparse.ArgumentParser()
    ap.add_argument("--force", action="store_true")
    ap.add_argument("-v", action="store_true")
    ap.add_argument("--define", action="append", default=[])
    ap.add_argument("--out", default=LIB)
    a = ap.parse_args()
    print(build(force=a.force, verbose=a.v, defines=a.define, out=a.out))
