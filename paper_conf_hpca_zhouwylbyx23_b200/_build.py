"""Build libmpress.so (and the input generator's libsynth.so) in-tree with nvcc.

Every CUDA source is compiled for sm_100a only
(``-gencode arch=compute_100a,code=sm_100a -lineinfo``); cudart is linked
statically and the driver API is reached through cudaGetDriverEntryPoint, so
the library loads on a host without a GPU driver (the CPU test suite checks
its exports and runs the planner there).
"""
import os
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
# MPRESS_BUILD_TAG + MPRESS_NVCC_FLAGS: an experimental build (tools/ab.py)
# into build/<tag>/ and build/ab/libmpress_<tag>.so; the product build is untagged.
_TAG = os.environ.get("MPRESS_BUILD_TAG", "")
BUILD = os.path.join(ROOT, "build", _TAG) if _TAG else os.path.join(ROOT, "build")
LIB = os.path.join(ROOT, "build", "ab", "libmpress_%s.so" % _TAG) if _TAG else os.path.join(PKG, "libmpress.so")
SYNTH_SRC = os.path.join(ROOT, "synth", "fill.cu")
SYNTH_LIB = os.path.join(ROOT, "synth", "libsynth.so")

NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
CFLAGS = ["-O3", "-std=c++17", "-lineinfo", "-Xcompiler", "-fPIC,-fvisibility=hidden,-Wall,-Wextra",
          "-I" + os.path.join(ROOT, "include")] + os.environ.get("MPRESS_NVCC_FLAGS", "").split()


def _sources():
    return sorted(os.path.join(CSRC, f) for f in os.listdir(CSRC)
                  if f.endswith((".cpp", ".cu")))


def _headers():
    hs = [os.path.join(CSRC, f) for f in os.listdir(CSRC) if f.endswith(".h")]
    return hs + [os.path.join(ROOT, "include", "mpress.h")]


def _stale(target, deps):
    if not os.path.exists(target):
        return True
    t = os.path.getmtime(target)
    return any(os.path.getmtime(d) > t for d in deps)


def _run(cmd, verbose):
    if verbose:
        print(" ".join(cmd), file=sys.stderr)
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        raise RuntimeError("build failed:\n" + " ".join(cmd) + "\n" + r.stdout + r.stderr)
    return r.stdout + r.stderr


def build_mpress(verbose=False, force=False):
    os.makedirs(BUILD, exist_ok=True)
    os.makedirs(os.path.dirname(LIB), exist_ok=True)
    hdrs = _headers()
    objs = []
    for src in _sources():
        obj = os.path.join(BUILD, os.path.basename(src) + ".o")
        objs.append(obj)
        if force or _stale(obj, [src] + hdrs):
            extra = ["-Xptxas", "-v"] if src.endswith(".cu") else []
            out = _run([NVCC] + ARCH + CFLAGS + extra + ["-c", src, "-o", obj], verbose)
            if src.endswith(".cu"):
                with open(os.path.join(BUILD, os.path.basename(src) + ".ptxas.txt"), "w") as f:
                    f.write(out)
    exports = os.path.join(BUILD, "exports.map")
    with open(exports, "w") as f:
        f.write("{ global: mpress_*; local: *; };\n")
    if force or _stale(LIB, objs):
        _run([NVCC] + ARCH + ["-shared", "-o", LIB] + objs +
             ["-Xlinker", "--version-script=" + exports, "-lpthread", "-ldl", "-lrt"], verbose)
    return LIB


def build_synth(verbose=False, force=False):
    if force or _stale(SYNTH_LIB, [SYNTH_SRC]):
        _run([NVCC] + ARCH + ["-O3", "-std=c++17", "-Xcompiler", "-fPIC", "-shared",
                              SYNTH_SRC, "-o", SYNTH_LIB], verbose)
    return SYNTH_LIB


def build_all(verbose=False, force=False):
    return build_mpress(verbose, force), build_synth(verbose, force)


if __name__ == "__main__":
    print(build_all(verbose=True, force="--force" in sys.argv))
