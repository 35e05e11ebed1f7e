"""Build libgmbe.so in-tree with nvcc for sm_100a (no JIT cache; the .so travels with the repo)."""
import os
import subprocess

HERE = os.path.dirname(os.path.abspath(__file__))
SRC = [os.path.join(HERE, "csrc", f) for f in ("gmbe_api.cu", "gmbe_graph.cu", "gmbe_enum.cu")]
DEPS = SRC + [os.path.join(HERE, "csrc", "gmbe_internal.cuh"), os.path.join(HERE, "csrc", "gmbe_block.cuh"),
              os.path.join(os.path.dirname(HERE), "include", "gmbe.h")]
LIB = os.path.join(HERE, "libgmbe.so")
LIB_PROF = os.path.join(HERE, "libgmbe_prof.so")  # phase-profiling variant (-DGMBE_PROFILE)
NVCC_FLAGS = ["-gencode", "arch=compute_100a,code=sm_100a", "-lineinfo", "-O3", "-std=c++17",
              "-Xcompiler", "-fPIC", "-shared", "-Xptxas", "-v"]


def nvcc():
    for c in (os.environ.get("NVCC"), "/usr/local/cuda/bin/nvcc", "nvcc"):
        if c and (os.path.sep not in c or os.path.exists(c)):
            return c
    return "nvcc"


def build(force=False, verbose=False, profile=False):
    """Compile every CUDA source into libgmbe.so (and, with profile=True, libgmbe_prof.so).
    Skipped when up to date."""
    if profile:
        build(force, verbose)
    lib = LIB_PROF if profile else LIB
    if not force and os.path.exists(lib):
        t = os.path.getmtime(lib)
        if all(os.path.getmtime(d) <= t for d in DEPS):
            return lib
    tmp = lib + ".tmp.%d" % os.getpid()
    cmd = [nvcc()] + NVCC_FLAGS + (["-DGMBE_PROFILE"] if profile else []) + ["-o", tmp] + SRC
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        raise RuntimeError("nvcc failed:\n" + r.stdout + r.stderr)
    if not profile:
        with open(os.path.join(HERE, "ptxas_report.txt"), "w") as f:
            f.write(r.stdout + r.stderr)
    if verbose:
        print(r.stderr)
    os.replace(tmp, lib)
    return lib
