"""Build libgmbe variants with extra -D flags into build_variants/ (experiments; git-ignored).
    python scripts/build_variants.py name1:"-DFOO=1 -DBAR" name2:"" ...
Run one with GMBE_LIB=build_variants/libgmbe_<name>.so python scripts/sweep.py ..."""
import os
import subprocess
import sys
from concurrent.futures import ThreadPoolExecutor

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, os.path.join(ROOT, "paper_conf_sc_panhlzwc23_b200"))
import _build  # noqa: E402

os.makedirs(os.path.join(ROOT, "build_variants"), exist_ok=True)


def one(spec):
    name, flags = spec.split(":", 1)
    out = os.path.join(ROOT, "build_variants", "libgmbe_%s.so" % name)
    cmd = [_build.nvcc()] + _build.NVCC_FLAGS + flags.split() + ["-o", out] + _build.SRC
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode:
        return name + " FAILED\n" + r.stderr[-3000:]
    lines = [l for l in (r.stdout + r.stderr).splitlines() if "6k_enumEN" in l or "spill" in l or "Used" in l]
    ke = [i for i, l in enumerate(lines) if "Function properties" in l and "6k_enumEN" in l]
    info = " | ".join(lines[ke[0] + 1: ke[0] + 3]) if ke else ""
    return "%s: %s" % (name, info)


with ThreadPoolExecutor(4) as ex:
    for r in ex.map(one, sys.argv[1:]):
        print(r)
