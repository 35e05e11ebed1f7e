"""C-ABI library checks that need no GPU: the .so loads, exports every function include/gmbe.h
declares, the ctypes struct layouts equal the C compiler's, and the paper's sizing formulas."""
import os
import re
import subprocess
import ctypes

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HDR = os.path.join(ROOT, "include", "gmbe.h")


@pytest.fixture(scope="module")
def gmbe():
    import paper_conf_sc_panhlzwc23_b200 as m
    return m


def _declared():
    src = open(HDR).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(gmbe_[a-z0-9_]+)\s*\(", src)))


def test_exports_every_declared_symbol(gmbe):
    lib = ctypes.CDLL(gmbe.LIB_PATH)
    names = _declared()
    assert len(names) >= 8
    for n in names:
        assert hasattr(lib, n), n
    assert set(names) == set(gmbe.EXPORTS)
    out = subprocess.run(["nm", "-D", "--defined-only", gmbe.LIB_PATH], capture_output=True, text=True).stdout
    for n in names:
        assert re.search(r" T %s$" % n, out, flags=re.M), n


def test_struct_layouts_match_c(gmbe, tmp_path):
    c = tmp_path / "sz.c"
    c.write_text('#include <stdio.h>\n#include <stddef.h>\n#include "gmbe.h"\nint main(){'
                 'printf("%zu %zu %zu %zu %zu %zu %zu\\n", sizeof(gmbe_load_opts), sizeof(gmbe_graph_info),'
                 ' sizeof(gmbe_opts), sizeof(gmbe_result), offsetof(gmbe_opts, out_offsets),'
                 ' offsetof(gmbe_result, kernel_ms), offsetof(gmbe_opts, root_cursor));return 0;}')
    exe = tmp_path / "sz"
    subprocess.check_call(["gcc", "-I", os.path.dirname(HDR), str(c), "-o", str(exe)])
    got = list(map(int, subprocess.check_output([str(exe)]).split()))
    want = [ctypes.sizeof(gmbe.LoadOpts), ctypes.sizeof(gmbe.GraphInfo), ctypes.sizeof(gmbe.Opts),
            ctypes.sizeof(gmbe.CResult), gmbe.Opts.out_offsets.offset, gmbe.CResult.kernel_ms.offset,
            gmbe.Opts.root_cursor.offset]
    assert got == want


def test_paper_sizing_formulas(gmbe):
    # Sec 4.1: BookCrossing Δ(V)=13,601, Δ2(V)=53,915 -> 595 KB per procedure vs
    # 3.67 GB without node reuse, 6,178x.
    a = gmbe.node_buf_bound_bytes(13601, 53915)
    b = gmbe.naive_alloc_bytes(13601, 53915)
    assert a == 594532 and round(a / 1000) == 595
    assert b == 3673140464 and round(b / 1e9, 2) == 3.67
    assert int(b / a) == 6178


def test_import_fails_loudly_without_library(tmp_path):
    """The product path has no fallback: a package copy without libgmbe.so refuses to import."""
    import shutil
    import sys
    pkg = tmp_path / "paper_conf_sc_panhlzwc23_b200"
    shutil.copytree(os.path.join(ROOT, "paper_conf_sc_panhlzwc23_b200"), pkg,
                    ignore=shutil.ignore_patterns("*.so", "csrc", "__pycache__"))
    r = subprocess.run([sys.executable, "-c", "import paper_conf_sc_panhlzwc23_b200"], cwd=tmp_path,
                       capture_output=True, text=True)
    assert r.returncode != 0 and "libgmbe.so is not built" in r.stderr


def test_enum_constants_match_c(gmbe, tmp_path):
    """The binding's copies of the header's enums (cursor slots, IPC handle size, part modes,
    schedulers)."""
    c = tmp_path / "en.c"
    c.write_text('#include <stdio.h>\n#include "gmbe.h"\nint main(){printf("%d %d %d %d\\n",'
                 ' GMBE_CURSOR_SLOTS, GMBE_IPC_HANDLE_BYTES, GMBE_PART_INTERLEAVE, GMBE_PART_COST);'
                 'printf("%d %d %d\\n", GMBE_SCHED_TASK, GMBE_SCHED_WARP, GMBE_SCHED_BLOCK);'
                 'return 0;}')
    exe = tmp_path / "en"
    subprocess.check_call(["gcc", "-I", os.path.dirname(HDR), str(c), "-o", str(exe)])
    got = list(map(int, subprocess.check_output([str(exe)]).split()))
    assert got == [gmbe.CURSOR_SLOTS, gmbe.IPC_HANDLE_BYTES, gmbe.PART_MODE["interleave"],
                   gmbe.PART_MODE["cost"], gmbe.SCHEDULER["task"], gmbe.SCHEDULER["warp"],
                   gmbe.SCHEDULER["block"]]
    assert ctypes.sizeof(ctypes.c_uint64) * 16 == 128  # one cursor slot per 128-byte line (slot_ptr)
