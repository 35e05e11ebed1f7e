"""CPU oracle for maximal biclique enumeration -- TEST INFRASTRUCTURE ONLY.

Only tests/, __graft_entry__.smoke() and bench.py (cpu_baseline leg, --impl reference) may import
this package.  It shares no code with the CUDA path (paper_conf_sc_panhlzwc23_b200) and neither
imports the other.  `oracle_mbe` wraps the plain C++ oracle (gmbe_oracle.cpp);
`brute` holds the literal brute force (O3) used to pin the oracle itself.

Parity pins: see gmbe_oracle.cpp header and tests/test_oracle.py.  No function here is
"parity unpinned".
"""
import ctypes
import os
import subprocess
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "gmbe_oracle.cpp")
_LIB = os.path.join(_HERE, "liboracle.so")
_lib = None


def build(force=False):
    """Compile the oracle shared library with g++ (plain -O2, no SIMD flags)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + ".tmp.%d" % os.getpid()
        subprocess.check_call(["g++", "-O2", "-std=c++17", "-shared", "-fPIC", "-o", tmp, _SRC,
                               "-lpthread"])
        os.replace(tmp, _LIB)
    return _LIB


class _Res(ctypes.Structure):
    _fields_ = [(n, ctypes.c_uint64) for n in (
        "count", "checksum", "roots_run", "nodes", "nonmax", "algo_bytes", "algo_bytes_qfull",
        "n_written", "ids_written", "truncated", "closure_failures", "algo_bytes_cand")]


def _load():
    global _lib
    if _lib is None:
        _lib = ctypes.CDLL(build())
        f = _lib.oracle_mbe
        u32, u64, ptr = ctypes.c_uint32, ctypes.c_uint64, ctypes.c_void_p
        f.argtypes = [u32, u32, ptr, u64, ctypes.c_int, ctypes.c_int, u32, u32, ctypes.c_int,
                      ptr, u64, ptr, u64, ptr, ptr, ptr, ctypes.POINTER(_Res)]
        f.restype = ctypes.c_int
    return _lib


@dataclass
class OracleResult:
    count: int
    checksum: int
    roots_run: int
    nodes: int
    nonmax: int
    algo_bytes: int
    algo_bytes_qfull: int
    truncated: int
    closure_failures: int
    algo_bytes_cand: int = 0
    bicliques: list = None      # list of (tuple(L), tuple(R)) in caller ids, if requested
    per_root_count: np.ndarray = None
    per_root_ns: np.ndarray = None


def oracle_mbe(n_u, n_v, edges, order="degree", prune=True, shard=(0, 1), check_closure=False,
               records=False, rec_cap=1 << 20, ids_cap=1 << 24, per_root=False, root_mask=None,
               root_times=False):
    """Run the oracle on edge list `edges` (uint32 [m,2], rows (u,v), caller ids).
    root_mask: optional bool array over the internal V side (the smaller side; caller V unless
    n_u < n_v): only those roots are enumerated.  root_times: also return per-root wall ns."""
    lib = _load()
    e = np.ascontiguousarray(np.asarray(edges, dtype=np.uint32).reshape(-1, 2))
    res = _Res()
    offs = ids = None
    if records:
        offs = np.zeros(rec_cap, np.uint64)
        ids = np.zeros(ids_cap, np.uint32)
    nv_int = n_u if n_u < n_v else n_v
    prc = np.zeros(max(nv_int, 1), np.uint64) if per_root else None
    msk = None
    if root_mask is not None:
        msk = np.ascontiguousarray(np.asarray(root_mask, dtype=np.uint8))
        if len(msk) != nv_int:
            raise ValueError("root_mask: length %d != |internal V| %d" % (len(msk), nv_int))
    rns = np.zeros(max(nv_int, 1), np.uint64) if root_times else None
    rc = lib.oracle_mbe(n_u, n_v, e.ctypes.data if len(e) else None, len(e),
                        0 if order == "degree" else 1, 1 if prune else 0, shard[0], shard[1],
                        1 if check_closure else 0,
                        offs.ctypes.data if records else None, rec_cap if records else 0,
                        ids.ctypes.data if records else None, ids_cap if records else 0,
                        prc.ctypes.data if per_root else None,
                        msk.ctypes.data if msk is not None and len(msk) else None,
                        rns.ctypes.data if root_times else None, ctypes.byref(res))
    if rc != 0:
        raise ValueError("oracle_mbe: invalid arguments")
    out = OracleResult(res.count, res.checksum, res.roots_run, res.nodes, res.nonmax,
                       res.algo_bytes, res.algo_bytes_qfull, res.truncated, res.closure_failures,
                       res.algo_bytes_cand)
    if records:
        out.bicliques = decode_records(offs[:res.n_written], ids)
    if per_root:
        out.per_root_count = prc[:nv_int]
    if root_times:
        out.per_root_ns = rns[:nv_int]
    return out


def decode_records(offsets, ids):
    """Record = [|L|, |R|, L ids..., R ids...] (caller roles).  Returns sorted tuples."""
    out = []
    for o in offsets.tolist():
        nl, nr = int(ids[o]), int(ids[o + 1])
        l_ = tuple(sorted(ids[o + 2:o + 2 + nl].tolist()))
        r_ = tuple(sorted(ids[o + 2 + nl:o + 2 + nl + nr].tolist()))
        out.append((l_, r_))
    return out
