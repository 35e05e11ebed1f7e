"""Python binding of libgmbe.so -- the B200 (sm_100a) maximal biclique enumeration library.

Argument marshalling only: every step of the path (graph build, root generation, search,
splitting, reduction) runs in the CUDA kernels behind the C ABI declared in include/gmbe.h.
There is no CPU fallback: importing this package fails loudly if libgmbe.so is missing.

    import paper_conf_sc_panhlzwc23_b200 as gmbe
    g = gmbe.load(n_u, n_v, edges)          # edges: uint32 [m, 2] numpy (host) or torch (cuda)
    r = g.enumerate()                        # -> Result(count, checksum, ...)
"""
import ctypes
import os
from dataclasses import dataclass, field

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("GMBE_LIB") or os.path.join(_HERE, "libgmbe.so")  # GMBE_LIB: experiments only
if not os.path.exists(LIB_PATH):
    raise ImportError("libgmbe.so is not built (run `python -c 'import __graft_entry__ as e; e.build()'`); "
                      "there is no CPU fallback")
_lib = ctypes.CDLL(LIB_PATH)

GMBE_OK, GMBE_EINVAL, GMBE_ENOMEM, GMBE_ECUDA, GMBE_EUNSUPPORTED, GMBE_EINTERNAL = 0, -1, -2, -3, -4, -5
ORDER = {"degree": 0, "identity": 1}
PHASES = ("root_wedges", "classify", "sort", "root_finish", "cand_scan", "maximality", "emit", "queue",
          "root_emit", "col_transpose", "root_entries", "root_pass2", "root_mask_hdr", "pool_alloc",
          "lprime", "dequeue")
EXPORTS = ("gmbe_load_bipartite", "gmbe_graph_info_get", "gmbe_free_graph", "gmbe_node_buf_bound_bytes",
           "gmbe_kernel_launch_count",
           "gmbe_naive_alloc_bytes", "gmbe_enumerate", "gmbe_enumerate_stream", "gmbe_release_workspace",
           "gmbe_last_error", "gmbe_shared_cursor_create", "gmbe_shared_cursor_open",
           "gmbe_shared_cursor_reset", "gmbe_shared_cursor_close")
CURSOR_SLOTS, IPC_HANDLE_BYTES = 16, 64
PART_MODE = {"interleave": 0, "cost": 1}
SCHEDULER = {"task": 0, "warp": 1, "block": 2}  # GMBE (Alg 4), GMBE-WARP, GMBE-BLOCK

_u32, _i32, _u64, _vp = ctypes.c_uint32, ctypes.c_int32, ctypes.c_uint64, ctypes.c_void_p


class LoadOpts(ctypes.Structure):
    _fields_ = [("struct_size", _u32), ("device", _i32), ("cuda_stream", _vp),
                ("edges_on_device", _u32), ("order", _u32)]


class GraphInfo(ctypes.Structure):
    _fields_ = [("n_u", _u64), ("n_v", _u64), ("n_edges_unique", _u64), ("delta_u", _u32),
                ("delta_v", _u32), ("wedge_bound_v", _u32), ("swapped", _u32), ("order", _u32),
                ("device", _u32)]


class Opts(ctypes.Structure):
    _fields_ = [("struct_size", _u32), ("no_prune", _u32), ("no_split", _u32), ("bound_height", _u32),
                ("bound_size", _u32), ("warps_per_sm", _u32), ("part_index", _u32),
                ("part_count", _u32), ("reserved0", _u32), ("scheduler", _u32),
                ("out_offsets", _vp), ("out_offsets_cap", _u64), ("out_ids", _vp),
                ("out_ids_cap", _u64), ("per_root_count", _vp), ("per_root_cycles", _vp), ("phase_cycles", _vp), ("timeline", _vp), ("timeline_cap", _u64),
                ("arena_words", _u64),
                ("pool_words", _u64), ("queue_cap", _u64), ("cuda_stream", _vp),
                ("split_wide", _u32), ("thr_min", _u32), ("root_cursor", _vp),
                ("part_mode", _u32), ("root_chunk", _u32)]


class CResult(ctypes.Structure):
    _fields_ = [(n, _u64) for n in ("count", "checksum", "n_written", "truncated", "roots_run",
                                     "nodes", "nonmax", "algo_bytes_cand", "splits",
                                     "tasks", "donations")] + [("kernel_ms", ctypes.c_double), ("retries", _u64)]


_lib.gmbe_load_bipartite.argtypes = [_u32, _u32, _vp, _u64, ctypes.POINTER(LoadOpts), ctypes.POINTER(_vp)]
_lib.gmbe_load_bipartite.restype = ctypes.c_int
_lib.gmbe_graph_info_get.argtypes = [_vp, ctypes.POINTER(GraphInfo)]
_lib.gmbe_graph_info_get.restype = ctypes.c_int
_lib.gmbe_free_graph.argtypes = [_vp]
_lib.gmbe_free_graph.restype = None
_lib.gmbe_release_workspace.argtypes = [_vp]
_lib.gmbe_release_workspace.restype = None
_lib.gmbe_node_buf_bound_bytes.argtypes = [_u64, _u64]
_lib.gmbe_node_buf_bound_bytes.restype = _u64
_lib.gmbe_naive_alloc_bytes.argtypes = [_u64, _u64]
_lib.gmbe_naive_alloc_bytes.restype = _u64
_lib.gmbe_shared_cursor_create.argtypes = [_i32, ctypes.POINTER(_vp), _vp]
_lib.gmbe_shared_cursor_create.restype = ctypes.c_int
_lib.gmbe_shared_cursor_open.argtypes = [_vp, _i32, ctypes.POINTER(_vp)]
_lib.gmbe_shared_cursor_open.restype = ctypes.c_int
_lib.gmbe_shared_cursor_reset.argtypes = [_vp, _u32, _vp]
_lib.gmbe_shared_cursor_reset.restype = ctypes.c_int
_lib.gmbe_shared_cursor_close.argtypes = [_vp, _i32]
_lib.gmbe_shared_cursor_close.restype = None
_lib.gmbe_enumerate.argtypes = [_vp, ctypes.POINTER(Opts), ctypes.POINTER(CResult)]
_lib.gmbe_enumerate.restype = ctypes.c_int
SINK_FN = ctypes.CFUNCTYPE(ctypes.c_int, ctypes.POINTER(ctypes.c_uint32), ctypes.c_uint64, ctypes.c_uint64, ctypes.c_void_p)
_lib.gmbe_enumerate_stream.argtypes = [_vp, ctypes.POINTER(Opts), SINK_FN, _vp, _u64, ctypes.POINTER(CResult)]
_lib.gmbe_enumerate_stream.restype = ctypes.c_int
_lib.gmbe_kernel_launch_count.argtypes = []
_lib.gmbe_kernel_launch_count.restype = _u64
_lib.gmbe_last_error.argtypes = []
_lib.gmbe_last_error.restype = ctypes.c_char_p


class GmbeError(RuntimeError):
    def __init__(self, code, msg):
        super().__init__("%s (code %d)" % (msg, code))
        self.code = code


def _check(rc):
    if rc != GMBE_OK:
        raise GmbeError(rc, _lib.gmbe_last_error().decode(errors="replace"))


def kernel_launch_count():
    """Number of libgmbe kernels launched so far in this process."""
    return int(_lib.gmbe_kernel_launch_count())


def node_buf_bound_bytes(delta_v, delta2_v):
    """Paper's per-procedure node_buf bound (3Δ(V)+2Δ2(V))·4 B."""
    return int(_lib.gmbe_node_buf_bound_bytes(delta_v, delta2_v))


def naive_alloc_bytes(delta_v, delta2_v):
    """Paper's per-subtree allocation without node reuse Δ(V)(Δ(V)+Δ2(V))·4 B."""
    return int(_lib.gmbe_naive_alloc_bytes(delta_v, delta2_v))


@dataclass
class Result:
    count: int
    checksum: int
    n_written: int
    truncated: int
    roots_run: int
    nodes: int
    nonmax: int
    algo_bytes_cand: int
    splits: int
    tasks: int
    donations: int
    kernel_ms: float
    retries: int = 0
    bicliques: list = field(default=None, repr=False)
    per_root_count: np.ndarray = field(default=None, repr=False)
    per_root_cycles: np.ndarray = field(default=None, repr=False)
    phase_cycles: dict = field(default=None, repr=False)
    timeline: np.ndarray = field(default=None, repr=False)


CUDA_STREAM_LEGACY = 0x1  # cudaStreamLegacy: the legacy default stream as an explicit handle


def _stream_ptr(stream):
    """cudaStream_t of a torch stream (or a raw handle).  torch's default stream has handle 0, which
    the library reads as "no stream given" (its own non-blocking stream, NOT ordered after torch's
    work), so it is passed as cudaStreamLegacy instead."""
    if stream is None:
        return None
    h = int(getattr(stream, "cuda_stream", stream))
    return h if h else CUDA_STREAM_LEGACY


class Graph:
    """Device-resident bipartite graph (opaque gmbe_graph handle)."""

    def __init__(self, handle):
        self._h = handle

    @property
    def handle(self):
        return self._h

    def info(self):
        gi = GraphInfo()
        _check(_lib.gmbe_graph_info_get(self._h, ctypes.byref(gi)))
        return {k: getattr(gi, k) for k, _ in GraphInfo._fields_}

    def enumerate(self, prune=True, split=True, bound_height=0, bound_size=0, warps_per_sm=0,
                  part=(0, 1), records=False, rec_cap=1 << 16, ids_cap=1 << 22,
                  per_root=False, root_cycles=False, phases=False, timeline=0, debug=0, thr_min=0, split_wide=0, arena_words=0, pool_words=0, queue_cap=0, stream=None,
                  root_cursor=None, part_mode="interleave", scheduler="task", root_chunk=0):
        """gmbe_enumerate.  records=True allocates device output buffers (torch) and decodes them.
        root_cursor: device address (int) of a shared root-cursor slot (SharedCursor.slot_ptr).
        part_mode: how `part` splits the roots -- "interleave" (degree rank mod N) or "cost" (N4).
        scheduler: "task" (GMBE, default), "warp" (GMBE-WARP) or "block" (GMBE-BLOCK), Sec 4.3."""
        o = Opts()
        o.struct_size = ctypes.sizeof(Opts)
        o.no_prune = 0 if prune else 1
        o.no_split = 0 if split else 1
        o.bound_height, o.bound_size, o.warps_per_sm = bound_height, bound_size, warps_per_sm
        o.part_index, o.part_count = part
        o.arena_words, o.pool_words, o.queue_cap = arena_words, pool_words, queue_cap
        o.cuda_stream = _stream_ptr(stream)
        o.reserved0 = debug
        o.thr_min, o.split_wide = thr_min, split_wide
        o.root_cursor = root_cursor
        o.part_mode = PART_MODE[part_mode]
        o.scheduler = SCHEDULER[scheduler]
        o.root_chunk = root_chunk
        bufs = None
        if records:
            import torch
            dev = torch.device("cuda", self.info()["device"])
            offs = torch.empty(rec_cap, dtype=torch.int64, device=dev)
            ids = torch.empty(ids_cap, dtype=torch.int32, device=dev)
            o.out_offsets, o.out_offsets_cap = offs.data_ptr(), rec_cap
            o.out_ids, o.out_ids_cap = ids.data_ptr(), ids_cap
            bufs = (offs, ids)
        prc = None
        if per_root:
            inf = self.info()
            nv_int = inf["n_u"] if inf["swapped"] else inf["n_v"]
            prc = np.zeros(max(nv_int, 1), np.uint64)
            o.per_root_count = prc.ctypes.data
        prcy = None
        if root_cycles:
            inf = self.info()
            prcy = np.zeros(max(inf["n_u"] if inf["swapped"] else inf["n_v"], 1), np.uint64)
            o.per_root_cycles = prcy.ctypes.data
        tl = None
        if timeline:
            import torch
            tdev = torch.device("cuda", self.info()["device"])
            tl = torch.zeros(1 + 4 * timeline, dtype=torch.int64, device=tdev)
            torch.cuda.current_stream(tdev).synchronize()  # the fill is on torch's stream, not the library's
            o.timeline, o.timeline_cap = tl.data_ptr(), 1 + 4 * timeline
        phc = None
        if phases:
            phc = np.zeros(16, np.uint64)
            o.phase_cycles = phc.ctypes.data
        cr = CResult()
        _check(_lib.gmbe_enumerate(self._h, ctypes.byref(o), ctypes.byref(cr)))
        res = Result(**{k: getattr(cr, k) for k, _ in CResult._fields_})
        if records:
            offs = bufs[0][: res.n_written].cpu().numpy().view(np.uint64)
            ids = bufs[1].cpu().numpy().view(np.uint32)
            res.bicliques = decode_records(offs, ids)
        if root_cycles:
            res.per_root_cycles = prcy
        if timeline:
            t = tl.cpu().numpy().view(np.uint64)
            nrec = min(int(t[0]), timeline)
            res.timeline = t[1:1 + 4 * nrec].reshape(-1, 4)
        if phases:
            res.phase_cycles = dict(zip(PHASES, phc.tolist()))
        if per_root:
            res.per_root_count = prc[: (self.info()["n_u"] if self.info()["swapped"] else self.info()["n_v"])]
        return res

    def enumerate_stream(self, sink, ring_words=0, prune=True, split=True, bound_height=0, bound_size=0,
                         part=(0, 1), debug=0, thr_min=0, split_wide=0, stream=None):
        """gmbe_enumerate_stream: every maximal biclique record is handed to sink(words, n_records)
        (words: uint32 numpy array of whole records [|L|, |R|, L ids, R ids], valid during the call)
        while the kernel runs, through a bounded ring in pinned host memory."""
        o = Opts()
        o.struct_size = ctypes.sizeof(Opts)
        o.no_prune = 0 if prune else 1
        o.no_split = 0 if split else 1
        o.bound_height, o.bound_size = bound_height, bound_size
        o.part_index, o.part_count = part
        o.cuda_stream = _stream_ptr(stream)
        o.reserved0 = debug
        o.thr_min, o.split_wide = thr_min, split_wide
        err = []

        def _cb(words, n_words, n_records, user):
            try:
                sink(np.ctypeslib.as_array(words, shape=(int(n_words),)), int(n_records))
                return 0
            except Exception as ex:  # reported after the call; the ring is drained
                err.append(ex)
                return 1

        cb = SINK_FN(_cb)
        cr = CResult()
        rc = _lib.gmbe_enumerate_stream(self._h, ctypes.byref(o), cb, None, ring_words, ctypes.byref(cr))
        if err:
            raise err[0]
        _check(rc)
        return Result(**{k: getattr(cr, k) for k, _ in CResult._fields_})

    def release_workspace(self):
        if self._h:
            _lib.gmbe_release_workspace(self._h)

    def free(self):
        if self._h:
            _lib.gmbe_free_graph(self._h)
            self._h = None

    def __del__(self):
        try:
            self.free()
        except Exception:
            pass


class SharedCursor:
    """A block of CURSOR_SLOTS root cursors in one GPU's memory, shareable across processes through
    CUDA IPC (gmbe_shared_cursor_*).  create() on the owner, handle() -> bytes to
    broadcast, open(handle) on the others."""

    def __init__(self, ptr, owner):
        self.ptr, self.owner = ptr, owner

    @classmethod
    def create(cls, device):
        p, h = _vp(), ctypes.create_string_buffer(IPC_HANDLE_BYTES)
        _check(_lib.gmbe_shared_cursor_create(device, ctypes.byref(p), h))
        c = cls(p.value, 1)
        c._handle = h.raw
        return c

    @classmethod
    def open(cls, handle, device):
        p = _vp()
        buf = ctypes.create_string_buffer(bytes(handle), IPC_HANDLE_BYTES)
        _check(_lib.gmbe_shared_cursor_open(buf, device, ctypes.byref(p)))
        return cls(p.value, 0)

    def handle(self):
        return self._handle

    def slot_ptr(self, k):
        return self.ptr + 128 * (k % CURSOR_SLOTS)

    def reset(self, k, stream=None):
        _check(_lib.gmbe_shared_cursor_reset(self.ptr, k % CURSOR_SLOTS, _stream_ptr(stream)))

    def close(self):
        if self.ptr:
            _lib.gmbe_shared_cursor_close(self.ptr, self.owner)
            self.ptr = None


def decode_records(offsets, ids):
    """Records [|L|, |R|, L ids, R ids] (caller roles) -> sorted list of (tuple(L), tuple(R)).
    Records that did not fit (offset == UINT64_MAX) are skipped."""
    out = []
    for o in offsets.tolist():
        if o == 0xFFFFFFFFFFFFFFFF:
            continue
        nl, nr = int(ids[o]), int(ids[o + 1])
        out.append((tuple(sorted(ids[o + 2:o + 2 + nl].tolist())),
                    tuple(sorted(ids[o + 2 + nl:o + 2 + nl + nr].tolist()))))
    return sorted(out)


def iter_records(words):
    """Split a batch of streamed records into (L ids, R ids) array pairs (caller roles)."""
    i, n = 0, len(words)
    while i < n:
        nl, nr = int(words[i]), int(words[i + 1])
        yield words[i + 2:i + 2 + nl], words[i + 2 + nl:i + 2 + nl + nr]
        i += 2 + nl + nr


def load(n_u, n_v, edges, order="degree", device=None, stream=None):
    """gmbe_load_bipartite.  `edges`: uint32/int32 [m, 2] rows (u, v) -- numpy (host) or a CUDA
    torch tensor (device pointer, no host copy)."""
    lo = LoadOpts()
    lo.struct_size = ctypes.sizeof(LoadOpts)
    lo.device = -1 if device is None else int(device)
    lo.cuda_stream = _stream_ptr(stream)
    lo.order = ORDER[order]
    keep = None
    if hasattr(edges, "is_cuda") and edges.is_cuda:
        import torch
        e = edges.contiguous()
        if e.element_size() != 4:
            raise TypeError("device edges must be a 32-bit integer tensor")
        ptr, m = e.data_ptr(), e.numel() // 2
        lo.edges_on_device = 1
        if device is None:
            lo.device = e.device.index
        if stream is None:
            # the edges were produced (or made contiguous) on torch's current stream: build on it
            lo.cuda_stream = _stream_ptr(torch.cuda.current_stream(e.device))
        keep = e
    else:
        a = np.asarray(edges)
        if a.dtype == np.int32:
            a = a.view(np.uint32)  # zero-copy (e.g. a pinned int32 buffer stays pinned)
        e = np.ascontiguousarray(a.astype(np.uint32, copy=False).reshape(-1, 2))
        ptr, m = (e.ctypes.data if len(e) else None), len(e)
        keep = e
    h = _vp()
    _check(_lib.gmbe_load_bipartite(n_u, n_v, ptr, m, ctypes.byref(lo), ctypes.byref(h)))
    del keep
    return Graph(h.value)


def enumerate_bicliques(n_u, n_v, edges, **kw):
    """Convenience: load + enumerate + free."""
    order = kw.pop("order", "degree")
    g = load(n_u, n_v, edges, order=order)
    try:
        return g.enumerate(**kw)
    finally:
        g.free()
