"""Multi-GPU root sharding (Sec 5 "MBE on multiple GPUs",
P:1039-1056).

Roots v_s are independent sub-problems.  Rank i of a world of N enumerates the roots
whose degree rank r satisfies r % N == i (a degree-aware interleave: V is sorted by degree, so every
rank gets the same mix of light and heavy roots), with no exchange during the search.  The only
collective is one all-reduce (SUM) of the per-rank [count, checksum, ...] vector -- NCCL over NVLink /
NVSwitch on the B200 box, gloo in the CPU tests.  uint64 sums travel as int64 views: two's-complement
addition is bit-identical mod 2^64, so the reduced checksum equals the single-GPU one exactly.

DynamicRoots (the paper's GPUs draw root tasks from one shared pool):
instead of the fixed interleave, every rank draws positions of the (identical, replicated) root
issue list from ONE counter in rank 0's HBM, mapped into the other processes through CUDA IPC and
advanced with system-scope atomics over NVLink / NVSwitch.  Heavy roots are issued first, so the
ranks finish together whatever the degree tail.  The per-call all-reduce doubles as the one
synchronisation the rotating cursor slots need (gmbe.h, gmbe_shared_cursor_*).  If any rank cannot
map the cursor, every rank falls back to the static interleave (agreed by one MIN all-reduce).
"""
import torch
import torch.distributed as dist

FIELDS = ("count", "checksum", "roots_run", "nodes", "nonmax", "algo_bytes_cand")
_M64 = 1 << 64


def _i64(v):
    v %= _M64
    return v - _M64 if v >= (1 << 63) else v


def to_tensor(res, device="cpu"):
    """Pack a Result (or any object with FIELDS attributes / dict) into an int64 tensor."""
    get = (lambda f: res[f]) if isinstance(res, dict) else (lambda f: getattr(res, f))
    return torch.tensor([_i64(int(get(f))) for f in FIELDS], dtype=torch.int64, device=device)


def from_tensor(t):
    """Inverse of to_tensor: int64 tensor -> dict of uint64 values (mod 2^64)."""
    return {f: int(v) % _M64 for f, v in zip(FIELDS, t.cpu().tolist())}


def allreduce_result(res, group=None, device="cpu"):
    """Sum the per-rank results over the process group (one collective)."""
    t = to_tensor(res, device)
    if dist.is_available() and dist.is_initialized():
        dist.all_reduce(t, op=dist.ReduceOp.SUM, group=group)
    return from_tensor(t)


def shard_of(rank, world):
    """The enumerate() `part` argument of this rank."""
    if not 0 <= rank < world:
        raise ValueError("rank %d outside world %d" % (rank, world))
    return (rank, world)


def enumerate_sharded(graph, rank, world, group=None, device="cpu", **kw):
    """Enumerate this rank's root shard of `graph` and all-reduce the totals."""
    r = graph.enumerate(part=shard_of(rank, world), **kw)
    return r, allreduce_result(r, group=group, device=device)


class DynamicRoots:
    """Per-process handle of the shared root cursor (N1).  Collective constructor: every rank of
    `group` must build it, in the same order.  `device`: this rank's CUDA device index; `dev`:
    the torch device of the NCCL tensors (cpu for gloo)."""

    def __init__(self, rank, world, device, group=None, dev="cpu", cursor_factory=None,
                 fallback="interleave"):
        self.rank, self.world, self.group, self.dev = rank, world, group, dev
        self.fallback = fallback  # part_mode of the static split if the cursor is unavailable
        self.k = 0
        self.cursor = None
        if cursor_factory is None:
            from paper_conf_sc_panhlzwc23_b200 import SharedCursor
            cursor_factory = SharedCursor
        err = None
        box = [None]
        if rank == 0:
            try:
                self.cursor = cursor_factory.create(device)
                box[0] = self.cursor.handle()
            except Exception as ex:  # no CUDA IPC here: everyone falls back
                err = ex
        if world > 1:
            dist.broadcast_object_list(box, src=0, group=group)
            if rank != 0 and box[0] is not None:
                try:
                    self.cursor = cursor_factory.open(box[0], device)
                except Exception as ex:
                    err = ex
            ok = torch.tensor([0 if self.cursor is None else 1], dtype=torch.int64, device=dev)
            dist.all_reduce(ok, op=dist.ReduceOp.MIN, group=group)
            agreed = bool(ok.item())
        else:
            agreed = self.cursor is not None
        if not agreed:
            # ranks that mapped the owner's block unmap it first; only then may the owner free it
            if self.cursor is not None and rank != 0:
                self.cursor.close()
            if world > 1:
                dist.barrier(group=group)
            if self.cursor is not None and rank == 0:
                self.cursor.close()
            self.cursor = None
        self.error = None if agreed else str(err or "a peer rank could not map the cursor")

    @property
    def dynamic(self):
        return self.cursor is not None

    def enumerate(self, graph, stream=None, **kw):
        """One collective call: enumerate this rank's share of the roots and all-reduce the totals.
        Returns (this rank's Result, the reduced dict)."""
        k = self.k
        self.k += 1
        if self.cursor is None:
            if self.fallback != "interleave":
                kw["part_mode"] = self.fallback
            r = graph.enumerate(part=shard_of(self.rank, self.world), stream=stream, **kw)
        else:
            if self.rank == 0:  # slot k+1 is zero before any rank can reach call k+1
                self.cursor.reset(k + 1, stream=stream)
            r = graph.enumerate(root_cursor=self.cursor.slot_ptr(k), stream=stream, **kw)
        return r, allreduce_result(r, group=self.group, device=self.dev)

    def close(self):
        if self.cursor is not None:
            self.cursor.close()
            self.cursor = None
