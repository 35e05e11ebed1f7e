"""Multi-GPU root sharding (Sec 5 "MBE on multiple GPUs",
P:1039-1056).

Roots v_s are independent sub-problems.  Rank i of a world of N enumerates the roots
whose degree rank r satisfies r % N == i (a degree-aware interleave: V is sorted by degree, so every
rank gets the same mix of light and heavy roots), with no exchange during the search.  The only
collective is one all-reduce (SUM) of the per-rank [count, checksum, ...] vector -- NCCL over NVLink /
NVSwitch on the B200 box, gloo in the CPU tests.  uint64 sums travel as int64 views: two's-complement
addition is bit-identical mod 2^64, so the reduced checksum equals the single-GPU one exactly.
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
