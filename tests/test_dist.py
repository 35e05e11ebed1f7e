"""Multi-process (world_size 2, gloo, CPU) checks of the multi-GPU host logic: root shards partition
the output and one all-reduce of the int64-viewed [count, checksum, ...] vector reproduces the
single-process totals bit-exactly (including mod-2^64 wraparound).  Per-rank shard results come from
the oracle here (no GPU); on the B200 box the same reduction runs over NCCL in bench.py."""
import os
import socket

import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle
from gmbe_inputs import make_config

try:
    from paper_conf_sc_panhlzwc23_b200 import dist as gdist
except ImportError as e:  # the .so must be built (build() runs first in the driver)
    pytest.skip(str(e), allow_module_level=True)


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _worker(rank, world, port, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        nu, nv, e = make_config("er40")
        part = gdist.shard_of(rank, world)
        r = oracle.oracle_mbe(nu, nv, e, shard=part)
        tot = gdist.allreduce_result(r)
        # wraparound: both ranks contribute 2^63 + 5 -> 10 (mod 2^64)
        wrap = gdist.allreduce_result({"count": 0, "checksum": (1 << 63) + 5, "roots_run": 0,
                                       "nodes": 0, "nonmax": 0, "algo_bytes_cand": 0})
        q.put((rank, tot, wrap["checksum"]))
    finally:
        dist.destroy_process_group()


def test_two_rank_allreduce_matches_single():
    world, port = 2, _free_port()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    ps = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in ps:
        p.start()
    out = [q.get(timeout=120) for _ in range(world)]
    for p in ps:
        p.join(timeout=60)
        assert p.exitcode == 0
    nu, nv, e = make_config("er40")
    full = oracle.oracle_mbe(nu, nv, e)
    for rank, tot, wrap in out:
        assert tot["count"] == full.count == 211
        assert tot["checksum"] == full.checksum
        assert tot["nodes"] == full.nodes and tot["algo_bytes_cand"] == full.algo_bytes_cand
        assert wrap == 10


def test_tensor_roundtrip_and_shard_validation():
    vals = {"count": 7, "checksum": (1 << 64) - 1, "roots_run": 3, "nodes": 9, "nonmax": 2,
            "algo_bytes_cand": 1 << 40}
    t = gdist.to_tensor(vals)
    assert t.dtype == torch.int64
    assert gdist.from_tensor(t) == vals
    assert gdist.shard_of(1, 4) == (1, 4)
    with pytest.raises(ValueError):
        gdist.shard_of(4, 4)


# ---- N1 dynamic root distribution: host protocol (slot rotation, handle broadcast, agreement) ----
class _FileCursor:
    """Stand-in for SharedCursor on CPU: the slots live in a file, increments under flock, so two
    processes really race on one counter (the GPU version: system-scope atomics over NVLink)."""
    SLOTS = 16

    def __init__(self, path, owner):
        self.path, self.owner = path, owner

    @classmethod
    def create(cls, device):
        import tempfile
        fd, path = tempfile.mkstemp(prefix="gmbe_cursor_")
        os.write(fd, b"\0" * 8 * cls.SLOTS)
        os.close(fd)
        return cls(path, 1)

    @classmethod
    def open(cls, handle, device):
        if os.environ.get("GMBE_TEST_FAIL_OPEN") == str(dist.get_rank()):
            raise RuntimeError("simulated: no peer access")
        return cls(handle, 0)

    def handle(self):
        return self.path

    def slot_ptr(self, k):
        return (self.path, k % self.SLOTS)

    def reset(self, k, stream=None):
        self._rw(k % self.SLOTS, lambda v: 0)

    def _rw(self, slot, f):
        import fcntl
        with open(self.path, "r+b") as fh:
            fcntl.flock(fh, fcntl.LOCK_EX)
            fh.seek(8 * slot)
            v = int.from_bytes(fh.read(8), "little")
            fh.seek(8 * slot)
            fh.write(int(f(v)).to_bytes(8, "little"))
            fh.flush()
            fcntl.flock(fh, fcntl.LOCK_UN)
            return v

    def close(self):
        if self.owner:
            os.unlink(self.path)


class _OracleGraph:
    """Graph stand-in: part=(i, n) -> the oracle's static shard; root_cursor -> draw root ranks
    from the shared counter one at a time (shard (t, n_v) is exactly root rank t)."""

    def __init__(self, nu, nv, e):
        self.nu, self.nv, self.e = nu, nv, e

    def enumerate(self, part=(0, 1), root_cursor=None, stream=None):
        if root_cursor is None:
            return oracle.oracle_mbe(self.nu, self.nv, self.e, shard=part)
        path, slot = root_cursor
        cur = _FileCursor(path, 0)
        tot = dict(count=0, checksum=0, roots_run=0, nodes=0, nonmax=0, algo_bytes_cand=0)
        n_roots = min(self.nu, self.nv)
        while True:
            t = cur._rw(slot, lambda v: v + 1)
            if t >= n_roots:
                return tot
            r = oracle.oracle_mbe(self.nu, self.nv, self.e, shard=(t, n_roots))
            for f in tot:
                tot[f] = (tot[f] + getattr(r, f)) % (1 << 64)


def _dyn_worker(rank, world, port, fail_rank, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    if fail_rank is not None:
        os.environ["GMBE_TEST_FAIL_OPEN"] = str(fail_rank)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        dr = gdist.DynamicRoots(rank, world, device=0, cursor_factory=_FileCursor)
        g = _OracleGraph(*make_config("er40"))
        outs = []
        for _ in range(3):  # consecutive calls rotate slots; only the all-reduce separates them
            r, tot = dr.enumerate(g)
            mine = r["count"] if isinstance(r, dict) else r.count
            outs.append((mine, tot["count"], tot["checksum"], tot["nodes"]))
        q.put((rank, dr.dynamic, outs))
        dist.barrier()
        dr.close()
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world,fail_rank", [(2, None), (2, 1), (3, None), (3, 2)])
def test_dynamic_roots_protocol(world, fail_rank):
    port = _free_port()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    ps = [ctx.Process(target=_dyn_worker, args=(r, world, port, fail_rank, q)) for r in range(world)]
    for p in ps:
        p.start()
    out = sorted(q.get(timeout=300) for _ in range(world))
    for p in ps:
        p.join(timeout=60)
        assert p.exitcode == 0
    full = oracle.oracle_mbe(*make_config("er40"))
    for step in range(3):
        assert sum(o[2][step][0] for o in out) == full.count  # the ranks' draws partition the roots
    for rank, dyn, outs in out:
        assert dyn == (fail_rank is None)  # one failing rank -> both fall back to the interleave
        for mine, cnt, cks, nodes in outs:
            assert (cnt, cks, nodes) == (full.count, full.checksum, full.nodes)
