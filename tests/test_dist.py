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
