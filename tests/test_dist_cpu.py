"""Host-side multi-process checks on CPU (gloo, world size 2): the sharding invariant the distributed check
relies on — races are a property of one location, so checking each location-owner shard separately (with global
record indices) and merging equals checking the whole trace — and the shard/index_base plumbing of bench.py."""
import os

import numpy as np
import pytest

import sesagen as G
from oracle import oracle as O

torch = pytest.importorskip("torch")
import torch.distributed as dist  # noqa: E402
import torch.multiprocessing as mp  # noqa: E402


def location_owner(r, world, G_=4):
    """owner rank of each record's first granule location (records here never span granules)."""
    g = (r["addr"] // G_).astype(np.uint64)
    key = np.where(r["space"] == 0, (r["block"].astype(np.uint64) << np.uint64(40)) ^ (r["interval"].astype(np.uint64) << np.uint64(32)) ^ g, g)
    h = (key * np.uint64(0x9E3779B97F4A7C15)) >> np.uint64(40)
    return (h % np.uint64(world)).astype(np.int64)


def _worker(rank, world, port, out):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    r = G.random_trace(6000, 42, threads=100, words=300, sizes=(4,), unaligned=False)
    n = len(r)
    lo, hi = rank * n // world, (rank + 1) * n // world
    # index_base = exclusive prefix of shard sizes, agreed by all-gather (what bench.py / callers pass)
    sizes = [None] * world
    dist.all_gather_object(sizes, hi - lo)
    assert sum(sizes[:rank]) == lo
    # owner partition of the whole trace (every rank computes the same mapping from its own shard's view)
    owner = location_owner(r, world)
    mine = np.flatnonzero(owner == rank)
    sub = r[mine]
    races = O.check(sub)  # indices are local to `sub`: map back to global record indices
    races["first"] = mine[races["first"].astype(np.int64)]
    races["second"] = mine[races["second"].astype(np.int64)]
    gathered = [None] * world
    dist.all_gather_object(gathered, races.tobytes())
    if rank == 0:
        merged = np.concatenate([np.frombuffer(b, dtype=O.RACE_DTYPE) for b in gathered])
        order = np.lexsort((merged["kind"], merged["addr"], merged["interval"], merged["block"], merged["space"]))
        out.put(bool(merged[order].tobytes() == O.check(r).tobytes()))
    dist.destroy_process_group()


def test_sharded_oracle_merge_equals_whole_gloo():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = 29500 + os.getpid() % 1000
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    ok = q.get(timeout=120)
    for p in procs:
        p.join(timeout=60)
    assert ok
