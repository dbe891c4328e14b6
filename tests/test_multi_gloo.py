"""Multi-process (world_size 2, gloo, CPU) coverage of the N>1 path
(SURVEY.md 8(e)): contiguous RHS shards, no data-path collective, the
max-over-ranks time reduction, and shard results equal to the unsharded
solve bit for bit (the per-RHS arithmetic does not depend on the shard).
The per-shard solve here is the host run of the library's plan (no GPU)."""
import os
import socket

import numpy as np
import pytest
import torch.multiprocessing as mp

from paper_conf_sc_asahilbpbgo24_b200 import inputs
from paper_conf_sc_asahilbpbgo24_b200.shard import max_over_ranks, shard_bounds, weak_bounds


def test_shard_bounds_cover_and_balance():
    for total in (0, 1, 7, 100, 100001, 8_000_000):
        for world in (1, 2, 3, 4, 8):
            spans = [shard_bounds(r, world, total) for r in range(world)]
            assert spans[0][0] == 0 and spans[-1][1] == total
            assert all(a[1] == b[0] for a, b in zip(spans, spans[1:]))
            sizes = [b - a for a, b in spans]
            assert max(sizes) - min(sizes) <= 1
    assert weak_bounds(3, 100000) == (300000, 400000)
    with pytest.raises(ValueError):
        shard_bounds(2, 2, 10)


def test_rhs_shards_are_independent_of_sharding():
    n, total = 50, 10000
    full = inputs.rhs(n, total, seed=1234)
    for world in (2, 3, 5):
        parts = [inputs.rhs(n, b - a, seed=1234, first=a) for a, b in
                 (shard_bounds(r, world, total) for r in range(world))]
        assert np.array_equal(np.concatenate(parts, axis=1), full)


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _worker(rank, world, port, out):
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    from paper_conf_sc_asahilbpbgo24_b200 import SplineBuilder
    n_points, total = 200, 37
    sb = SplineBuilder(3, n_points, 0, host_only=True)
    a, b = shard_bounds(rank, world, total)
    x = inputs.rhs(sb.n, b - a, seed=7, first=a)
    sb.solve_cpu_plan_(x)
    t = max_over_ranks(float(rank + 1))  # the bench's max-over-ranks timing reduction
    np.save(os.path.join(out, f"shard{rank}.npy"), x)
    with open(os.path.join(out, f"t{rank}.txt"), "w") as f:
        f.write(repr(t))
    dist.barrier()
    dist.destroy_process_group()


def test_gloo_world2_shards_match_unsharded(tmp_path):
    world = 2
    mp.spawn(_worker, args=(world, _free_port(), str(tmp_path)), nprocs=world, join=True)
    from paper_conf_sc_asahilbpbgo24_b200 import SplineBuilder
    sb = SplineBuilder(3, 200, 0, host_only=True)
    full = inputs.rhs(sb.n, 37, seed=7)
    sb.solve_cpu_plan_(full)
    got = np.concatenate([np.load(tmp_path / f"shard{r}.npy") for r in range(world)], axis=1)
    assert np.array_equal(got, full)
    for r in range(world):
        assert float(open(tmp_path / f"t{r}.txt").read()) == float(world)
