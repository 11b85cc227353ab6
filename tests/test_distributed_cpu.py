"""Data-parallel host logic on CPU with gloo, world size 2.

The only cross-rank step of the method is the sum of each layer's filter
gradient (dL/dw = sum over samples): sharding N over ranks and
summing the per-rank dw must equal the full-batch dw.  Checked with the fp64
oracle providing the per-rank partial gradients (the GPU kernels are not
needed for the host-side reduction logic)."""
import os
import socket
import tempfile

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _worker(rank, world, port, out_dir):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port), RANK=str(rank), WORLD_SIZE=str(world),
                      LOCAL_RANK=str(rank))
    import sys
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    import oracle
    from paper_conf_cluster_oyamabhm18_b200.distributed import (GradAllreduce, init_from_env, max_over_ranks,
                                                               shard_range)
    from synthetic import conv_inputs
    assert init_from_env("gloo")
    n, c, h, w, k, r, s, pad, st = 6, 3, 9, 9, 4, 3, 3, 1, 2
    x, _, dy = conv_inputs(n, c, h, w, k, r, s, pad, st, seed=21)
    lo, hi = shard_range(n, rank, world)
    dw_local = torch.from_numpy(oracle.conv_backward_filter(x[lo:hi], dy[lo:hi], r, s, pad, st))
    ar = GradAllreduce()
    ar(0, dw_local)
    ar.wait()
    t = max_over_ranks(float(rank + 1))
    np.save(os.path.join(out_dir, f"dw{rank}.npy"), dw_local.numpy())
    np.save(os.path.join(out_dir, f"t{rank}.npy"), np.array([t]))
    dist.barrier()
    dist.destroy_process_group()


def test_shard_range_covers_batch():
    from paper_conf_cluster_oyamabhm18_b200.distributed import shard_range
    for n in (1, 7, 256, 2048):
        for world in (1, 2, 3, 8):
            rng = [shard_range(n, r, world) for r in range(world)]
            assert rng[0][0] == 0 and rng[-1][1] == n
            assert all(a[1] == b[0] for a, b in zip(rng, rng[1:]))
            assert max(b - a for a, b in rng) - min(b - a for a, b in rng) <= 1


@pytest.mark.timeout(180)
def test_gloo_dw_allreduce_equals_full_batch():
    import oracle
    from synthetic import conv_inputs
    world = 2
    with tempfile.TemporaryDirectory() as d:
        mp.spawn(_worker, args=(world, _free_port(), d), nprocs=world, join=True)
        n, c, h, w, k, r, s, pad, st = 6, 3, 9, 9, 4, 3, 3, 1, 2
        x, _, dy = conv_inputs(n, c, h, w, k, r, s, pad, st, seed=21)
        full = oracle.conv_backward_filter(x, dy, r, s, pad, st)
        for rank in range(world):
            got = np.load(os.path.join(d, f"dw{rank}.npy"))
            assert np.max(np.abs(got - full)) <= 1e-12 * max(1.0, np.max(np.abs(full)))
            assert float(np.load(os.path.join(d, f"t{rank}.npy"))[0]) == world  # max over ranks
