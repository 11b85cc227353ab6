"""I7 on a multi-GPU box: the global mini-batch sharded
over 2 GPUs (NCCL, one process per GPU) gives per-sample forward / backward-data
outputs bitwise equal to the single-GPU run of the same plan, and the allreduced
dW equal to the single-GPU full-batch dW (exact on integer data).  Skipped when
fewer than 2 GPUs are visible (the round's GPU box has one)."""
import os
import socket
import tempfile

import numpy as np
import pytest
import torch

pytestmark = pytest.mark.gpu

N_GLOBAL = 16


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _run(rank, world, port, out_dir):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port), RANK=str(rank), WORLD_SIZE=str(world),
                      LOCAL_RANK=str(rank))
    import sys
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    import torch.distributed as dist
    import paper_conf_cluster_oyamabhm18_b200 as mu
    from paper_conf_cluster_oyamabhm18_b200.distributed import GradAllreduce, init_from_env, shard_range
    from paper_conf_cluster_oyamabhm18_b200.network import ConvNet
    from synthetic import network
    if world > 1:
        assert init_from_env("nccl")
    torch.cuda.set_device(rank)
    layers = network("alexnet")[:3]
    lo, hi = shard_range(N_GLOBAL, rank, world)
    h = mu.Handle(rank)
    net = ConvNet(h, layers, hi - lo, mu.MATH_BF16, device=f"cuda:{rank}")
    net.allocate(seed=0, kind="int")
    # same global data on every world size: slice the global batch
    full = ConvNet(h, layers, N_GLOBAL, mu.MATH_BF16, device=f"cuda:{rank}")
    full.allocate(seed=0, kind="int")
    for t, f in zip(net.tensors, full.tensors):
        t["x"].copy_(f["x"][lo:hi]); t["dy"].copy_(f["dy"][lo:hi]); t["w"].copy_(f["w"])
    del full
    for k in net.kernels.values():  # one fixed plan per kernel: IG over the shard
        k.plan = [(mu.IMPLICIT_GEMM, hi - lo)]
    net.workspaces = {key: None for key in net.kernels}
    ar = GradAllreduce()
    net.iteration(grad_hook=ar)
    ar.wait()
    torch.cuda.synchronize()
    for i, t in enumerate(net.tensors):
        for k in ("y", "dx", "dw"):
            np.save(os.path.join(out_dir, f"w{world}_{k}{i}_{rank}.npy"), t[k].float().cpu().numpy())
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()


@pytest.mark.skipif(torch.cuda.device_count() < 2, reason="needs 2 GPUs")
def test_i7_sharded_equals_single_gpu():
    import torch.multiprocessing as mp
    with tempfile.TemporaryDirectory() as d:
        mp.spawn(_run, args=(1, _free_port(), d), nprocs=1, join=True)
        mp.spawn(_run, args=(2, _free_port(), d), nprocs=2, join=True)
        for i in range(3):
            for k in ("y", "dx"):
                one = np.load(os.path.join(d, f"w1_{k}{i}_0.npy"))
                two = np.concatenate([np.load(os.path.join(d, f"w2_{k}{i}_{r}.npy")) for r in range(2)])
                assert np.array_equal(one, two), (i, k)
            one = np.load(os.path.join(d, f"w1_dw{i}_0.npy"))
            for r in range(2):
                assert np.array_equal(np.load(os.path.join(d, f"w2_dw{i}_{r}.npy")), one), (i, r)
