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


def _bench_worker(rank, world, port, out_dir):
    """Sharded benchmark pass with a stand-in benchmark:
    host logic only (sharding, all-gather, fan-out to identical kernels)."""
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port), RANK=str(rank), WORLD_SIZE=str(world),
                      LOCAL_RANK=str(rank))
    import sys
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    import json
    import paper_conf_cluster_oyamabhm18_b200 as mu
    from paper_conf_cluster_oyamabhm18_b200 import network as N
    from paper_conf_cluster_oyamabhm18_b200 import torch_api as T
    from paper_conf_cluster_oyamabhm18_b200.distributed import init_from_env
    from synthetic.networks import resnet18
    assert init_from_env("gloo")
    calls = []

    class FakeHandle:
        def benchmark(self, d, conv_type, ws_limit, scratch, nbytes, stream):
            calls.append(f"{d.c},{d.h},{d.k},{d.r},{d.stride}|{conv_type}")
            t = np.full((mu.NUM_ALGOS, d.n + 1), -1, dtype=np.int64)
            t[:, 1:] = (d.c * 7 + d.k * 3 + d.h + conv_type) * np.arange(1, d.n + 1)
            return t, np.zeros((mu.NUM_ALGOS, d.n + 1), dtype=np.uint64)

    N.L.benchmark_scratch_size = lambda *a: 0
    T.make_scratch = lambda *a: torch.empty(1, dtype=torch.uint8)
    T._stream = lambda: 0
    net = N.ConvNet(FakeHandle(), resnet18(), 8, mu.MATH_BF16, device="cpu")
    net.benchmark_all(1 << 20)
    tables = {f"{k[0]}/{k[1]}": v.table[0][0].tolist() for k, v in net.kernels.items()}
    json.dump({"calls": calls, "tables": tables}, open(os.path.join(out_dir, f"b{rank}.json"), "w"))
    dist.barrier()
    dist.destroy_process_group()


def test_sharded_benchmark_pass_gloo():
    import json
    from synthetic.networks import resnet18
    with tempfile.TemporaryDirectory() as d:
        mp.spawn(_bench_worker, args=(2, _free_port(), d), nprocs=2, join=True)
        r = [json.load(open(os.path.join(d, f"b{i}.json"))) for i in range(2)]
    layers = resnet18()
    uniq = {(l.c, l.h, l.k, l.r, l.stride, t) for l in layers for t in range(3)}
    c0, c1 = set(r[0]["calls"]), set(r[1]["calls"])
    assert not (c0 & c1)                                    # each unique kernel benchmarked on one rank
    assert len(r[0]["calls"]) + len(r[1]["calls"]) == len(uniq)
    assert abs(len(c0) - len(c1)) <= len(uniq) // 2         # both ranks work
    assert r[0]["tables"] == r[1]["tables"]                 # identical tables everywhere after the gather
    for i, l in enumerate(layers):                          # fan-out to identical kernels is the right table
        for t in range(3):
            v = r[0]["tables"][f"{i}/{t}"]
            assert v[1] == l.c * 7 + l.k * 3 + l.h + t


def test_shard_benchmark_lpt():
    from paper_conf_cluster_oyamabhm18_b200.network import shard_benchmark
    costs = {"a": 10, "b": 9, "c": 5, "d": 4, "e": 1}
    s = shard_benchmark(costs, 2)
    assert sorted(sum(s, [])) == sorted(costs)
    assert s == [["a", "d", "e"], ["b", "c"]]
    assert shard_benchmark(costs, 1) == [["a", "b", "c", "d", "e"]]


def _iteration_worker(rank, world, port, out_dir):
    """ConvNet.iteration + GradAllreduce over gloo: each rank runs
    its shard of a global batch through the network executor; the conv calls are
    routed to the fp64 oracle on CPU (test stand-in for the GPU kernels) so the
    executor order, zero_grad, the grad hook and the allreduce are exercised."""
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port), RANK=str(rank), WORLD_SIZE=str(world),
                      LOCAL_RANK=str(rank))
    import sys
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    import oracle
    import paper_conf_cluster_oyamabhm18_b200 as mu
    from paper_conf_cluster_oyamabhm18_b200 import network as N
    from paper_conf_cluster_oyamabhm18_b200.distributed import GradAllreduce, init_from_env, shard_range
    from synthetic import conv_inputs
    from synthetic.networks import ConvLayer
    assert init_from_env("gloo")
    layers = [ConvLayer("a", 3, 11, 11, 8, 3, 3, 1, 2), ConvLayer("b", 8, 6, 6, 6, 3, 3, 1, 1)]
    n_global = 6
    lo, hi = shard_range(n_global, rank, world)

    def fwd(h, d, plan, x, w, y, workspace=None):
        y.copy_(torch.from_numpy(oracle.conv_forward(x.numpy(), w.numpy(), d.pad, d.stride)).float())

    def dgrad(h, d, plan, dy, w, dx, workspace=None):
        dx.copy_(torch.from_numpy(oracle.conv_backward_data(dy.numpy(), w.numpy(), d.h, d.w, d.pad, d.stride)).float())

    def wgrad(h, d, plan, x, dy, dw, beta=0.0, workspace=None):
        dw.copy_(torch.from_numpy(oracle.conv_backward_filter(x.numpy(), dy.numpy(), d.r, d.s, d.pad, d.stride, 1.0,
                                                              beta, dw.numpy().astype(np.float64))).float())

    N.T.conv_forward, N.T.conv_backward_data, N.T.conv_backward_filter = fwd, dgrad, wgrad
    net = N.ConvNet(None, layers, hi - lo, mu.MATH_F32, device="cpu")
    net.tensors = []
    sizes = [l.k * l.r * l.s * l.c for l in layers]
    net.dw_flat = torch.zeros(sum(sizes))
    off = 0
    for i, l in enumerate(layers):
        x, w, dy = conv_inputs(n_global, l.c, l.h, l.w, l.k, l.r, l.s, l.pad, l.stride, seed=40 + i, kind="int")
        p_, q_ = (l.h + 2 * l.pad - l.r) // l.stride + 1, (l.w + 2 * l.pad - l.s) // l.stride + 1
        net.tensors.append(dict(x=torch.from_numpy(x[lo:hi].copy()), w=torch.from_numpy(w),
                                dy=torch.from_numpy(dy[lo:hi].copy()), y=torch.empty(hi - lo, p_, q_, l.k),
                                dx=torch.empty(hi - lo, l.h, l.w, l.c),
                                dw=net.dw_flat[off:off + sizes[i]].view(l.k, l.r, l.s, l.c)))
        off += sizes[i]
    for k in net.kernels.values():
        k.plan = [(mu.IMPLICIT_GEMM, hi - lo)]
    seen = []
    ar = GradAllreduce()

    def hook(i, dw):
        seen.append(i)
        ar(i, dw)
    net.iteration(grad_hook=hook)
    ar.wait()
    assert seen == [1, 0]  # dW handed over as soon as each layer's BackwardFilter is done
    for i in range(len(layers)):
        t = net.tensors[i]
        np.save(os.path.join(out_dir, f"y{i}_{rank}.npy"), t["y"].numpy())
        np.save(os.path.join(out_dir, f"dw{i}_{rank}.npy"), t["dw"].numpy())
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.timeout(240)
def test_gloo_convnet_iteration_allreduce():
    import oracle
    from synthetic import conv_inputs
    from synthetic.networks import ConvLayer
    from paper_conf_cluster_oyamabhm18_b200.distributed import shard_range
    layers = [ConvLayer("a", 3, 11, 11, 8, 3, 3, 1, 2), ConvLayer("b", 8, 6, 6, 6, 3, 3, 1, 1)]
    world = 2
    with tempfile.TemporaryDirectory() as d:
        mp.spawn(_iteration_worker, args=(world, _free_port(), d), nprocs=world, join=True)
        for i, l in enumerate(layers):
            x, w, dy = conv_inputs(6, l.c, l.h, l.w, l.k, l.r, l.s, l.pad, l.stride, seed=40 + i, kind="int")
            full_dw = oracle.conv_backward_filter(x, dy, l.r, l.s, l.pad, l.stride)
            full_y = oracle.conv_forward(x, w, l.pad, l.stride)
            for rank in range(world):
                lo, hi = shard_range(6, rank, world)
                # dW summed over ranks == full-batch dW (exact on integer data)
                assert np.array_equal(np.load(os.path.join(d, f"dw{i}_{rank}.npy")), full_dw.astype(np.float32))
                # I7: per-sample forward identical to the single-device full batch
                assert np.array_equal(np.load(os.path.join(d, f"y{i}_{rank}.npy")), full_y[lo:hi].astype(np.float32))


def _fd_worker(rank, world, port, out_dir):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port), RANK=str(rank), WORLD_SIZE=str(world),
                      LOCAL_RANK=str(rank))
    import sys
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    from paper_conf_cluster_oyamabhm18_b200.distributed import init_from_env, share_fd
    assert init_from_env("gloo")
    fd = None
    if rank == 0:
        # an anonymous object only rank 0 holds (like the exported multicast handle)
        fd = os.memfd_create("nvls-probe")
        os.write(fd, b"multicast handle of rank 0")
    got = share_fd(fd)
    if rank == 0:
        assert got == fd
    os.lseek(got, 0, os.SEEK_SET)
    data = os.read(got, 64)
    with open(os.path.join(out_dir, f"fd{rank}.txt"), "wb") as f:
        f.write(data)
    dist.barrier()
    os.close(got)
    dist.destroy_process_group()


def test_share_fd_gloo():
    """NEXT-3 setup: rank 0's exported handle (a POSIX fd) reaches every rank
    through pidfd_getfd over the process group (world size 2)."""
    if not hasattr(os, "pidfd_open") or not hasattr(os, "memfd_create"):
        pytest.skip("pidfd_open / memfd_create unavailable")
    world = 2
    with tempfile.TemporaryDirectory() as d:
        mp.spawn(_fd_worker, args=(world, _free_port(), d), nprocs=world, join=True)
        for r in range(world):
            with open(os.path.join(d, f"fd{r}.txt"), "rb") as f:
                assert f.read() == b"multicast handle of rank 0"
