"""Executor invariants on a whole network (GPU): the concurrent backward
(each BackwardFilter on a side stream next to its BackwardData,
ConvNet.iteration(concurrent=True), the bench.py step) computes exactly what the
sequential order computes.  Integer-valued inputs make every tensor-core path
exact, so y, dx and dW must match bit for bit (the split-K reduction order of
BackwardFilter is then irrelevant)."""
import numpy as np
import pytest
import torch

import paper_conf_cluster_oyamabhm18_b200 as mu
from paper_conf_cluster_oyamabhm18_b200.network import ConvNet
from synthetic import network

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("config,math,policy", [("alexnet", mu.MATH_TF32, "wr"), ("resnet18", mu.MATH_BF16, "wr"),
                                                ("alexnet", mu.MATH_BF16, "wd")],
                         ids=["alexnet-tf32-wr", "resnet18-bf16-wr", "alexnet-bf16-wd"])
def test_concurrent_backward_matches_sequential(config, math, policy):
    h = mu.Handle(0)
    h.set_policy(mu.POLICY_POW2)
    net = ConvNet(h, network(config), 8, math, device="cuda")
    net.allocate(seed=5, kind="int")
    limit = 8 << 20                       # tight: micro-batched plans
    net.benchmark_all(limit)
    if policy == "wr":
        net.plan_wr(limit)
    else:  # one shared network workspace: concurrent kernels use disjoint segments
        net.plan_wd(len(net.kernels) * limit // 2)

    def outputs():
        torch.cuda.synchronize()
        return [{k: t[k].float().cpu().numpy().copy() for k in ("y", "dx", "dw")} for t in net.tensors]

    def reset():
        for t in net.tensors:
            for k in ("y", "dx", "dw"):
                t[k].fill_(float("nan") if k != "dw" else 0.0)

    reset()
    net.iteration()
    seq = outputs()
    reset()
    net.iteration(concurrent=True)
    con = outputs()
    for i, (a, b) in enumerate(zip(seq, con)):
        for k in ("y", "dx", "dw"):
            assert np.array_equal(a[k], b[k]), (config, i, k)
    if config == "alexnet" and policy == "wr":  # at 8 MiB some AlexNet kernels really are micro-batched
        assert any(len(k.plan) > 1 for k in net.kernels.values())
