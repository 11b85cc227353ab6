"""paper_conf_cluster_oyamabhm18_b200 -- B200-native micro-batched convolution
(the hot path of mu-cuDNN, Oyama et al., IEEE CLUSTER 2018).

* ``_lib``: ctypes binding of libmucudnn.so (C ABI in include/mucudnn.h).
* ``torch_api``: tensor-level wrappers (PyTorch supplies memory and streams).
* ``network``: per-network WR / WD planning and the fwd+bwd conv iteration.
* ``distributed``: data-parallel dW allreduce over NCCL.

There is no CPU fallback: importing fails if the native library is missing,
and every convolution runs in the library's sm_100a kernels.
"""
from ._lib import (ALGO_NAMES, BWD_DATA, BWD_FILTER, FFT, FFT_TILING, FWD, IM2COL_GEMM, IMPLICIT_GEMM, MATH_BF16, MATH_F32,  # noqa: F401
                   MATH_NAMES, MATH_TF32, NUM_ALGOS, POLICY_ALL, POLICY_POW2, POLICY_UNDIVIDED, TYPE_NAMES,
                   WINOGRAD, ConvDesc, Handle, MicroConfig, MucuError, Network, benchmark_scratch_size, desc,
                   output_dims, pareto_front, plan_wr, solve_wd, version, workspace_size)
from . import torch_api  # noqa: F401
