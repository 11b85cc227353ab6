"""Small parity shapes through every (algorithm x conv type x math) of the C ABI,
for compute-sanitizer (memcheck / racecheck / initcheck):

    compute-sanitizer --tool memcheck python tools/sanitize_probe.py
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tests"))

import numpy as np  # noqa: E402

import paper_conf_cluster_oyamabhm18_b200 as mu  # noqa: E402
from gpu_util import oracle_ref, run_gpu  # noqa: E402
from synthetic import conv_inputs  # noqa: E402

SHAPES = [(2, 32, 9, 9, 48, 3, 3, 1, 1), (2, 3, 35, 35, 64, 11, 11, 2, 4), (2, 64, 14, 14, 128, 3, 3, 1, 2),
          (3, 64, 10, 10, 96, 1, 1, 0, 1)]
bad = 0
for shape in SHAPES:
    x, w, dy = conv_inputs(*shape, seed=1, kind="int")
    for math in (mu.MATH_F32, mu.MATH_TF32, mu.MATH_BF16):
        d = mu.desc(*shape, math)
        for t in (mu.FWD, mu.BWD_DATA, mu.BWD_FILTER):
            for a in (mu.IMPLICIT_GEMM, mu.IM2COL_GEMM, mu.WINOGRAD):
                if a == mu.WINOGRAD and not (shape[5] == 3 and shape[8] == 1):
                    continue
                got, intact = run_gpu(d, t, [(a, 1), (a, shape[0] - 1)], x, w, dy, canary=True)
                ref = oracle_ref(shape, t, x, w, dy)
                ok = intact and np.max(np.abs(got - ref)) <= 1e-2 * max(1.0, np.max(np.abs(ref)))
                bad += not ok
                print(shape, math, mu.TYPE_NAMES[t], mu.ALGO_NAMES[a], "ok" if ok else "MISMATCH", flush=True)
print("probe done, mismatches:", bad)
