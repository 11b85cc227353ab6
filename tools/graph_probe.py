"""Host-overhead probe: one conv step eager (with / without per-op events) vs
replayed as a CUDA graph.  python tools/graph_probe.py --config resnet50 --math bf16"""
import argparse, os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_cluster_oyamabhm18_b200 as mu
from paper_conf_cluster_oyamabhm18_b200.network import ConvNet
from synthetic import network

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="resnet50")
ap.add_argument("--math", default="bf16")
ap.add_argument("--tables", default="")
a = ap.parse_args()
math = {"f32": 0, "tf32": 1, "bf16": 2}[a.math]
torch.cuda.set_device(0)
h = mu.Handle(0)
net = ConvNet(h, network(a.config), 256, math, device="cuda")
net.allocate()
lim = 64 << 20
if not (a.tables and net.load_tables(a.tables, lim, "pow2")):
    net.benchmark_all(lim)
net.plan_wr(lim)
flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
st = torch.cuda.current_stream()

def timeit(fn, n=10):
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    ts = []
    for _ in range(n):
        flush.zero_()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(st); fn(); e1.record(st); e1.synchronize()
        ts.append(e0.elapsed_time(e1))
    return sum(ts) / len(ts)

evs = []
def with_events():
    def on_op(i, t, w):
        e = torch.cuda.Event(enable_timing=True); e.record(st); evs.append(e)
    net.iteration(on_op=on_op)
print("eager, no events   %.4f ms" % timeit(lambda: net.iteration()))
print("concurrent WGRAD   %.4f ms" % timeit(lambda: net.iteration(concurrent=True)))
print("eager, no events   %.4f ms" % timeit(lambda: net.iteration()))
print("concurrent WGRAD   %.4f ms" % timeit(lambda: net.iteration(concurrent=True)))
print("eager, op events   %.4f ms" % timeit(with_events))
t0 = time.perf_counter(); net.iteration(); torch.cuda.synchronize()
t1 = time.perf_counter(); net.iteration(); t2 = time.perf_counter(); torch.cuda.synchronize()
print("host enqueue time  %.4f ms (wall of one iteration without sync)" % ((t2 - t1) * 1e3))
