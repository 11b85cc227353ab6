"""Probe: NVLink multicast (NVLS) availability on this box at world size 1.

Prints the driver's multicast attribute, whether torch symmetric memory
rendezvous gives a multicast address, and whether a multimem all-reduce of a
1-rank group runs.  Run via gpurun (MASTER_ADDR=127.0.0.1).
"""
import os

import torch
import torch.distributed as dist

os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
os.environ.setdefault("MASTER_PORT", "29533")
os.environ.setdefault("RANK", "0")
os.environ.setdefault("WORLD_SIZE", "1")

try:
    from cuda.bindings import driver as cu
    cu.cuInit(0)
    err, dev = cu.cuDeviceGet(0)
    err, v = cu.cuDeviceGetAttribute(cu.CUdevice_attribute.CU_DEVICE_ATTRIBUTE_MULTICAST_SUPPORTED, dev)
    print("CU_DEVICE_ATTRIBUTE_MULTICAST_SUPPORTED", err, v)
    err, v = cu.cuDeviceGetAttribute(
        cu.CUdevice_attribute.CU_DEVICE_ATTRIBUTE_HANDLE_TYPE_FABRIC_SUPPORTED, dev)
    print("HANDLE_TYPE_FABRIC_SUPPORTED", err, v)
except Exception as e:  # noqa: BLE001
    print("driver probe failed:", repr(e))

torch.cuda.set_device(0)
dist.init_process_group("nccl", device_id=torch.device("cuda:0"))
import torch.distributed._symmetric_memory as symm_mem  # noqa: E402

try:
    t = symm_mem.empty(1 << 20, dtype=torch.float32, device="cuda:0")
    h = symm_mem.rendezvous(t, dist.group.WORLD.group_name)
    print("rendezvous ok; multicast_ptr", hex(h.multicast_ptr), "buffer_ptrs", [hex(x) for x in h.buffer_ptrs])
    print("signal_pad_ptrs", [hex(x) for x in h.signal_pad_ptrs])
    t.fill_(1.5)
    torch.ops.symm_mem.multimem_all_reduce_(t, "sum", dist.group.WORLD.group_name)
    torch.cuda.synchronize()
    print("multimem_all_reduce_ ok, t[0] =", t[0].item())
except Exception as e:  # noqa: BLE001
    print("symm mem failed:", repr(e))
dist.destroy_process_group()
