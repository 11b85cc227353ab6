"""Probe cuMulticastCreate parameter combinations on this box (NEXT-3 setup)."""
from cuda.bindings import driver as cu

cu.cuInit(0)
err, dev = cu.cuDeviceGet(0)
err, ctx = cu.cuDevicePrimaryCtxRetain(dev)
cu.cuCtxSetCurrent(ctx)
H = cu.CUmemAllocationHandleType
for nd in (1, 2):
    for ht_name in ("CU_MEM_HANDLE_TYPE_NONE", "CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR", "CU_MEM_HANDLE_TYPE_FABRIC"):
        ht = getattr(H, ht_name)
        p = cu.CUmulticastObjectProp()
        p.numDevices = nd
        p.handleTypes = ht
        p.size = 2 << 20
        e1, g = cu.cuMulticastGetGranularity(p, cu.CUmulticastGranularity_flags.CU_MULTICAST_GRANULARITY_MINIMUM)
        e1r, gr = cu.cuMulticastGetGranularity(p, cu.CUmulticastGranularity_flags.CU_MULTICAST_GRANULARITY_RECOMMENDED)
        for size in (g if g else 2 << 20, 32 << 20, gr if gr else 512 << 20):
            p.size = size
            e, h = cu.cuMulticastCreate(p)
            msg = ""
            if e == 0:
                e2 = cu.cuMulticastAddDevice(h, dev)[0]
                msg = f" add={e2}"
                if ht_name.endswith("FILE_DESCRIPTOR"):
                    ee, fd = cu.cuMemExportToShareableHandle(h, ht, 0)
                    msg += f" export={ee} fd={fd}"
                cu.cuMemRelease(h)
            print(f"nd={nd} {ht_name} gran={e1}:{g} rec={e1r}:{gr} size={size} -> {e}{msg}", flush=True)
