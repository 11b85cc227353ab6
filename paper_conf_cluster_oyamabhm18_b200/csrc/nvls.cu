// nvls.cu -- NEXT-3: the cross-rank dW reduction fused
// into the BackwardFilter epilogue.
//
// P:L17 motivates micro-batching with "hiding the communication of parameter
// gradients": in data-parallel training every rank's dW must be summed across the
// ranks.  Instead of a separate NCCL all-reduce after the layer's last micro-batch,
// the kernel that writes a dw element's FINAL value (the last micro-batch's epilogue,
// or its last ordered split group, or the partial-slot reduction) also adds that value
// to the reduction target: with NVLink SHARP (NVLS), one `multimem.red.add` to the
// multicast address of a symmetric fp32 buffer, which NVSwitch adds into every rank's
// copy; without multicast, one `red.global.add` per rank buffer through NVLink P2P
// pointers.  When all ranks have passed the barrier below, every rank's buffer holds
// sum_ranks dw_rank.
//
// This file: the multicast object (driver VMM + multicast API, entry points resolved at
// run time through the runtime -- no -lcuda), the push kernel for dw writers that do
// not fuse (F32 SIMT, Winograd, FFT, atomic split-K), and the barrier kernel.
#include <cuda.h>
#include <cuda_runtime.h>

#include <cstdarg>
#include <cstring>

#include "mucudnn_internal.h"

namespace mucu {
namespace {

// ------------------------------------------------------------ kernels ----
__global__ void reduce_push_kernel(const float* __restrict__ src, const RedTarget t, int64_t n) {
    bool al = ((uintptr_t)src & 15) == 0;
    for (int r = 0; r < (t.mc ? 1 : t.n); ++r) al = al && ((uintptr_t)t.dst[r] & 15) == 0;
    const int64_t nv = al ? n / 4 : 0;
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < nv; i += stride)
        red_add4(t, 4 * i, __ldg(reinterpret_cast<const float4*>(src) + i));
    for (int64_t i = 4 * nv + blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += stride)
        red_add(t, i, __ldg(src + i));
}

// One thread: publish this rank's earlier reductions (the kernels before this one on
// the stream have completed; the system-scope release orders their writes before the
// flag increment), add 1 to every rank's flag (one multicast address or each rank's
// flag word), then wait until this rank's own flag reaches `target`.
__global__ void reduce_barrier_kernel(const RedTarget flags, const unsigned* own, unsigned target) {
    asm volatile("fence.proxy.alias;" ::: "memory");
    asm volatile("fence.acq_rel.sys;" ::: "memory");
    if (flags.mc) {
        asm volatile("multimem.red.release.sys.global.add.u32 [%0], %1;" ::"l"(flags.dst[0]), "r"(1u) : "memory");
    } else {
        for (int r = 0; r < flags.n; ++r)
            asm volatile("red.release.sys.global.add.u32 [%0], %1;" ::"l"(flags.dst[r]), "r"(1u) : "memory");
    }
    const unsigned long long t0 = global_ns();
    for (;;) {
        unsigned v;
        asm volatile("ld.acquire.sys.global.u32 %0, [%1];" : "=r"(v) : "l"(own) : "memory");
        if ((int)(v - target) >= 0) break;
        if (global_ns() - t0 > kWatchdogNs) watchdog_trap("reduce barrier", (unsigned long long)own, target, v);
        __nanosleep(64);
    }
    asm volatile("fence.proxy.alias;" ::: "memory");
}

// ------------------------------------------------------ driver entry ----
template <class F>
F entry(const char* name) {
    void* p = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint(name, &p, cudaEnableDefault, &q) != cudaSuccess || q != cudaDriverEntryPointSuccess)
        return nullptr;
    return (F)p;
}

struct Drv {
    CUresult (*mcCreate)(CUmemGenericAllocationHandle*, const CUmulticastObjectProp*);
    CUresult (*mcAddDevice)(CUmemGenericAllocationHandle, CUdevice);
    CUresult (*mcBindMem)(CUmemGenericAllocationHandle, size_t, CUmemGenericAllocationHandle, size_t, size_t,
                          unsigned long long);
    CUresult (*mcUnbind)(CUmemGenericAllocationHandle, CUdevice, size_t, size_t);
    CUresult (*mcGran)(size_t*, const CUmulticastObjectProp*, CUmulticastGranularity_flags);
    CUresult (*memCreate)(CUmemGenericAllocationHandle*, size_t, const CUmemAllocationProp*, unsigned long long);
    CUresult (*memGran)(size_t*, const CUmemAllocationProp*, CUmemAllocationGranularity_flags);
    CUresult (*memRelease)(CUmemGenericAllocationHandle);
    CUresult (*addrReserve)(CUdeviceptr*, size_t, size_t, CUdeviceptr, unsigned long long);
    CUresult (*addrFree)(CUdeviceptr, size_t);
    CUresult (*memMap)(CUdeviceptr, size_t, size_t, CUmemGenericAllocationHandle, unsigned long long);
    CUresult (*memUnmap)(CUdeviceptr, size_t);
    CUresult (*setAccess)(CUdeviceptr, size_t, const CUmemAccessDesc*, size_t);
    CUresult (*exportH)(void*, CUmemGenericAllocationHandle, CUmemAllocationHandleType, unsigned long long);
    CUresult (*importH)(CUmemGenericAllocationHandle*, void*, CUmemAllocationHandleType);
    CUresult (*devGet)(CUdevice*, int);
    CUresult (*devAttr)(int*, CUdevice_attribute, CUdevice);
    bool ok = false;
};

const Drv& drv() {
    static Drv d = [] {
        Drv x;
        x.mcCreate = entry<decltype(x.mcCreate)>("cuMulticastCreate");
        x.mcAddDevice = entry<decltype(x.mcAddDevice)>("cuMulticastAddDevice");
        x.mcBindMem = entry<decltype(x.mcBindMem)>("cuMulticastBindMem");
        x.mcUnbind = entry<decltype(x.mcUnbind)>("cuMulticastUnbind");
        x.mcGran = entry<decltype(x.mcGran)>("cuMulticastGetGranularity");
        x.memCreate = entry<decltype(x.memCreate)>("cuMemCreate");
        x.memGran = entry<decltype(x.memGran)>("cuMemGetAllocationGranularity");
        x.memRelease = entry<decltype(x.memRelease)>("cuMemRelease");
        x.addrReserve = entry<decltype(x.addrReserve)>("cuMemAddressReserve");
        x.addrFree = entry<decltype(x.addrFree)>("cuMemAddressFree");
        x.memMap = entry<decltype(x.memMap)>("cuMemMap");
        x.memUnmap = entry<decltype(x.memUnmap)>("cuMemUnmap");
        x.setAccess = entry<decltype(x.setAccess)>("cuMemSetAccess");
        x.exportH = entry<decltype(x.exportH)>("cuMemExportToShareableHandle");
        x.importH = entry<decltype(x.importH)>("cuMemImportFromShareableHandle");
        x.devGet = entry<decltype(x.devGet)>("cuDeviceGet");
        x.devAttr = entry<decltype(x.devAttr)>("cuDeviceGetAttribute");
        x.ok = x.mcCreate && x.mcAddDevice && x.mcBindMem && x.mcUnbind && x.mcGran && x.memCreate && x.memGran &&
               x.memRelease && x.addrReserve && x.addrFree && x.memMap && x.memUnmap && x.setAccess && x.exportH &&
               x.importH && x.devGet && x.devAttr;
        return x;
    }();
    return d;
}

}  // namespace

int launch_reduce_push(const float* src, const RedTarget& t, int64_t n, cudaStream_t st) {
    if (n <= 0 || t.n <= 0) return 0;
    const int64_t work = std::max<int64_t>(1, n / 4);
    const int grid = (int)std::min<int64_t>((work + 255) / 256, 148 * 8);
    reduce_push_kernel<<<grid, 256, 0, st>>>(src, t, n);
    count_launch();
    return (int)cudaGetLastError();
}

int launch_reduce_barrier(const RedTarget& flags, const unsigned* own, unsigned target, cudaStream_t st) {
    reduce_barrier_kernel<<<1, 1, 0, st>>>(flags, own, target);
    count_launch();
    return (int)cudaGetLastError();
}

}  // namespace mucu

using namespace mucu;

// The multicast object of one rank: `data` bytes of user data + one 256-B flag block,
// rounded up to the multicast granularity; mapped twice into this device's address
// space (unicast: this rank's physical copy; multicast: every rank's copy).
struct mucu_nvls {
    int device = 0;
    int32_t ranks = 1;
    uint64_t data = 0, total = 0;
    CUmemGenericAllocationHandle mc = 0, mem = 0;
    CUdeviceptr uc_va = 0, mc_va = 0;
    bool have_mc = false, have_mem = false, bound = false;
    unsigned epoch = 0;
};

static mucu_status_t cu_fail(CUresult r, const char* what) {
    return set_error(MUCU_ERR_CUDA, "%s failed (CUresult %d)", what, (int)r);
}

static CUmulticastObjectProp mc_prop(int32_t ranks, uint64_t total) {
    CUmulticastObjectProp p;
    std::memset(&p, 0, sizeof(p));
    p.numDevices = (unsigned)ranks;
    p.size = total;
    p.handleTypes = CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR;
    return p;
}

// Size of the object: user bytes (rounded to 256) + flag block, multiple of both the
// multicast and the physical allocation granularity (identical on every rank).
static mucu_status_t nvls_sizes(int device, int32_t ranks, uint64_t bytes, uint64_t* data, uint64_t* total) {
    const Drv& d = drv();
    if (!d.ok) return set_error(MUCU_ERR_CUDA, "driver multicast / VMM entry points not available");
    CUdevice dev;
    CUresult r = d.devGet(&dev, device);
    if (r) return cu_fail(r, "cuDeviceGet");
    int sup = 0;
    r = d.devAttr(&sup, CU_DEVICE_ATTRIBUTE_MULTICAST_SUPPORTED, dev);
    if (r) return cu_fail(r, "cuDeviceGetAttribute(MULTICAST_SUPPORTED)");
    if (!sup) return set_error(MUCU_ERR_UNSUPPORTED, "device %d does not support NVLink multicast", device);
    *data = (bytes + 255) & ~255ull;
    uint64_t need = *data + 256;
    CUmulticastObjectProp mp = mc_prop(ranks, need);
    size_t g1 = 0, g2 = 0;
    if ((r = d.mcGran(&g1, &mp, CU_MULTICAST_GRANULARITY_MINIMUM))) return cu_fail(r, "cuMulticastGetGranularity");
    CUmemAllocationProp ap;
    std::memset(&ap, 0, sizeof(ap));
    ap.type = CU_MEM_ALLOCATION_TYPE_PINNED;
    ap.location.type = CU_MEM_LOCATION_TYPE_DEVICE;
    ap.location.id = device;
    if ((r = d.memGran(&g2, &ap, CU_MEM_ALLOC_GRANULARITY_MINIMUM))) return cu_fail(r, "cuMemGetAllocationGranularity");
    const uint64_t g = std::max<uint64_t>(g1, g2);
    *total = (need + g - 1) / g * g;
    return MUCU_OK;
}

extern "C" mucu_status_t mucu_nvls_supported(int device, int32_t* supported) {
    if (!supported) return set_error(MUCU_ERR_INVALID_VALUE, "supported is NULL");
    *supported = 0;
    const Drv& d = drv();
    if (!d.ok) return MUCU_OK;
    CUdevice dev;
    int sup = 0;
    if (d.devGet(&dev, device) == CUDA_SUCCESS && d.devAttr(&sup, CU_DEVICE_ATTRIBUTE_MULTICAST_SUPPORTED, dev) ==
                                                       CUDA_SUCCESS)
        *supported = sup ? 1 : 0;
    return MUCU_OK;
}

static mucu_status_t nvls_open(int device, int32_t ranks, uint64_t bytes, int32_t fd, mucu_nvls_t* out) {
    if (!out) return set_error(MUCU_ERR_INVALID_VALUE, "out is NULL");
    *out = nullptr;
    if (ranks < 1 || bytes == 0) return set_error(MUCU_ERR_INVALID_VALUE, "ranks < 1 or bytes == 0");
    if (cudaSetDevice(device) != cudaSuccess) return set_error(MUCU_ERR_CUDA, "cudaSetDevice(%d) failed", device);
    cudaFree(nullptr);  // the primary context exists before any driver call
    uint64_t data, total;
    mucu_status_t s = nvls_sizes(device, ranks, bytes, &data, &total);
    if (s) return s;
    const Drv& d = drv();
    mucu_nvls* nv = new mucu_nvls;
    nv->device = device; nv->ranks = ranks; nv->data = data; nv->total = total;
    CUresult r;
    if (fd < 0) {
        CUmulticastObjectProp mp = mc_prop(ranks, total);
        r = d.mcCreate(&nv->mc, &mp);
        if (r) { delete nv; return cu_fail(r, "cuMulticastCreate"); }
    } else {
        r = d.importH(&nv->mc, (void*)(uintptr_t)fd, CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR);
        if (r) { delete nv; return cu_fail(r, "cuMemImportFromShareableHandle(multicast)"); }
    }
    nv->have_mc = true;
    CUdevice dev;
    d.devGet(&dev, device);
    if ((r = d.mcAddDevice(nv->mc, dev))) { mucu_nvls_destroy(nv); return cu_fail(r, "cuMulticastAddDevice"); }
    *out = nv;
    return MUCU_OK;
}

extern "C" mucu_status_t mucu_nvls_create(int device, int32_t ranks, uint64_t bytes, mucu_nvls_t* out) {
    return nvls_open(device, ranks, bytes, -1, out);
}

extern "C" mucu_status_t mucu_nvls_import(int device, int32_t ranks, uint64_t bytes, int32_t fd, mucu_nvls_t* out) {
    if (fd < 0) return set_error(MUCU_ERR_INVALID_VALUE, "fd < 0");
    return nvls_open(device, ranks, bytes, fd, out);
}

extern "C" mucu_status_t mucu_nvls_export(mucu_nvls_t nv, int32_t* fd) {
    if (!nv || !fd) return set_error(MUCU_ERR_INVALID_VALUE, "nv or fd is NULL");
    int h = -1;
    CUresult r = drv().exportH(&h, nv->mc, CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR, 0);
    if (r) return cu_fail(r, "cuMemExportToShareableHandle(multicast)");
    *fd = h;
    return MUCU_OK;
}

extern "C" mucu_status_t mucu_nvls_bind(mucu_nvls_t nv, void** local, void** multicast) {
    if (!nv) return set_error(MUCU_ERR_INVALID_VALUE, "nv is NULL");
    const Drv& d = drv();
    CUresult r;
    if (!nv->bound) {
        cudaSetDevice(nv->device);
        CUmemAllocationProp ap;
        std::memset(&ap, 0, sizeof(ap));
        ap.type = CU_MEM_ALLOCATION_TYPE_PINNED;
        ap.location.type = CU_MEM_LOCATION_TYPE_DEVICE;
        ap.location.id = nv->device;
        if ((r = d.memCreate(&nv->mem, nv->total, &ap, 0))) return cu_fail(r, "cuMemCreate");
        nv->have_mem = true;
        // blocks until every rank has added its device
        if ((r = d.mcBindMem(nv->mc, 0, nv->mem, 0, nv->total, 0))) return cu_fail(r, "cuMulticastBindMem");
        CUmemAccessDesc acc;
        std::memset(&acc, 0, sizeof(acc));
        acc.location.type = CU_MEM_LOCATION_TYPE_DEVICE;
        acc.location.id = nv->device;
        acc.flags = CU_MEM_ACCESS_FLAGS_PROT_READWRITE;
        if ((r = d.addrReserve(&nv->uc_va, nv->total, 0, 0, 0))) return cu_fail(r, "cuMemAddressReserve");
        if ((r = d.memMap(nv->uc_va, nv->total, 0, nv->mem, 0))) return cu_fail(r, "cuMemMap(unicast)");
        if ((r = d.setAccess(nv->uc_va, nv->total, &acc, 1))) return cu_fail(r, "cuMemSetAccess(unicast)");
        if ((r = d.addrReserve(&nv->mc_va, nv->total, 0, 0, 0))) return cu_fail(r, "cuMemAddressReserve");
        if ((r = d.memMap(nv->mc_va, nv->total, 0, nv->mc, 0))) return cu_fail(r, "cuMemMap(multicast)");
        if ((r = d.setAccess(nv->mc_va, nv->total, &acc, 1))) return cu_fail(r, "cuMemSetAccess(multicast)");
        if (cudaMemset((void*)nv->uc_va, 0, nv->total) != cudaSuccess || cudaDeviceSynchronize() != cudaSuccess)
            return set_error(MUCU_ERR_CUDA, "zeroing the NVLS buffer failed");
        nv->bound = true;
    }
    if (local) *local = (void*)nv->uc_va;
    if (multicast) *multicast = (void*)nv->mc_va;
    return MUCU_OK;
}

extern "C" mucu_status_t mucu_nvls_barrier(mucu_nvls_t nv, void* stream) {
    if (!nv || !nv->bound) return set_error(MUCU_ERR_INVALID_VALUE, "NVLS object not bound");
    ++nv->epoch;
    RedTarget f = {};
    f.dst[0] = (float*)(nv->mc_va + nv->data);
    f.n = 1;
    f.mc = 1;
    const int e = launch_reduce_barrier(f, (const unsigned*)(nv->uc_va + nv->data), nv->epoch * (unsigned)nv->ranks,
                                        (cudaStream_t)stream);
    return e ? set_error(MUCU_ERR_CUDA, "nvls barrier launch: %s", cudaGetErrorString((cudaError_t)e)) : MUCU_OK;
}

extern "C" mucu_status_t mucu_peer_barrier(const mucu_reduce_target_t* flags, const uint32_t* own, uint32_t target,
                                           void* stream) {
    if (!flags || !own || flags->count < 1 || flags->count > MUCU_MAX_REDUCE_RANKS || (flags->multicast && flags->count != 1))
        return set_error(MUCU_ERR_INVALID_VALUE, "peer_barrier: bad flag target");
    RedTarget f = {};
    for (int r = 0; r < flags->count; ++r) {
        if (!flags->dst[r] || ((uintptr_t)flags->dst[r] & 3)) return set_error(MUCU_ERR_MISALIGNED, "flag %d", r);
        f.dst[r] = flags->dst[r];
    }
    f.n = flags->count;
    f.mc = flags->multicast ? 1 : 0;
    const int e = launch_reduce_barrier(f, (const unsigned*)own, target, (cudaStream_t)stream);
    return e ? set_error(MUCU_ERR_CUDA, "peer barrier launch: %s", cudaGetErrorString((cudaError_t)e)) : MUCU_OK;
}

extern "C" mucu_status_t mucu_nvls_destroy(mucu_nvls_t nv) {
    if (!nv) return MUCU_OK;
    const Drv& d = drv();
    cudaSetDevice(nv->device);
    cudaDeviceSynchronize();
    if (nv->mc_va) { d.memUnmap(nv->mc_va, nv->total); d.addrFree(nv->mc_va, nv->total); }
    if (nv->uc_va) { d.memUnmap(nv->uc_va, nv->total); d.addrFree(nv->uc_va, nv->total); }
    CUdevice dev;
    d.devGet(&dev, nv->device);
    if (nv->bound) d.mcUnbind(nv->mc, dev, 0, nv->total);
    if (nv->have_mem) d.memRelease(nv->mem);
    if (nv->have_mc) d.memRelease(nv->mc);
    delete nv;
    return MUCU_OK;
}
