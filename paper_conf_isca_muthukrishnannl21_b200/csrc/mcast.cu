// mcast.cu -- NVLS multicast replicas: one agent store reaches every
// peer's replica through the NVSwitch (multimem.st), instead of one store per destination.
//
// the transfer threads "perform remote writes to the target GPU(s)"; L82: NVLink
// efficiency needs >= 128-byte writes.  With full replication every chunk goes to all G-1 peers,
// so a unicast agent issues (G-1) stores per byte; a multicast object binds the replica of every
// rank to one multicast address, and a multimem.st.global.v4 to it is delivered by the switch to
// all bound replicas (the writer's own included, which already holds the same bytes).  Ingress per
// GPU is unchanged; the agent's egress instructions and SM time drop by (G-1)x.
//
// Scope: ranks that are threads of ONE process on distinct devices of an NVSwitch system whose
// devices report CU_DEVICE_ATTRIBUTE_MULTICAST_SUPPORTED (the multicast handle is then a process
// handle every rank can use).  Elsewhere proact_alloc_replica still returns a usable replica
// (cudaMalloc) and the multicast push falls back to 16-byte unicast stores.  Driver entry points
// are resolved through the runtime (no link dependency on libcuda).
#include <cuda.h>
#include <cuda_runtime.h>
#include <unistd.h>

#include <cstdio>
#include <cstring>
#include <mutex>
#include <vector>

#include "proact.h"

namespace {

struct Drv {
    CUresult (*MulticastCreate)(CUmemGenericAllocationHandle *, const CUmulticastObjectProp *);
    CUresult (*MulticastAddDevice)(CUmemGenericAllocationHandle, CUdevice);
    CUresult (*MulticastBindMem)(CUmemGenericAllocationHandle, size_t, CUmemGenericAllocationHandle, size_t, size_t,
                                 unsigned long long);
    CUresult (*MulticastUnbind)(CUmemGenericAllocationHandle, CUdevice, size_t, size_t);
    CUresult (*MulticastGetGranularity)(size_t *, const CUmulticastObjectProp *, CUmulticastGranularity_flags);
    CUresult (*MemCreate)(CUmemGenericAllocationHandle *, size_t, const CUmemAllocationProp *, unsigned long long);
    CUresult (*MemRelease)(CUmemGenericAllocationHandle);
    CUresult (*MemAddressReserve)(CUdeviceptr *, size_t, size_t, CUdeviceptr, unsigned long long);
    CUresult (*MemAddressFree)(CUdeviceptr, size_t);
    CUresult (*MemMap)(CUdeviceptr, size_t, size_t, CUmemGenericAllocationHandle, unsigned long long);
    CUresult (*MemUnmap)(CUdeviceptr, size_t);
    CUresult (*MemSetAccess)(CUdeviceptr, size_t, const CUmemAccessDesc *, size_t);
    CUresult (*MemGetAllocationGranularity)(size_t *, const CUmemAllocationProp *, CUmemAllocationGranularity_flags);
    CUresult (*DeviceGetAttribute)(int *, CUdevice_attribute, CUdevice);
    bool ok = false;
};

Drv g_drv;
std::once_flag g_drv_once;

template <class F>
bool sym(const char *name, F &f)
{
    void *p = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint(name, &p, cudaEnableDefault, &q) != cudaSuccess || !p) return false;
    f = reinterpret_cast<F>(p);
    return true;
}

Drv &drv()
{
    std::call_once(g_drv_once, [] {
        Drv &d = g_drv;
        d.ok = sym("cuMulticastCreate", d.MulticastCreate) && sym("cuMulticastAddDevice", d.MulticastAddDevice) &&
               sym("cuMulticastBindMem", d.MulticastBindMem) && sym("cuMulticastUnbind", d.MulticastUnbind) &&
               sym("cuMulticastGetGranularity", d.MulticastGetGranularity) && sym("cuMemCreate", d.MemCreate) &&
               sym("cuMemRelease", d.MemRelease) && sym("cuMemAddressReserve", d.MemAddressReserve) &&
               sym("cuMemAddressFree", d.MemAddressFree) && sym("cuMemMap", d.MemMap) &&
               sym("cuMemUnmap", d.MemUnmap) && sym("cuMemSetAccess", d.MemSetAccess) &&
               sym("cuMemGetAllocationGranularity", d.MemGetAllocationGranularity) &&
               sym("cuDeviceGetAttribute", d.DeviceGetAttribute);
    });
    return g_drv;
}

struct McAlloc {
    char *ptr = nullptr;          // unicast replica (what the caller gets)
    size_t bytes = 0, size = 0;   // requested / mapped
    int device = -1, world = 0;
    bool vmm = false;             // ptr is a VMM mapping of `mem` (else cudaMalloc)
    CUmemGenericAllocationHandle mem = 0, mc = 0;
    CUdeviceptr mc_va = 0;        // this rank's mapping of the multicast object (0: none)
};
std::mutex g_mu;
std::vector<McAlloc> g_allocs;

}  // namespace

// runtime.cu: job rendezvous of the calling rank (all-gather of n <= 4096 bytes), rank, world
extern "C" __attribute__((visibility("hidden"))) int proact_internal_allgather(const void *mine, size_t n, void *all);
extern "C" __attribute__((visibility("hidden"))) int proact_internal_same_process_devices(int *devices);

extern "C" {

int proact_mcast_supported(void)
{
    const int world = proact_world();
    if (world < 2) return 0;
    int devs[PROACT_MAX_RANKS];
    if (!proact_internal_same_process_devices(devs)) return 0;   // ranks in several processes
    for (int a = 0; a < world; ++a)
        for (int b = a + 1; b < world; ++b)
            if (devs[a] == devs[b]) return 0;                       // loopback: no switch involved
    Drv &d = drv();
    if (!d.ok) return 0;
    for (int r = 0; r < world; ++r) {
        int v = 0;
        if (d.DeviceGetAttribute(&v, CU_DEVICE_ATTRIBUTE_MULTICAST_SUPPORTED, (CUdevice)devs[r]) != CUDA_SUCCESS || !v)
            return 0;
    }
    return 1;
}

int proact_alloc_replica(size_t bytes, void **out)
{
    const int world = proact_world(), rank = proact_rank();
    if (world <= 0) return PROACT_ERR_STATE;
    if (!out || bytes == 0) return PROACT_ERR_INVALID;
    int dev = 0;
    cudaGetDevice(&dev);
    // every rank decides the same way (a collective)
    int32_t can = proact_mcast_supported();
    std::vector<int32_t> cans(world);
    int rc = proact_internal_allgather(&can, sizeof(can), cans.data());
    if (rc) return rc;
    for (int32_t x : cans) can = can && x;
    McAlloc A;
    A.bytes = bytes;
    A.device = dev;
    A.world = world;
    if (!can) {   // a plain replica (IPC-able); pushes fall back to unicast
        if (cudaMalloc((void **)&A.ptr, bytes) != cudaSuccess) return PROACT_ERR_NOMEM;
        A.size = bytes;
        std::lock_guard<std::mutex> g(g_mu);
        g_allocs.push_back(A);
        *out = A.ptr;
        return PROACT_OK;
    }
    Drv &d = drv();
    CUmulticastObjectProp mp = {};
    mp.numDevices = (unsigned)world;
    mp.handleTypes = CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR;
    size_t mg = 0, ag = 0;
    CUmemAllocationProp ap = {};
    ap.type = CU_MEM_ALLOCATION_TYPE_PINNED;
    ap.location.type = CU_MEM_LOCATION_TYPE_DEVICE;
    ap.location.id = dev;
    ap.requestedHandleTypes = CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR;
    if (d.MulticastGetGranularity(&mg, &mp, CU_MULTICAST_GRANULARITY_RECOMMENDED) != CUDA_SUCCESS ||
        d.MemGetAllocationGranularity(&ag, &ap, CU_MEM_ALLOC_GRANULARITY_RECOMMENDED) != CUDA_SUCCESS)
        return PROACT_ERR_CUDA;
    const size_t gran = mg > ag ? mg : ag;
    A.size = (bytes + gran - 1) / gran * gran;
    mp.size = A.size;
    // rank 0 creates the multicast object; the handle is a process handle (all ranks are threads
    // of this process, proact_mcast_supported)
    uint64_t h = 0;
    if (rank == 0 && d.MulticastCreate(&A.mc, &mp) != CUDA_SUCCESS) A.mc = 0;
    h = (uint64_t)A.mc;
    std::vector<uint64_t> hs(world);
    if ((rc = proact_internal_allgather(&h, sizeof(h), hs.data()))) return rc;
    A.mc = (CUmemGenericAllocationHandle)hs[0];
    if (!A.mc) return PROACT_ERR_CUDA;
    int32_t bad = d.MulticastAddDevice(A.mc, (CUdevice)dev) != CUDA_SUCCESS;
    std::vector<int32_t> bads(world);
    if ((rc = proact_internal_allgather(&bad, sizeof(bad), bads.data()))) return rc;   // all added
    for (int32_t x : bads) bad |= x;
    if (bad) return PROACT_ERR_CUDA;
    // my physical replica, bound to the multicast object and mapped for unicast access by every
    // device of the job (peers push into it with plain stores too)
    CUmemAccessDesc ad[PROACT_MAX_RANKS];
    int devs[PROACT_MAX_RANKS];
    proact_internal_same_process_devices(devs);
    for (int r = 0; r < world; ++r) {
        ad[r] = {};
        ad[r].location.type = CU_MEM_LOCATION_TYPE_DEVICE;
        ad[r].location.id = devs[r];
        ad[r].flags = CU_MEM_ACCESS_FLAGS_PROT_READWRITE;
    }
    CUdeviceptr va = 0;
    bad = d.MemCreate(&A.mem, A.size, &ap, 0) != CUDA_SUCCESS ||
          d.MulticastBindMem(A.mc, 0, A.mem, 0, A.size, 0) != CUDA_SUCCESS ||
          d.MemAddressReserve(&va, A.size, gran, 0, 0) != CUDA_SUCCESS || d.MemMap(va, A.size, 0, A.mem, 0) != CUDA_SUCCESS ||
          d.MemSetAccess(va, A.size, ad, (size_t)world) != CUDA_SUCCESS ||
          d.MemAddressReserve(&A.mc_va, A.size, gran, 0, 0) != CUDA_SUCCESS ||
          d.MemMap(A.mc_va, A.size, 0, A.mc, 0) != CUDA_SUCCESS || d.MemSetAccess(A.mc_va, A.size, &ad[rank], 1) != CUDA_SUCCESS;
    if ((rc = proact_internal_allgather(&bad, sizeof(bad), bads.data()))) return rc;
    for (int32_t x : bads) bad |= x;
    if (bad) return PROACT_ERR_CUDA;
    A.ptr = (char *)va;
    A.vmm = true;
    std::lock_guard<std::mutex> g(g_mu);
    g_allocs.push_back(A);
    *out = A.ptr;
    return PROACT_OK;
}

int proact_free_replica(void *ptr)
{
    McAlloc A;
    {
        std::lock_guard<std::mutex> g(g_mu);
        size_t k = 0;
        for (; k < g_allocs.size() && g_allocs[k].ptr != ptr; ++k) {}
        if (k == g_allocs.size()) return PROACT_ERR_INVALID;
        A = g_allocs[k];
        g_allocs.erase(g_allocs.begin() + (long)k);
    }
    cudaDeviceSynchronize();
    if (!A.vmm) return cudaFree(A.ptr) == cudaSuccess ? PROACT_OK : PROACT_ERR_CUDA;
    Drv &d = drv();
    int32_t x = 0;
    std::vector<int32_t> xs(A.world);
    proact_internal_allgather(&x, sizeof(x), xs.data());   // nobody stores through the object
    d.MemUnmap(A.mc_va, A.size);
    d.MemAddressFree(A.mc_va, A.size);
    d.MulticastUnbind(A.mc, (CUdevice)A.device, 0, A.size);
    d.MemUnmap((CUdeviceptr)A.ptr, A.size);
    d.MemAddressFree((CUdeviceptr)A.ptr, A.size);
    d.MemRelease(A.mem);
    proact_internal_allgather(&x, sizeof(x), xs.data());
    if (proact_rank() == 0) d.MemRelease(A.mc);
    return PROACT_OK;
}

}  // extern "C"

// runtime.cu: the multicast address of [ptr, ptr + bytes) of a replica from proact_alloc_replica,
// or 0 if that replica has no multicast binding
extern "C" __attribute__((visibility("hidden"))) void *proact_internal_mcast_lookup(const void *ptr, size_t bytes)
{
    std::lock_guard<std::mutex> g(g_mu);
    for (const McAlloc &A : g_allocs) {
        const char *p = (const char *)ptr;
        if (A.mc_va && p >= A.ptr && p + bytes <= A.ptr + A.bytes) return (char *)A.mc_va + (p - A.ptr);
    }
    return nullptr;
}
