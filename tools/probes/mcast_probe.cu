// NVLS multicast probe: does this box expose switch multicast to one process?
// Checks CU_DEVICE_ATTRIBUTE_MULTICAST_SUPPORTED, builds a 1-device multicast object, binds
// memory, maps the multicast address and stores through it with multimem.st; verifies the
// unicast view.  nvcc -gencode arch=compute_100a,code=sm_100a -o mcast_probe mcast_probe.cu -lcuda
#include <cuda.h>
#include <cuda_runtime.h>
#include <cstdio>

#define CU(x) do { CUresult r_ = (x); if (r_ != CUDA_SUCCESS) { const char *s; cuGetErrorString(r_, &s); \
    printf("FAIL %s: %s\n", #x, s); return 1; } } while (0)

__global__ void mc_store(float *mc, int n)
{
    int i = (blockIdx.x * blockDim.x + threadIdx.x) * 4;
    if (i < n) {
        float a = i, b = i + 1, c = i + 2, d = i + 3;
        asm volatile("multimem.st.global.v4.f32 [%0], {%1, %2, %3, %4};" ::"l"(mc + i), "f"(a), "f"(b), "f"(c), "f"(d)
                     : "memory");
    }
}

int main()
{
    CU(cuInit(0));
    CUdevice dev;
    CU(cuDeviceGet(&dev, 0));
    int mc = 0, ndev = 0;
    CU(cuDeviceGetAttribute(&mc, CU_DEVICE_ATTRIBUTE_MULTICAST_SUPPORTED, dev));
    cudaGetDeviceCount(&ndev);
    printf("devices %d multicast_supported %d\n", ndev, mc);
    if (!mc) return 0;
    cudaSetDevice(0);
    CUmulticastObjectProp p = {};
    p.numDevices = 1;
    p.handleTypes = CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR;
    size_t gran = 0;
    CU(cuMulticastGetGranularity(&gran, &p, CU_MULTICAST_GRANULARITY_RECOMMENDED));
    const size_t bytes = gran > (4u << 20) ? gran : (4u << 20);
    p.size = bytes;
    CUmemGenericAllocationHandle mh, uh;
    CU(cuMulticastCreate(&mh, &p));
    CU(cuMulticastAddDevice(mh, dev));
    CUmemAllocationProp ap = {};
    ap.type = CU_MEM_ALLOCATION_TYPE_PINNED;
    ap.location.type = CU_MEM_LOCATION_TYPE_DEVICE;
    ap.location.id = 0;
    ap.requestedHandleTypes = CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR;
    CU(cuMemCreate(&uh, bytes, &ap, 0));
    CU(cuMulticastBindMem(mh, 0, uh, 0, bytes, 0));
    CUdeviceptr ua, ma;
    CUmemAccessDesc ad = {};
    ad.location = ap.location;
    ad.flags = CU_MEM_ACCESS_FLAGS_PROT_READWRITE;
    CU(cuMemAddressReserve(&ua, bytes, gran, 0, 0));
    CU(cuMemMap(ua, bytes, 0, uh, 0));
    CU(cuMemSetAccess(ua, bytes, &ad, 1));
    CU(cuMemAddressReserve(&ma, bytes, gran, 0, 0));
    CU(cuMemMap(ma, bytes, 0, mh, 0));
    CU(cuMemSetAccess(ma, bytes, &ad, 1));
    const int n = (int)(bytes / 4);
    cudaMemset((void *)ua, 0, bytes);
    mc_store<<<(n / 4 + 255) / 256, 256>>>((float *)ma, n);
    cudaError_t e = cudaDeviceSynchronize();
    printf("kernel: %s\n", cudaGetErrorString(e));
    float h[8];
    cudaMemcpy(h, (void *)(ua + 4096), sizeof(h), cudaMemcpyDeviceToHost);
    int ok = 1;
    for (int k = 0; k < 8; ++k) ok &= h[k] == (float)(1024 + k);
    printf("unicast view after multimem.st: %s (gran %zu)\n", ok ? "OK" : "MISMATCH", gran);
    return 0;
}
