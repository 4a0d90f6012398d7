// TMA bulk-copy throughput probe: global -> smem -> global with NCTA CTAs, each with W issuing
// warps (lane 0), each warp a ring of NS stages of SB bytes.  Copies `bytes` per CTA.
// Also a SIMT 16-B vector copy for comparison.  Prints GB/s (read+write counted once: copy rate).
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t su(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

__global__ void tma_copy(const char* src, char* dst, size_t per_cta, int W, int NS, int SB, int wait_read_n)
{
    extern __shared__ __align__(128) unsigned char sm[];
    int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    if (warp >= W || lane) return;
    unsigned char* ring = sm + (size_t)warp * NS * SB;
    uint64_t* bars = (uint64_t*)(sm + (size_t)W * NS * SB) + warp * 16;
    for (int s = 0; s < NS; ++s) asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" :: "r"(su(&bars[s])));
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    size_t base = (size_t)blockIdx.x * per_cta;
    size_t per_w = per_cta / W;
    const char* s0 = src + base + warp * per_w;
    char* d0 = dst + base + warp * per_w;
    int nst = (int)(per_w / SB);
    uint32_t parity = 0;
    int issued = 0;
    auto load = [&](int k) {
        int b = k % NS;
        asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" :: "r"(su(&bars[b])), "r"(SB) : "memory");
        asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                     :: "r"(su(ring + (size_t)b * SB)), "l"(s0 + (size_t)k * SB), "r"(SB), "r"(su(&bars[b])) : "memory");
    };
    while (issued < NS - 1 && issued < nst) load(issued++);
    for (int k = 0; k < nst; ++k) {
        int b = k % NS;
        uint32_t done = 0;
        do {
            asm volatile("{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\tselp.u32 %0,1,0,p;\n\t}"
                         : "=r"(done) : "r"(su(&bars[b])), "r"((parity >> b) & 1u) : "memory");
        } while (!done);
        parity ^= 1u << b;
        asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" :: "l"(d0 + (size_t)k * SB), "r"(su(ring + (size_t)b * SB)), "r"(SB) : "memory");
        asm volatile("cp.async.bulk.commit_group;" ::: "memory");
        if (issued < nst) {
            if (wait_read_n == 0) asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");
            else if (wait_read_n == 1) asm volatile("cp.async.bulk.wait_group.read 1;" ::: "memory");
            else asm volatile("cp.async.bulk.wait_group.read 2;" ::: "memory");
            load(issued++);
        }
    }
    asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
}

__global__ void simt_copy(const uint4* src, uint4* dst, size_t per_cta_vec, int U)
{
    size_t base = (size_t)blockIdx.x * per_cta_vec;
    for (size_t i = threadIdx.x; i < per_cta_vec; i += (size_t)blockDim.x * 8) {
        uint4 v[8];
#pragma unroll
        for (int k = 0; k < 8; ++k) if (i + k * blockDim.x < per_cta_vec) v[k] = src[base + i + k * blockDim.x];
#pragma unroll
        for (int k = 0; k < 8; ++k) if (i + k * blockDim.x < per_cta_vec) dst[base + i + k * blockDim.x] = v[k];
    }
}

int main()
{
    size_t total = 1ull << 30;
    char *a, *b;
    cudaMalloc(&a, total); cudaMalloc(&b, total);
    cudaMemset(a, 1, total);
    cudaFuncSetAttribute(tma_copy, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
    cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
    int ncta_list[] = {1, 8, 16, 32, 148};
    struct Cfg { int W, NS, SB, wr; } cfgs[] = {{1,4,16384,0},{1,8,16384,1},{1,8,16384,0},{1,4,32768,1},{2,4,16384,1},{4,4,16384,1},{4,2,16384,0},{1,12,16384,2},{8,2,8192,0}};
    for (int nc : ncta_list) {
        for (auto c : cfgs) {
            size_t smem = (size_t)c.W * c.NS * c.SB + c.W * 128;
            if (smem > 200 * 1024) continue;
            size_t per_cta = (256ull << 20) / nc;   // 256 MiB total per test
            per_cta = per_cta / ((size_t)c.W * c.SB) * ((size_t)c.W * c.SB);
            tma_copy<<<nc, 32 * c.W, smem>>>(a, b, per_cta, c.W, c.NS, c.SB, c.wr);
            cudaEventRecord(e0);
            tma_copy<<<nc, 32 * c.W, smem>>>(a, b, per_cta, c.W, c.NS, c.SB, c.wr);
            cudaEventRecord(e1);
            cudaEventSynchronize(e1);
            float ms; cudaEventElapsedTime(&ms, e0, e1);
            printf("TMA ncta=%d W=%d NS=%d SB=%d waitread=%d : %.1f GB/s copy (%.2f per CTA)\n", nc, c.W, c.NS, c.SB, c.wr,
                   per_cta * nc / ms / 1e6, per_cta / ms / 1e6);
        }
        size_t per_cta = (256ull << 20) / nc / 16;
        simt_copy<<<nc, 256>>>((uint4*)a, (uint4*)b, per_cta, 8);
        cudaEventRecord(e0);
        simt_copy<<<nc, 256>>>((uint4*)a, (uint4*)b, per_cta, 8);
        cudaEventRecord(e1);
        cudaEventSynchronize(e1);
        float ms; cudaEventElapsedTime(&ms, e0, e1);
        printf("SIMT ncta=%d 256thr U=8 : %.1f GB/s copy (%.2f per CTA)\n", nc, per_cta * 16 * nc / ms / 1e6, per_cta * 16 / ms / 1e6);
    }
    printf("err=%s\n", cudaGetErrorString(cudaGetLastError()));
    return 0;
}
