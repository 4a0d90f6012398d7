// gather_peak.cu -- measured ceiling of the graph kernels' bound: random 4-byte gathers from an
// L2-resident vector, driven by a streamed index array (the PageRank / SSSP pull inner loop with
// nothing else).  Prints one JSON line per configuration: gathers/s.
//
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o gather_peak gather_peak.cu && ./gather_peak
//
// V = 2^24 floats (64 MiB, the RMAT-24 contribution vector), E = 2^28 - 2^26 random indices
// (the cold in-edges of PageRank at RMAT-24: 209.6 M), index loads 16 bytes per thread (4 edges
// per run, as pagerank_hot_kernel), gathers with the same cache policy (.nc, L1::no_allocate,
// L2 evict_last).  Sweeps CTA size x CTAs per SM x runs per thread in flight.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t mix(uint32_t x)
{
    x ^= x >> 16; x *= 0x85EBCA6Bu; x ^= x >> 13; x *= 0xC2B2AE35u; x ^= x >> 16;
    return x;
}
__global__ void fill_idx(uint32_t *idx, uint64_t E, uint32_t V)
{
    for (uint64_t e = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; e < E; e += (uint64_t)gridDim.x * blockDim.x)
        idx[e] = mix((uint32_t)e * 2654435761u + 12345u) & (V - 1);
}
__global__ void fill_val(float *v, uint32_t V)
{
    for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < V; i += gridDim.x * blockDim.x) v[i] = 1e-7f * (i & 1023);
}

template <int R>   // runs of 4 edges per thread in flight
__global__ void gather(const uint32_t *__restrict__ idx, uint64_t E, const float *__restrict__ val, float *out)
{
    uint64_t pl, pf;
    asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(pl));
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pf));
    float acc = 0.f;
    const uint64_t nrun = E / 4, T = (uint64_t)gridDim.x * blockDim.x;
    for (uint64_t r0 = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; r0 < nrun; r0 += T * R) {
        uint32_t x[R][4];
#pragma unroll
        for (int k = 0; k < R; ++k) {
            const uint64_t r = r0 + k * T;
            if (r < nrun)
                asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.v4.u32 {%0,%1,%2,%3}, [%4], %5;"
                             : "=r"(x[k][0]), "=r"(x[k][1]), "=r"(x[k][2]), "=r"(x[k][3]) : "l"(idx + 4 * r), "l"(pf));
            else
                x[k][0] = x[k][1] = x[k][2] = x[k][3] = 0u;
        }
#pragma unroll
        for (int k = 0; k < R; ++k)
#pragma unroll
            for (int q = 0; q < 4; ++q) {
                float g;
                asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.f32 %0, [%1], %2;" : "=f"(g) : "l"(val + x[k][q]), "l"(pl));
                acc += g;
            }
    }
    if (acc == 12345.f) out[0] = acc;   // keep the loads
}

template <int R>
float run(const uint32_t *idx, uint64_t E, const float *val, float *out, int block, int ctas)
{
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    gather<R><<<ctas, block>>>(idx, E, val, out);
    cudaEventRecord(a);
    const int reps = 5;
    for (int k = 0; k < reps; ++k) gather<R><<<ctas, block>>>(idx, E, val, out);
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms = 0;
    cudaEventElapsedTime(&ms, a, b);
    return ms / reps;
}

int main()
{
    const uint32_t V = 1u << 24;
    const uint64_t E = 209626978ull & ~3ull;   // PageRank RMAT-24's cold in-edges
    int nsm = 0, clk = 0;
    cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0);
    cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
    uint32_t *idx;
    float *val, *out;
    cudaMalloc(&idx, 4 * E);
    cudaMalloc(&val, 4ull * V);
    cudaMalloc(&out, 4);
    fill_idx<<<4096, 256>>>(idx, E, V);
    fill_val<<<1024, 256>>>(val, V);
    cudaDeviceSynchronize();
    const int blocks[] = {256, 512, 1024};
    for (int bi = 0; bi < 3; ++bi) {
        const int block = blocks[bi];
        for (int per = 512; per <= 2048; per *= 2) {   // threads per SM
            const int ctas = nsm * per / block;
            for (int R = 1; R <= 4; R *= 2) {
                float ms = R == 1 ? run<1>(idx, E, val, out, block, ctas)
                         : R == 2 ? run<2>(idx, E, val, out, block, ctas) : run<4>(idx, E, val, out, block, ctas);
                const cudaError_t e = cudaGetLastError();
                if (e != cudaSuccess) { printf("{\"error\": \"%s\"}\n", cudaGetErrorString(e)); return 1; }
                printf("{\"block\": %d, \"ctas\": %d, \"runs_in_flight\": %d, \"ms\": %.4f, \"gathers_per_s\": %.4e, "
                       "\"gathers_per_clk_per_sm_at_max_clock\": %.3f}\n",
                       block, ctas, R, ms, E / (ms * 1e-3), E / (ms * 1e-3) / (nsm * (double)clk * 1e3));
            }
        }
    }
    return 0;
}
