// Dependent-round-trip latency under the per-insertion kernel's launch shape
// (diagnostic microbenchmark): G CTAs x 512 threads, 2 per SM; every CTA runs
// "levels" in which its first A threads each do R dependent ld.cg of random
// words of its own region of a large array, then a CTA barrier.  Prints SM
// cycles per round trip for several footprints and access patterns.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 rt_load.cu -o rt_load
#include <cstdio>
#include <cstdint>
#include <vector>
#include <cuda_runtime.h>

__global__ void __launch_bounds__(512, 2) levels(const int *__restrict__ p, size_t region, int nlev, int active,
                                                 int rts, int stride_regions, long long *cyc, int *sink) {
    const size_t base = (size_t)blockIdx.x * region * stride_regions;
    unsigned x = blockIdx.x * 2654435761u + threadIdx.x * 40503u;
    int acc = 0;
    __syncthreads();
    long long t0 = clock64();
    for (int l = 0; l < nlev; ++l) {
        if (threadIdx.x < active) {
            int i = (int)(x % region);
            for (int r = 0; r < rts; ++r) {
                const int v = __ldcg(p + base + i);
                acc += v;
                i = (int)((unsigned)(v + i * 2654435761u + r) % region);
            }
            x = x * 1664525u + 1013904223u;
        }
        __syncthreads();
    }
    long long t1 = clock64();
    if (threadIdx.x == 0) cyc[blockIdx.x] = (t1 - t0);
    if (acc == 0x7fffffff) sink[0] = acc;
}

int main() {
    int nsm = 0;
    cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0);
    const size_t total = (size_t)1 << 29;  // 2 GB of ints
    int *p;
    cudaMalloc(&p, total * 4);
    std::vector<int> h((size_t)1 << 24);
    uint64_t s = 88172645463325252ull;
    for (auto &v : h) { s ^= s << 13; s ^= s >> 7; s ^= s << 17; v = (int)(s & 0x7fffffff); }
    for (size_t o = 0; o < total; o += h.size()) cudaMemcpy(p + o, h.data(), h.size() * 4, cudaMemcpyHostToDevice);
    long long *cyc;
    int *sink;
    cudaMalloc(&cyc, 4096 * 8);
    cudaMalloc(&sink, 4);
    struct Case { const char *name; int grid; size_t region; int stride; int active; int rts; };
    const Case cases[] = {
        {"256 CTAs, 64 KB region each (16 MB, L2)", 256, 1 << 14, 1, 32, 4},
        {"256 CTAs, 1 MB region each (256 MB)", 256, 1 << 18, 1, 32, 4},
        {"256 CTAs, 1 MB regions 8 MB apart (2 GB)", 256, 1 << 18, 8, 32, 4},
        {"256 CTAs, 1 MB region, 1 thread", 256, 1 << 18, 1, 1, 4},
        {"256 CTAs, 1 MB region, 256 threads", 256, 1 << 18, 1, 256, 4},
        {"1 CTA, 1 MB region", 1, 1 << 18, 1, 32, 4},
        {"1 CTA, 64 KB region", 1, 1 << 14, 1, 32, 4},
    };
    for (const Case &c : cases) {
        const int nlev = 200;
        levels<<<c.grid, 512>>>(p, c.region, 20, c.active, c.rts, c.stride, cyc, sink);
        levels<<<c.grid, 512>>>(p, c.region, nlev, c.active, c.rts, c.stride, cyc, sink);
        cudaDeviceSynchronize();
        std::vector<long long> hc(c.grid);
        cudaMemcpy(hc.data(), cyc, c.grid * 8, cudaMemcpyDeviceToHost);
        double m = 0;
        for (auto v : hc) m += (double)v;
        m /= c.grid;
        printf("%-48s %7.0f cycles per level, %6.0f per round trip (+barrier share)\n", c.name, m / nlev,
               m / nlev / c.rts);
    }
    printf("err: %s\n", cudaGetErrorString(cudaGetLastError()));
    return 0;
}
