// Memory-op latency on B200 (diagnostic microbenchmark): one thread, dependent
// chains; cycles per step.  nvcc -gencode arch=compute_100a,code=sm_100a -O3
#include <cstdio>
#include <cstdint>
#include <vector>
#include <cuda_runtime.h>

__global__ void chase(const int *__restrict__ p, int steps, int mode, int *out, long long *cyc,
                      unsigned *mk, double *acc) {
    int i = 0;
    long long t0 = clock64();
    for (int s = 0; s < steps; ++s) {
        if (mode == 0) i = __ldcg(p + i);                          // L2-only load chain
        else if (mode == 1) i = p[i];                              // default load chain
        else if (mode == 2) i = (int)(atomicMax(mk + i, 1u) & 0) + __ldcg(p + i);  // atomic then load
        else if (mode == 3) { atomicAdd(acc + i, 1.0); i = __ldcg(p + i); }       // RED then load
        else if (mode == 4) i = (int)atomicAdd((unsigned *)mk + (i & 1023), 0u) * 0 + __ldcg(p + i);
    }
    long long t1 = clock64();
    out[0] = i;
    cyc[0] = (t1 - t0) / steps;
}

int main() {
    for (size_t n : {size_t(1) << 16, size_t(1) << 26}) {  // 256 KB (L2), 256 MB (DRAM)
        std::vector<int> h(n);
        uint64_t x = 88172645463325252ull;
        // random cyclic permutation (Sattolo)
        for (size_t i = 0; i < n; ++i) h[i] = (int)i;
        for (size_t i = n - 1; i > 0; --i) {
            x ^= x << 13; x ^= x >> 7; x ^= x << 17;
            size_t j = x % i;
            std::swap(h[i], h[j]);
        }
        int *d; unsigned *mk; double *acc; int *out; long long *cyc;
        cudaMalloc(&d, n * 4); cudaMalloc(&mk, n * 4); cudaMalloc(&acc, n * 8);
        cudaMalloc(&out, 4); cudaMalloc(&cyc, 8);
        cudaMemcpy(d, h.data(), n * 4, cudaMemcpyHostToDevice);
        cudaMemset(mk, 0, n * 4); cudaMemset(acc, 0, n * 8);
        const char *names[] = {"ld.cg chain", "ld chain", "atomicMax+ld.cg", "RED f64+ld.cg", "atomicAdd(hot)+ld.cg"};
        for (int mode = 0; mode < 5; ++mode) {
            chase<<<1, 1>>>(d, 1000, mode, out, cyc, mk, acc);  // warm
            chase<<<1, 1>>>(d, 20000, mode, out, cyc, mk, acc);
            long long c; cudaMemcpy(&c, cyc, 8, cudaMemcpyDeviceToHost);
            printf("%10zu ints  %-24s %lld cycles/step\n", n, names[mode], c);
        }
        cudaFree(d); cudaFree(mk); cudaFree(acc); cudaFree(out); cudaFree(cyc);
    }
    return 0;
}
