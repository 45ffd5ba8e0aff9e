// Random 64-byte record reads (gather) vs random 64-byte record writes
// (scatter) vs a streaming copy, n = 20.1 M records (C4's entry count).
// nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o /tmp/sgp scatter_gather_probe.cu
#include <cstdio>
#include <cstdint>
#include <vector>
#include <random>
#include <algorithm>
#include <cuda_runtime.h>

struct __align__(32) R4 { double a, b, c, d; };
__device__ __forceinline__ R4 ld(const R4* p) { return *p; }

__global__ void k_copy(const R4* __restrict__ D, R4* __restrict__ out, size_t n) {
    size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (i < n) { out[2 * i] = D[2 * i]; out[2 * i + 1] = D[2 * i + 1]; }
}
__global__ void k_gather(const R4* __restrict__ D, const uint32_t* __restrict__ perm, R4* __restrict__ out, size_t n) {
    size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (i < n) { uint32_t r = perm[i]; R4 x = D[2 * (size_t)r], y = D[2 * (size_t)r + 1]; out[2 * i] = x; out[2 * i + 1] = y; }
}
template <int IT>
__global__ void k_gather_it(const R4* __restrict__ D, const uint32_t* __restrict__ perm, R4* __restrict__ out, size_t n) {
    size_t b = (size_t)blockIdx.x * blockDim.x * IT + threadIdx.x;
    uint32_t r[IT]; R4 x[IT], y[IT];
#pragma unroll
    for (int k = 0; k < IT; ++k) { size_t i = b + (size_t)k * blockDim.x; r[k] = i < n ? perm[i] : 0; }
#pragma unroll
    for (int k = 0; k < IT; ++k) { size_t i = b + (size_t)k * blockDim.x; if (i < n) { x[k] = D[2 * (size_t)r[k]]; y[k] = D[2 * (size_t)r[k] + 1]; } }
#pragma unroll
    for (int k = 0; k < IT; ++k) { size_t i = b + (size_t)k * blockDim.x; if (i < n) { out[2 * i] = x[k]; out[2 * i + 1] = y[k]; } }
}
__global__ void k_scatter(const R4* __restrict__ D, const uint32_t* __restrict__ perm, R4* __restrict__ out, size_t n) {
    size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (i < n) { uint32_t r = perm[i]; R4 x = D[2 * i], y = D[2 * i + 1]; out[2 * (size_t)r] = x; out[2 * (size_t)r + 1] = y; }
}
__global__ void k_scatter_u32(const uint32_t* __restrict__ perm, uint32_t* __restrict__ pos, size_t n) {
    size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (i < n) pos[perm[i]] = (uint32_t)i;
}
__global__ void k_flush(uint4* p, size_t n) { size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x; if (i < n) p[i] = make_uint4(i, 0, 0, 0); }

int main() {
    const size_t n = 20132736;
    std::vector<uint32_t> perm(n);
    for (size_t i = 0; i < n; ++i) perm[i] = (uint32_t)i;
    std::mt19937_64 g(1);
    std::shuffle(perm.begin(), perm.end(), g);
    // permutations made of runs of R consecutive targets in random order
    auto runs_perm = [&](size_t R) {
        std::vector<uint32_t> pr(n), runs(n / R);
        for (size_t i = 0; i < runs.size(); ++i) runs[i] = (uint32_t)i;
        std::shuffle(runs.begin(), runs.end(), g);
        for (size_t i = 0; i < n; ++i) pr[i] = i / R < runs.size() ? runs[i / R] * R + (i % R) : (uint32_t)i;
        return pr;
    };
    std::vector<uint32_t> bperm = runs_perm(8), p2 = runs_perm(2), p4 = runs_perm(4);
    R4 *D, *out; uint32_t *dp, *dbp, *pos, *d2, *d4; uint4* fl;
    cudaMalloc(&D, n * 64); cudaMalloc(&out, n * 64); cudaMalloc(&dp, n * 4); cudaMalloc(&dbp, n * 4); cudaMalloc(&pos, n * 4);
    cudaMalloc(&d2, n * 4); cudaMalloc(&d4, n * 4);
    cudaMemcpy(d2, p2.data(), n * 4, cudaMemcpyHostToDevice);
    cudaMemcpy(d4, p4.data(), n * 4, cudaMemcpyHostToDevice);
    const size_t nf = (256u << 20) / 16; cudaMalloc(&fl, nf * 16);
    cudaMemset(D, 1, n * 64);
    cudaMemcpy(dp, perm.data(), n * 4, cudaMemcpyHostToDevice);
    cudaMemcpy(dbp, bperm.data(), n * 4, cudaMemcpyHostToDevice);
    cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
    const int T = 256; const unsigned G = (unsigned)((n + T - 1) / T);
    auto run = [&](const char* name, auto f, double bytes) {
        float best = 1e9, tot = 0; int reps = 10;
        for (int r = 0; r < reps + 2; ++r) {
            k_flush<<<(unsigned)((nf + 255) / 256), 256>>>(fl, nf);
            cudaEventRecord(e0); f(); cudaEventRecord(e1); cudaEventSynchronize(e1);
            float ms; cudaEventElapsedTime(&ms, e0, e1);
            if (r >= 2) { best = std::min(best, ms); tot += ms; }
        }
        printf("%-28s mean %.3f ms  best %.3f ms  %.0f GB/s (mean)\n", name, tot / reps, best, bytes / (tot / reps) / 1e6);
    };
    run("copy 64B", [&] { k_copy<<<G, T>>>(D, out, n); }, n * 128.0);
    run("gather 64B random", [&] { k_gather<<<G, T>>>(D, dp, out, n); }, n * 132.0);
    run("gather 64B random IT=2", [&] { k_gather_it<2><<<(G + 1) / 2, T>>>(D, dp, out, n); }, n * 132.0);
    run("gather 64B random IT=4", [&] { k_gather_it<4><<<(G + 3) / 4, T>>>(D, dp, out, n); }, n * 132.0);
    run("scatter 64B random", [&] { k_scatter<<<G, T>>>(D, dp, out, n); }, n * 132.0);
    run("scatter 64B runs of 8", [&] { k_scatter<<<G, T>>>(D, dbp, out, n); }, n * 132.0);
    run("gather 64B runs of 8", [&] { k_gather<<<G, T>>>(D, dbp, out, n); }, n * 132.0);
    run("gather 64B runs of 4", [&] { k_gather<<<G, T>>>(D, d4, out, n); }, n * 132.0);
    run("gather 64B runs of 2", [&] { k_gather<<<G, T>>>(D, d2, out, n); }, n * 132.0);
    run("scatter u32 random", [&] { k_scatter_u32<<<G, T>>>(dp, pos, n); }, n * 8.0);
    run("scatter u32 runs of 8", [&] { k_scatter_u32<<<G, T>>>(dbp, pos, n); }, n * 8.0);
    cudaError_t e = cudaDeviceSynchronize();
    printf("%s\n", cudaGetErrorString(e));
    return 0;
}
