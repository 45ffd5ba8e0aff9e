// Measurement probe (not product code): time CUB's onesweep radix sort on the
// entry-sort shape of C4 (20.1 M packed u64 keys, key bits [25, 59)) as a
// target for libdts's own onesweep (build phase "sort").
#include <cub/cub.cuh>
#include <cstdio>
#include <vector>
#include <random>
int main() {
    const size_t n = 20132736;
    std::vector<unsigned long long> h(n);
    std::mt19937_64 r(1);
    for (size_t i = 0; i < n; ++i) h[i] = ((r() & ((1ull << 34) - 1)) << 25) | i;
    unsigned long long *a, *b;
    cudaMalloc(&a, n * 8); cudaMalloc(&b, n * 8);
    cudaMemcpy(a, h.data(), n * 8, cudaMemcpyHostToDevice);
    size_t tb = 0;
    cub::DeviceRadixSort::SortKeys(nullptr, tb, a, b, n, 25, 59);
    void* t; cudaMalloc(&t, tb);
    cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
    for (int bits : {34, 32, 24, 16, 8}) {
        float best = 1e9;
        for (int it = 0; it < 10; ++it) {
            cudaEventRecord(e0);
            cub::DeviceRadixSort::SortKeys(t, tb, a, b, n, 25, 25 + bits);
            cudaEventRecord(e1); cudaEventSynchronize(e1);
            float ms; cudaEventElapsedTime(&ms, e0, e1); if (ms < best) best = ms;
        }
        printf("cub SortKeys u64 n=%zu bits=%d: %.3f ms\n", n, bits, best);
    }
    return 0;
}
