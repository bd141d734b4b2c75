// sort_bench.cu - standalone timing + check of the radix sorts in radix_sort.cuh
// (tools only; not part of the product).  nvcc -gencode arch=compute_100a,code=sm_100a -O3
//   -std=c++17 -o tools/sort_bench tools/sort_bench.cu;  ./tools/sort_bench
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdio>
#include <cstdlib>
#include <vector>

#include "../paper_conf_edbt_jibrilabs23_b200/csrc/radix_sort.cuh"
#ifndef SB_ITEMS
#define SB_ITEMS 12
#endif

using namespace h2tap;

#define CK(x)                                                                          \
    do {                                                                               \
        cudaError_t e = (x);                                                           \
        if (e != cudaSuccess) { printf("%s:%d %s\n", __FILE__, __LINE__, cudaGetErrorString(e)); exit(1); } \
    } while (0)

__global__ void k_empty(unsigned int* bar, int reps) {
    unsigned int target = 0;
    for (int i = 0; i < reps; ++i) rs_grid_sync(bar, target);
}

template <int ITEMS>
float run_coop(uint64_t* k0, uint32_t* v0, uint64_t* k1, uint32_t* v1, uint64_t n, int passes, uint32_t* scratch) {
    constexpr int tile = kRsThreads * ITEMS, smem = tile * 12;
    const uint64_t T = (n + tile - 1) / tile;
    uint32_t* cnt = scratch;
    uint32_t* tot = cnt + T * 256;
    unsigned int* bar = tot + 256;
    const unsigned long long* nd = nullptr;
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    CK(cudaMemset(bar, 0, 4));
    void* args[] = {&k0, &v0, &k1, &v1, &n, &nd, &passes, &cnt, &tot, &bar};
    cudaEventRecord(a);
    CK(cudaLaunchCooperativeKernel((void*)rs_coop<ITEMS>, dim3((unsigned)T), dim3(kRsThreads), args, smem, 0));
    cudaEventRecord(b);
    CK(cudaEventSynchronize(b));
    float ms;
    cudaEventElapsedTime(&ms, a, b);
    return ms;
}

int main() {
    const uint64_t maxn = 1 << 21;
    uint64_t *k0, *k1;
    uint32_t *v0, *v1, *scratch;
    CK(cudaMalloc(&k0, maxn * 8));
    CK(cudaMalloc(&k1, maxn * 8));
    CK(cudaMalloc(&v0, maxn * 4));
    CK(cudaMalloc(&v1, maxn * 4));
    CK(cudaMalloc(&scratch, (maxn / 1024 + 2) * 256 * 4 + 4096));
    int occ4 = 0, occ12 = 0, sms = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ4, rs_coop<4>, kRsThreads, 1024 * 12);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ12, rs_coop<SB_ITEMS>, kRsThreads, 256 * SB_ITEMS * 12);
    printf("SMs %d occ<4> %d occ<12> %d\n", sms, occ4, occ12);
    // barrier cost
    for (int g : {10, 100, 296, 444}) {
        unsigned int* bar = scratch;
        CK(cudaMemset(bar, 0, 4));
        int reps = 100;
        void* args[] = {&bar, &reps};
        cudaEvent_t a, b;
        cudaEventCreate(&a);
        cudaEventCreate(&b);
        cudaEventRecord(a);
        CK(cudaLaunchCooperativeKernel((void*)k_empty, dim3(g), dim3(256), args, 0, 0));
        cudaEventRecord(b);
        CK(cudaEventSynchronize(b));
        float ms;
        cudaEventElapsedTime(&ms, a, b);
        printf("grid barrier, %d CTAs: %.2f us each\n", g, ms * 1e3 / reps);
    }
    for (uint64_t n : {10000ull, 25000ull, 100000ull, 262144ull, 1000000ull, 1300000ull}) {
        for (int bits : {32, 40, 50}) {
            const int passes = (bits + 7) / 8;
            std::vector<uint64_t> hk(n);
            std::vector<uint32_t> hv(n);
            uint64_t x = 88172645463325252ull;
            for (uint64_t i = 0; i < n; ++i) {
                x ^= x << 13; x ^= x >> 7; x ^= x << 17;
                hk[i] = x & ((1ull << bits) - 1);
                hv[i] = (uint32_t)i;
            }
            float best = 1e9;
            for (int rep = 0; rep < 5; ++rep) {
                CK(cudaMemcpy(k0, hk.data(), n * 8, cudaMemcpyHostToDevice));
                CK(cudaMemcpy(v0, hv.data(), n * 4, cudaMemcpyHostToDevice));
#ifndef SB_ITEMS
#define SB_ITEMS 12
#endif
                float ms = n <= (1u << 18) ? run_coop<4>(k0, v0, k1, v1, n, passes, scratch)
                                           : run_coop<SB_ITEMS>(k0, v0, k1, v1, n, passes, scratch);
                best = std::min(best, ms);
            }
            std::vector<uint64_t> ok(n);
            std::vector<uint32_t> ov(n);
            CK(cudaMemcpy(ok.data(), (passes & 1) ? k1 : k0, n * 8, cudaMemcpyDeviceToHost));
            CK(cudaMemcpy(ov.data(), (passes & 1) ? v1 : v0, n * 4, cudaMemcpyDeviceToHost));
            std::vector<uint32_t> idx(n);
            for (uint64_t i = 0; i < n; ++i) idx[i] = (uint32_t)i;
            std::stable_sort(idx.begin(), idx.end(), [&](uint32_t a, uint32_t b) { return hk[a] < hk[b]; });
            bool good = true;
            for (uint64_t i = 0; i < n && good; ++i) good = ok[i] == hk[idx[i]] && ov[i] == idx[i];
            printf("n=%8llu bits=%d passes=%d: %.1f us (%.1f us/pass) %s\n", (unsigned long long)n, bits, passes,
                   best * 1e3, best * 1e3 / passes, good ? "OK" : "WRONG");
        }
    }
    return 0;
}
