// Microbenchmark: cost breakdown of the grid insert (1M objects, one step).
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -I paper_conf_ipps_hellwigcmbw23_b200/csrc -o /tmp/ib tools/micro/insert_bench.cu
#include <cstdio>
#include <cstdlib>
#include <vector>
#include <cuda_runtime.h>
#include "cd_device.cuh"
using namespace cdk;

__global__ void k_init(Entry* E, int n, unsigned long long seed)
{
    int i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= n) return;
    unsigned long long x = seed ^ (i * 0x9E3779B97F4A7C15ull);
    auto rnd = [&]() { x ^= x >> 12; x ^= x << 25; x ^= x >> 27; return (double)((x * 2685821657736338717ull) >> 11) * (1.0 / 9007199254740992.0); };
    double r = 6900 + 600 * rnd(), u = 2 * rnd() - 1, ph = 6.283185307 * rnd();
    double s = sqrt(1 - u * u);
    E[i].x = r * s * cos(ph); E[i].y = r * s * sin(ph); E[i].z = r * u; E[i].next = kNil;
}

template <int V>
__global__ void __launch_bounds__(256) k_ins(GridGeom g, GridTab tab, Entry* ents, int n, uint64_t mask, uint32_t epoch, uint32_t tag)
{
    const int r = blockIdx.x * blockDim.x + threadIdx.x;
    if (r >= n) return;
    Entry* en = ents + r;
    const double p[3] = {en->x, en->y, en->z};
    int64_t c[3];
    cell_of(g, p, c);
    const unsigned long long key = pack_key(c[0], c[1], c[2]);
    if (V == 0) { en->pad = (uint32_t)key; return; }                 // no atomics
    if (V == 1 || V == 4) { const uint32_t hb = bit_of(key) & tab.bmask; atomicOr(tab.bits + (hb >> 5), 1u << (hb & 31)); }
    if (V == 1) { en->pad = (uint32_t)key; return; }                  // bitmap RED only
    uint64_t slot;
    if (V == 5) {   // plain CAS on the hashed slot, no probing loop (upper bound of a perfect table)
        slot = fmix64(key) & mask;
        atomicCAS(tab.keys + slot, 0ull, key | (1ull << 57));
    } else {
        slot = insert_key(tab.keys, mask, key, tag);
    }
    if (V == 2) { en->next = (uint32_t)slot; return; }                // CAS only
    const unsigned long long old = atomicExch(tab.heads + slot, ((unsigned long long)epoch << 32) | (unsigned long long)r);
    en->next = (old >> 32) == epoch ? (uint32_t)old : kNil;          // V3: CAS+EXCH, V4: +RED
}

int main()
{
    const int n = 1 << 20;
    const uint64_t M = 2ull * n;
    Entry* E; unsigned long long *keys, *heads; uint32_t* bits;
    cudaMalloc(&E, sizeof(Entry) * n); cudaMalloc(&keys, 8 * M); cudaMalloc(&heads, 8 * M); cudaMalloc(&bits, 4 * (32ull * n / 32));
    cudaMemset(keys, 0, 8 * M); cudaMemset(heads, 0, 8 * M);
    k_init<<<n / 256, 256>>>(E, n, 12345);
    GridGeom g{0, 0, 0, 1.0 / (3 * 9.8), 9.8 * 9.8, 9.8, 0};
    GridTab tab{keys, heads, bits, (uint32_t)(32ull * n - 1), (uint32_t)n};
    cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
    const char* names[] = {"no atomics", "bitmap RED", "key CAS (probe loop)", "CAS + head EXCH", "CAS + EXCH + RED", "single CAS (no loop)"};
    for (int V = 0; V < 6; ++V) {
        float best = 1e9;
        for (int it = 0; it < 20; ++it) {
            cudaMemsetAsync(bits, 0, 4ull * n);
            uint32_t tag = 1 + (it % 120);
            cudaEventRecord(a);
            switch (V) {
            case 0: k_ins<0><<<n / 256, 256>>>(g, tab, E, n, M - 1, it + 1, tag); break;
            case 1: k_ins<1><<<n / 256, 256>>>(g, tab, E, n, M - 1, it + 1, tag); break;
            case 2: k_ins<2><<<n / 256, 256>>>(g, tab, E, n, M - 1, it + 1, tag); break;
            case 3: k_ins<3><<<n / 256, 256>>>(g, tab, E, n, M - 1, it + 1, tag); break;
            case 4: k_ins<4><<<n / 256, 256>>>(g, tab, E, n, M - 1, it + 1, tag); break;
            case 5: k_ins<5><<<n / 256, 256>>>(g, tab, E, n, M - 1, it + 1, tag); break;
            }
            cudaEventRecord(b); cudaEventSynchronize(b);
            float ms; cudaEventElapsedTime(&ms, a, b); if (ms < best) best = ms;
        }
        printf("%-28s %8.2f us\n", names[V], best * 1e3);
    }
    printf("err: %s\n", cudaGetErrorString(cudaGetLastError()));
    return 0;
}
