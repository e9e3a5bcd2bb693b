// probe_bench.cu -- per-thread vs warp-cooperative probing of the open-addressing cell map
// (Eq. 2: MurmurHash3 slot, linear probing, CAS insert), on real positions.
//
// The north star names "a lock-free open-addressing map in HBM built on atomicCAS, with a
// warp-cooperative probe".  This measures both probe schemes on the same table and queries:
//   A  one thread per object, its lookups resolved one after another by that thread
//      (s, s+1, ... until the key or an empty slot: the library's grid_find);
//   B  warp-cooperative: for each lookup of any lane, the whole warp reads 32 consecutive slots
//      s..s+31 (one coalesced 512-byte load) and a ballot finds the key or the first empty slot.
// Queries: each object's own cell and its 13 half-shell neighbours (the paper's 27-cell scan,
// each cell pair once).  Table: M = next_pow2(2n) 16-byte slots {key, count}.
//
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o probe_bench tools/micro/probe_bench.cu
//   ./probe_bench positions.f64 n cell_km [reps]       (positions: n x 3 float64, km)
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <vector>

#include <cuda_runtime.h>

#define CK(x)                                                                                  \
    do {                                                                                       \
        cudaError_t e_ = (x);                                                                  \
        if (e_ != cudaSuccess) {                                                               \
            fprintf(stderr, "%s: %s\n", #x, cudaGetErrorString(e_));                           \
            exit(1);                                                                           \
        }                                                                                      \
    } while (0)

struct __align__(16) Slot {
    unsigned long long key;
    unsigned long long cnt;
};
constexpr unsigned long long kEmpty = ~0ull;

__device__ __forceinline__ uint64_t fmix64(uint64_t k)
{
    k ^= k >> 33;
    k *= 0xff51afd7ed558ccdull;
    k ^= k >> 33;
    k *= 0xc4ceb9fe1a85ec53ull;
    k ^= k >> 33;
    return k;
}

__device__ __forceinline__ unsigned long long pack(int x, int y, int z)
{
    const int b = 1 << 20;
    return (unsigned long long)(x + b) | ((unsigned long long)(y + b) << 21) | ((unsigned long long)(z + b) << 42);
}

__constant__ int8_t kOff[14][3] = {{0, 0, 0},  {1, -1, -1}, {1, -1, 0}, {1, -1, 1}, {1, 0, -1},
                                   {1, 0, 0},  {1, 0, 1},   {1, 1, -1}, {1, 1, 0},  {1, 1, 1},
                                   {0, 1, -1}, {0, 1, 0},   {0, 1, 1},  {0, 0, 1}};

__global__ void k_cells(const double* p, int n, double inv, int* c)
{
    const int i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= n) return;
    for (int a = 0; a < 3; ++a) c[3 * i + a] = (int)floor(p[3 * i + a] * inv);
}

__global__ void k_insert(const int* c, int n, Slot* s, uint64_t mask)
{
    const int i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= n) return;
    const unsigned long long key = pack(c[3 * i], c[3 * i + 1], c[3 * i + 2]);
    uint64_t h = fmix64(key) & mask;
    while (true) {
        const unsigned long long prev = atomicCAS(&s[h].key, kEmpty, key);
        if (prev == kEmpty || prev == key) {
            atomicAdd(&s[h].cnt, 1ull);
            return;
        }
        h = (h + 1) & mask;
    }
}

// A: per-thread probing
__global__ void k_probe_thread(const int* c, int n, const Slot* __restrict__ s, uint64_t mask,
                               unsigned long long* found, unsigned long long* probes)
{
    const int i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= n) return;
    unsigned f = 0, pr = 0;
    for (int o = 0; o < 14; ++o) {
        const unsigned long long key = pack(c[3 * i] + kOff[o][0], c[3 * i + 1] + kOff[o][1], c[3 * i + 2] + kOff[o][2]);
        uint64_t h = fmix64(key) & mask;
        while (true) {
            ++pr;
            const unsigned long long k = __ldg(&s[h].key);
            if (k == key) { f += (unsigned)__ldg(&s[h].cnt) > 0; break; }
            if (k == kEmpty) break;
            h = (h + 1) & mask;
        }
    }
    for (int o = 16; o; o >>= 1) {
        f += __shfl_down_sync(__activemask(), f, o);
        pr += __shfl_down_sync(__activemask(), pr, o);
    }
    if ((threadIdx.x & 31) == 0) {
        atomicAdd(found, (unsigned long long)f);
        atomicAdd(probes, (unsigned long long)pr);
    }
}

// B: warp-cooperative probing (every lane of the warp executes the loops; n padded to 32)
__global__ void k_probe_warp(const int* c, int n, const Slot* __restrict__ s, uint64_t mask,
                             unsigned long long* found)
{
    const int i = blockIdx.x * blockDim.x + threadIdx.x;
    const unsigned lane = threadIdx.x & 31;
    const bool valid = i < n;
    unsigned f = 0;
    for (int o = 0; o < 14; ++o) {
        unsigned long long key = valid ? pack(c[3 * i] + kOff[o][0], c[3 * i + 1] + kOff[o][1], c[3 * i + 2] + kOff[o][2]) : 0;
        unsigned pend = __ballot_sync(0xffffffffu, valid);
        while (pend) {
            const int src = __ffs(pend) - 1;
            pend &= pend - 1;
            const unsigned long long k = __shfl_sync(0xffffffffu, key, src);
            uint64_t h = fmix64(k) & mask;
            while (true) {
                const unsigned long long w = __ldg(&s[(h + lane) & mask].key);
                const unsigned hit = __ballot_sync(0xffffffffu, w == k);
                const unsigned emp = __ballot_sync(0xffffffffu, w == kEmpty);
                if (hit && (!emp || __ffs(hit) < __ffs(emp))) {
                    if (lane == (unsigned)src) ++f;
                    break;
                }
                if (emp) break;
                h = (h + 32) & mask;
            }
        }
    }
    for (int o = 16; o; o >>= 1) f += __shfl_down_sync(0xffffffffu, f, o);
    if (lane == 0) atomicAdd(found, (unsigned long long)f);
}

int main(int argc, char** argv)
{
    if (argc < 4) {
        fprintf(stderr, "usage: %s positions.f64 n cell_km [reps]\n", argv[0]);
        return 2;
    }
    const int n = atoi(argv[2]);
    const double cell = atof(argv[3]);
    const int reps = argc > 4 ? atoi(argv[4]) : 20;
    std::vector<double> hp(3 * (size_t)n);
    FILE* fp = fopen(argv[1], "rb");
    if (!fp || fread(hp.data(), sizeof(double), hp.size(), fp) != hp.size()) {
        fprintf(stderr, "cannot read %s\n", argv[1]);
        return 1;
    }
    fclose(fp);
    uint64_t M = 1;
    while (M < 2 * (uint64_t)n) M <<= 1;
    double* p;
    int* c;
    Slot* s;
    unsigned long long *cnt;
    CK(cudaMalloc(&p, sizeof(double) * hp.size()));
    CK(cudaMalloc(&c, sizeof(int) * hp.size()));
    CK(cudaMalloc(&s, sizeof(Slot) * M));
    CK(cudaMalloc(&cnt, 3 * sizeof(unsigned long long)));
    CK(cudaMemcpy(p, hp.data(), sizeof(double) * hp.size(), cudaMemcpyHostToDevice));
    const int T = 256, Bn = (n + T - 1) / T;
    k_cells<<<Bn, T>>>(p, n, 1.0 / cell, c);
    CK(cudaMemset(s, 0xff, sizeof(Slot) * M));
    CK(cudaMemset2D(reinterpret_cast<char*>(s) + 8, sizeof(Slot), 0, 8, M));
    k_insert<<<Bn, T>>>(c, n, s, M - 1);
    CK(cudaDeviceSynchronize());
    cudaEvent_t e0, e1;
    CK(cudaEventCreate(&e0));
    CK(cudaEventCreate(&e1));
    float msA = 0, msB = 0;
    unsigned long long h[3], fa = 0, fb = 0, pa = 0;
    for (int variant = 0; variant < 2; ++variant) {
        CK(cudaMemset(cnt, 0, 3 * sizeof(unsigned long long)));
        if (variant == 0) k_probe_thread<<<Bn, T>>>(c, n, s, M - 1, cnt, cnt + 2);
        else k_probe_warp<<<Bn, T>>>(c, n, s, M - 1, cnt + 1);
        CK(cudaEventRecord(e0));
        for (int r = 0; r < reps; ++r) {
            if (variant == 0) k_probe_thread<<<Bn, T>>>(c, n, s, M - 1, cnt, cnt + 2);
            else k_probe_warp<<<Bn, T>>>(c, n, s, M - 1, cnt + 1);
        }
        CK(cudaEventRecord(e1));
        CK(cudaEventSynchronize(e1));
        float ms;
        CK(cudaEventElapsedTime(&ms, e0, e1));
        (variant == 0 ? msA : msB) = ms / reps;
        CK(cudaMemcpy(h, cnt, sizeof h, cudaMemcpyDeviceToHost));
        if (variant == 0) {
            fa = h[0] / (reps + 1);
            pa = h[2] / (reps + 1);
        } else {
            fb = h[1] / (reps + 1);
        }
    }
    const double lookups = 14.0 * n;
    printf("{\"n\": %d, \"cell_km\": %g, \"slots\": %llu, \"lookups\": %.0f, \"found_thread\": %llu, "
           "\"found_warp\": %llu, \"avg_probe_len\": %.3f, \"us_thread\": %.2f, \"us_warp\": %.2f}\n",
           n, cell, (unsigned long long)M, lookups, fa, fb, (double)pa / lookups, 1e3 * msA, 1e3 * msB);
    return 0;
}
