// Microbenchmark: random-address L2 primitive rates on B200 (1M threads, 16-32 MB tables).
#include <cstdio>
#include <cuda_runtime.h>
__device__ __forceinline__ unsigned long long mix(unsigned long long k) {
    k ^= k >> 33; k *= 0xff51afd7ed558ccdull; k ^= k >> 33; k *= 0xc4ceb9fe1a85ec53ull; k ^= k >> 33; return k; }

template <int V, int ILP>
__global__ void __launch_bounds__(256) k(unsigned long long* t, unsigned* t32, unsigned long long mask, unsigned seed, unsigned long long* sink)
{
    const unsigned long long i = blockIdx.x * (unsigned long long)blockDim.x + threadIdx.x;
    unsigned long long acc = 0;
#pragma unroll
    for (int u = 0; u < ILP; ++u) {
        const unsigned long long h = mix(i * ILP + u + ((unsigned long long)seed << 40)) & mask;
        if (V == 0) acc += atomicCAS(t + h, 0ull, i + 1);                        // 64-bit CAS
        if (V == 1) acc += atomicCAS(t32 + h, 0u, (unsigned)i + 1);              // 32-bit CAS
        if (V == 2) acc += atomicExch(t + h, i + 1);                             // 64-bit EXCH
        if (V == 3) atomicOr(t32 + (h >> 5), 1u << (h & 31));                    // RED.OR (no return)
        if (V == 4) acc += *(volatile unsigned long long*)(t + h);               // plain L2 load
        if (V == 5) acc += __ldg(t + h);                                         // read-only load
        if (V == 6) {                                                            // 128-bit CAS
            unsigned long long lo, hi;
            unsigned long long* a = t + (h & ~1ull);
            asm volatile("{ .reg .b128 d, b, c;\n\t"
                         "mov.b128 b, {%2, %3};\n\t"
                         "mov.b128 c, {%4, %5};\n\t"
                         "atom.global.cas.b128 d, [%6], b, c;\n\t"
                         "mov.b128 {%0, %1}, d; }"
                         : "=l"(lo), "=l"(hi) : "l"(0ull), "l"(0ull), "l"(i + 1), "l"(i), "l"(a) : "memory");
            acc += lo + hi;
        }
        if (V == 7) t[h] = i;                                                    // plain random store
    }
    if (acc == 0x1234567) *sink = acc;
}

int main()
{
    const unsigned long long n = 1ull << 20, M = 1ull << 21;
    unsigned long long *t, *sink; unsigned* t32;
    cudaMalloc(&t, 8 * M); cudaMalloc(&t32, 4 * M); cudaMalloc(&sink, 8);
    cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
    const char* nm[] = {"CAS64", "CAS32", "EXCH64", "RED.OR32", "LD64 volatile", "LDG64", "CAS128", "ST64"};
    for (int V = 0; V < 8; ++V)
        for (int ilp = 1; ilp <= 4; ilp *= 2) {
            float best = 1e9;
            for (int it = 0; it < 10; ++it) {
                cudaMemsetAsync(t, 0, 8 * M); cudaMemsetAsync(t32, 0, 4 * M);
                cudaEventRecord(a);
                unsigned blocks = (unsigned)(n / ilp / 256);
#define L(VV, II) if (V == VV && ilp == II) k<VV, II><<<blocks, 256>>>(t, t32, M - 1, it, sink);
#define LL(VV) L(VV, 1) L(VV, 2) L(VV, 4)
                LL(0) LL(1) LL(2) LL(3) LL(4) LL(5) LL(6) LL(7)
                cudaEventRecord(b); cudaEventSynchronize(b);
                float ms; cudaEventElapsedTime(&ms, a, b); if (ms < best) best = ms;
            }
            printf("%-14s ILP %d: %7.2f us for 1M ops -> %6.1f Gop/s\n", nm[V], ilp, best * 1e3, 1e-9 * n / (best * 1e-3));
        }
    printf("err: %s\n", cudaGetErrorString(cudaGetLastError()));
}
