// Atomic costs in the k_step context: 1M objects, 128-bit CAS on a slot table of S MB (fresh
// zeroed vs stale lines), RED.OR on a 4 MB bitmap, both together, 64-bit CAS, atomicExch u32.
#include <cstdio>
#include <cuda_runtime.h>
__device__ __forceinline__ unsigned long long mix(unsigned long long k) {
    k ^= k >> 33; k *= 0xff51afd7ed558ccdull; k ^= k >> 33; k *= 0xc4ceb9fe1a85ec53ull; k ^= k >> 33; return k; }
__device__ __forceinline__ bool cas128(unsigned long long* s, unsigned long long e0, unsigned long long e1,
                                       unsigned long long d0, unsigned long long d1) {
    unsigned long long o0, o1;
    asm volatile("{ .reg .b128 d, b, c;\n\tmov.b128 b, {%2, %3};\n\tmov.b128 c, {%4, %5};\n\t"
                 "atom.relaxed.gpu.global.cas.b128 d, [%6], b, c;\n\tmov.b128 {%0, %1}, d; }"
                 : "=l"(o0), "=l"(o1) : "l"(e0), "l"(e1), "l"(d0), "l"(d1), "l"(s) : "memory");
    return o0 == e0 && o1 == e1;
}
template <int V>
__global__ void __launch_bounds__(256) k(unsigned long long* tab, unsigned long long mask, unsigned* bits,
                                         unsigned bmask, unsigned* heads, unsigned seed, unsigned long long* sink)
{
    const unsigned long long i = blockIdx.x * 256ull + threadIdx.x;
    const unsigned long long h = mix(i + ((unsigned long long)seed << 40));
    unsigned long long acc = 0;
    if (V == 0 || V == 2) acc += cas128(tab + 2 * (h & mask), 0, 0, h | 1, i);           // blind CAS128
    if (V == 1 || V == 2) atomicOr(bits + ((h >> 20) & bmask), 1u << (h & 31));         // RED.OR
    if (V == 3) acc += atomicCAS(tab + (h & mask), 0ull, h | 1);                         // CAS64
    if (V == 4) acc += atomicExch(heads + (h & mask), (unsigned)i);                      // EXCH32
    if (V == 5) { unsigned long long w0 = *(volatile unsigned long long*)(tab + 2 * (h & mask));  // load+CAS128
                  acc += cas128(tab + 2 * (h & mask), w0, 0, h | 1, i); }
    if (acc == 0x123456789ull) *sink = acc;
}
int main()
{
    const unsigned long long n = 1 << 20;
    unsigned long long *tab, *sink; unsigned *bits, *heads, *junk;
    cudaMalloc(&tab, 256ull << 20); cudaMalloc(&bits, 4 << 20); cudaMalloc(&heads, 64 << 20);
    cudaMalloc(&junk, 512ull << 20); cudaMalloc(&sink, 8);
    cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
    const char* nm[] = {"CAS128 blind", "RED.OR 4MB", "CAS128+RED", "CAS64 blind", "EXCH32", "load+CAS128"};
    for (int slotsMB : {16, 32, 64}) {
        const unsigned long long nslots = (unsigned long long)slotsMB << 20 >> 4;   // 16 B slots
        for (int V = 0; V < 6; ++V) for (int mode = 0; mode < 2; ++mode) {
            float best = 1e9;
            for (int it = 0; it < 5; ++it) {
                cudaMemset(tab, 0, (size_t)slotsMB << 20); cudaMemset(bits, 0, 4 << 20); cudaMemset(heads, 0, 64 << 20);
                if (mode == 1) cudaMemset(junk, 1, 512ull << 20);   // evict the table from L2 (cold)
                cudaEventRecord(a);
                unsigned long long m = (V == 3 || V == 4) ? (nslots * 2 - 1) : (nslots - 1);
                switch (V) {
                case 0: k<0><<<n / 256, 256>>>(tab, m, bits, (1u << 20) - 1, heads, it, sink); break;
                case 1: k<1><<<n / 256, 256>>>(tab, m, bits, (1u << 20) - 1, heads, it, sink); break;
                case 2: k<2><<<n / 256, 256>>>(tab, m, bits, (1u << 20) - 1, heads, it, sink); break;
                case 3: k<3><<<n / 256, 256>>>(tab, m, bits, (1u << 20) - 1, heads, it, sink); break;
                case 4: k<4><<<n / 256, 256>>>(tab, m < (16ull << 20) - 1 ? m : (16ull << 20) - 1, bits, (1u << 20) - 1, heads, it, sink); break;
                case 5: k<5><<<n / 256, 256>>>(tab, m, bits, (1u << 20) - 1, heads, it, sink); break;
                }
                cudaEventRecord(b); cudaEventSynchronize(b);
                float ms; cudaEventElapsedTime(&ms, a, b); if (ms < best) best = ms;
            }
            printf("table %3d MB  %-14s %s: %7.2f us\n", slotsMB, nm[V], mode ? "cold(L2 evicted)" : "warm(zeroed)   ", best * 1e3);
        }
    }
    printf("err %s\n", cudaGetErrorString(cudaGetLastError()));
}
