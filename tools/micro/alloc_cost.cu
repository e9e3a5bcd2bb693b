// Cost of growing device memory: cudaMalloc vs stream-ordered pool growth (cudaMallocAsync),
// with and without a release threshold.  nvcc -arch=sm_100a -O2 alloc_cost.cu -o alloc_cost
#include <chrono>
#include <cstdio>
#include <cuda_runtime.h>
static double ms_since(std::chrono::steady_clock::time_point t)
{
    return std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t).count();
}
int main()
{
    cudaFree(0);
    cudaStream_t st;
    cudaStreamCreate(&st);
    const size_t sizes[] = {size_t(64) << 20, size_t(256) << 20, size_t(550) << 20, size_t(1200) << 20};
    for (size_t b : sizes) {
        void* p;
        auto t = std::chrono::steady_clock::now();
        cudaMalloc(&p, b);
        double a = ms_since(t);
        t = std::chrono::steady_clock::now();
        cudaFree(p);
        double f = ms_since(t);
        printf("cudaMalloc %6zu MB: %8.3f ms (free %.3f ms)\n", b >> 20, a, f);
    }
    cudaMemPool_t pool;
    cudaDeviceGetDefaultMemPool(&pool, 0);
    uint64_t thr = ~0ull;
    cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &thr);
    for (size_t b : sizes) {
        void* p;
        auto t = std::chrono::steady_clock::now();
        cudaMallocAsync(&p, b, st);
        double a = ms_since(t);
        cudaStreamSynchronize(st);
        double a2 = ms_since(t);
        cudaFreeAsync(p, st);
        cudaStreamSynchronize(st);
        t = std::chrono::steady_clock::now();
        cudaMallocAsync(&p, b, st);
        double r = ms_since(t);
        cudaFreeAsync(p, st);
        cudaStreamSynchronize(st);
        printf("cudaMallocAsync %6zu MB: grow %8.3f ms (+sync %.3f), reuse %.3f ms\n", b >> 20, a, a2, r);
    }
    // a pool created with explicit properties
    cudaMemPoolProps props = {};
    props.allocType = cudaMemAllocationTypePinned;
    props.location.type = cudaMemLocationTypeDevice;
    props.location.id = 0;
    cudaMemPool_t own;
    cudaMemPoolCreate(&own, &props);
    cudaMemPoolSetAttribute(own, cudaMemPoolAttrReleaseThreshold, &thr);
    for (size_t b : sizes) {
        void* p;
        auto t = std::chrono::steady_clock::now();
        cudaMallocFromPoolAsync(&p, b * 2, own, st);
        double a = ms_since(t);
        cudaStreamSynchronize(st);
        cudaFreeAsync(p, st);
        cudaStreamSynchronize(st);
        printf("own pool %6zu MB: grow %8.3f ms\n", (b * 2) >> 20, a);
    }
    return 0;
}
