// cd_sort.cu -- a10 finalize: map internal object order to the caller's ids and sort the
// records by (i, j, step) on the device (CUB radix sort, stable, two passes), plus the
// eccentricity-class sort used by the precompute.
#include <cub/cub.cuh>

#include "cd_internal.h"

using namespace cdk;

namespace cdh {

#define CD_TRY(x)                                  \
    do {                                           \
        cudaError_t _e = (x);                      \
        if (_e != cudaSuccess) return _e;          \
    } while (0)

template <typename T>
static cudaError_t dalloc(T** p, size_t count, cudaStream_t st)
{
    return dev_malloc((void**)p, sizeof(T) * (count ? count : 1), st);
}

cudaError_t sort_pairs_u32(const uint32_t* kin, uint32_t* kout, const uint32_t* vin, uint32_t* vout,
                           size_t count, int end_bit, cudaStream_t st, LaunchCount& lc)
{
    size_t tmp_bytes = 0;
    CD_TRY(cub::DeviceRadixSort::SortPairs(nullptr, tmp_bytes, kin, kout, vin, vout, (int64_t)count,
                                           0, end_bit, st));
    void* tmp = nullptr;
    CD_TRY(dev_malloc(&tmp, tmp_bytes ? tmp_bytes : 1, st));
    CD_TRY(cub::DeviceRadixSort::SortPairs(tmp, tmp_bytes, kin, kout, vin, vout, (int64_t)count, 0,
                                           end_bit, st));
    lc.bump(4);   // CUB onesweep: histogram + exclusive scan + one pass per 8-bit digit (upper bound)
    dev_free(tmp, st);
    return cudaGetLastError();
}

template <typename Rec>
__global__ void k_map_keys(const Rec* __restrict__ in, size_t n, const uint32_t* __restrict__ perm,
                           uint32_t* __restrict__ step_key, uint32_t* __restrict__ idx)
{
    const size_t q = blockIdx.x * (size_t)blockDim.x + threadIdx.x;
    if (q >= n) return;
    step_key[q] = in[q].step;
    idx[q] = (uint32_t)q;
}

template <typename Rec>
__global__ void k_pair_keys(const Rec* __restrict__ in, const uint32_t* __restrict__ idx, size_t n,
                            const uint32_t* __restrict__ perm, unsigned long long* __restrict__ key)
{
    const size_t q = blockIdx.x * (size_t)blockDim.x + threadIdx.x;
    if (q >= n) return;
    const Rec r = in[idx[q]];
    uint32_t a = perm ? perm[r.i] : r.i, b = perm ? perm[r.j] : r.j;
    if (a > b) { uint32_t t = a; a = b; b = t; }
    key[q] = ((unsigned long long)a << 32) | b;
}

template <typename Rec>
__global__ void k_gather(const Rec* __restrict__ in, const uint32_t* __restrict__ idx, size_t n,
                         const uint32_t* __restrict__ perm, Rec* __restrict__ out)
{
    const size_t q = blockIdx.x * (size_t)blockDim.x + threadIdx.x;
    if (q >= n) return;
    Rec r = in[idx[q]];
    uint32_t a = perm ? perm[r.i] : r.i, b = perm ? perm[r.j] : r.j;
    if (a > b) { uint32_t t = a; a = b; b = t; }
    r.i = a;
    r.j = b;
    out[q] = r;
}

template <typename Rec>
static cudaError_t finalize_impl(const Rec* in, size_t n, const uint32_t* perm, Rec* out,
                                 cudaStream_t st, LaunchCount& lc)
{
    if (n == 0) return cudaSuccess;
    if (n >= (size_t(1) << 32)) return cudaErrorInvalidValue;
    uint32_t *k1 = nullptr, *k1o = nullptr, *i1 = nullptr, *i1o = nullptr, *i2o = nullptr;
    unsigned long long *k2 = nullptr, *k2o = nullptr;
    CD_TRY(dalloc(&k1, n, st));
    CD_TRY(dalloc(&k1o, n, st));
    CD_TRY(dalloc(&i1, n, st));
    CD_TRY(dalloc(&i1o, n, st));
    CD_TRY(dalloc(&i2o, n, st));
    CD_TRY(dalloc(&k2, n, st));
    CD_TRY(dalloc(&k2o, n, st));
    const unsigned blocks = (unsigned)((n + 255) / 256);
    // pass 1: by step
    k_map_keys<Rec><<<blocks, 256, 0, st>>>(in, n, perm, k1, i1);
    lc.bump();
    CD_TRY(cudaGetLastError());
    size_t tb = 0;
    CD_TRY(cub::DeviceRadixSort::SortPairs(nullptr, tb, k1, k1o, i1, i1o, (int64_t)n, 0, 32, st));
    size_t tb2 = 0;
    CD_TRY(cub::DeviceRadixSort::SortPairs(nullptr, tb2, k2, k2o, i1o, i2o, (int64_t)n, 0, 64, st));
    if (tb2 > tb) tb = tb2;
    void* tmp = nullptr;
    CD_TRY(dev_malloc(&tmp, tb ? tb : 1, st));
    CD_TRY(cub::DeviceRadixSort::SortPairs(tmp, tb, k1, k1o, i1, i1o, (int64_t)n, 0, 32, st));
    lc.bump(6);
    // pass 2 (stable): by (i, j) in caller ids
    k_pair_keys<Rec><<<blocks, 256, 0, st>>>(in, i1o, n, perm, k2);
    lc.bump();
    CD_TRY(cudaGetLastError());
    CD_TRY(cub::DeviceRadixSort::SortPairs(tmp, tb, k2, k2o, i1o, i2o, (int64_t)n, 0, 64, st));
    lc.bump(10);
    k_gather<Rec><<<blocks, 256, 0, st>>>(in, i2o, n, perm, out);
    lc.bump();
    CD_TRY(cudaGetLastError());
    dev_free(tmp, st);
    dev_free(k1, st);
    dev_free(k1o, st);
    dev_free(i1, st);
    dev_free(i1o, st);
    dev_free(i2o, st);
    dev_free(k2, st);
    dev_free(k2o, st);
    return cudaGetLastError();
}

// ---------------------------------------------------------------------------------------
// Spatial slot order (DESIGN.md section 5 "Spatial order"): every R steps the objects are
// renumbered in Morton order of their current position (within their eccentricity class), so a
// warp's objects -- and the grid heads, cells and list entries they touch -- are neighbours in
// space and memory.  The hot build records, the class bytes and the slot -> internal id map are
// gathered into the new order.
// ---------------------------------------------------------------------------------------
__device__ __forceinline__ uint64_t spread3(uint32_t v)   // 16 bits -> every third of 48
{
    uint64_t x = v & 0xffffu;
    x = (x | (x << 32)) & 0x1f00000000ffffull;
    x = (x | (x << 16)) & 0x1f0000ff0000ffull;
    x = (x | (x << 8)) & 0x100f00f00f00f00full;
    x = (x | (x << 4)) & 0x10c30c30c30c30c3ull;
    x = (x | (x << 2)) & 0x1249249249249249ull;
    return x;
}

__device__ __forceinline__ uint32_t quant16(double x)   // [-65536, 65536) km in 2 km steps
{
    const double q = floor((x + 65536.0) * 0.5);
    return q < 0.0 ? 0u : q > 65535.0 ? 65535u : (uint32_t)q;
}

__global__ void k_space_keys(const Entry* __restrict__ E, const uint8_t* __restrict__ cls, int64_t n,
                             unsigned long long* __restrict__ key, uint32_t* __restrict__ val)
{
    const int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (t >= n) return;
    const Entry e = E[t];
    const uint64_t m = spread3(quant16(e.x)) | (spread3(quant16(e.y)) << 1) | (spread3(quant16(e.z)) << 2);
    key[t] = ((unsigned long long)cls[t] << 48) | m;   // class first (class-0 slots stay [0, n0))
    val[t] = (uint32_t)t;
}

// new slot u takes old slot t = perm[u]: its build-record columns (the 9 that the build reads,
// plus the J2 rates), class byte and internal id
__global__ void k_resort_gather(const double* __restrict__ Hold, const uint8_t* __restrict__ cold,
                                const uint32_t* __restrict__ sold, const uint32_t* __restrict__ perm,
                                int64_t n, int ncol, int j2, double* __restrict__ Hnew,
                                uint8_t* __restrict__ cnew, uint32_t* __restrict__ snew)
{
    const int64_t u = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (u >= n) return;
    const uint32_t t = perm[u];
    cnew[u] = cold[t];
    snew[u] = sold ? sold[t] : t;
    for (int k = 0; k <= kBQz; ++k) Hnew[k * n + u] = Hold[k * n + t];
    if (j2)
        for (int k = kDOm; k < ncol; ++k) Hnew[k * n + u] = Hold[k * n + t];
}

cudaError_t space_sort_temp_bytes(int64_t n, size_t* bytes)
{
    *bytes = 0;
    return cub::DeviceRadixSort::SortPairs(nullptr, *bytes, (const unsigned long long*)nullptr,
                                           (unsigned long long*)nullptr, (const uint32_t*)nullptr,
                                           (uint32_t*)nullptr, n, 0, 51);
}

cudaError_t space_resort(const SpaceSort& S, const Entry* E, const double* Hold, const uint8_t* cold,
                         const uint32_t* sold, int64_t n, int ncol, int j2, double* Hnew,
                         uint8_t* cnew, uint32_t* snew, cudaStream_t st, LaunchCount& lc)
{
    const unsigned blocks = (unsigned)((n + 255) / 256);
    k_space_keys<<<blocks, 256, 0, st>>>(E, cold, n, S.key, S.val);
    lc.bump();
    CD_TRY(cudaGetLastError());
    size_t tb = S.tmp_bytes;
    CD_TRY(cub::DeviceRadixSort::SortPairs(S.tmp, tb, S.key, S.key2, S.val, S.val2, n, 0, 51, st));
    lc.bump(8);
    k_resort_gather<<<blocks, 256, 0, st>>>(Hold, cold, sold, S.val2, n, ncol, j2, Hnew, cnew, snew);
    lc.bump();
    return cudaGetLastError();
}

cudaError_t finalize_conj(const Conj* in, size_t count, const uint32_t* perm, Conj* out,
                          cudaStream_t st, LaunchCount& lc)
{
    return finalize_impl<Conj>(in, count, perm, out, st, lc);
}

cudaError_t finalize_cand(const Cand* in, size_t count, const uint32_t* perm, Cand* out,
                          cudaStream_t st, LaunchCount& lc)
{
    return finalize_impl<Cand>(in, count, perm, out, st, lc);
}

}  // namespace cdh
