// cd_internal.h -- host-side declarations shared by the library's translation units.
#pragma once
#include <cuda_runtime.h>

#include <atomic>
#include <cstddef>
#include <cstdint>

#include "cd_device.cuh"

namespace cdh {

extern std::atomic<uint64_t> g_launches;   // kernels launched by this process

// Per-call launch counter: every launcher bumps both the global and the per-call count.
struct LaunchCount {
    uint64_t n = 0;
    void bump(uint64_t k = 1) { n += k; g_launches.fetch_add(k, std::memory_order_relaxed); }
};

// Device scratch memory of the current call (thread-local, set by the call for its duration):
// the caller's allocator (cd_options.alloc / free / alloc_ctx, e.g. PyTorch's caching allocator)
// when given, else the device's stream-ordered pool.
struct DevAlloc {
    void* (*alloc)(size_t bytes, void* ctx) = nullptr;
    void (*free)(void* p, void* ctx) = nullptr;
    void* ctx = nullptr;
};
extern thread_local DevAlloc g_dev_alloc;

// The library's own stream-ordered pool of the call's device (created on first use with
// cudaMemPoolCreate; the device's default pool and its settings are left alone).  It keeps its
// memory between calls (release threshold = max) so back-to-back screens do not re-map pages;
// cd_release_caches() trims it.
extern thread_local cudaMemPool_t g_pool;

inline cudaError_t dev_malloc(void** p, size_t bytes, cudaStream_t st)
{
    if (bytes == 0) bytes = 1;
    if (g_dev_alloc.alloc) {
        *p = g_dev_alloc.alloc(bytes, g_dev_alloc.ctx);
        return *p ? cudaSuccess : cudaErrorMemoryAllocation;
    }
    if (g_pool) return cudaMallocFromPoolAsync(p, bytes, g_pool, st);
    return cudaMallocAsync(p, bytes, st);
}

inline void dev_free(void* p, cudaStream_t st)
{
    if (!p) return;
    if (g_dev_alloc.free) g_dev_alloc.free(p, g_dev_alloc.ctx);
    else cudaFreeAsync(p, st);
}

struct Elements {   // device pointers (external order)
    const double *a, *e, *inc, *raan, *argp, *nu0;
};

// Refinement work item: a candidate (or a hybrid time window) for Brent's search.
struct Work {
    uint32_t i, j, step, flags;
    double lo, hi;   // search interval relative to t_k (inside [t0, t1])
};

// Optional persisting-L2 window applied to a launch (the per-step grid arena: slots, bitmap,
// entries), so the random-access structures stay resident while the orbit records stream.
struct L2Win {
    bool on = false;
    cudaAccessPolicyWindow w{};
};

struct RefineParams {
    double t0, t1, dt, d, gc;
    const void* hrec = nullptr;   // hybrid: compact per-object filter records
};

// ---- precompute (a1) -------------------------------------------------------------------
// min_cls: minimum eccentricity class (Contour point count) of every object, from
// cd_options.kepler_points (kepler_class_of_points)
cudaError_t launch_classify(const Elements& el, int64_t n, uint32_t* key, uint32_t* idx,
                            unsigned long long* n0, int min_cls, cudaStream_t st, LaunchCount& lc);
cudaError_t launch_build_records(const Elements& el, const uint32_t* perm, int64_t n,
                                 double* rec, double* arec, uint8_t* cls, int j2, int min_cls,
                                 cudaStream_t st, LaunchCount& lc);
cudaError_t launch_propagate_out(const cdk::Orbits& O, const uint32_t* perm, const double* t,
                                 int64_t nt, double* xyz, double* vxyz, cudaStream_t st,
                                 LaunchCount& lc);

// ---- radial L2 shards (screen_sharded) ----------------------------------------------------
cudaError_t launch_gather_elements(const Elements& src, const uint32_t* idx, int64_t m, double* dst,
                                   cudaStream_t st, LaunchCount& lc);
cudaError_t launch_compose_perm(uint32_t* perm, const uint32_t* idx, int64_t m, cudaStream_t st,
                                LaunchCount& lc);
cudaError_t launch_conj_to_global(const cdk::Conj* in, size_t n, const uint32_t* perm,
                                  cdk::Conj* out, cudaStream_t st, LaunchCount& lc);

// ---- grid build + scan (a2-a6) ---------------------------------------------------------
// One batch launch of the fused step kernel: build batch b+1 into build_tab (slots tagged
// build_tag, bitmap zero on entry), scan batch b in scan_tab (tag scan_tag), zero the bitmap set
// zero_bits (zero_depth tables) for batch b+2.
struct StepArgs {
    cdk::Orbits O;
    cdk::GridGeom g;
    uint64_t mask;
    double t0, dt;
    int64_t build_B, build_k0;   // build_B = 0: no build role
    cdk::GridTab build_tab;
    cdk::Entry* build_ents;
    uint32_t build_tag;
    int64_t scan_B, scan_k0;     // scan_B = 0: no scan role
    cdk::GridTab scan_tab;
    const cdk::Entry* scan_ents;
    uint32_t scan_tag;
    uint32_t* zero_bits;
    int64_t zero_bits_words;     // words per table
    int64_t zero_depth;          // tables to zero (0: none)
    cdk::Cand* q;
    size_t qcap;
    cdk::Ctrl* ctrl;
    int64_t nbA, nbB, nbC;       // blocks per step of roles A, B, C (filled by launch_step)
    int64_t nCblocks;            // role-C blocks in the launch
    int chained;                 // 1: chained spatial hash (heads in the bitmap arrays)
    int pdl;                     // 1: programmatic dependent launch (chained grid only)
    int csr;                     // 1: CSR grid (counting sort by cell): build_ents = per-object
                                 // (slot, rank) entries, scan_ents = the scanned batch's segments
    const uint32_t* scan_start;  // CSR: segment start per slot of the scanned batch
};
// CSR grid: segments of a built batch (B steps): k_csr_alloc + k_csr_scatter (cd_kernels.cu)
cudaError_t launch_csr_segments(const cdk::Slot* slots, uint32_t* start, uint64_t M,
                                const cdk::Entry* tmp, cdk::Entry* csr, int64_t n, int B, uint32_t tag,
                                unsigned long long* total, cudaStream_t st, LaunchCount& lc);
cudaError_t launch_step(StepArgs a, const L2Win* win, cudaStream_t st, LaunchCount& lc);

// ---- refinement (a7) -------------------------------------------------------------------
cudaError_t launch_prefilter(const cdk::Orbits& O, const RefineParams& p, const cdk::Cand* q,
                             size_t qcap, Work* w, size_t wcap, unsigned long long* n_work,
                             cdk::Conj* out, size_t ocap, cdk::Ctrl* ctrl, cudaStream_t st,
                             LaunchCount& lc);
cudaError_t launch_brent(const cdk::Orbits& O, const RefineParams& p, const Work* w,
                         const unsigned long long* n_work, size_t wcap, cdk::Conj* out,
                         size_t ocap, cdk::Ctrl* ctrl, cudaStream_t st, LaunchCount& lc);

// digest_only: fold a round's records into Ctrl's digest and empty the buffer (k_conj_digest,
// k_conj_reset; skipped for an overflowed round)
cudaError_t launch_conj_digest(const cdk::Conj* c, size_t ocap, const uint32_t* perm, cdk::Ctrl* ctrl,
                               cudaStream_t st, LaunchCount& lc);

// ---- finalize (a10) --------------------------------------------------------------------
// Map internal indices to external ids (i < j) and sort by (i, j, step).  Returns the sorted
// array in `out` (device).  Scratch is allocated on the stream.
cudaError_t finalize_conj(const cdk::Conj* in, size_t count, const uint32_t* perm, cdk::Conj* out,
                          cudaStream_t st, LaunchCount& lc);
cudaError_t finalize_cand(const cdk::Cand* in, size_t count, const uint32_t* perm, cdk::Cand* out,
                          cudaStream_t st, LaunchCount& lc);
// spatial slot order (cd_sort.cu): scratch of one re-sort, allocated once per call
struct SpaceSort {
    unsigned long long *key, *key2;
    uint32_t *val, *val2;
    void* tmp;
    size_t tmp_bytes;
};
cudaError_t space_sort_temp_bytes(int64_t n, size_t* bytes);
// renumber the n slots in Morton order (within class) of the positions in E (one built step,
// slot-indexed in the old order); gather the old hot build records / classes / slot -> internal
// id map (sold: nullptr = identity) into the new order
cudaError_t space_resort(const SpaceSort& S, const cdk::Entry* E, const double* Hold, const uint8_t* cold,
                         const uint32_t* sold, int64_t n, int ncol, int j2, double* Hnew,
                         uint8_t* cnew, uint32_t* snew, cudaStream_t st, LaunchCount& lc);
// stable sort of (key, value) pairs with CUB, used by classify
cudaError_t sort_pairs_u32(const uint32_t* kin, uint32_t* kout, const uint32_t* vin, uint32_t* vout,
                           size_t count, int end_bit, cudaStream_t st, LaunchCount& lc);

}  // namespace cdh
