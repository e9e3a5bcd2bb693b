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

struct Elements {   // device pointers (external order)
    const double *a, *e, *inc, *raan, *argp, *nu0;
};

// Refinement work item: a candidate that survived the linear pre-filter.
struct Work {
    uint32_t i, j, step, pad;
    double tw;   // Brent half-window t_w = 2 g_c / min(|v_i|, |v_j|)
};

// Optional persisting-L2 window applied to a launch (the per-step grid arena: slots, bitmap,
// entries), so the random-access structures stay resident while the orbit records stream.
struct L2Win {
    bool on = false;
    cudaAccessPolicyWindow w{};
};

struct RefineParams {
    double t0, t1, dt, d, gc;
};

// ---- precompute (a1) -------------------------------------------------------------------
cudaError_t launch_classify(const Elements& el, int64_t n, uint32_t* key, uint32_t* idx,
                            cudaStream_t st, LaunchCount& lc);
cudaError_t launch_build_records(const Elements& el, const uint32_t* perm, int64_t n,
                                 double* rec, uint8_t* cls, cudaStream_t st, LaunchCount& lc);
cudaError_t launch_propagate_out(const cdk::Orbits& O, const uint32_t* perm, const double* t,
                                 int64_t nt, double* xyz, double* vxyz, cudaStream_t st,
                                 LaunchCount& lc);

// ---- grid build + scan (a2-a6) ---------------------------------------------------------
cudaError_t launch_fill_u64(unsigned long long* p, size_t count, unsigned long long v,
                            cudaStream_t st, LaunchCount& lc);
// Fused propagate + cell key + insert; the tables of `tab` must be zero on entry.
cudaError_t launch_prop_insert(const cdk::Orbits& O, const cdk::GridGeom& g, const cdk::GridTab& tab,
                               cdk::Entry* ents, uint64_t mask, int64_t k0, int B, double t0,
                               double dt, cdk::Ctrl* ctrl, const L2Win* win, cudaStream_t st,
                               LaunchCount& lc);
// Neighbour scan of the batch in `tab`; also zeroes the ping-pong set `clr` for the next batch.
cudaError_t launch_scan(const cdk::GridGeom& g, const cdk::GridTab& tab, const cdk::GridTab& clr,
                        int nclr, const cdk::Entry* ents, int64_t n, uint64_t mask, int64_t k0, uint32_t tag,
                        int B, cdk::Cand* q, size_t qcap, cdk::Ctrl* ctrl, const L2Win* win,
                        cudaStream_t st, LaunchCount& lc);

// ---- refinement (a7) -------------------------------------------------------------------
cudaError_t launch_prefilter(const cdk::Orbits& O, const RefineParams& p, const cdk::Cand* q,
                             size_t qcap, Work* w, size_t wcap, unsigned long long* n_work,
                             cdk::Conj* out, size_t ocap, cdk::Ctrl* ctrl, cudaStream_t st,
                             LaunchCount& lc);
cudaError_t launch_brent(const cdk::Orbits& O, const RefineParams& p, const Work* w,
                         const unsigned long long* n_work, size_t wcap, cdk::Conj* out,
                         size_t ocap, cdk::Ctrl* ctrl, cudaStream_t st, LaunchCount& lc);

// ---- finalize (a10) --------------------------------------------------------------------
// Map internal indices to external ids (i < j) and sort by (i, j, step).  Returns the sorted
// array in `out` (device).  Scratch is allocated on the stream.
cudaError_t finalize_conj(const cdk::Conj* in, size_t count, const uint32_t* perm, cdk::Conj* out,
                          cudaStream_t st, LaunchCount& lc);
cudaError_t finalize_cand(const cdk::Cand* in, size_t count, const uint32_t* perm, cdk::Cand* out,
                          cudaStream_t st, LaunchCount& lc);
// stable sort of (key, value) pairs with CUB, used by classify
cudaError_t sort_pairs_u32(const uint32_t* kin, uint32_t* kout, const uint32_t* vin, uint32_t* vout,
                           size_t count, int end_bit, cudaStream_t st, LaunchCount& lc);

}  // namespace cdh
