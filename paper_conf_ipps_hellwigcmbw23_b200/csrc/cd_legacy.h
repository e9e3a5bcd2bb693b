// cd_legacy.h -- legacy full-window filter chain launchers (P:43, P:189,
// P:315-318).  See cd_legacy.cu.
#pragma once
#include "cd_internal.h"

namespace cdh {

struct LegacyParams {
    double t0, t1, dt, d;
    int64_t K;   // steps in [t0, t1] (reading R4); a minimum is reported by its owner step k < K
};

// Filter pairs [p0, p1) of the row-major upper triangle (i < j) of n objects; surviving
// intervals become work items in w (n_work counts past wcap on overflow); rejections are counted
// in ctrl (n_ap, n_coplanar, n_path, n_time), intervals in ctrl->n_refined.
cudaError_t launch_legacy_filter(const LegacyParams& p, const void* hrec, int64_t n, uint64_t p0,
                                 uint64_t p1, Work* w, size_t wcap, unsigned long long* n_work,
                                 cdk::Ctrl* ctrl, cudaStream_t st, LaunchCount& lc);
// Search the work items for minima below d (next_item: zeroed work counter).
cudaError_t launch_legacy_search(const cdk::Orbits& O, const LegacyParams& p, const void* hrec,
                                 const Work* w, const unsigned long long* n_work, size_t wcap,
                                 unsigned long long* next_item, cdk::Conj* out, size_t ocap,
                                 cdk::Ctrl* ctrl, cudaStream_t st, LaunchCount& lc);

}  // namespace cdh
