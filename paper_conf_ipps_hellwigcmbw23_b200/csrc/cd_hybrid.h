// cd_hybrid.h -- hybrid-variant filter chain launchers.
#pragma once
#include "cd_internal.h"

namespace cdh {

cudaError_t launch_hybrid_filter(const cdk::Orbits& O, const RefineParams& p, const cdk::Cand* q,
                                 size_t qcap, Work* w, size_t wcap, unsigned long long* n_work,
                                 cdk::Conj* out, size_t ocap, cdk::Ctrl* ctrl, cudaStream_t st,
                                 LaunchCount& lc);
cudaError_t launch_hybrid_brent(const cdk::Orbits& O, const RefineParams& p, const Work* w,
                                const unsigned long long* n_work, size_t wcap, cdk::Conj* out,
                                size_t ocap, cdk::Ctrl* ctrl, cudaStream_t st, LaunchCount& lc);

}  // namespace cdh
