// cd_hybrid.h -- hybrid-variant filter chain launcher.
#pragma once
#include "cd_internal.h"

namespace cdh {

// Compact per-object filter records (one 128-byte line each), built once per call.
size_t hybrid_record_bytes();
cudaError_t launch_build_hybrid_records(const cdk::Orbits& O, void* hrec, cudaStream_t st,
                                        LaunchCount& lc);

// Filters the coarse candidates in q; survivors become Brent work items in w (refined by the
// grid variant's k_brent); rejections are counted in ctrl (n_ap, n_coplanar, n_path, n_time).
cudaError_t launch_hybrid_filter(const cdk::Orbits& O, const RefineParams& p, const cdk::Cand* q,
                                 size_t qcap, Work* w, size_t wcap, unsigned long long* n_work,
                                 cdk::Conj* out, size_t ocap, cdk::Ctrl* ctrl, cudaStream_t st,
                                 LaunchCount& lc);

}  // namespace cdh
