// cd_hybrid.cu -- hybrid variant filter chain (not yet built: returns cudaErrorNotSupported).
#include "cd_hybrid.h"

namespace cdh {

cudaError_t launch_hybrid_filter(const cdk::Orbits&, const RefineParams&, const cdk::Cand*, size_t,
                                 Work*, size_t, unsigned long long*, cdk::Conj*, size_t, cdk::Ctrl*,
                                 cudaStream_t, LaunchCount&)
{
    return cudaErrorNotSupported;
}

cudaError_t launch_hybrid_brent(const cdk::Orbits&, const RefineParams&, const Work*,
                                const unsigned long long*, size_t, cdk::Conj*, size_t, cdk::Ctrl*,
                                cudaStream_t, LaunchCount&)
{
    return cudaErrorNotSupported;
}

}  // namespace cdh
