// cd_hybrid.cu -- hybrid variant: the classical orbital filter chain applied to the coarse grid's
// candidates, on the device.
//
// The grid (k_step) runs at the coarse step dt_h with cell g_c,h = d + 7.8 dt_h (9 s).
// Per coarse candidate (i, j, k) this kernel evaluates (reading R17):
//   apogee/perigee  exclude iff max(q_i, q_j) - min(Q_i, Q_j) > d                   (Hoots [13])
//   coplanarity     |r_A - r_B| >= |r_A . h_B| = |r_A| |sin u_A| sin D: a conjunction needs
//                   |sin u_A| < s_A = d / (q_A sin D) and the same for B; if s_A >= 1, s_B >= 1
//                   or q_A cos(asin s_A) + q_B cos(asin s_B) <= d the windows cannot separate
//                   the mutual nodes -> "coplanar": the grid-variant refinement
//   orbit path      per mutual node: radial ranges over the two windows more than d apart
//                   excludes the node; both nodes excluded excludes the pair       (Hoots [13])
//   time filter     windows in time (true anomaly -> eccentric -> mean anomaly -> t, no Kepler
//                   solve) of both objects at the same node, intersected with each other and
//                   with the coarse step's owner cell; empty excludes the pair    (Woodburn [15])
// Surviving intervals become Brent work items (k_brent, shared with the grid variant); because
// every filter is conservative the result is the set of minima below d owned by coarse steps.
#include "cd_hybrid.h"
#ifdef CD_DEBUG_FILTER
#include <cstdio>
#endif
#include "cd_filters.cuh"

using namespace cdk;

namespace cdh {

using namespace filt;


__global__ void k_build_hrec(Orbits O, HOrbit* __restrict__ hr)
{
    const int64_t r = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (r >= O.n) return;
    HOrbit o;
    horbit(O, r, o);
    hr[r] = o;
}

#ifndef CD_FILTER_MINB
#define CD_FILTER_MINB 2
#endif
__global__ void __launch_bounds__(256, CD_FILTER_MINB) k_hybrid_filter(Orbits O, RefineParams P, const Cand* __restrict__ q,
                                                       size_t qcap, Work* __restrict__ w, size_t wcap,
                                                       unsigned long long* n_work,
                                                       Conj* __restrict__ out, size_t ocap, Ctrl* ctrl)
{
    const HOrbit* __restrict__ hr = static_cast<const HOrbit*>(P.hrec);
    unsigned long long nc = ctrl->n_cand;
    if (nc > qcap) nc = qcap;
    const size_t stride = (size_t)gridDim.x * blockDim.x;
    for (size_t idx = blockIdx.x * (size_t)blockDim.x + threadIdx.x; idx < nc; idx += stride) {
        const Cand cd = q[idx];
        const double d = P.d;
        // apogee / perigee first, from 16 bytes of each record
        if (fmax(hr[cd.i].q, hr[cd.j].q) - fmin(hr[cd.i].Q, hr[cd.j].Q) > d) {
            count1(&ctrl->n_ap);
            continue;
        }
        // records by reference: fields are loaded where used (94 instead of 118 registers)
        const HOrbit& A = hr[cd.i];
        const HOrbit& B = hr[cd.j];
        bool coplanar;
        NodeGeom gA, gB;
        if (pair_geometry(A, B, d, coplanar, gA, gB)) {   // apogee / perigee
            count1(&ctrl->n_ap);
            continue;
        }
        if (coplanar) {   // same procedure as the grid-based variant (set-up in k_brent)
            count1(&ctrl->n_coplanar);
            Work it;
            it.i = cd.i; it.j = cd.j; it.step = cd.step;
            it.flags = 4u /* CD_FLAG_COPLANAR */ | kWorkSetup;
            it.lo = it.hi = 0.0;
            append(w, wcap, n_work, it);
            continue;
        }
        // owner cell of the coarse step, relative to t_k
        const double tk = fma((double)cd.step, P.dt, P.t0);
        const double lo = fmax(tk - 0.5 * P.dt, P.t0) - tk, hi = fmin(tk + 0.5 * P.dt, P.t1) - tk;
        bool any_node = false;
        int nwin = 0;
        for (int node = 0; node < 2; ++node) {
            const double sg = node ? -1.0 : 1.0;   // mutual node / opposite node (f + pi)
            if (node_closed(A, B, d, gA, gB, sg)) continue;   // orbit path: node closed
            any_node = true;
            // the copies k T of each periodic window that meet the owner cell [lo, hi] (windows
            // are shorter than half a period and the cell far shorter than a period: at most two
            // of three consecutive copies), intersected pairwise.  A's window first: B's is only
            // computed when one of A's copies meets the cell (most pairs end here)
            double atl, ath, btl, bth;
            node_window(A, gA, sg, atl, ath);
            const double TA = kTwoPiH * A.inm, TB = kTwoPiH * B.inm;
            const double ka = floor((lo - (ath - tk)) * (A.nm * (1.0 / kTwoPiH)));
            bool a_meets = false;
            for (int x = 0; x < 3; ++x)
                a_meets = a_meets || fmin(ath - tk + (ka + x) * TA, hi) >= fmax(atl - tk + (ka + x) * TA, lo);
            if (!a_meets) continue;
            node_window(B, gB, sg, btl, bth);
            const double kb = floor((lo - (bth - tk)) * (B.nm * (1.0 / kTwoPiH)));
            for (int x = 0; x < 3; ++x) {
                const double al = fmax(atl - tk + (ka + x) * TA, lo), ah = fmin(ath - tk + (ka + x) * TA, hi);
                if (!(ah >= al)) continue;
                for (int y = 0; y < 3; ++y) {
                    const double bl = fmax(btl - tk + (kb + y) * TB, lo), bh = fmin(bth - tk + (kb + y) * TB, hi);
                    if (!(bh >= bl)) continue;
                    const double l = fmax(al, bl), h = fmin(ah, bh);
                    if (h > l) {
                        Work it;
                        it.i = cd.i; it.j = cd.j; it.step = cd.step; it.flags = 0u;
                        it.lo = l;
                        it.hi = h;
                        append(w, wcap, n_work, it);
                        ++nwin;
                    }
                }
            }
        }
#ifdef CD_DEBUG_FILTER
        printf("filter i=%u j=%u k=%u lo=%g hi=%g any=%d nwin=%d\n", cd.i, cd.j, cd.step, lo, hi,
               (int)any_node, nwin);
#endif
        if (!any_node) count1(&ctrl->n_path);
        else if (nwin == 0) count1(&ctrl->n_time);
    }
}

size_t hybrid_record_bytes() { return sizeof(HOrbit); }

cudaError_t launch_build_hybrid_records(const Orbits& O, void* hrec, cudaStream_t st, LaunchCount& lc)
{
    k_build_hrec<<<(unsigned)((O.n + 127) / 128), 128, 0, st>>>(O, static_cast<HOrbit*>(hrec));
    lc.bump();
    return cudaGetLastError();
}

cudaError_t launch_hybrid_filter(const Orbits& O, const RefineParams& p, const Cand* q, size_t qcap,
                                 Work* w, size_t wcap, unsigned long long* n_work, Conj* out,
                                 size_t ocap, Ctrl* ctrl, cudaStream_t st, LaunchCount& lc)
{
    k_hybrid_filter<<<148 * 8, 256, 0, st>>>(O, p, q, qcap, w, wcap, n_work, out, ocap, ctrl);
    lc.bump();
    return cudaGetLastError();
}

}  // namespace cdh
