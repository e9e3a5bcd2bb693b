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
    HHot h;
    horbit(O, r, o, h);
    hr[r] = o;
    reinterpret_cast<HHot*>(hr + O.n)[r] = h;   // the stage-1 lines follow the full records
}

#ifndef CD_FILTER_MINB
#define CD_FILTER_MINB 2
#endif
// Two stages with a per-warp queue between them.  Stage 1 (every candidate): apogee/perigee,
// coplanarity, orbit path -- a pair survives with the mask of its open mutual nodes (~8 % of the
// coarse candidates at 1M objects).  Survivors are queued in shared memory (ballot + prefix) and
// stage 2 (node windows in time: 2-4 atan2 per node, the chain's costliest part) runs only when
// the warp holds 32 of them, so its lanes are converged instead of ~2.6 of 32 active.
constexpr int kFQ = 64;   // per-warp ring: < 32 left over + <= 32 pushed
__device__ __forceinline__ void filter_windows(const HOrbit* __restrict__ hr, const RefineParams& P,
                                               const Cand* __restrict__ q, uint64_t item,
                                               Work* __restrict__ w, size_t wcap,
                                               unsigned long long* n_work, Ctrl* ctrl)
{
    const Cand cd = q[item >> 2];
    const unsigned open = (unsigned)item & 3u;
    const double d = P.d;
    const HOrbit& A = hr[cd.i];
    const HOrbit& B = hr[cd.j];
    bool coplanar;
    NodeGeom gA, gB;
    pair_geometry(A, B, d, coplanar, gA, gB);   // (stage 1's result: not rejected, not coplanar)
    // owner cell of the coarse step, relative to t_k
    const double tk = fma((double)cd.step, P.dt, P.t0);
    const double lo = fmax(tk - 0.5 * P.dt, P.t0) - tk, hi = fmin(tk + 0.5 * P.dt, P.t1) - tk;
    int nwin = 0;
    for (int node = 0; node < 2; ++node) {
        if (!((open >> node) & 1u)) continue;   // orbit path: node closed
        const double sg = node ? -1.0 : 1.0;   // mutual node / opposite node (f + pi)
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
    printf("filter i=%u j=%u k=%u lo=%g hi=%g open=%u nwin=%d\n", cd.i, cd.j, cd.step, lo, hi, open, nwin);
#endif
    if (nwin == 0) count1(&ctrl->n_time);
}

__global__ void __launch_bounds__(256, CD_FILTER_MINB) k_hybrid_filter(Orbits O, RefineParams P, const Cand* __restrict__ q,
                                                       size_t qcap, Work* __restrict__ w, size_t wcap,
                                                       unsigned long long* n_work,
                                                       Conj* __restrict__ out, size_t ocap, Ctrl* ctrl)
{
    __shared__ uint64_t s_fq[8][kFQ];   // per warp: (candidate index << 2) | open-node mask
    const HOrbit* __restrict__ hr = static_cast<const HOrbit*>(P.hrec);
    const HHot* __restrict__ hot = reinterpret_cast<const HHot*>(hr + O.n);
    unsigned long long nc = ctrl->n_cand;
    if (nc > qcap) nc = qcap;
    const unsigned lane = threadIdx.x & 31u, wid = threadIdx.x >> 5;
    uint64_t* fq = s_fq[wid];
    unsigned qh = 0, qt = 0;   // warp-uniform ring head / tail
    const size_t wstride = (size_t)gridDim.x * (blockDim.x >> 5) * 32u;
    for (size_t base = ((size_t)blockIdx.x * (blockDim.x >> 5) + wid) * 32u; base < nc; base += wstride) {
        const size_t idx = base + lane;
        unsigned open = 0;
        if (idx < nc) {
            const Cand cd = q[idx];
            const double d = P.d;
            const HHot ha = hot[cd.i], hb = hot[cd.j];   // one 64-byte line each
            // apogee / perigee first
            if (fmax(ha.a * (1.0 - ha.e), hb.a * (1.0 - hb.e)) - fmin(ha.a * (1.0 + ha.e), hb.a * (1.0 + hb.e)) > d) {
                count1(&ctrl->n_ap);
            } else {
                const HGeo A = geo_of(ha), B = geo_of(hb);
                bool coplanar;
                NodeGeom gA, gB;
                if (pair_geometry(A, B, d, coplanar, gA, gB)) {   // apogee / perigee
                    count1(&ctrl->n_ap);
                } else if (coplanar) {   // same procedure as the grid-based variant (set-up in k_brent)
                    count1(&ctrl->n_coplanar);
                    Work it;
                    it.i = cd.i; it.j = cd.j; it.step = cd.step;
                    it.flags = 4u /* CD_FLAG_COPLANAR */ | kWorkSetup;
                    it.lo = it.hi = 0.0;
                    append(w, wcap, n_work, it);
                } else {
                    open = (node_closed(A, B, d, gA, gB, 1.0) ? 0u : 1u) |
                           (node_closed(A, B, d, gA, gB, -1.0) ? 0u : 2u);
                    if (!open) count1(&ctrl->n_path);
                }
            }
        }
        const unsigned bal = __ballot_sync(0xffffffffu, open != 0);
        if (open) fq[(qt + __popc(bal & ((1u << lane) - 1u))) % kFQ] = ((uint64_t)idx << 2) | open;
        qt += __popc(bal);
        __syncwarp();
        if (qt - qh >= 32u) {
            filter_windows(hr, P, q, fq[(qh + lane) % kFQ], w, wcap, n_work, ctrl);
            qh += 32u;
            __syncwarp();
        }
    }
    if (lane < qt - qh) filter_windows(hr, P, q, fq[(qh + lane) % kFQ], w, wcap, n_work, ctrl);
}

size_t hybrid_record_bytes() { return sizeof(HOrbit) + sizeof(HHot); }

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
