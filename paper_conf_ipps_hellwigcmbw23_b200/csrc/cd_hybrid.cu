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
#include "cd_refine.cuh"

using namespace cdk;

namespace cdh {

namespace {

constexpr double kPiH = 3.14159265358979323846;
constexpr double kTwoPiH = 6.28318530717958647692;

struct __align__(128) HOrbit {   // one 128-byte line per object (compact gather in the filter)
    double e, q, Q, p, nm, M0;
    double P[3], Qv[3], h[3];
    double pad;
};
static_assert(sizeof(HOrbit) == 128, "HOrbit must be one 128-byte line");

__device__ __forceinline__ void horbit(const Orbits& O, int64_t r, HOrbit& o)
{
    const double ap[3] = {O.at(kAPx, r), O.at(kAPy, r), O.at(kAPz, r)};
    const double bq[3] = {O.at(kBQx, r), O.at(kBQy, r), O.at(kBQz, r)};
    const double a = sqrt(ap[0] * ap[0] + ap[1] * ap[1] + ap[2] * ap[2]);
    const double b = sqrt(bq[0] * bq[0] + bq[1] * bq[1] + bq[2] * bq[2]);
    for (int c = 0; c < 3; ++c) {
        o.P[c] = ap[c] / a;
        o.Qv[c] = bq[c] / b;
    }
    o.h[0] = o.P[1] * o.Qv[2] - o.P[2] * o.Qv[1];
    o.h[1] = o.P[2] * o.Qv[0] - o.P[0] * o.Qv[2];
    o.h[2] = o.P[0] * o.Qv[1] - o.P[1] * o.Qv[0];
    o.e = O.at(kE, r);
    o.q = a * (1.0 - o.e);
    o.Q = a * (1.0 + o.e);
    o.p = a * (1.0 - o.e) * (1.0 + o.e);
    o.nm = O.at(kNm, r);
    o.M0 = O.at(kM0, r);
    o.pad = 0.0;
}

// mean anomaly of true anomaly f, in [-pi, pi]: f is reduced to [-pi, pi] first so the half-angle
// formula stays on its principal branch (window ends on different branches would cancel a window)
__device__ __forceinline__ double mean_of_true(double f, double e)
{
    f = remainder(f, kTwoPiH);
    double sf, cf;
    sincos(0.5 * f, &sf, &cf);
    const double E = 2.0 * atan2(sqrt(1.0 - e) * sf, sqrt(1.0 + e) * cf);
    return E - e * sin(E);
}

// radius range over true anomalies [f1, f2], f2 - f1 < pi
__device__ __forceinline__ void radius_range(const HOrbit& o, double f1, double f2, double& rmin,
                                             double& rmax)
{
    const double r1 = o.p / (1.0 + o.e * cos(f1)), r2 = o.p / (1.0 + o.e * cos(f2));
    rmin = fmin(r1, r2);
    rmax = fmax(r1, r2);
    if (ceil(f1 / kTwoPiH) * kTwoPiH <= f2) rmin = o.q;                  // perigee inside
    if (kPiH + ceil((f1 - kPiH) / kTwoPiH) * kTwoPiH <= f2) rmax = o.Q;  // apogee inside
}

// first-occurrence time window [tl, th] (mod T) of true anomaly in (fc - al, fc + al)
__device__ __forceinline__ void node_window(const HOrbit& o, double fc, double al, double& tl,
                                            double& th)
{
    const double Ml = mean_of_true(fc - al, o.e);
    double Mh = mean_of_true(fc + al, o.e);
    if (Mh < Ml) Mh += kTwoPiH;
    tl = (Ml - o.M0) / o.nm;
    th = (Mh - o.M0) / o.nm;
}

// the (at most one per period) copy of the periodic window [tl, th] + k T overlapping [lo, hi];
// windows are shorter than half a period and [lo, hi] (one coarse cell) is far shorter than a
// period, so at most two copies can touch it
__device__ __forceinline__ int window_copies(double tl, double th, double T, double lo, double hi,
                                             double out[4])
{
    int c = 0;
    const double k0 = floor((lo - th) / T);
    for (int q = 0; q < 3; ++q) {
        const double a = tl + (k0 + q) * T, b = th + (k0 + q) * T;
        if (b < lo || a > hi) continue;
        if (c < 2) {
            out[2 * c] = fmax(a, lo);
            out[2 * c + 1] = fmin(b, hi);
            ++c;
        }
    }
    return c;
}

// warp-aggregated counter increment (one atomic per group of converged lanes)
__device__ __forceinline__ void count1(unsigned long long* cnt)
{
    cg::coalesced_group g = cg::coalesced_threads();
    if (g.thread_rank() == 0) atomicAdd(cnt, (unsigned long long)g.size());
}

}  // namespace

__global__ void k_build_hrec(Orbits O, HOrbit* __restrict__ hr)
{
    const int64_t r = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (r >= O.n) return;
    HOrbit o;
    horbit(O, r, o);
    hr[r] = o;
}

__global__ void __launch_bounds__(256) k_hybrid_filter(Orbits O, RefineParams P, const Cand* __restrict__ q,
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
        const HOrbit A = hr[cd.i], B = hr[cd.j];
        const double d = P.d;
        // apogee / perigee
        if (fmax(A.q, B.q) - fmin(A.Q, B.Q) > d) {
            count1(&ctrl->n_ap);
            continue;
        }
        // mutual inclination and node line
        const double c[3] = {A.h[1] * B.h[2] - A.h[2] * B.h[1], A.h[2] * B.h[0] - A.h[0] * B.h[2],
                             A.h[0] * B.h[1] - A.h[1] * B.h[0]};
        const double sD = sqrt(c[0] * c[0] + c[1] * c[1] + c[2] * c[2]);
        const double sA = sD > 0.0 ? d / (A.q * sD) : 2.0;
        const double sB = sD > 0.0 ? d / (B.q * sD) : 2.0;
        bool coplanar = sA >= 1.0 || sB >= 1.0;
        double aA = 0.0, aB = 0.0;
        if (!coplanar) {
            aA = asin(sA);
            aB = asin(sB);
            coplanar = A.q * cos(aA) + B.q * cos(aB) <= d;
        }
        if (coplanar) {   // same procedure as the grid-based variant
            count1(&ctrl->n_coplanar);
            grid_refine_item(O, P, cd, 4u /* CD_FLAG_COPLANAR */, w, wcap, n_work, out, ocap, ctrl);
            continue;
        }
        const double nn[3] = {c[0] / sD, c[1] / sD, c[2] / sD};
        const double fA = atan2(nn[0] * A.Qv[0] + nn[1] * A.Qv[1] + nn[2] * A.Qv[2],
                                nn[0] * A.P[0] + nn[1] * A.P[1] + nn[2] * A.P[2]);
        const double fB = atan2(nn[0] * B.Qv[0] + nn[1] * B.Qv[1] + nn[2] * B.Qv[2],
                                nn[0] * B.P[0] + nn[1] * B.P[1] + nn[2] * B.P[2]);
        // owner cell of the coarse step, relative to t_k
        const double tk = fma((double)cd.step, P.dt, P.t0);
        const double lo = fmax(tk - 0.5 * P.dt, P.t0) - tk, hi = fmin(tk + 0.5 * P.dt, P.t1) - tk;
        bool any_node = false;
        int nwin = 0;
        for (int node = 0; node < 2; ++node) {
            const double off = node ? kPiH : 0.0;
            double rAl, rAh, rBl, rBh;
            radius_range(A, fA + off - aA, fA + off + aA, rAl, rAh);
            radius_range(B, fB + off - aB, fB + off + aB, rBl, rBh);
            if (fmax(rAl, rBl) - fmin(rAh, rBh) > d) continue;   // orbit path: node closed
            any_node = true;
            double atl, ath, btl, bth;
            node_window(A, fA + off, aA, atl, ath);
            node_window(B, fB + off, aB, btl, bth);
            double wa[4], wb[4];
            const int na = window_copies(atl - tk, ath - tk, kTwoPiH / A.nm, lo, hi, wa);
            const int nb = window_copies(btl - tk, bth - tk, kTwoPiH / B.nm, lo, hi, wb);
            for (int x = 0; x < na; ++x)
                for (int y = 0; y < nb; ++y) {
                    const double l = fmax(wa[2 * x], wb[2 * y]), h = fmin(wa[2 * x + 1], wb[2 * y + 1]);
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
#ifdef CD_DEBUG_FILTER
        printf("filter i=%u j=%u k=%u sD=%.17g sA=%.17g sB=%.17g fA=%.17g fB=%.17g lo=%g hi=%g any=%d nwin=%d A.M0=%.17g A.nm=%.17g B.M0=%.17g B.nm=%.17g\n",
               cd.i, cd.j, cd.step, sD, sA, sB, fA, fB, lo, hi, (int)any_node, nwin, A.M0, A.nm, B.M0, B.nm);
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
