// cd_filters.cuh -- classical orbital filter geometry shared by the hybrid variant (cd_hybrid.cu,
// coarse-step candidates) and the legacy full-window chain (cd_legacy.cu, all pairs): compact
// per-object records and the apogee/perigee, orbit-path and time-filter formulas of reading R17
// (PAPER.md:43 names the filters [13], [15]).
#pragma once
#include "cd_refine.cuh"

namespace cdh {
namespace filt {

using namespace cdk;


constexpr double kPiH = 3.14159265358979323846;
constexpr double kTwoPiH = 6.28318530717958647692;

struct __align__(128) HOrbit {   // one 128-byte line per object (compact gather in the filter)
    double e, q, Q, p, nm, M0;
    double P[3], Qv[3], h[3];
    double inm;   // 1 / nm
};
static_assert(sizeof(HOrbit) == 128, "HOrbit must be one 128-byte line");

// The hybrid filter's stage 1 (apogee/perigee, coplanarity, orbit path) reads only a, e and the
// perifocal unit vectors: one 64-byte line per object (64 MB at 1M objects, L2-resident), loaded
// whole into registers; q, Q, p and h are derived there with horbit's own expressions (so the
// values are bit-identical to HOrbit's).
struct __align__(64) HHot {
    double a, e, P[3], Qv[3];
};
static_assert(sizeof(HHot) == 64, "HHot must be one 64-byte line");

// the HOrbit fields stage 1 uses, in registers
struct HGeo {
    double e, q, Q, p;
    double P[3], Qv[3], h[3];
};
__device__ __forceinline__ HGeo geo_of(const HHot& o)
{
    HGeo g;
    g.e = o.e;
    g.q = o.a * (1.0 - o.e);
    g.Q = o.a * (1.0 + o.e);
    g.p = o.a * (1.0 - o.e) * (1.0 + o.e);
    for (int c = 0; c < 3; ++c) {
        g.P[c] = o.P[c];
        g.Qv[c] = o.Qv[c];
    }
    g.h[0] = g.P[1] * g.Qv[2] - g.P[2] * g.Qv[1];
    g.h[1] = g.P[2] * g.Qv[0] - g.P[0] * g.Qv[2];
    g.h[2] = g.P[0] * g.Qv[1] - g.P[1] * g.Qv[0];
    return g;
}

__device__ __forceinline__ void horbit(const Orbits& O, int64_t r, HOrbit& o, HHot& hot)
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
    o.inm = 1.0 / o.nm;
    hot.a = a;
    hot.e = o.e;
    for (int c = 0; c < 3; ++c) {
        hot.P[c] = o.P[c];
        hot.Qv[c] = o.Qv[c];
    }
}

// Divisions are reciprocal estimates refined to full precision (rcp_fast: two Newton steps) times
// the numerator -- the filters' decisions have km margins, 2 roundings instead of 1 are immaterial.
// Node geometry of one orbit of a pair (reading R17), all algebraic: the mutual node line is a
// unit vector in the orbit plane, so its components along P and Q are the cosine and sine of its
// true anomaly f; the window half-angle a = asin(s) has sin a = s, cos a = sqrt(1 - s^2).  The
// opposite node (f + pi) flips the sign of (cos f, sin f).
struct NodeGeom {
    double cf, sf;   // cos f, sin f of the ascending mutual node
    double sa, ca;   // sin a, cos a of the window half-angle
};

// Mean anomaly of the true anomaly with cosine c and sine s, in [-pi, pi] (principal branch):
//   sin E = sqrt(1 - e^2) s / (1 + e c),  cos E = (e + c) / (1 + e c),  M = E - e sin E
__device__ __forceinline__ double mean_of_true_cs(double c, double s, double e)
{
    const double w = sqrt((1.0 - e) * (1.0 + e));
    const double E = atan2(w * s, e + c);
    return E - e * (w * s * rcp_fast(fma(e, c, 1.0)));
}

// radius range over the true anomalies (f - a, f + a) of node `sg` (+1: f, -1: f + pi), a < pi/2:
// the ends r = p / (1 + e cos(f -+ a)), widened to the perigee radius if the interval contains
// f = 0 (cos f >= cos a) and to the apogee radius if it contains f = pi (-cos f >= cos a)
template <typename R>
__device__ __forceinline__ void radius_range(const R& o, const NodeGeom& g, double sg,
                                             double& rmin, double& rmax)
{
    const double cf = sg * g.cf, sf = sg * g.sf;
    const double c1 = fma(cf, g.ca, sf * g.sa), c2 = fma(cf, g.ca, -sf * g.sa);
    const double r1 = o.p * rcp_fast(fma(o.e, c1, 1.0)), r2 = o.p * rcp_fast(fma(o.e, c2, 1.0));
    rmin = fmin(r1, r2);
    rmax = fmax(r1, r2);
    if (cf >= g.ca) rmin = o.q;    // perigee inside
    if (-cf >= g.ca) rmax = o.Q;   // apogee inside
}

// first-occurrence time window [tl, th] (mod T) of the true anomaly in (f - a, f + a) of node sg
__device__ __forceinline__ void node_window(const HOrbit& o, const NodeGeom& g, double sg,
                                            double& tl, double& th)
{
    const double cf = sg * g.cf, sf = sg * g.sf;
    const double Ml = mean_of_true_cs(fma(cf, g.ca, sf * g.sa), fma(sf, g.ca, -cf * g.sa), o.e);
    double Mh = mean_of_true_cs(fma(cf, g.ca, -sf * g.sa), fma(sf, g.ca, cf * g.sa), o.e);
    if (Mh < Ml) Mh += kTwoPiH;
    tl = (Ml - o.M0) * o.inm;
    th = (Mh - o.M0) * o.inm;
}

// Pair geometry of the filter chain (reading R17).  Returns 1 if the apogee/perigee filter
// rejects the pair; otherwise 0 with coplanar set, and for non-coplanar pairs the node geometry
// of each orbit.
//   AP:        exclude iff max(q_A, q_B) - min(Q_A, Q_B) > d
//   coplanar:  s_X = d / (q_X sin D) >= 1 for A or B, or q_A cos(asin s_A) + q_B cos(asin s_B) <= d
template <typename R>
__device__ __forceinline__ int pair_geometry(const R& A, const R& B, double d,
                                             bool& coplanar, NodeGeom& gA, NodeGeom& gB)
{
    if (fmax(A.q, B.q) - fmin(A.Q, B.Q) > d) return 1;
    const double c[3] = {A.h[1] * B.h[2] - A.h[2] * B.h[1], A.h[2] * B.h[0] - A.h[0] * B.h[2],
                         A.h[0] * B.h[1] - A.h[1] * B.h[0]};
    const double sD = sqrt(c[0] * c[0] + c[1] * c[1] + c[2] * c[2]);
    const double sA = sD > 0.0 ? d * rcp_fast(A.q * sD) : 2.0;
    const double sB = sD > 0.0 ? d * rcp_fast(B.q * sD) : 2.0;
    coplanar = sA >= 1.0 || sB >= 1.0;
    if (coplanar) return 0;
    gA.sa = sA;
    gB.sa = sB;
    gA.ca = sqrt((1.0 - sA) * (1.0 + sA));
    gB.ca = sqrt((1.0 - sB) * (1.0 + sB));
    coplanar = A.q * gA.ca + B.q * gB.ca <= d;
    if (coplanar) return 0;
    const double isD = rcp_fast(sD);
    const double nn[3] = {c[0] * isD, c[1] * isD, c[2] * isD};
    double x = nn[0] * A.P[0] + nn[1] * A.P[1] + nn[2] * A.P[2];
    double y = nn[0] * A.Qv[0] + nn[1] * A.Qv[1] + nn[2] * A.Qv[2];
    double k = rcp_fast(sqrt(x * x + y * y));
    gA.cf = x * k;
    gA.sf = y * k;
    x = nn[0] * B.P[0] + nn[1] * B.P[1] + nn[2] * B.P[2];
    y = nn[0] * B.Qv[0] + nn[1] * B.Qv[1] + nn[2] * B.Qv[2];
    k = rcp_fast(sqrt(x * x + y * y));
    gB.cf = x * k;
    gB.sf = y * k;
    return 0;
}

// orbit-path filter at node sg (+1 / -1): true iff the radial ranges of A and B over their node
// windows are more than d apart (|r_A - r_B| >= ||r_A| - |r_B||)
template <typename R>
__device__ __forceinline__ bool node_closed(const R& A, const R& B, double d,
                                            const NodeGeom& gA, const NodeGeom& gB, double sg)
{
    double rAl, rAh, rBl, rBh;
    radius_range(A, gA, sg, rAl, rAh);
    radius_range(B, gB, sg, rBl, rBh);
    return fmax(rAl, rBl) - fmin(rAh, rBh) > d;
}

// warp-aggregated counter increment (one atomic per group of converged lanes)
__device__ __forceinline__ void count1(unsigned long long* cnt)
{
    cg::coalesced_group g = cg::coalesced_threads();
    if (g.thread_rank() == 0) atomicAdd(cnt, (unsigned long long)g.size());
}


}  // namespace filt
}  // namespace cdh
