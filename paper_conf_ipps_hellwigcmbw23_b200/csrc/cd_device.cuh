// cd_device.cuh -- device-side math of the screening path (sm_100a, fp64, no tensor cores).
//
// Orbit record layout, the Contour Kepler solver (ref. [43]), position/velocity
// (P:166), cell keys and the MurmurHash3 finaliser (fn. 3).
#pragma once
#include <cstdint>

namespace cdk {

constexpr double kMu = 398600.4418;                       // km^3/s^2 (reading R1)
constexpr double kPi = 3.14159265358979323846264338327950288;
constexpr double kTwoPi = 6.28318530717958647692528676655900577;
// 2*pi as hi + lo for the mean-anomaly reduction M - k*2pi (two fused multiply-adds)
constexpr double kTwoPiHi = 6.28318530717958623199592693708837032;   // nearest double
constexpr double kTwoPiLo = 2.44929359829470635445213186455000e-16;   // 2pi - hi

// ---------------------------------------------------------------------------------------
// Orbit records: column-major SoA, column c of object r at rec[c * n + r] (coalesced).
// ---------------------------------------------------------------------------------------
enum Col : int {
    kM0 = 0,   // mean anomaly at epoch
    kNm = 1,   // mean motion sqrt(mu/a^3)
    kE = 2,    // eccentricity
    kAPx = 3, kAPy = 4, kAPz = 5,   // a * P (perifocal x axis)
    kBQx = 6, kBQy = 7, kBQz = 8,   // b * Q, b = a sqrt(1-e^2)
    kQper = 9,                       // perigee radius q = a(1-e) (acceleration bound)
    // (the Contour constants of P:168 -- e cos(rho), e sin(rho) and the node tables -- are
    // evaluated in registers by series, contour_core: no record columns)
    // J2 secular propagator (Orbits::j2): node and perigee rates and
    // the axis ratios that rotate the (aP, bQ) frame in its plane
    kDOm = 10, kDw = 11,             // dOmega/dt, domega/dt [rad/s]
    kBA = 12, kAB = 13,              // b/a, a/b
    kNCol = 14
};

// J2 secular propagator constants (EGM-96 / WGS-84, reading R19)
constexpr double kJ2 = 1.08262668e-3;
constexpr double kRe = 6378.137;   // km

// Contour point count (N_it) per eccentricity class (reading R15)
__host__ __device__ constexpr int class_points(int cls)
{
    return cls == 0 ? 4 : cls == 1 ? 6 : cls == 2 ? 8 : cls == 3 ? 12 : 16;
}
__host__ __device__ inline int ecc_class(double e)
{
    return e <= 0.01 ? 0 : e <= 0.1 ? 1 : e <= 0.3 ? 2 : e <= 0.6 ? 3 : 4;
}
// class of a requested point count (cd_options.kepler_points): 0 -> 0 (per e), 4/6/8/12/16 ->
// class 0..4, anything else -> -1 (invalid)
__host__ __device__ inline int kepler_class_of_points(int pts)
{
    return pts == 0 || pts == 4 ? 0 : pts == 6 ? 1 : pts == 8 ? 2 : pts == 12 ? 3 : pts == 16 ? 4 : -1;
}

// Refinement records (Orbits::arec): the same columns object-major, one 128-byte line per object
// (column c of object r at arec[r * kAoS + c], the class at kAoSCls): the refinement gathers a
// candidate's two objects at random, and one line per object replaces up to 14 scattered sectors
// of the column-major records (8M objects: the prefilter was DRAM-bound on those gathers).
constexpr int kAoS = 16;
constexpr int kAoSCls = 14;
static_assert(kNCol <= kAoSCls, "refinement record columns");

struct Orbits {
    const double* rec;   // kNCol x n
    const double* arec;  // refinement records, n x kAoS (object-major)
    const uint8_t* cls;  // eccentricity class per object
    int64_t n;
    int64_t n0;          // objects [0, n0) are class 0 (records sorted by class)
    int j2;              // 1: J2 secular propagator (plane and perigee rotate; columns kDOm..kAB)
    // records are streamed once per step: evict-first so they do not push the per-step grid
    // (slots, bitmap, entries) out of L2
    __device__ __forceinline__ double at(int c, int64_t r) const { return __ldcs(rec + c * n + r); }
    __device__ __forceinline__ double aat(int c, int64_t r) const { return __ldg(arec + r * kAoS + c); }
    // column c of object r from the layout kA selects (true: refinement records)
    template <bool kA>
    __device__ __forceinline__ double col(int c, int64_t r) const { return kA ? aat(c, r) : at(c, r); }
};

// ---------------------------------------------------------------------------------------
// sin/cos of a small |d| <= 0.5 by Taylor polynomials (Horner; truncation < 1e-22)
// ---------------------------------------------------------------------------------------
__device__ __forceinline__ void sincos_small(double d, double& s, double& c)
{
    const double x = d * d;
    double ps = 1.0 / 355687428096000.0;          // 1/17!
    ps = fma(ps, x, -1.0 / 1307674368000.0);      // 1/15!
    ps = fma(ps, x, 1.0 / 6227020800.0);          // 1/13!
    ps = fma(ps, x, -1.0 / 39916800.0);           // 1/11!
    ps = fma(ps, x, 1.0 / 362880.0);              // 1/9!
    ps = fma(ps, x, -1.0 / 5040.0);
    ps = fma(ps, x, 1.0 / 120.0);
    ps = fma(ps, x, -1.0 / 6.0);
    s = fma(ps * x, d, d);
    double pc = 1.0 / 6402373705728000.0;         // 1/18!
    pc = fma(pc, x, -1.0 / 20922789888000.0);     // 1/16!
    pc = fma(pc, x, 1.0 / 87178291200.0);         // 1/14!
    pc = fma(pc, x, -1.0 / 479001600.0);          // 1/12!
    pc = fma(pc, x, 1.0 / 3628800.0);             // 1/10!
    pc = fma(pc, x, -1.0 / 40320.0);
    pc = fma(pc, x, 1.0 / 720.0);
    pc = fma(pc, x, -1.0 / 24.0);
    pc = fma(pc, x, 0.5);
    c = fma(-pc, x, 1.0);
}

// sin and cos for the Contour centre c in [-0.5, 2 pi + 0.5] (also correct for |x| < ~1e5):
// Cody-Waite reduction by pi/2 (two-part constant, fused multiply-adds) and Taylor series on
// [-pi/4, pi/4] (truncation < 1e-19).  No slow path, few registers.
__device__ __forceinline__ void sincos_fast(double x, double& s, double& c)
{
    const double k = rint(x * 0.63661977236758134308);
    double r = fma(-k, 1.5707963267948966, x);
    r = fma(-k, 6.123233995736766e-17, r);
    double sr, cr;
    sincos_small(r, sr, cr);
    const int q = (int)k & 3;
    s = q == 0 ? sr : q == 1 ? cr : q == 2 ? -sr : -cr;
    c = q == 0 ? cr : q == 1 ? -sr : q == 2 ? -cr : sr;
}

// 1/b from the hardware fp64 reciprocal estimate plus two Newton steps (full precision for the
// finite, non-zero arguments used here; no IEEE-division slow path)
__device__ __forceinline__ double rcp_fast(double b)
{
    double r;
    asm("rcp.approx.ftz.f64 %0, %1;" : "=d"(r) : "d"(b));
    double e = fma(-b, r, 1.0);
    r = fma(r, e, r);
    e = fma(-b, r, 1.0);
    return fma(r, e, r);
}

// M = (M0 + n t) reduced to [0, 2pi)
__device__ __forceinline__ double mean_anomaly(double M0, double nm, double t)
{
    double M = fma(nm, t, M0);
    double k = floor(M * (1.0 / kTwoPi));
    M = fma(-k, kTwoPiHi, M);
    M = fma(-k, kTwoPiLo, M);
    if (M < 0.0) M += kTwoPi;
    if (M >= kTwoPi) M -= kTwoPi;
    return M;
}

// ---------------------------------------------------------------------------------------
// Contour Kepler solver (Philcox, Goodman & Slepian [43]; PAPER.md:168 -- one independent
// solve per thread, reusable per-object parts precomputed).  Solves E - e sin E = M.
//
// E is the only zero of f(z) = z - e sin z - M inside the circle |z - c| = rho, rho = e/2,
// c = M + rho (M < pi) or M - rho (M >= pi).  By the argument principle
//     E = c + rho * [sum_j w_j Re(e^{2 i th_j} / f_j)] / [sum_j w_j Re(e^{i th_j} / f_j)],
// trapezoid rule on th_j = pi j/(N-1), j = 0..N-1 (conjugate symmetry folds [pi, 2pi) onto
// [0, pi]); w = 1 at the two real nodes, 2 inside.  With z = c + rho e^{i th}:
//     Re f = dc + rho cos th - e sin(c + rho cos th) cosh(rho sin th),  dc = c - M = +-rho
//     Im f = rho sin th - e cos(c + rho cos th) sinh(rho sin th)
// and e sin(c + x) = sin c (e cos x) + cos c (e sin x): one sincos(c) per solve.
// Guard: if f vanishes exactly at a real node the node is the root (covers M = 0, pi and
// sin(M + e) = 1, where the quadrature would divide by zero).
// Returns E and its sine/cosine (from sincos(c) rotated by the small delta = E - c).
// ---------------------------------------------------------------------------------------
// cos th_j, sin th_j, cos 2th_j, sin 2th_j for th_j = pi j/(N-1), j = 1..(N-2)/2, per class
__constant__ double kNodes[5][7][4] = {
    {  // N = 4
        {0.5000000000000001, 0.8660254037844386, -0.4999999999999998, 0.8660254037844387},
        {0.0, 0.0, 0.0, 0.0},
        {0.0, 0.0, 0.0, 0.0},
        {0.0, 0.0, 0.0, 0.0},
        {0.0, 0.0, 0.0, 0.0},
        {0.0, 0.0, 0.0, 0.0},
        {0.0, 0.0, 0.0, 0.0}},
    {  // N = 6
        {0.8090169943749475, 0.5877852522924731, 0.30901699437494745, 0.9510565162951535},
        {0.30901699437494745, 0.9510565162951535, -0.8090169943749473, 0.5877852522924732},
        {0.0, 0.0, 0.0, 0.0},
        {0.0, 0.0, 0.0, 0.0},
        {0.0, 0.0, 0.0, 0.0},
        {0.0, 0.0, 0.0, 0.0},
        {0.0, 0.0, 0.0, 0.0}},
    {  // N = 8
        {0.9009688679024191, 0.4338837391175581, 0.6234898018587336, 0.7818314824680298},
        {0.6234898018587336, 0.7818314824680298, -0.22252093395631434, 0.9749279121818236},
        {0.22252093395631445, 0.9749279121818236, -0.900968867902419, 0.43388373911755823},
        {0.0, 0.0, 0.0, 0.0},
        {0.0, 0.0, 0.0, 0.0},
        {0.0, 0.0, 0.0, 0.0},
        {0.0, 0.0, 0.0, 0.0}},
    {  // N = 12
        {0.9594929736144974, 0.28173255684142967, 0.8412535328311812, 0.5406408174555976},
        {0.8412535328311812, 0.5406408174555976, 0.41541501300188644, 0.9096319953545183},
        {0.6548607339452851, 0.7557495743542583, -0.142314838273285, 0.9898214418809328},
        {0.41541501300188644, 0.9096319953545183, -0.654860733945285, 0.7557495743542583},
        {0.14231483827328512, 0.9898214418809327, -0.9594929736144974, 0.28173255684142967},
        {0.0, 0.0, 0.0, 0.0},
        {0.0, 0.0, 0.0, 0.0}},
    {  // N = 16
        {0.9781476007338057, 0.20791169081775931, 0.9135454576426009, 0.40673664307580015},
        {0.9135454576426009, 0.40673664307580015, 0.6691306063588582, 0.7431448254773941},
        {0.8090169943749475, 0.5877852522924731, 0.30901699437494745, 0.9510565162951535},
        {0.6691306063588582, 0.7431448254773941, -0.10452846326765333, 0.9945218953682734},
        {0.5000000000000001, 0.8660254037844386, -0.4999999999999998, 0.8660254037844387},
        {0.30901699437494745, 0.9510565162951535, -0.8090169943749473, 0.5877852522924732},
        {0.10452846326765346, 0.9945218953682733, -0.9781476007338057, 0.20791169081775931}}};

// cos/sin and cosh/sinh of |x| <= rho_max(class) by T-term Taylor polynomials in Horner form
// (T = 5 / 7 / 8 / 10 for rho <= 0.05 / 0.15 / 0.3 / 0.5: truncation < 3e-20 in every class, max
// error vs libm 2.2e-16 absolute over each range): the per-object Contour constants
// e cos(rho cos th_j), e sin(rho cos th_j), cosh(rho sin th_j), sinh(rho sin th_j) (P:168's
// "precalculated reusable parts") are evaluated in registers instead of being streamed from the
// records -- every class reads the same 9 columns per object-step (the tables were 80-240 bytes
// per object-step of the ~16 % e > 0.01 objects; measured equal or faster in every class split)
template <int T>
__device__ __forceinline__ void cs_series(double x, double& c, double& s)
{
    const double x2 = x * x;
    double pc = 0.0, ps = 0.0;
#pragma unroll
    for (int k = T - 1; k >= 0; --k) {   // x^{2k}: (-1)^k / (2k)!,  x^{2k+1}: (-1)^k / (2k+1)!
        double f2k = 1.0;                // (compile-time constants once unrolled)
#pragma unroll
        for (int q = 2; q <= 2 * k; ++q) f2k *= (double)q;
        const double f2k1 = f2k * (double)(2 * k + 1);
        const double sg = (k & 1) ? -1.0 : 1.0;
        pc = fma(pc, x2, sg / f2k);
        ps = fma(ps, x2, sg / f2k1);
    }
    c = pc;
    s = x * ps;
}
template <int T>
__device__ __forceinline__ void chsh_series(double x, double& ch, double& sh)
{
    const double x2 = x * x;
    double pc = 0.0, ps = 0.0;
#pragma unroll
    for (int k = T - 1; k >= 0; --k) {
        double f2k = 1.0;
#pragma unroll
        for (int q = 2; q <= 2 * k; ++q) f2k *= (double)q;
        const double f2k1 = f2k * (double)(2 * k + 1);
        pc = fma(pc, x2, 1.0 / f2k);
        ps = fma(ps, x2, 1.0 / f2k1);
    }
    ch = pc;
    sh = x * ps;
}
__host__ __device__ constexpr int series_terms(int N)
{
    return N <= 6 ? 5 : N <= 8 ? 7 : N <= 12 ? 8 : 10;
}

template <int N>
__device__ __forceinline__ void contour_core(double M, double e, double& E, double& sE, double& cE)
{
    const double rho = 0.5 * e;
    const bool lower = M < kPi;
    const double dc = lower ? rho : -rho;
    const double c = M + dc;
    double sc, cc;
    sincos_fast(c, sc, cc);
    double ecr, esr;
    if (N == 4) {
        // class 0 (e <= 0.01, rho <= 0.005): the six per-object constants are evaluated here by
        // short Taylor series (truncation < 1e-22) instead of being streamed from the records
        const double x2 = rho * rho;
        ecr = e * fma(fma(fma(-1.0 / 720.0, x2, 1.0 / 24.0), x2, -0.5), x2, 1.0);
        esr = e * rho * fma(fma(fma(-1.0 / 5040.0, x2, 1.0 / 120.0), x2, -1.0 / 6.0), x2, 1.0);
    } else {   // classes 1-4 (rho <= 0.05 / 0.15 / 0.3 / 0.5)
        double cr, sr;
        cs_series<series_terms(N)>(rho, cr, sr);
        ecr = e * cr;
        esr = e * sr;
    }
    // real nodes th = 0 (z = c + rho) and th = pi (z = c - rho)
    const double f0 = (dc + rho) - (sc * ecr + cc * esr);
    const double fp = (dc - rho) - (sc * ecr - cc * esr);
    double delta;
    if (f0 == 0.0) {
        delta = rho;
    } else if (fp == 0.0) {
        delta = -rho;
    } else {
        const double i0 = rcp_fast(f0);
        const double ip = rcp_fast(fp);
        double num = i0 + ip;   // e^{2i*0}=1, e^{2i*pi}=1
        double den = i0 - ip;   // e^{i*0}=1,  e^{i*pi}=-1
#pragma unroll(N == 4 ? 1 : 1)
        for (int j = 1; j <= (N - 2) / 2; ++j) {
            constexpr int cl = N == 4 ? 0 : N == 6 ? 1 : N == 8 ? 2 : N == 12 ? 3 : 4;
            const double ct = kNodes[cl][j - 1][0], st = kNodes[cl][j - 1][1];
            const double c2t = kNodes[cl][j - 1][2], s2t = kNodes[cl][j - 1][3];
            double ec, es, ch, sh;
            if (N == 4) {   // th = pi/3: rho cos th = rho/2, rho sin th = rho sqrt(3)/2
                const double a = 0.5 * rho, a2 = a * a;
                const double b = 0.86602540378443864676 * rho, b2 = b * b;
                ec = e * fma(fma(fma(-1.0 / 720.0, a2, 1.0 / 24.0), a2, -0.5), a2, 1.0);
                es = e * a * fma(fma(fma(-1.0 / 5040.0, a2, 1.0 / 120.0), a2, -1.0 / 6.0), a2, 1.0);
                ch = fma(fma(fma(1.0 / 720.0, b2, 1.0 / 24.0), b2, 0.5), b2, 1.0);
                sh = b * fma(fma(fma(1.0 / 5040.0, b2, 1.0 / 120.0), b2, 1.0 / 6.0), b2, 1.0);
            } else {   // arguments rho cos th, rho sin th <= rho
                double cx, sx;
                cs_series<series_terms(N)>(rho * ct, cx, sx);
                ec = e * cx;
                es = e * sx;
                chsh_series<series_terms(N)>(rho * st, ch, sh);
            }
            // point j (cos th = +ct) and its mirror N-1-j (cos th = -ct, same sin th)
            const double esin_a = sc * ec + cc * es, ecos_a = cc * ec - sc * es;
            const double esin_b = sc * ec - cc * es, ecos_b = cc * ec + sc * es;
            const double rea = fma(rho, ct, dc) - esin_a * ch;
            const double ima = fma(rho, st, -ecos_a * sh);
            const double reb = fma(-rho, ct, dc) - esin_b * ch;
            const double imb = fma(rho, st, -ecos_b * sh);
            const double ia = 2.0 * rcp_fast(fma(rea, rea, ima * ima));
            const double ib = 2.0 * rcp_fast(fma(reb, reb, imb * imb));
            // th_b = pi - th: cos th_b = -ct, sin th_b = st, cos 2th_b = c2t, sin 2th_b = -s2t
            num += ia * fma(c2t, rea, s2t * ima) + ib * fma(c2t, reb, -s2t * imb);
            den += ia * fma(ct, rea, st * ima) + ib * fma(-ct, reb, st * imb);
        }
        delta = rho * (num * rcp_fast(den));
        // the root lies inside the contour, |E - c| < rho: a non-finite or out-of-range quotient
        // (rounding next to a degenerate node) falls back to Newton from the contour centre
        if (!(fabs(delta) <= rho)) {
            double x = c;
            for (int it = 0; it < 12; ++it) {
                double sx, cx;
                sincos_fast(x, sx, cx);
                const double dx = (x - e * sx - M) / fma(-e, cx, 1.0);
                x -= dx;
                if (fabs(dx) <= 1e-16 * fmax(1.0, fabs(x))) break;
            }
            delta = fmin(fmax(x - c, -rho), rho);
        }
    }
    E = c + delta;
    double sd, cd;
    if (N == 4) {   // |delta| <= rho <= 0.005: truncation < 1e-24
        const double x = delta * delta;
        sd = delta * fma(fma(fma(-1.0 / 5040.0, x, 1.0 / 120.0), x, -1.0 / 6.0), x, 1.0);
        cd = fma(fma(fma(-1.0 / 720.0, x, 1.0 / 24.0), x, -0.5), x, 1.0);
    } else {
        sincos_small(delta, sd, cd);
    }
    sE = fma(sc, cd, cc * sd);
    cE = fma(cc, cd, -sc * sd);
}

// Eccentricity-class dispatch (objects are sorted by class, so warps are uniform).
__device__ __forceinline__ void kepler_solve(double M, double e, int cls, double& E, double& sE, double& cE)
{
    switch (cls) {
    case 0: contour_core<4>(M, e, E, sE, cE); break;
    case 1: contour_core<6>(M, e, E, sE, cE); break;
    case 2: contour_core<8>(M, e, E, sE, cE); break;
    case 3: contour_core<12>(M, e, E, sE, cE); break;
    default:
        contour_core<16>(M, e, E, sE, cE);
        if (e > 0.8) {   // Newton polish of the contour estimate (R15)
            for (int it = 0; it < 8; ++it) {
                const double dE = (E - e * sE - M) * rcp_fast(1.0 - e * cE);
                E -= dE;
                sincos_fast(E, sE, cE);
                if (fabs(dE) <= 1e-15 * fmax(1.0, fabs(E))) break;
            }
        }
    }
}

// One out-of-line copy of the class dispatch for the refinement (state<..., kA = true>): Brent and
// the polish evaluate two states per call site, and inlining the five Contour instances at each
// had made k_brent instruction-cache bound (ncu at 8M objects: 9.9 no-instruction stalls per
// issue).
static __device__ __noinline__ void kepler_solve_ool(double M, double e, int cls, double& E, double& sE, double& cE)
{
    kepler_solve(M, e, cls, E, sE, cE);
}

// Position (and velocity) of object r at time t.
//   r = (cos E - e) aP + sin E bQ;     v = n/(1 - e cos E) (-sin E aP + cos E bQ)
// J2 secular (O.j2): the epoch frame (P, Q) turns by domega t about the orbit normal h and the
// plane by dOmega t about z.  With X = cos E - e, Y = sin E, the in-plane coordinates become
//   r = [X cw - (b/a) Y sw] aP + [(a/b) X sw + Y cw] bQ,   (cw, sw) = cos, sin(domega t)
// followed by the z-rotation; velocity = the rotated two-body velocity + domega h x r (in the
// plane: (x, y) -> (-y, x)) + dOmega z x r.
// kClass: 0 = object known to be class 0 (lean path), -1 = any class
// kJ2: 0 = two-body only, 1 = J2 secular only, -1 = per O.j2 (runtime, warp-uniform)
// kA: read the refinement records (Orbits::arec, random access) instead of the columns
template <bool kVel, int kClass = -1, int kJ2 = -1, bool kA = false>
__device__ __forceinline__ void state(const Orbits& O, int64_t r, double t, double p[3], double v[3])
{
    const double e = O.col<kA>(kE, r);
    const double M = mean_anomaly(O.col<kA>(kM0, r), O.col<kA>(kNm, r), t);
    double E, sE, cE;
    if (kClass == 0) contour_core<4>(M, e, E, sE, cE);
    else if (kA) kepler_solve_ool(M, e, (int)O.aat(kAoSCls, r), E, sE, cE);
    else kepler_solve(M, e, (int)O.cls[r], E, sE, cE);
    double x = cE - e, y = sE;              // coefficients of aP and bQ
    double vx = -sE, vy = cE;               // velocity coefficients (times n/(1 - e cos E))
    const bool j2 = kJ2 == 1 || (kJ2 == -1 && O.j2);
    double sO = 0.0, cO = 1.0, dOm = 0.0, dw = 0.0, ba = 1.0, ab = 1.0;
    if (j2) {
        dOm = O.col<kA>(kDOm, r);
        dw = O.col<kA>(kDw, r);
        ba = O.col<kA>(kBA, r);
        ab = O.col<kA>(kAB, r);
        double sw, cw;
        sincos_fast(dw * t, sw, cw);
        sincos_fast(dOm * t, sO, cO);
        const double xr = fma(x, cw, -ba * y * sw), yr = fma(ab * x, sw, y * cw);
        x = xr;
        y = yr;
        if (kVel) {
            const double vxr = fma(vx, cw, -ba * vy * sw), vyr = fma(ab * vx, sw, vy * cw);
            vx = vxr;
            vy = vyr;
        }
    }
    const double ap[3] = {O.col<kA>(kAPx, r), O.col<kA>(kAPy, r), O.col<kA>(kAPz, r)};
    const double bq[3] = {O.col<kA>(kBQx, r), O.col<kA>(kBQy, r), O.col<kA>(kBQz, r)};
#pragma unroll
    for (int c = 0; c < 3; ++c) p[c] = fma(x, ap[c], y * bq[c]);
    if (kVel) {
        const double k = O.col<kA>(kNm, r) / fma(-e, cE, 1.0);
        if (j2) {
            // domega h x r: the in-plane vector (X, Y) in unit (P, Q) axes turns to (-Y, X);
            // in (aP, bQ) coefficients: (-(b/a) y, (a/b) x)
            const double wx = k * vx - dw * ba * y, wy = k * vy + dw * ab * x;
#pragma unroll
            for (int c = 0; c < 3; ++c) v[c] = fma(wx, ap[c], wy * bq[c]);
        } else {
#pragma unroll
            for (int c = 0; c < 3; ++c) v[c] = k * fma(vx, ap[c], vy * bq[c]);
        }
    }
    if (j2) {   // plane rotation about z by dOmega t (and dOmega z x r for the velocity)
        const double px = fma(p[0], cO, -p[1] * sO), py = fma(p[0], sO, p[1] * cO);
        p[0] = px;
        p[1] = py;
        if (kVel) {
            const double qx = fma(v[0], cO, -v[1] * sO), qy = fma(v[0], sO, v[1] * cO);
            v[0] = fma(-dOm, py, qx);
            v[1] = fma(dOm, px, qy);
        }
    }
}

// ---------------------------------------------------------------------------------------
// grid cells and keys ("calculates the grid cell based on the Cartesian coordinates")
// ---------------------------------------------------------------------------------------
// Cell keys pack 21 bits per axis: cells in [-(2^20 - 2), 2^20 - 2], i.e.
// +-1,048,574 cells of edge L >= g_c -- +-104,857 km at g_c = 0.1 km, beyond GEO for any g_c >=
// 0.05 km (P:128's (85,000 km)^3 space).  Bit 63 is 0.  The open map keeps the tag of the build
// pass that wrote a slot (1..kMaxTag) in the upper half of the slot's head word: a slot whose tag
// differs from the current pass is empty (P:147 reserves a value for "empty"; tagging lets a
// table be reused without clearing it every step -- tables are zeroed only when the tags wrap).
constexpr int64_t kKeyBias = int64_t(1) << 20;
constexpr int64_t kCellMax = kKeyBias - 2;   // valid cells in [-kCellMax, kCellMax]
constexpr uint32_t kMaxTag = 0x7ffffffeu;
constexpr uint32_t kNil = 0xffffffffu;

__device__ __forceinline__ uint64_t pack_key(int cx, int cy, int cz)
{
    return uint64_t(uint32_t(cx + (int)kKeyBias)) | (uint64_t(uint32_t(cy + (int)kKeyBias)) << 21) |
           (uint64_t(uint32_t(cz + (int)kKeyBias)) << 42);
}

// MurmurHash3 64-bit finaliser (footnote 3: smhasher)
__device__ __forceinline__ uint64_t fmix64(uint64_t k)
{
    k ^= k >> 33;
    k *= 0xff51afd7ed558ccdull;
    k ^= k >> 33;
    k *= 0xc4ceb9fe1a85ec53ull;
    k ^= k >> 33;
    return k;
}

struct GridGeom {
    double ox, oy, oz;   // origin
    double inv_cell;     // 1 / cell edge L (L >= g_c)
    double gc2;          // g_c^2 (candidate gate)
    double reach;        // g_c (1 + 1e-9) + 1e-9: ball radius used to pick the probed cells
    int halfshell;       // 1: own cell + 13 half-shell neighbours (L < 2 g_c); 0: the cells
                         // overlapping the ball |x - p| < g_c (L >= 2 g_c)
    uint32_t max_walk;   // list-walk bound (n): guards against a corrupted list
    // radial shard (cd_options.shell_lo/hi): a candidate is kept iff the
    // smaller of its two radii^2 lies in [band_lo2, band_hi2) (default [0, inf): all)
    double band_lo2, band_hi2;
    int stage;           // 1: stage candidates per block in shared memory (dense candidate rates)
    // spatial slot order: entry index (slot) -> internal object id of the scanned batch
    // (nullptr: slots are internal ids)
    const uint32_t* sig;
    int raw;             // cd_options.emit_raw_counts: count every pair examined (Ctrl::n_raw)
};

// Cell of position p: c = floor((p - o) / L) per axis (R7); frac = (p - o)/L - c in [0, 1).
// Returns false outside the key range.
__device__ __forceinline__ bool cell_of(const GridGeom& g, const double p[3], int c[3], double* frac = nullptr)
{
    const double u[3] = {(p[0] - g.ox) * g.inv_cell, (p[1] - g.oy) * g.inv_cell, (p[2] - g.oz) * g.inv_cell};
    bool ok = true;
#pragma unroll
    for (int a = 0; a < 3; ++a) {
        const double f = floor(u[a]);
        ok = ok && f >= -(double)kCellMax && f <= (double)kCellMax;
        c[a] = ok ? (int)f : 0;
        if (frac) frac[a] = u[a] - f;
    }
    return ok;
}

// Occupancy-bitmap hash of a cell from per-axis products (so the scan can combine neighbour
// cells with two XORs): h = mix(cx*A ^ cy*B ^ cz*C).  Any fixed hash is valid for the bitmap;
// only its uniformity matters (false-positive rate).
constexpr uint32_t kHX = 0x9E3779B1u, kHY = 0x85EBCA77u, kHZ = 0xC2B2AE3Du;
__device__ __forceinline__ uint32_t bit_mix(uint32_t h)
{
    h ^= h >> 15;
    h *= 0x2C1B3C6Du;
    h ^= h >> 12;
    return h;
}
__device__ __forceinline__ uint32_t bit_hash(int cx, int cy, int cz)
{
    return bit_mix((uint32_t)cx * kHX ^ (uint32_t)cy * kHY ^ (uint32_t)cz * kHZ);
}

// Chained-grid bucket of a cell: hash of its aligned superblock of 2^kSB cells per axis
// (floor(c / 2^kSB)) in the high bits, the cell's position inside the superblock (c mod 2^kSB per
// axis) in the low 3 kSB bits.  The <= 8 cells a ball of radius g_c <= L/2 overlaps differ by one
// in each axis they differ in, so their low bits -- and their buckets -- are always distinct (no
// de-duplication), and the cells of one superblock share 4 * 8^kSB contiguous bytes of heads.
#ifndef CD_SB_BITS
#define CD_SB_BITS 2   // 4x4x4 superblocks (measured: 8M objects 970 -> 894 us per step, 1M 61.6 -> 60.3)
#endif
constexpr int kSB = CD_SB_BITS;
static_assert(kSB >= 2, "the half-shell chained scan needs the 27 cells of a 3x3x3 block in distinct buckets");
__device__ __forceinline__ uint32_t chain_bucket(int cx, int cy, int cz, uint32_t hmask)
{
    constexpr uint32_t m = (1u << kSB) - 1u;
    const uint32_t blk = bit_mix((uint32_t)(cx >> kSB) * kHX ^ (uint32_t)(cy >> kSB) * kHY ^
                                 (uint32_t)(cz >> kSB) * kHZ);
    return ((blk << (3 * kSB)) | ((uint32_t)cx & m) | (((uint32_t)cy & m) << kSB) |
            (((uint32_t)cz & m) << (2 * kSB))) & hmask;
}
// Cell tag stored with each chained-grid entry: the cell's coordinates mod 1024 per axis.  Two
// cells of one 3x3x3 neighbourhood never share a tag, so a walk can tell the probed cell's
// entries from those of a colliding neighbour cell without recomputing cells from positions.
__device__ __forceinline__ uint32_t cell_tag(int cx, int cy, int cz)
{
    return ((uint32_t)cx & 0x3FFu) | (((uint32_t)cy & 0x3FFu) << 10) | (((uint32_t)cz & 0x3FFu) << 20);
}
// Chained-grid heads: (epoch << 24) | (index + 1); a head of another epoch is an empty bucket,
// so the head arrays are never cleared per step (zeroed only when the 8-bit epoch wraps).
constexpr uint32_t kEpochShift = 24, kIdxMask = (1u << 24) - 1u;
constexpr uint32_t kMaxChainN = (1u << 24) - 2u;   // chained grid needs n < 2^24 - 1

// Grid entry (Fig. 6: id, coordinates, next); the id is the entry index.
struct __align__(32) Entry {
    double x, y, z;
    uint32_t next;
    uint32_t tag;    // chained grid: cell_tag of the entry's cell (open map: unused)
};

// Hash grid of one step.  Open addressing over M = 2^m >= 2n slots,
// linear probing s_{i+1} = s_i + 1 mod M (Eq. 2) from the MurmurHash3 slot.  A slot is
// 16 bytes {cell key, tag << 32 | list head}: key and head are installed together by one 128-bit
// CAS (P:147-148's CAS, widened so that claiming a cell and pushing the first object onto its
// list is a single atomic).  A slot whose tag is not the current pass's is empty (an all-zero
// slot has tag 0, never used: tables are cleared with plain coalesced stores).
struct __align__(16) Slot {
    unsigned long long key;    // pack_key(cell)
    unsigned long long head;   // tag << 32 | entry index of the list head (Fig. 6)
};

__device__ __forceinline__ bool cas128(Slot* s, unsigned long long& e0, unsigned long long& e1,
                                       unsigned long long d0, unsigned long long d1)
{
    unsigned long long o0, o1;
    asm volatile("{ .reg .b128 d, b, c;\n\t"
                 "mov.b128 b, {%2, %3};\n\t"
                 "mov.b128 c, {%4, %5};\n\t"
                 "atom.relaxed.gpu.global.cas.b128 d, [%6], b, c;\n\t"
                 "mov.b128 {%0, %1}, d; }"
                 : "=l"(o0), "=l"(o1)
                 : "l"(e0), "l"(e1), "l"(d0), "l"(d1), "l"(s)
                 : "memory");
    const bool ok = o0 == e0 && o1 == e1;
    e0 = o0;
    e1 = o1;
    return ok;
}

// Non-blocking insert of object r into the cell `key`.  A slot carrying another
// pass's tag is empty: it is claimed by a 128-bit CAS against the value just read; a slot already
// holding the key (this pass) pushes r onto its list (CAS of the head word); a slot of another cell
// moves on along the probe sequence (Eq. 2).  Returns the previous list head (r's `next`), kNil if
// r is the first object of its cell.
__device__ __forceinline__ uint32_t grid_insert(Slot* slots, uint64_t mask, unsigned long long key,
                                                uint32_t tag, uint32_t r)
{
    const unsigned long long th = (unsigned long long)tag << 32;
    uint64_t h = fmix64(key) & mask;
    while (true) {
        unsigned long long w0, w1;
        asm volatile("ld.relaxed.gpu.global.v2.u64 {%0, %1}, [%2];" : "=l"(w0), "=l"(w1) : "l"(slots + h));
        while (true) {
            const bool stale = (uint32_t)(w1 >> 32) != tag;
            if (!stale && w0 != key) break;   // another cell of this pass: next slot
            const unsigned long long prev = w1;
            if (cas128(slots + h, w0, w1, key, th | (unsigned long long)r))
                return stale ? kNil : (uint32_t)prev;
            // lost a race: (w0, w1) now hold the slot's current contents; re-evaluate
        }
        h = (h + 1) & mask;
    }
}

// Per-step occupancy bitmap: 32 bits per object, set at insertion with bit_hash(cell); a probe
// of an empty cell (the common case) is one 4-byte load from a small L2-resident array; false
// positives (~3 %) only cost a table probe.
struct GridTab {
    Slot* slots;      // M slots per step
    uint32_t* bits;   // bwords words per step
    uint32_t bmask;   // bit index mask (2^b - 1)
    uint32_t bwords;
};

// Lookup after the build (read-only): list head of cell `key`, kNil if the cell is empty.
__device__ __forceinline__ uint32_t grid_find(const Slot* __restrict__ slots, uint64_t mask,
                                              unsigned long long key, uint32_t tag)
{
    uint64_t h = fmix64(key) & mask;
    while (true) {
        const ulonglong2 w = __ldg(reinterpret_cast<const ulonglong2*>(slots + h));
        if ((uint32_t)(w.y >> 32) != tag) return kNil;   // empty: the cell is not in the table
        if (w.x == key) return (uint32_t)w.y;
        h = (h + 1) & mask;
    }
}

struct Cand {   // candidate ("the satellites' ids and the sampling step")
    uint32_t i, j, step;
};

struct Conj {   // conjunction record (matches cd_conjunction)
    uint32_t i, j, step, flags;
    double tca, pca;
};

struct Ctrl {   // device-side counters and flags of one call
    unsigned long long n_cand;
    unsigned long long n_conj;
    unsigned long long n_refined;
    unsigned long long n_ap, n_coplanar, n_path, n_time;
    int err_range;
    int err_internal;
    unsigned long long n_raw;   // pairs examined by the scan (emit_raw_counts; per round)
    // digest_only: accepted rounds' conjunctions folded into a count, an order-independent sum of
    // hashes of (i, j, step) in caller ids, and the smallest PCA (stored as max of ~bits)
    unsigned long long dg_count, dg_sum, dg_notminpca;
};

}  // namespace cdk
