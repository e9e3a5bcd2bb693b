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
    kEcr = 10, kEsr = 11,            // e cos(rho), e sin(rho), rho = e/2   (real nodes)
    kTab = 12,                       // 4 per symmetric interior pair: e cos(rho c_j),
                                     // e sin(rho c_j), cosh(rho s_j), sinh(rho s_j)
    kNCol = 12 + 28
};

// Contour point count (N_it) per eccentricity class (reading R15)
__host__ __device__ constexpr int class_points(int cls)
{
    return cls == 0 ? 4 : cls == 1 ? 6 : cls == 2 ? 8 : cls == 3 ? 12 : 16;
}
__host__ __device__ inline int ecc_class(double e)
{
    return e <= 0.01 ? 0 : e <= 0.1 ? 1 : e <= 0.3 ? 2 : e <= 0.6 ? 3 : 4;
}

struct Orbits {
    const double* rec;   // kNCol x n
    const uint8_t* cls;  // eccentricity class per object
    int64_t n;
    __device__ __forceinline__ double at(int c, int64_t r) const { return __ldg(rec + c * n + r); }
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

template <int N>
__device__ __forceinline__ void contour_core(double M, double e, const Orbits& O, int64_t r,
                                             double& E, double& sE, double& cE)
{
    const double rho = 0.5 * e;
    const bool lower = M < kPi;
    const double dc = lower ? rho : -rho;
    const double c = M + dc;
    double sc, cc;
    sincos(c, &sc, &cc);
    const double ecr = O.at(kEcr, r), esr = O.at(kEsr, r);
    // real nodes th = 0 (z = c + rho) and th = pi (z = c - rho)
    const double f0 = (dc + rho) - (sc * ecr + cc * esr);
    const double fp = (dc - rho) - (sc * ecr - cc * esr);
    double delta;
    if (f0 == 0.0) {
        delta = rho;
    } else if (fp == 0.0) {
        delta = -rho;
    } else {
        double num = 1.0 / f0 + 1.0 / fp;   // e^{2i*0}=1, e^{2i*pi}=1
        double den = 1.0 / f0 - 1.0 / fp;   // e^{i*0}=1,  e^{i*pi}=-1
#pragma unroll
        for (int j = 1; j <= (N - 2) / 2; ++j) {
            constexpr int cl = N == 4 ? 0 : N == 6 ? 1 : N == 8 ? 2 : N == 12 ? 3 : 4;
            const double ct = kNodes[cl][j - 1][0], st = kNodes[cl][j - 1][1];
            const double c2t = kNodes[cl][j - 1][2], s2t = kNodes[cl][j - 1][3];
            const double ec = O.at(kTab + 4 * (j - 1) + 0, r);
            const double es = O.at(kTab + 4 * (j - 1) + 1, r);
            const double ch = O.at(kTab + 4 * (j - 1) + 2, r);
            const double sh = O.at(kTab + 4 * (j - 1) + 3, r);
            // point j (cos th = +ct) and its mirror N-1-j (cos th = -ct, same sin th)
            const double esin_a = sc * ec + cc * es, ecos_a = cc * ec - sc * es;
            const double esin_b = sc * ec - cc * es, ecos_b = cc * ec + sc * es;
            const double rea = fma(rho, ct, dc) - esin_a * ch;
            const double ima = fma(rho, st, -ecos_a * sh);
            const double reb = fma(-rho, ct, dc) - esin_b * ch;
            const double imb = fma(rho, st, -ecos_b * sh);
            const double ia = 2.0 / fma(rea, rea, ima * ima);
            const double ib = 2.0 / fma(reb, reb, imb * imb);
            // th_b = pi - th: cos th_b = -ct, sin th_b = st, cos 2th_b = c2t, sin 2th_b = -s2t
            num += ia * fma(c2t, rea, s2t * ima) + ib * fma(c2t, reb, -s2t * imb);
            den += ia * fma(ct, rea, st * ima) + ib * fma(-ct, reb, st * imb);
        }
        delta = rho * (num / den);
    }
    E = c + delta;
    double sd, cd;
    sincos_small(delta, sd, cd);
    sE = fma(sc, cd, cc * sd);
    cE = fma(cc, cd, -sc * sd);
}

__device__ __forceinline__ void kepler_solve(double M, double e, int cls, const Orbits& O,
                                             int64_t r, double& E, double& sE, double& cE)
{
    switch (cls) {
    case 0: contour_core<4>(M, e, O, r, E, sE, cE); break;
    case 1: contour_core<6>(M, e, O, r, E, sE, cE); break;
    case 2: contour_core<8>(M, e, O, r, E, sE, cE); break;
    case 3: contour_core<12>(M, e, O, r, E, sE, cE); break;
    default: {
        contour_core<16>(M, e, O, r, E, sE, cE);
        // e > 0.6: Newton polish of the contour estimate (R15)
        for (int it = 0; it < 8; ++it) {
            const double dE = (E - e * sE - M) / (1.0 - e * cE);
            E -= dE;
            sincos(E, &sE, &cE);
            if (fabs(dE) <= 1e-15 * fmax(1.0, fabs(E))) break;
        }
    }
    }
}

// Position (and velocity) of object r at time t.
//   r = (cos E - e) aP + sin E bQ;     v = n/(1 - e cos E) (-sin E aP + cos E bQ)
template <bool kVel>
__device__ __forceinline__ void state(const Orbits& O, int64_t r, double t, double p[3], double v[3])
{
    const double e = O.at(kE, r);
    const double M = mean_anomaly(O.at(kM0, r), O.at(kNm, r), t);
    double E, sE, cE;
    kepler_solve(M, e, O.cls[r], O, r, E, sE, cE);
    const double x = cE - e;
    const double ap[3] = {O.at(kAPx, r), O.at(kAPy, r), O.at(kAPz, r)};
    const double bq[3] = {O.at(kBQx, r), O.at(kBQy, r), O.at(kBQz, r)};
#pragma unroll
    for (int c = 0; c < 3; ++c) p[c] = fma(x, ap[c], sE * bq[c]);
    if (kVel) {
        const double k = O.at(kNm, r) / fma(-e, cE, 1.0);
#pragma unroll
        for (int c = 0; c < 3; ++c) v[c] = k * fma(-sE, ap[c], cE * bq[c]);
    }
}

// ---------------------------------------------------------------------------------------
// grid cells and keys ("calculates the grid cell based on the Cartesian coordinates")
// ---------------------------------------------------------------------------------------
constexpr int64_t kKeyBias = int64_t(1) << 20;
constexpr int64_t kCellMax = kKeyBias - 2;   // valid cells in [-kCellMax, kCellMax]
constexpr uint64_t kEmpty = ~uint64_t(0);    // the maximum 64-bit value marks empty
constexpr uint32_t kNil = 0xffffffffu;

__device__ __forceinline__ uint64_t pack_key(int64_t cx, int64_t cy, int64_t cz)
{
    return uint64_t(cx + kKeyBias) | (uint64_t(cy + kKeyBias) << 21) | (uint64_t(cz + kKeyBias) << 42);
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
    double inv_cell;     // 1 / cell edge
    double gc2;          // g_c^2 (candidate gate)
};

__device__ __forceinline__ bool cell_of(const GridGeom& g, const double p[3], int64_t c[3])
{
    c[0] = (int64_t)floor((p[0] - g.ox) * g.inv_cell);
    c[1] = (int64_t)floor((p[1] - g.oy) * g.inv_cell);
    c[2] = (int64_t)floor((p[2] - g.oz) * g.inv_cell);
    return c[0] >= -kCellMax && c[0] <= kCellMax && c[1] >= -kCellMax && c[1] <= kCellMax &&
           c[2] >= -kCellMax && c[2] <= kCellMax;
}

// Grid entry (Fig. 6: id, coordinates, next); the id is the entry index.
struct __align__(32) Entry {
    double x, y, z;
    uint32_t next;
    uint32_t pad;
};

// Hash-map slot: 64-bit cell key + head of the cell's entry list.
struct __align__(16) Slot {
    unsigned long long key;
    uint32_t head;
    uint32_t pad;
};

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
    int pad;
};

}  // namespace cdk
