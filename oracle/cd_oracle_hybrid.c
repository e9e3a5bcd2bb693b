/*
 * cd_oracle_hybrid.c -- TEST INFRASTRUCTURE ONLY.  Oracle level O4: the hybrid variant.
 *
 * PAPER.md:66 / P:72 / P:95 / P:183: the grid (with a larger step and cell) is a coarse pre-filter;
 * its pairs pass "classical orbital filters" (apogee/perigee filter [13], orbit path filter
 * [13], time filter [15]); "For the hybrid variant, we distinguish between coplanar and
 * non-coplanar pairs.  The orbital filters determine the interval to search in for non-coplanar
 * pairs.  For the coplanar ones, the procedure is the same as for the grid-based variant."
 * The filters are only named in the paper; reading R17 fixes these conservative
 * formulas (plain geometry, each step below is one formula):
 *
 *   AP        exclude iff max(q_A, q_B) - min(Q_A, Q_B) > d         (q = a(1-e), Q = a(1+e))
 *   plane     |r_A - r_B| >= |r_A . h_B| = |r_A| |sin u_A| sin D   (u_A: angle of r_A from the
 *             mutual node line n = h_A x h_B / sin D, D = mutual inclination)
 *             => D < d needs |sin u_A| < s_A = d / (q_A sin D), same for B
 *   coplanar  s_A >= 1 or s_B >= 1, or q_A cos a_A + q_B cos a_B <= d (a = asin s): the node
 *             windows cannot separate the nodes -> grid-variant refinement of the owner cell
 *   path      per node (u = 0 and u = pi): radial ranges of A and B over their windows; the node
 *             is excluded iff the ranges are more than d apart (|r_A - r_B| >= ||r_A|-|r_B||);
 *             the pair is excluded iff both nodes are
 *   time      windows (in time) of A and B at the same surviving node, intersected with each
 *             other and with the coarse step's owner cell; empty -> excluded
 *
 * Conjunctions: the local minima of D below d inside the intervals (sign changes of
 * g = dr.dv, 32 samples per interval, bisection to 1e-10 s), TCA in the owner cell.  Because
 * the filters are conservative the final set equals level O3 on the coarse candidates --
 * including O3's degenerate rows (R#14), which the coplanar path reports as O3 does (twins are
 * coplanar: D = 0).
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#ifdef _OPENMP
#include <omp.h>
#endif

#include "cd_oracle.h"

#define HY_PI 3.14159265358979323846
#define HY_TWO_PI 6.28318530717958647692

/* per-object geometry (independent of the propagator's internal struct in cd_oracle.c) */
typedef struct {
    double a, e, q, Q, p, nmean, M0;
    double P[3], Qv[3], h[3];
} hy_orbit;

static void hy_make(const orc_elements* el, int64_t i, hy_orbit* o)
{
    double a = el->a[i], e = el->e[i], inc = el->inc[i];
    double raan = el->raan[i], argp = el->argp[i], nu0 = el->nu0[i];
    double cO = cos(raan), sO = sin(raan), cw = cos(argp), sw = sin(argp), ci = cos(inc), si = sin(inc);
    o->P[0] = cO * cw - sO * sw * ci;
    o->P[1] = sO * cw + cO * sw * ci;
    o->P[2] = sw * si;
    o->Qv[0] = -cO * sw - sO * cw * ci;
    o->Qv[1] = -sO * sw + cO * cw * ci;
    o->Qv[2] = cw * si;
    o->h[0] = si * sO;   /* orbit normal h = P x Q */
    o->h[1] = -si * cO;
    o->h[2] = ci;
    o->a = a;
    o->e = e;
    o->q = a * (1.0 - e);
    o->Q = a * (1.0 + e);
    o->p = a * (1.0 - e * e);
    o->nmean = sqrt(orc_mu() / (a * a * a));
    double E0 = 2.0 * atan2(sqrt(1.0 - e) * sin(0.5 * nu0), sqrt(1.0 + e) * cos(0.5 * nu0));
    o->M0 = E0 - e * sin(E0);
}

/* mean anomaly of true anomaly f (forward Kepler relation, no solve), in [-pi, pi]: f is first
 * reduced to [-pi, pi], so that f/2 lies in [-pi/2, pi/2] and the half-angle formula returns the
 * principal E (an unreduced f beyond pi would land E -- and M -- on another branch, 2 pi or 4 pi
 * away, and a window whose ends fall on different branches would come out empty) */
static double hy_mean_of_true(double f, double e)
{
    f = remainder(f, HY_TWO_PI);
    double E = 2.0 * atan2(sqrt(1.0 - e) * sin(0.5 * f), sqrt(1.0 + e) * cos(0.5 * f));
    return E - e * sin(E);
}

/* radius range of an orbit over true anomalies [f1, f2] (f2 - f1 < 2 pi) */
static void hy_radius_range(const hy_orbit* o, double f1, double f2, double* rmin, double* rmax)
{
    double r1 = o->p / (1.0 + o->e * cos(f1));
    double r2 = o->p / (1.0 + o->e * cos(f2));
    *rmin = fmin(r1, r2);
    *rmax = fmax(r1, r2);
    /* perigee (f = 0 mod 2pi) or apogee (f = pi mod 2pi) inside the interval */
    double k0 = ceil(f1 / HY_TWO_PI);
    if (k0 * HY_TWO_PI <= f2) *rmin = o->q;
    double k1 = ceil((f1 - HY_PI) / HY_TWO_PI);
    if (HY_PI + k1 * HY_TWO_PI <= f2) *rmax = o->Q;
}

/* the time intervals (within [tlo, thi]) during which the object's true anomaly lies in
 * (fc - al, fc + al) (periodic); appends to iv (pairs), returns the count */
static int hy_time_windows(const hy_orbit* o, double fc, double al, double tlo, double thi,
                           double* iv, int cap)
{
    double Ml = hy_mean_of_true(fc - al, o->e);
    double Mh = hy_mean_of_true(fc + al, o->e);
    if (Mh < Ml) Mh += HY_TWO_PI;
    double T = HY_TWO_PI / o->nmean;
    /* t(M) = (M - M0)/n + k T */
    double tl = (Ml - o->M0) / o->nmean, th = (Mh - o->M0) / o->nmean;
    double kmin = floor((tlo - th) / T), kmax = ceil((thi - tl) / T);
    int c = 0;
    for (double k = kmin; k <= kmax; k += 1.0) {
        double a = tl + k * T, b = th + k * T;
        if (b < tlo || a > thi) continue;
        if (c < cap) {
            iv[2 * c] = fmax(a, tlo);
            iv[2 * c + 1] = fmin(b, thi);
            c++;
        }
    }
    return c;
}

static double hy_dot(const double* a, const double* b) { return a[0] * b[0] + a[1] * b[1] + a[2] * b[2]; }

/* Filter chain for pair (A, B) and search range [tlo, thi].  Returns flags
 * (ORC_H_AP | ORC_H_COPLANAR | ORC_H_PATH | ORC_H_TIME) and, for non-coplanar pairs that pass,
 * up to `cap` intervals in iv. */
static int hy_filter(const hy_orbit* A, const hy_orbit* B, double d, double tlo, double thi,
                     double* iv, int cap, int* niv)
{
    *niv = 0;
    if (fmax(A->q, B->q) - fmin(A->Q, B->Q) > d) return ORC_H_AP;
    double c[3] = {A->h[1] * B->h[2] - A->h[2] * B->h[1], A->h[2] * B->h[0] - A->h[0] * B->h[2],
                   A->h[0] * B->h[1] - A->h[1] * B->h[0]};
    double sD = sqrt(hy_dot(c, c));
    double sA = sD > 0.0 ? d / (A->q * sD) : 2.0;
    double sB = sD > 0.0 ? d / (B->q * sD) : 2.0;
    if (sA >= 1.0 || sB >= 1.0) return ORC_H_COPLANAR;
    double aA = asin(sA), aB = asin(sB);
    if (A->q * cos(aA) + B->q * cos(aB) <= d) return ORC_H_COPLANAR;
    double nn[3] = {c[0] / sD, c[1] / sD, c[2] / sD};
    /* true anomaly of the node direction in each orbit */
    double fA = atan2(hy_dot(nn, A->Qv), hy_dot(nn, A->P));
    double fB = atan2(hy_dot(nn, B->Qv), hy_dot(nn, B->P));
    int any = 0;
    for (int node = 0; node < 2; ++node) {
        double off = node ? HY_PI : 0.0;
        double rAl, rAh, rBl, rBh;
        hy_radius_range(A, fA + off - aA, fA + off + aA, &rAl, &rAh);
        hy_radius_range(B, fB + off - aB, fB + off + aB, &rBl, &rBh);
        double gap = fmax(rAl, rBl) - fmin(rAh, rBh);
        if (gap > d) continue; /* orbit-path filter: this node cannot host an approach below d */
        any |= 1;
        double wa[32], wb[32];
        int na = hy_time_windows(A, fA + off, aA, tlo, thi, wa, 16);
        int nb = hy_time_windows(B, fB + off, aB, tlo, thi, wb, 16);
        for (int x = 0; x < na; ++x)
            for (int y = 0; y < nb; ++y) {
                double lo = fmax(wa[2 * x], wb[2 * y]), hi = fmin(wa[2 * x + 1], wb[2 * y + 1]);
                if (hi > lo && *niv < cap) {
                    iv[2 * *niv] = lo;
                    iv[2 * *niv + 1] = hi;
                    (*niv)++;
                }
            }
    }
    if (!any) return ORC_H_PATH;
    if (*niv == 0) return ORC_H_TIME;
    return 0;
}

int orc_pair_filter(const orc_elements* el, int64_t i, int64_t j, double d, double tlo, double thi,
                    double* iv, int cap, int* niv)
{
    if (el->model != ORC_PROP_KEPLER)   /* the filters assume fixed orbit planes (Kepler) */
        return -1;
    hy_orbit A, B;
    hy_make(el, i, &A);
    hy_make(el, j, &B);
    return hy_filter(&A, &B, d, tlo, thi, iv, cap, niv);
}

/* g = dr.dv (and D) via the O1 propagator (cd_oracle.c) */
static double hy_g(const orc_elements* el, int64_t i, int64_t j, double t, double* D)
{
    double g;
    orc_pair_distance(el, i, j, &t, 1, D, &g);
    return g;
}

/* local minima below d of D(t) on [lo, hi] (sign changes of g sampled at 32 sub-intervals,
 * bisected to 1e-10 s) whose time lies in the owner cell [oa, ob) */
static int hy_minima(const orc_elements* el, int64_t i, int64_t j, double lo, double hi, double oa,
                     double ob, double d, double* tca, double* pca, int cap)
{
    int c = 0;
    const int NS = 32;
    double tprev = lo, gprev = hy_g(el, i, j, lo, NULL);
    for (int s = 1; s <= NS; ++s) {
        double t = lo + (hi - lo) * (double)s / (double)NS;
        double g = hy_g(el, i, j, t, NULL);
        if (gprev < 0.0 && g >= 0.0) {
            double a = tprev, b = t;
            for (int it = 0; it < 200 && b - a > 1e-10; ++it) {
                double m = 0.5 * (a + b);
                if (hy_g(el, i, j, m, NULL) < 0.0) a = m;
                else b = m;
            }
            double tm = 0.5 * (a + b), D;
            hy_g(el, i, j, tm, &D);
            if (tm >= oa && tm < ob && D < d && c < cap) {
                tca[c] = tm;
                pca[c] = D;
                c++;
            }
        }
        tprev = t;
        gprev = g;
    }
    return c;
}

static int hy_cmp(const void* x, const void* y)
{
    const orc_conjunction* a = (const orc_conjunction*)x;
    const orc_conjunction* b = (const orc_conjunction*)y;
    if (a->i != b->i) return a->i < b->i ? -1 : 1;
    if (a->j != b->j) return a->j < b->j ? -1 : 1;
    if (a->step != b->step) return a->step < b->step ? -1 : 1;
    if (a->tca != b->tca) return a->tca < b->tca ? -1 : 1;
    return 0;
}

int64_t orc_hybrid(const orc_elements* el, int64_t n, double t0, double t1, double dt, double d,
                   double gc, int64_t k_begin, int64_t k_end, void** out, int64_t* counts)
{
    if (el->model != ORC_PROP_KEPLER) {   /* the filters assume fixed orbit planes (Kepler) */
        *out = NULL;
        return -1;
    }
    orc_candidate* cand = NULL;
    int64_t nc = orc_candidates_grid(el, n, t0, t1, dt, gc, 0.0, NULL, k_begin, k_end, &cand);
    /* plain serial-per-candidate evaluation, OpenMP over candidates */
    int nt = orc_num_threads();
    orc_conjunction** bufs = (orc_conjunction**)calloc((size_t)nt, sizeof(void*));
    int64_t* bn = (int64_t*)calloc((size_t)nt, sizeof(int64_t));
    int64_t* bc = (int64_t*)calloc((size_t)nt, sizeof(int64_t));
    int64_t st[5] = {0, 0, 0, 0, 0};
#pragma omp parallel
    {
#ifdef _OPENMP
        int tid = omp_get_thread_num();
#else
        int tid = 0;
#endif
        int64_t ls[5] = {0, 0, 0, 0, 0};
#pragma omp for schedule(dynamic, 64)
        for (int64_t qd = 0; qd < nc; ++qd) {
            const orc_candidate* c = &cand[qd];
            double tk = fma((double)c->step, dt, t0);
            /* owner cell; a single instant when t1 == t0, where only a degenerate coplanar
             * pair has a row (R#14, as in O3) and the minima searches below find nothing */
            double oa = fmax(tk - 0.5 * dt, t0), ob = fmin(tk + 0.5 * dt, t1);
            hy_orbit A, B;
            hy_make(el, c->i, &A);
            hy_make(el, c->j, &B);
            double iv[64];
            int niv = 0;
            int fl = hy_filter(&A, &B, d, oa, ob, iv, 32, &niv);
            double tca[8], pca[8];
            int m = 0;
            uint32_t flags = 0;
            if (fl == ORC_H_AP) { ls[0]++; continue; }
            if (fl == ORC_H_PATH) { ls[2]++; continue; }
            if (fl == ORC_H_TIME) { ls[3]++; continue; }
            if (fl == ORC_H_COPLANAR) {
                ls[1]++;
                flags = ORC_COPLANAR;
                /* "the procedure is the same as for the grid-based variant", so a
                 * degenerate pair (D stationary) is reported as there: tca = t_k, pca = D(t_k)
                 * (reading R#14) */
                double Dk;
                if (orc_pair_degenerate(el, c->i, c->j, tk, &Dk)) {
                    if (Dk < d) {
                        flags |= ORC_DEGENERATE;
                        tca[0] = tk;
                        pca[0] = Dk;
                        m = 1;
                    }
                } else {
                    m = hy_minima(el, c->i, c->j, oa, ob, oa, ob, d, tca, pca, 8);
                }
            } else {
                ls[4]++;
                for (int w = 0; w < niv && m < 8; ++w)
                    m += hy_minima(el, c->i, c->j, iv[2 * w], iv[2 * w + 1], oa, ob, d, tca + m, pca + m, 8 - m);
            }
            for (int x = 0; x < m; ++x) {
                if (bn[tid] == bc[tid]) {
                    bc[tid] = bc[tid] ? 2 * bc[tid] : 256;
                    bufs[tid] = (orc_conjunction*)realloc(bufs[tid], sizeof(orc_conjunction) * (size_t)bc[tid]);
                }
                orc_conjunction* r = &bufs[tid][bn[tid]++];
                r->i = c->i; r->j = c->j; r->step = c->step; r->flags = flags;
                r->tca = tca[x]; r->pca = pca[x];
            }
        }
#pragma omp critical
        for (int q = 0; q < 5; ++q) st[q] += ls[q];
    }
    int64_t total = 0;
    for (int q = 0; q < nt; ++q) total += bn[q];
    orc_conjunction* res = (orc_conjunction*)malloc(sizeof(orc_conjunction) * (size_t)(total > 0 ? total : 1));
    int64_t off = 0;
    for (int q = 0; q < nt; ++q) {
        if (bn[q]) memcpy(res + off, bufs[q], sizeof(orc_conjunction) * (size_t)bn[q]);
        off += bn[q];
        free(bufs[q]);
    }
    free(bufs); free(bn); free(bc);
    orc_free(cand);
    qsort(res, (size_t)total, sizeof(orc_conjunction), hy_cmp);
    if (counts) {
        counts[0] = nc;     /* coarse candidates                 */
        counts[1] = st[0];  /* rejected by apogee/perigee        */
        counts[2] = st[1];  /* coplanar (grid refinement path)   */
        counts[3] = st[2];  /* rejected by the orbit-path filter */
        counts[4] = st[3];  /* rejected by the time filter       */
        counts[5] = st[4];  /* time-window work                  */
    }
    *out = res;
    return total;
}

/* ------------------------------------------------------------------------------------------
 * O5: legacy full-window filter chain.  The paper's comparison baseline
 * screens every pair with the "classical orbital filters" alone, without a grid (P:43, P:189,
 * P:315-318 accuracy comparison, "not possible with the legacy variant to calculate more
 * than 64,000 satellites").  Per pair i < j, the O4 formulas over the whole window [t0, t1]:
 *   AP -> coplanar (search all of [t0, t1]) -> orbit path -> time filter: every window of A at a
 *   surviving node intersected with every window of B at the same node (both lists are sorted
 *   in time and each object's windows are disjoint, so a merge visits each once)
 * Conjunctions: every local minimum of D below d inside the intervals = every - -> + sign
 * change of g = dr.dv sampled at spacing <= dt/8 (at least 8 samples per interval), bisected
 * to 1e-10 s, with D < d and TCA in [t0, t1].  Each row is labelled with the nearest step
 * k = floor((TCA - t0)/dt + 1/2) (reading R9) and, as in the grid variant, reported only if that
 * step exists (k < K, reading R4); MULTI flags a second sign change within 2 dt
 * (two minima the method's per-sample search may not separate); COPLANAR the coplanar path.
 * Degenerate pairs (g identically 0) have no sign change and are not reported.
 * counts: pairs, ap_rejected, coplanar, path_rejected, time_rejected, intervals.
 * ------------------------------------------------------------------------------------------ */

typedef struct {
    double* v;
    int64_t n, cap;
} lg_buf;

static void lg_push(lg_buf* b, double x, double y)
{
    if (b->n + 2 > b->cap) {
        b->cap = b->cap ? 2 * b->cap : 64;
        b->v = (double*)realloc(b->v, sizeof(double) * (size_t)b->cap);
    }
    b->v[b->n++] = x;
    b->v[b->n++] = y;
}

/* every window of object o at node direction fc (half-angle al) within [t0, t1], in time order */
static void lg_windows(const hy_orbit* o, double fc, double al, double t0, double t1, lg_buf* out)
{
    out->n = 0;
    double Ml = hy_mean_of_true(fc - al, o->e);
    double Mh = hy_mean_of_true(fc + al, o->e);
    if (Mh < Ml) Mh += HY_TWO_PI;
    double T = HY_TWO_PI / o->nmean;
    double tl = (Ml - o->M0) / o->nmean, th = (Mh - o->M0) / o->nmean;
    double kmin = floor((t0 - th) / T), kmax = ceil((t1 - tl) / T);
    for (double k = kmin; k <= kmax; k += 1.0) {
        double a = tl + k * T, b = th + k * T;
        if (b < t0 || a > t1) continue;
        lg_push(out, fmax(a, t0), fmin(b, t1));
    }
}

/* filter chain of one pair over [t0, t1]; intervals appended to iv */
static int lg_filter(const hy_orbit* A, const hy_orbit* B, double d, double t0, double t1,
                     lg_buf* iv, lg_buf* wa, lg_buf* wb)
{
    iv->n = 0;
    if (fmax(A->q, B->q) - fmin(A->Q, B->Q) > d) return ORC_H_AP;
    double c[3] = {A->h[1] * B->h[2] - A->h[2] * B->h[1], A->h[2] * B->h[0] - A->h[0] * B->h[2],
                   A->h[0] * B->h[1] - A->h[1] * B->h[0]};
    double sD = sqrt(hy_dot(c, c));
    double sA = sD > 0.0 ? d / (A->q * sD) : 2.0;
    double sB = sD > 0.0 ? d / (B->q * sD) : 2.0;
    int coplanar = sA >= 1.0 || sB >= 1.0;
    double aA = 0.0, aB = 0.0;
    if (!coplanar) {
        aA = asin(sA);
        aB = asin(sB);
        coplanar = A->q * cos(aA) + B->q * cos(aB) <= d;
    }
    if (coplanar) {
        lg_push(iv, t0, t1);
        return ORC_H_COPLANAR;
    }
    double nn[3] = {c[0] / sD, c[1] / sD, c[2] / sD};
    double fA = atan2(hy_dot(nn, A->Qv), hy_dot(nn, A->P));
    double fB = atan2(hy_dot(nn, B->Qv), hy_dot(nn, B->P));
    int any = 0;
    for (int node = 0; node < 2; ++node) {
        double off = node ? HY_PI : 0.0;
        double rAl, rAh, rBl, rBh;
        hy_radius_range(A, fA + off - aA, fA + off + aA, &rAl, &rAh);
        hy_radius_range(B, fB + off - aB, fB + off + aB, &rBl, &rBh);
        if (fmax(rAl, rBl) - fmin(rAh, rBh) > d) continue;   /* orbit path */
        any = 1;
        lg_windows(A, fA + off, aA, t0, t1, wa);
        lg_windows(B, fB + off, aB, t0, t1, wb);
        int64_t x = 0, y = 0;
        while (x < wa->n && y < wb->n) {
            double lo = fmax(wa->v[x], wb->v[y]), hi = fmin(wa->v[x + 1], wb->v[y + 1]);
            if (hi > lo) lg_push(iv, lo, hi);
            if (wa->v[x + 1] < wb->v[y + 1]) x += 2;
            else y += 2;
        }
    }
    if (!any) return ORC_H_PATH;
    if (iv->n == 0) return ORC_H_TIME;
    return 0;
}

int64_t orc_legacy(const orc_elements* el, int64_t n, double t0, double t1, double dt, double d,
                   void** out, int64_t* counts)
{
    if (el->model != ORC_PROP_KEPLER) {   /* the filters assume fixed orbit planes (Kepler) */
        *out = NULL;
        return -1;
    }
    hy_orbit* o = (hy_orbit*)malloc(sizeof(hy_orbit) * (size_t)(n > 0 ? n : 1));
    for (int64_t i = 0; i < n; ++i) hy_make(el, i, &o[i]);
    const double K = (double)orc_num_steps(t0, t1, dt);
    int nt = orc_num_threads();
    orc_conjunction** bufs = (orc_conjunction**)calloc((size_t)nt, sizeof(void*));
    int64_t* bn = (int64_t*)calloc((size_t)nt, sizeof(int64_t));
    int64_t* bc = (int64_t*)calloc((size_t)nt, sizeof(int64_t));
    int64_t st[6] = {0, 0, 0, 0, 0, 0};
#pragma omp parallel
    {
#ifdef _OPENMP
        int tid = omp_get_thread_num();
#else
        int tid = 0;
#endif
        int64_t ls[6] = {0, 0, 0, 0, 0, 0};
        lg_buf iv = {0}, wa = {0}, wb = {0}, mins = {0};
#pragma omp for schedule(dynamic, 1)
        for (int64_t i = 0; i < n; ++i) {
            for (int64_t j = i + 1; j < n; ++j) {
                ls[0]++;
                int fl = lg_filter(&o[i], &o[j], d, t0, t1, &iv, &wa, &wb);
                if (fl == ORC_H_AP) { ls[1]++; continue; }
                if (fl == ORC_H_PATH) { ls[3]++; continue; }
                if (fl == ORC_H_TIME) { ls[4]++; continue; }
                if (fl == ORC_H_COPLANAR) ls[2]++;
                ls[5] += iv.n / 2;
                /* every - -> + sign change of g in the intervals: (tca, D) in mins */
                mins.n = 0;
                for (int64_t w = 0; w < iv.n; w += 2) {
                    double lo = iv.v[w], hi = iv.v[w + 1];
                    int64_t ns = (int64_t)ceil((hi - lo) / (dt / 8.0));
                    if (ns < 8) ns = 8;
                    double tprev = lo, gprev = hy_g(el, i, j, lo, NULL);
                    for (int64_t s = 1; s <= ns; ++s) {
                        double t = lo + (hi - lo) * (double)s / (double)ns;
                        double g = hy_g(el, i, j, t, NULL);
                        if (gprev < 0.0 && g >= 0.0) {
                            double a = tprev, b = t;
                            for (int it = 0; it < 200 && b - a > 1e-10; ++it) {
                                double m = 0.5 * (a + b);
                                if (hy_g(el, i, j, m, NULL) < 0.0) a = m;
                                else b = m;
                            }
                            double tm = 0.5 * (a + b), D;
                            hy_g(el, i, j, tm, &D);
                            lg_push(&mins, tm, D);
                        }
                        tprev = t;
                        gprev = g;
                    }
                }
                for (int64_t x = 0; x < mins.n; x += 2) {
                    double tm = mins.v[x], D = mins.v[x + 1];
                    if (!(D < d) || tm < t0 || tm > t1) continue;
                    if (floor((tm - t0) / dt + 0.5) >= K) continue;   /* owner step beyond the last */
                    uint32_t flags = fl == ORC_H_COPLANAR ? ORC_COPLANAR : 0u;
                    for (int64_t y = 0; y < mins.n; y += 2)
                        if (y != x && fabs(mins.v[y] - tm) < 2.0 * dt) flags |= ORC_MULTI;
                    if (bn[tid] == bc[tid]) {
                        bc[tid] = bc[tid] ? 2 * bc[tid] : 256;
                        bufs[tid] = (orc_conjunction*)realloc(bufs[tid], sizeof(orc_conjunction) * (size_t)bc[tid]);
                    }
                    orc_conjunction* r = &bufs[tid][bn[tid]++];
                    r->i = (uint32_t)i;
                    r->j = (uint32_t)j;
                    r->step = (uint32_t)floor((tm - t0) / dt + 0.5);
                    r->flags = flags;
                    r->tca = tm;
                    r->pca = D;
                }
            }
        }
        free(iv.v);
        free(wa.v);
        free(wb.v);
        free(mins.v);
#pragma omp critical
        for (int q = 0; q < 6; ++q) st[q] += ls[q];
    }
    int64_t total = 0;
    for (int q = 0; q < nt; ++q) total += bn[q];
    orc_conjunction* res = (orc_conjunction*)malloc(sizeof(orc_conjunction) * (size_t)(total > 0 ? total : 1));
    int64_t off = 0;
    for (int q = 0; q < nt; ++q) {
        if (bn[q]) memcpy(res + off, bufs[q], sizeof(orc_conjunction) * (size_t)bn[q]);
        off += bn[q];
        free(bufs[q]);
    }
    free(bufs);
    free(bn);
    free(bc);
    free(o);
    qsort(res, (size_t)total, sizeof(orc_conjunction), hy_cmp);
    for (int q = 0; q < 6; ++q) counts[q] = st[q];
    *out = res;
    return total;
}
