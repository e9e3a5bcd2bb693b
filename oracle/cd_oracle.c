/*
 * cd_oracle.c -- TEST INFRASTRUCTURE ONLY (not the product path).
 *
 * Plain, slow, obviously-correct CPU oracle for the screening hot path of
 * Hellwig, Czappa, Michel, Bertrand, Wolf, "Satellite Collision Detection using Spatial Data
 * Structures", IPDPS 2023.  Only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline / --impl reference legs may load or execute this file.  It shares no code,
 * headers, tables or constants with the CUDA path under paper_conf_ipps_hellwigcmbw23_b200/.
 *
 * Citations "P:NN" are PAPER.md line numbers; "R#n" are the readings listed in DESIGN.md
 * (and SURVEY.md 8(c)) for passages the paper leaves silent or garbled.
 *
 * Levels:
 *   O1 propagate      -- two-body Kepler, Newton-Raphson on E - e sin E = M
 *   O1' J2 secular    -- the same with secular J2 rates of Omega, omega, M ("other
 *                        propagators"; Vallado [41] Section 9.6), orc_elements.model = 1
 *   O2 candidates     -- K = {(i,j,k): i<j, |r_i(t_k) - r_j(t_k)| < g_c}
 *                        brute force O(n^2) per step, and a plain sorted-cell grid with 27 neighbours
 *   O3 conjunctions   -- all local minima of D(t) = |r_i - r_j| inside the owner cell of step k
 *                        with D < d (Fig. 2; owner rule R#9)
 *   O4 hybrid filters -- see cd_oracle_hybrid.c
 *
 * Arithmetic is plain IEEE fp64 (compiled with -ffp-contract=off, no -ffast-math).
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#ifdef _OPENMP
#include <omp.h>
#endif

#include "cd_oracle.h"

#define ORC_PI 3.14159265358979323846
#define ORC_TWO_PI 6.28318530717958647692

/* ------------------------------------------------------------------------------------------
 * O1: propagation ("six values (semi-major-axis, eccentricity, inclination, longitude of
 * the ascending node, argument of perigee, true anomaly)"; Fig. 7/8 geometry).
 * Standard two-body formulas, mu = 398600.4418 km^3/s^2 (R#1),
 * epoch t = 0 for all objects (R#2).
 * ------------------------------------------------------------------------------------------ */

double orc_mu(void) { return 398600.4418; }

/* Kepler's equation E - e sin E = M by plain Newton-Raphson (the paper uses the Contour solver
 * [43]; both reach the same root of the same equation).  Start E = M for e < 0.8, else pi. */
double orc_kepler_newton(double M, double e)
{
    double E = (e < 0.8) ? M : ORC_PI;
    for (int it = 0; it < 200; ++it) {
        double f = E - e * sin(E) - M;
        double fp = 1.0 - e * cos(E);
        double dE = f / fp;
        E = E - dE;
        if (fabs(dE) <= 1e-15 * fmax(1.0, fabs(E)))
            break;
    }
    return E;
}

typedef struct {
    double a, e, b, nmean, M0;
    double P[3], Q[3];
    /* J2 secular model (ORC_PROP_J2): elements at epoch and their secular rates */
    int j2;
    double inc, raan0, argp0, draan, dargp;
} orc_orbit;

/* ------------------------------------------------------------------------------------------
 * O1': J2 secular propagator ("other propagators instead of the Kepler
 * Contour solver").  First-order secular effect of Earth's oblateness J2 on the mean
 * elements, Vallado & McClain [41] Section 9.6 (the paper's ref. [41]):
 *     p = a (1 - e^2),  n0 = sqrt(mu / a^3),  k = J2 (R_E / p)^2
 *     dM/dt     = n0 [1 + (3/2) k sqrt(1 - e^2) (1 - (3/2) sin^2 i)]
 *     dOmega/dt = -(3/2) n0 k cos i
 *     domega/dt =  (3/4) n0 k (4 - 5 sin^2 i)
 * a, e, i constant; the position at t is the two-body position of the elements
 * (a, e, i, Omega0 + dOmega/dt t, omega0 + domega/dt t, M0 + dM/dt t).  J2 and R_E: EGM-96 /
 * WGS-84 values (reading R19).
 * ------------------------------------------------------------------------------------------ */
double orc_j2(void) { return 1.08262668e-3; }
double orc_earth_radius(void) { return 6378.137; }

static void orc_perifocal(double raan, double inc, double argp, double P[3], double Q[3])
{
    double cO = cos(raan), sO = sin(raan), cw = cos(argp), sw = sin(argp);
    double ci = cos(inc), si = sin(inc);
    P[0] = cO * cw - sO * sw * ci;
    P[1] = sO * cw + cO * sw * ci;
    P[2] = sw * si;
    Q[0] = -cO * sw - sO * cw * ci;
    Q[1] = -sO * sw + cO * cw * ci;
    Q[2] = cw * si;
}

/* Per-object constants: perifocal unit vectors P, Q (Fig. 8: Omega, i, omega), mean motion,
 * mean anomaly at epoch from the true anomaly nu0 (P:166 element set; R#2). */
static void orc_make_orbit(const orc_elements* el, int64_t idx, orc_orbit* o)
{
    double a = el->a[idx], e = el->e[idx], inc = el->inc[idx];
    double raan = el->raan[idx], argp = el->argp[idx], nu0 = el->nu0[idx];
    orc_perifocal(raan, inc, argp, o->P, o->Q);
    o->a = a;
    o->e = e;
    o->b = a * sqrt(1.0 - e * e);
    o->nmean = sqrt(orc_mu() / (a * a * a));
    double E0 = 2.0 * atan2(sqrt(1.0 - e) * sin(0.5 * nu0), sqrt(1.0 + e) * cos(0.5 * nu0));
    o->M0 = E0 - e * sin(E0);
    o->j2 = el->model == ORC_PROP_J2;
    o->inc = inc;
    o->raan0 = raan;
    o->argp0 = argp;
    o->draan = 0.0;
    o->dargp = 0.0;
    if (o->j2) {   /* Vallado [41] Section 9.6, see O1' above */
        double p = a * (1.0 - e * e);
        double k = orc_j2() * (orc_earth_radius() / p) * (orc_earth_radius() / p);
        double n0 = o->nmean;
        double s2 = sin(inc) * sin(inc);
        o->nmean = n0 * (1.0 + 1.5 * k * sqrt(1.0 - e * e) * (1.0 - 1.5 * s2));
        o->draan = -1.5 * n0 * k * cos(inc);
        o->dargp = 0.75 * n0 * k * (4.0 - 5.0 * s2);
    }
}

/* Position (and optionally velocity) at time t (seconds from epoch). */
static void orc_state(const orc_orbit* o, double t, double r[3], double v[3])
{
    double M = fmod(o->M0 + o->nmean * t, ORC_TWO_PI);
    if (M < 0.0)
        M += ORC_TWO_PI;
    double E = orc_kepler_newton(M, o->e);
    double cE = cos(E), sE = sin(E);
    double x = o->a * (cE - o->e);
    double y = o->b * sE;
    double P[3], Q[3];
    if (o->j2) {   /* O1': the orbit plane and perigee at time t */
        orc_perifocal(o->raan0 + o->draan * t, o->inc, o->argp0 + o->dargp * t, P, Q);
    } else {
        for (int c = 0; c < 3; ++c) {
            P[c] = o->P[c];
            Q[c] = o->Q[c];
        }
    }
    for (int c = 0; c < 3; ++c)
        r[c] = x * P[c] + y * Q[c];
    if (v) {
        /* dE/dt = n / (1 - e cos E) with n the mean-anomaly rate (n0, or the J2 dM/dt) */
        double rr = 1.0 - o->e * cE;
        double k = o->nmean / rr;
        for (int c = 0; c < 3; ++c)
            v[c] = k * (-o->a * sE * P[c] + o->b * cE * Q[c]);
        if (o->j2) {
            /* d/dt of the rotating plane: dOmega/dt z x r + domega/dt h x r, h = P x Q */
            double h[3] = {P[1] * Q[2] - P[2] * Q[1], P[2] * Q[0] - P[0] * Q[2],
                           P[0] * Q[1] - P[1] * Q[0]};
            double hxr[3] = {h[1] * r[2] - h[2] * r[1], h[2] * r[0] - h[0] * r[2],
                             h[0] * r[1] - h[1] * r[0]};
            double zxr[3] = {-r[1], r[0], 0.0};
            for (int c = 0; c < 3; ++c)
                v[c] += o->draan * zxr[c] + o->dargp * hxr[c];
        }
    }
}

static orc_orbit* orc_make_orbits(const orc_elements* el, int64_t n)
{
    orc_orbit* o = (orc_orbit*)malloc(sizeof(orc_orbit) * (size_t)(n > 0 ? n : 1));
    for (int64_t i = 0; i < n; ++i)
        orc_make_orbit(el, i, &o[i]);
    return o;
}

void orc_propagate(const orc_elements* el, int64_t n, const double* t, int64_t nt,
                   double* xyz, double* vxyz)
{
    orc_orbit* o = orc_make_orbits(el, n);
#pragma omp parallel for schedule(static)
    for (int64_t q = 0; q < nt; ++q) {
        for (int64_t i = 0; i < n; ++i) {
            double r[3], v[3];
            orc_state(&o[i], t[q], r, vxyz ? v : NULL);
            for (int c = 0; c < 3; ++c) {
                xyz[(q * n + i) * 3 + c] = r[c];
                if (vxyz)
                    vxyz[(q * n + i) * 3 + c] = v[c];
            }
        }
    }
    free(o);
}

/* Step set (o = t / s_ps; R#4): t_k = t0 + k dt, k = 0 .. K-1, K = floor((t1-t0)/dt) + 1. */
int64_t orc_num_steps(double t0, double t1, double dt)
{
    if (!(dt > 0.0) || t1 < t0)
        return 0;
    return (int64_t)floor((t1 - t0) / dt) + 1;
}

static double orc_step_time(int64_t k, double t0, double dt) { return fma((double)k, dt, t0); }

/* ------------------------------------------------------------------------------------------
 * growable output buffers
 * ------------------------------------------------------------------------------------------ */
typedef struct { orc_candidate* p; int64_t n, cap; } cand_buf;
typedef struct { orc_conjunction* p; int64_t n, cap; } conj_buf;

static void cand_push(cand_buf* b, uint32_t i, uint32_t j, uint32_t k)
{
    if (b->n == b->cap) {
        b->cap = b->cap ? 2 * b->cap : 1024;
        b->p = (orc_candidate*)realloc(b->p, sizeof(orc_candidate) * (size_t)b->cap);
    }
    b->p[b->n].i = i;
    b->p[b->n].j = j;
    b->p[b->n].step = k;
    b->n++;
}

static void conj_push(conj_buf* b, const orc_conjunction* c)
{
    if (b->n == b->cap) {
        b->cap = b->cap ? 2 * b->cap : 1024;
        b->p = (orc_conjunction*)realloc(b->p, sizeof(orc_conjunction) * (size_t)b->cap);
    }
    b->p[b->n++] = *c;
}

static int cmp_cand(const void* x, const void* y)
{
    const orc_candidate* a = (const orc_candidate*)x;
    const orc_candidate* b = (const orc_candidate*)y;
    if (a->i != b->i) return a->i < b->i ? -1 : 1;
    if (a->j != b->j) return a->j < b->j ? -1 : 1;
    if (a->step != b->step) return a->step < b->step ? -1 : 1;
    return 0;
}

static int cmp_conj(const void* x, const void* y)
{
    const orc_conjunction* a = (const orc_conjunction*)x;
    const orc_conjunction* b = (const orc_conjunction*)y;
    if (a->i != b->i) return a->i < b->i ? -1 : 1;
    if (a->j != b->j) return a->j < b->j ? -1 : 1;
    if (a->step != b->step) return a->step < b->step ? -1 : 1;
    if (a->tca != b->tca) return a->tca < b->tca ? -1 : 1;
    return 0;
}

static int orc_threads(void)
{
#ifdef _OPENMP
    return omp_get_max_threads();
#else
    return 1;
#endif
}

static int orc_thread_id(void)
{
#ifdef _OPENMP
    return omp_get_thread_num();
#else
    return 0;
#endif
}

int orc_num_threads(void) { return orc_threads(); }

/* merge per-thread candidate buffers and sort by (i, j, step) */
static int64_t merge_cands(cand_buf* bufs, int nb, orc_candidate** out)
{
    int64_t total = 0;
    for (int q = 0; q < nb; ++q)
        total += bufs[q].n;
    orc_candidate* r = (orc_candidate*)malloc(sizeof(orc_candidate) * (size_t)(total > 0 ? total : 1));
    int64_t off = 0;
    for (int q = 0; q < nb; ++q) {
        if (bufs[q].n)
            memcpy(r + off, bufs[q].p, sizeof(orc_candidate) * (size_t)bufs[q].n);
        off += bufs[q].n;
        free(bufs[q].p);
    }
    qsort(r, (size_t)total, sizeof(orc_candidate), cmp_cand);
    *out = r;
    return total;
}

/* ------------------------------------------------------------------------------------------
 * O2a: candidate set by brute force.  K = {(i,j,k) : i < j, |r_i(t_k) - r_j(t_k)| < g_c}.
 * The grid of P:61-62/P:93-95 exists only to find exactly these pairs faster; the distance gate
 * |dr| < g_c (strict) is reading R#6 (the Eq. 1 argument).
 * ------------------------------------------------------------------------------------------ */
int64_t orc_candidates_brute(const orc_elements* el, int64_t n, double t0, double t1, double dt,
                             double gc, int64_t k_begin, int64_t k_end, orc_candidate** out)
{
    int64_t K = orc_num_steps(t0, t1, dt);
    if (k_end < 0 || k_end > K) k_end = K;
    if (k_begin < 0) k_begin = 0;
    orc_orbit* o = orc_make_orbits(el, n);
    int nt = orc_threads();
    cand_buf* bufs = (cand_buf*)calloc((size_t)nt, sizeof(cand_buf));
    double gc2 = gc * gc;
#pragma omp parallel
    {
        double* pos = (double*)malloc(sizeof(double) * 3 * (size_t)(n > 0 ? n : 1));
        cand_buf* mine = &bufs[orc_thread_id()];
#pragma omp for schedule(dynamic, 1)
        for (int64_t k = k_begin; k < k_end; ++k) {
            double tk = orc_step_time(k, t0, dt);
            for (int64_t i = 0; i < n; ++i)
                orc_state(&o[i], tk, &pos[3 * i], NULL);
            for (int64_t i = 0; i < n; ++i)
                for (int64_t j = i + 1; j < n; ++j) {
                    double dx = pos[3 * i] - pos[3 * j];
                    double dy = pos[3 * i + 1] - pos[3 * j + 1];
                    double dz = pos[3 * i + 2] - pos[3 * j + 2];
                    if (dx * dx + dy * dy + dz * dz < gc2)
                        cand_push(mine, (uint32_t)i, (uint32_t)j, (uint32_t)k);
                }
        }
        free(pos);
    }
    free(o);
    int64_t c = merge_cands(bufs, nt, out);
    free(bufs);
    return c;
}

/* ------------------------------------------------------------------------------------------
 * O2b: the same set through a plain CPU grid: cells of edge L >= g_c
 * (Eq. 1), cell index floor((r - origin)/L) per axis (R#7), objects sorted by cell,
 * and for every object the 3^3 = 27 cells around its own ("all 3^3 - 1 = 26 neighboring
 * cells" plus its own).  Every pair closer than g_c <= L lies in the same or an adjacent cell
 * on every axis, so this finds exactly K.  Each unordered pair is reported once (i < j).
 * ------------------------------------------------------------------------------------------ */
typedef struct { int64_t c[3]; int64_t id; } cell_item;

static int cmp_cell3(const int64_t* a, const int64_t* b)
{
    for (int q = 0; q < 3; ++q)
        if (a[q] != b[q]) return a[q] < b[q] ? -1 : 1;
    return 0;
}

static int cmp_item(const void* x, const void* y)
{
    const cell_item* a = (const cell_item*)x;
    const cell_item* b = (const cell_item*)y;
    int r = cmp_cell3(a->c, b->c);
    if (r) return r;
    return a->id < b->id ? -1 : (a->id > b->id);
}

/* first index in sorted items[0..m) whose cell is >= key */
static int64_t lower_bound_cell(const cell_item* items, int64_t m, const int64_t key[3])
{
    int64_t lo = 0, hi = m;
    while (lo < hi) {
        int64_t mid = lo + (hi - lo) / 2;
        if (cmp_cell3(items[mid].c, key) < 0) lo = mid + 1;
        else hi = mid;
    }
    return lo;
}

int64_t orc_candidates_grid(const orc_elements* el, int64_t n, double t0, double t1, double dt,
                            double gc, double cell, const double origin[3],
                            int64_t k_begin, int64_t k_end, orc_candidate** out)
{
    int64_t K = orc_num_steps(t0, t1, dt);
    if (k_end < 0 || k_end > K) k_end = K;
    if (k_begin < 0) k_begin = 0;
    double L = (cell > 0.0) ? cell : gc;
    /* a cell must be at least g_c wide; widen by a few ulps so that rounding of
     * (x - o)/L can never place two points closer than g_c two cells apart */
    if (L < gc * (1.0 + 1e-12)) L = gc * (1.0 + 1e-12);
    double o3[3] = {0.0, 0.0, 0.0};
    if (origin) { o3[0] = origin[0]; o3[1] = origin[1]; o3[2] = origin[2]; }
    orc_orbit* o = orc_make_orbits(el, n);
    int nt = orc_threads();
    cand_buf* bufs = (cand_buf*)calloc((size_t)nt, sizeof(cand_buf));
    double gc2 = gc * gc;
#pragma omp parallel
    {
        size_t nn = (size_t)(n > 0 ? n : 1);
        double* pos = (double*)malloc(sizeof(double) * 3 * nn);
        cell_item* items = (cell_item*)malloc(sizeof(cell_item) * nn);
        cand_buf* mine = &bufs[orc_thread_id()];
#pragma omp for schedule(dynamic, 1)
        for (int64_t k = k_begin; k < k_end; ++k) {
            double tk = orc_step_time(k, t0, dt);
            for (int64_t i = 0; i < n; ++i) {
                orc_state(&o[i], tk, &pos[3 * i], NULL);
                for (int q = 0; q < 3; ++q)
                    items[i].c[q] = (int64_t)floor((pos[3 * i + q] - o3[q]) / L);
                items[i].id = i;
            }
            qsort(items, (size_t)n, sizeof(cell_item), cmp_item);
            for (int64_t s = 0; s < n; ++s) {
                int64_t i = items[s].id;
                for (int dx = -1; dx <= 1; ++dx)
                    for (int dy = -1; dy <= 1; ++dy)
                        for (int dz = -1; dz <= 1; ++dz) {
                            int64_t key[3] = {items[s].c[0] + dx, items[s].c[1] + dy, items[s].c[2] + dz};
                            for (int64_t u = lower_bound_cell(items, n, key);
                                 u < n && cmp_cell3(items[u].c, key) == 0; ++u) {
                                int64_t j = items[u].id;
                                if (j <= i) continue;
                                double ddx = pos[3 * i] - pos[3 * j];
                                double ddy = pos[3 * i + 1] - pos[3 * j + 1];
                                double ddz = pos[3 * i + 2] - pos[3 * j + 2];
                                if (ddx * ddx + ddy * ddy + ddz * ddz < gc2)
                                    cand_push(mine, (uint32_t)i, (uint32_t)j, (uint32_t)k);
                            }
                        }
            }
        }
        free(pos);
        free(items);
    }
    free(o);
    int64_t c = merge_cands(bufs, nt, out);
    free(bufs);
    return c;
}

/* ------------------------------------------------------------------------------------------
 * O3: conjunctions.  P:57: "A PCA is a local minimum of the distance between two satellites in
 * orbit, and the TCA is the time when the PCA occurs."  P:59/P:65 (Fig. 2): encounters with a
 * minimal distance below the threshold d are reported.  P:181: the search for candidate
 * (i, j, k) is centred on the sample time t_k; a minimum found at the edge of the interval
 * belongs to the neighbouring interval.  Reading R#9 (owner rule): a minimum is reported by
 * the step whose owner cell [t_k - dt/2, t_k + dt/2) contains it, intersected with [t0, t1].
 *
 * Plain definition, evaluated directly: local minima of D^2(t) are the - -> + sign changes of
 * g(t) = (r_i - r_j) . (v_i - v_j) = (1/2) dD^2/dt.  g is sampled at 33 points across the
 * owner cell and each bracketed sign change is bisected to 1e-10 s.
 *
 * Flags: ORC_MULTI if g changes sign more than once (either direction) on
 * [t_k - t_w, t_k + t_w], t_w = 2 g_c / min(|v_i|, |v_j|) ("time it takes the slower of
 * both satellites to cross two cells"; R#10): there D^2 is not unimodal and a single-minimum
 * search may legitimately return another minimum.  ORC_DEGENERATE if |v_i - v_j| < 1e-9 km/s
 * at t_k (D stationary, e.g. co-located identical orbits; R#14): reported with tca = t_k,
 * pca = D(t_k) when D(t_k) < d.
 * ------------------------------------------------------------------------------------------ */
static double orc_g(const orc_orbit* A, const orc_orbit* B, double t, double* D)
{
    double ra[3], va[3], rb[3], vb[3];
    orc_state(A, t, ra, va);
    orc_state(B, t, rb, vb);
    double g = 0.0, d2 = 0.0;
    for (int c = 0; c < 3; ++c) {
        double dr = ra[c] - rb[c];
        g += dr * (va[c] - vb[c]);
        d2 += dr * dr;
    }
    if (D) *D = sqrt(d2);
    return g;
}

static int count_sign_changes(const orc_orbit* A, const orc_orbit* B, double ta, double tb, int ns)
{
    int changes = 0;
    double gprev = orc_g(A, B, ta, NULL);
    for (int s = 1; s <= ns; ++s) {
        double t = ta + (tb - ta) * (double)s / (double)ns;
        double g = orc_g(A, B, t, NULL);
        if ((gprev < 0.0 && g >= 0.0) || (gprev >= 0.0 && g < 0.0))
            changes++;
        gprev = g;
    }
    return changes;
}

static void orc_refine_one(const orc_orbit* o, const orc_candidate* c, double t0, double t1,
                           double dt, double d, double gc, conj_buf* out)
{
    const orc_orbit* A = &o[c->i];
    const orc_orbit* B = &o[c->j];
    double tk = orc_step_time((int64_t)c->step, t0, dt);
    double ra[3], va[3], rb[3], vb[3];
    orc_state(A, tk, ra, va);
    orc_state(B, tk, rb, vb);
    double dv2 = 0.0, dr2 = 0.0, sa = 0.0, sb = 0.0;
    for (int q = 0; q < 3; ++q) {
        dv2 += (va[q] - vb[q]) * (va[q] - vb[q]);
        dr2 += (ra[q] - rb[q]) * (ra[q] - rb[q]);
        sa += va[q] * va[q];
        sb += vb[q] * vb[q];
    }
    if (sqrt(dv2) < 1e-9) {
        if (sqrt(dr2) < d) {
            orc_conjunction r;
            r.i = c->i; r.j = c->j; r.step = c->step; r.flags = ORC_DEGENERATE;
            r.tca = tk; r.pca = sqrt(dr2);
            conj_push(out, &r);
        }
        return;
    }
    double vmin = sqrt(fmin(sa, sb));
    double tw = 2.0 * gc / vmin;
    uint32_t flags = 0;
    if (count_sign_changes(A, B, tk - tw, tk + tw, 64) > 1)
        flags |= ORC_MULTI;

    double ta = fmax(tk - 0.5 * dt, t0);
    double tb = fmin(tk + 0.5 * dt, t1);
    if (!(tb > ta)) return;
    const int NS = 32;
    double tprev = ta, gprev = orc_g(A, B, ta, NULL);
    for (int s = 1; s <= NS; ++s) {
        double t = ta + (tb - ta) * (double)s / (double)NS;
        double g = orc_g(A, B, t, NULL);
        if (gprev < 0.0 && g >= 0.0) {
            double lo = tprev, hi = t;
            for (int it = 0; it < 200 && hi - lo > 1e-10; ++it) {
                double mid = 0.5 * (lo + hi);
                if (orc_g(A, B, mid, NULL) < 0.0) lo = mid;
                else hi = mid;
            }
            double tca = 0.5 * (lo + hi);
            double D;
            orc_g(A, B, tca, &D);
            if (tca >= ta && tca < tb && D < d) {
                orc_conjunction r;
                r.i = c->i; r.j = c->j; r.step = c->step; r.flags = flags;
                r.tca = tca; r.pca = D;
                conj_push(out, &r);
            }
        }
        tprev = t;
        gprev = g;
    }
}

int64_t orc_conjunctions(const orc_elements* el, int64_t n, double t0, double t1, double dt,
                         double d, double gc, const orc_candidate* cand, int64_t ncand,
                         orc_conjunction** out)
{
    orc_orbit* o = orc_make_orbits(el, n);
    int nt = orc_threads();
    conj_buf* bufs = (conj_buf*)calloc((size_t)nt, sizeof(conj_buf));
#pragma omp parallel
    {
        conj_buf* mine = &bufs[orc_thread_id()];
#pragma omp for schedule(dynamic, 64)
        for (int64_t q = 0; q < ncand; ++q)
            orc_refine_one(o, &cand[q], t0, t1, dt, d, gc, mine);
    }
    free(o);
    int64_t total = 0;
    for (int q = 0; q < nt; ++q) total += bufs[q].n;
    orc_conjunction* r = (orc_conjunction*)malloc(sizeof(orc_conjunction) * (size_t)(total > 0 ? total : 1));
    int64_t off = 0;
    for (int q = 0; q < nt; ++q) {
        if (bufs[q].n) memcpy(r + off, bufs[q].p, sizeof(orc_conjunction) * (size_t)bufs[q].n);
        off += bufs[q].n;
        free(bufs[q].p);
    }
    free(bufs);
    qsort(r, (size_t)total, sizeof(orc_conjunction), cmp_conj);
    *out = r;
    return total;
}

/* D(t) and g(t) at arbitrary times for one pair (test helper: dense-sampling checks). */
void orc_pair_distance(const orc_elements* el, int64_t i, int64_t j, const double* t, int64_t nt,
                       double* D, double* g)
{
    orc_orbit A, B;
    orc_make_orbit(el, i, &A);
    orc_make_orbit(el, j, &B);
    for (int64_t q = 0; q < nt; ++q) {
        double dd;
        double gg = orc_g(&A, &B, t[q], &dd);
        if (D) D[q] = dd;
        if (g) g[q] = gg;
    }
}

/* R#14 test of one pair at time t: 1 iff |v_i - v_j| < 1e-9 km/s (D stationary); *D = D(t). */
int orc_pair_degenerate(const orc_elements* el, int64_t i, int64_t j, double t, double* D)
{
    orc_orbit A, B;
    orc_make_orbit(el, i, &A);
    orc_make_orbit(el, j, &B);
    double ra[3], va[3], rb[3], vb[3], dv2 = 0.0, dr2 = 0.0;
    orc_state(&A, t, ra, va);
    orc_state(&B, t, rb, vb);
    for (int q = 0; q < 3; ++q) {
        dv2 += (va[q] - vb[q]) * (va[q] - vb[q]);
        dr2 += (ra[q] - rb[q]) * (ra[q] - rb[q]);
    }
    if (D) *D = sqrt(dr2);
    return sqrt(dv2) < 1e-9;
}

void orc_free(void* p) { free(p); }

/* Flags of arbitrary candidates (test helper for parity exclusions): ORC_MULTI when g changes
 * sign more than once on [t_k - t_w, t_k + t_w], ORC_DEGENERATE when |v_i - v_j| < 1e-9 km/s
 * at t_k -- the same predicates orc_refine_one applies. */
void orc_candidate_flags(const orc_elements* el, int64_t n, double t0, double dt, double gc,
                         const orc_candidate* cand, int64_t ncand, uint32_t* flags)
{
    orc_orbit* o = orc_make_orbits(el, n);
#pragma omp parallel for schedule(dynamic, 16)
    for (int64_t q = 0; q < ncand; ++q) {
        const orc_orbit* A = &o[cand[q].i];
        const orc_orbit* B = &o[cand[q].j];
        double tk = orc_step_time((int64_t)cand[q].step, t0, dt);
        double ra[3], va[3], rb[3], vb[3];
        orc_state(A, tk, ra, va);
        orc_state(B, tk, rb, vb);
        double dv2 = 0.0, sa = 0.0, sb = 0.0;
        for (int c = 0; c < 3; ++c) {
            dv2 += (va[c] - vb[c]) * (va[c] - vb[c]);
            sa += va[c] * va[c];
            sb += vb[c] * vb[c];
        }
        uint32_t f = 0;
        if (sqrt(dv2) < 1e-9) {
            f |= ORC_DEGENERATE;
        } else {
            double tw = 2.0 * gc / sqrt(fmin(sa, sb));
            if (count_sign_changes(A, B, tk - tw, tk + tw, 64) > 1) f |= ORC_MULTI;
        }
        flags[q] = f;
    }
    free(o);
}
