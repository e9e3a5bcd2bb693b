/* cd_oracle.h -- TEST INFRASTRUCTURE ONLY.  Private header of the CPU oracle (oracle/*.c).
 * Shares nothing with include/cdscreen.h or the CUDA sources. */
#ifndef CD_ORACLE_H
#define CD_ORACLE_H
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

enum { ORC_PROP_KEPLER = 0, ORC_PROP_J2 = 1 };

typedef struct {
    const double *a, *e, *inc, *raan, *argp, *nu0; /* km, -, rad, rad, rad, rad */
    int model;                                     /* ORC_PROP_KEPLER or ORC_PROP_J2 */
} orc_elements;

typedef struct { uint32_t i, j, step; } orc_candidate;

enum { ORC_MULTI = 1u, ORC_DEGENERATE = 2u, ORC_COPLANAR = 4u };
/* hybrid filter outcomes (orc_pair_filter) */
enum { ORC_H_AP = 1, ORC_H_COPLANAR = 2, ORC_H_PATH = 4, ORC_H_TIME = 8 };

typedef struct {
    uint32_t i, j, step, flags;
    double tca, pca;
} orc_conjunction;

double  orc_mu(void);
double  orc_j2(void);
double  orc_earth_radius(void);
int     orc_num_threads(void);
double  orc_kepler_newton(double M, double e);
int64_t orc_num_steps(double t0, double t1, double dt);
void    orc_propagate(const orc_elements* el, int64_t n, const double* t, int64_t nt,
                      double* xyz, double* vxyz);
int64_t orc_candidates_brute(const orc_elements* el, int64_t n, double t0, double t1, double dt,
                             double gc, int64_t k_begin, int64_t k_end, orc_candidate** out);
int64_t orc_candidates_grid(const orc_elements* el, int64_t n, double t0, double t1, double dt,
                            double gc, double cell, const double origin[3],
                            int64_t k_begin, int64_t k_end, orc_candidate** out);
int64_t orc_conjunctions(const orc_elements* el, int64_t n, double t0, double t1, double dt,
                         double d, double gc, const orc_candidate* cand, int64_t ncand,
                         orc_conjunction** out);
void    orc_pair_distance(const orc_elements* el, int64_t i, int64_t j, const double* t, int64_t nt,
                          double* D, double* g);
int     orc_pair_degenerate(const orc_elements* el, int64_t i, int64_t j, double t, double* D);
void    orc_candidate_flags(const orc_elements* el, int64_t n, double t0, double dt, double gc,
                            const orc_candidate* cand, int64_t ncand, uint32_t* flags);
int     orc_pair_filter(const orc_elements* el, int64_t i, int64_t j, double d, double tlo,
                        double thi, double* iv, int cap, int* niv);
int64_t orc_hybrid(const orc_elements* el, int64_t n, double t0, double t1, double dt, double d,
                   double gc, int64_t k_begin, int64_t k_end, void** out, int64_t* counts);
int64_t orc_legacy(const orc_elements* el, int64_t n, double t0, double t1, double dt, double d,
                   void** out, int64_t* counts);
void    orc_free(void* p);

#ifdef __cplusplus
}
#endif
#endif
