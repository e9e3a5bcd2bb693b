/*
 * cdscreen.h -- C ABI of the B200-native conjunction-screening library (libcdscreen.so).
 *
 * Implements the data-parallel screening path of Hellwig, Czappa, Michel, Bertrand, Wolf,
 * "Satellite Collision Detection using Spatial Data Structures", IPDPS 2023:
 * per sampling step, propagate every object, hash its position into a
 * uniform grid of cell size g_c = d + 7.8 dt (Eq. 1) held in a non-blocking atomic
 * hash map (Eq. 2), scan each occupied cell and its 26 neighbours (P:62, P:95,
 * P:162), and refine every candidate's time and distance of closest approach with Brent's
 * method.  The hybrid variant reuses the grid as a coarse
 * pre-filter ahead of the apogee/perigee, orbit-path and time filters.
 *
 * Conventions for every call:
 *   Units      km, s, rad.  All floating point is IEEE fp64.
 *   Elements   osculating Kepler elements at epoch t = 0 (a, e, i, Omega, omega, true
 *              anomaly), structure of arrays, n entries each, caller-owned, read-only, never
 *              retained after the call returns.  Host pointers unless
 *              cd_options.inputs_on_device != 0 (then device pointers on cd_options.device).
 *   Steps      t_k = t0 + k dt (computed as fma(k, dt, t0)), k = 0 .. K-1,
 *              K = floor((t1 - t0)/dt) + 1 (P:242-246 o = t/s_ps; both ends included).
 *   Candidates (i, j, k), i < j, with |r_i(t_k) - r_j(t_k)| < g_c (strict).
 *   Conjunctions  local minima of D(t) = |r_i(t) - r_j(t)| with D < d (strict) and TCA in
 *              [t0, t1].  Each minimum is reported once, by its owner step
 *              k = floor((TCA - t0)/dt + 1/2) (the step whose half-open cell
 *              [t_k - dt/2, t_k + dt/2) contains it), and only if (i, j, k) is a candidate.
 *   Output     sorted by (i, j, step), i < j; identical for any thread schedule and
 *              independent of grid_origin and n_ranks (the union over ranks is the same set).
 *   Ownership  outputs are library-owned until released with the matching *_free call.
 *   Errors     every call returns cd_status; nothing throws across the ABI.  On error the output
 *              is {NULL, 0} and cd_last_error() (thread-local) explains.  CUDA errors map to
 *              CD_ECUDA with the driver's message.
 *   Threads    calls may be made from several host threads; each call uses its own stream and
 *              scratch memory.
 *   Streams    a call runs on cd_options.stream when given: device-resident inputs must be
 *              complete in that stream's order (e.g. written earlier on it), and device results
 *              are ready in its order when the call returns.  Without one the library runs on a
 *              stream of its own created blocking (cudaStreamDefault), so it is ordered after all
 *              work queued earlier on the legacy default stream.  With cd_options.alloc, the
 *              allocator's blocks are used on that same stream only.
 *   Memory     device scratch comes from cd_options.alloc when given, else from a private
 *              stream-ordered pool per device (the device's default pool is not touched) that
 *              keeps its memory between calls; a per-device cache keeps the largest result
 *              accumulation buffer (<= 1 GiB) between calls.  cd_release_caches() returns both.
 */
#ifndef CDSCREEN_H
#define CDSCREEN_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define CD_ABI_VERSION 3   /* 2: cd_options.propagator; 3: kepler_points honoured, cd_release_caches,
                              cd_stats.cell_factor / grid_table */

typedef enum {
    CD_OK = 0,
    CD_EINVAL = 1,    /* invalid argument (see validation rules below)                        */
    CD_ENOMEM = 2,    /* device or host allocation failed even after capacity retries         */
    CD_ECUDA = 3,     /* a CUDA runtime/driver error; cd_last_error() has the message          */
    CD_ENCCL = 4,     /* reserved: collective failure (the merge runs in the Python layer)     */
    CD_ERANGE = 5,    /* a position fell outside the key range +-(2^20 - 2) cells of the cell
                         edge L >= g_c per axis (>= +-104,857 km at g_c = 0.1 km)              */
    CD_EINTERNAL = 6, /* internal invariant violated                                           */
    CD_ENODEV = 7     /* no CUDA device / the library was not built for this device            */
} cd_status;

/* Propagator of the screen (two-body Kepler with the Contour solver [43]; P:333 names
 * "other propagators instead of the Kepler Contour solver" as future work). */
typedef enum {
    CD_PROP_KEPLER = 0, /* two-body Kepler, Contour solver (the paper's propagator)                */
    CD_PROP_J2 = 1      /* + first-order secular J2 drift of Omega, omega and M (Vallado &
                           McClain [41] Sec. 9.6; J2 = 1.08262668e-3, R_E = 6378.137 km):
                           dM/dt = n0 [1 + 1.5 k sqrt(1-e^2) (1 - 1.5 sin^2 i)],
                           dOmega/dt = -1.5 n0 k cos i, domega/dt = 0.75 n0 k (4 - 5 sin^2 i),
                           k = J2 (R_E / (a (1 - e^2)))^2, n0 = sqrt(mu/a^3); a, e, i constant.
                           Grid variant and cd_propagate only (the hybrid filters assume fixed
                           orbit planes: CD_HYBRID with CD_PROP_J2 is CD_EINVAL)                 */
} cd_propagator;

typedef enum {
    CD_GRID = 0,   /* grid-based variant                               */
    CD_HYBRID = 1, /* hybrid: coarse grid + orbital filter chain             */
    CD_LEGACY = 2  /* legacy full-window filter chain, no grid (P:43 filters, P:189 legacy variant,
                      P:315-318 accuracy comparison): every pair i < j passes apogee/perigee ->
                      coplanarity -> orbit path -> time windows over all of [t0, t1] (coplanar
                      pairs: all of [t0, t1]); the steps t_k inside the surviving intervals are
                      sampled and every minimum below d reported by its owner step, with no Eq. 1
                      speed assumption (gate d + (v_p,i + v_p,j) dt/2, perigee speeds): a superset
                      of CD_GRID's result.  O(n^2) pairs; cd_screen/cd_screen_ex only, Kepler
                      propagator only; pairs are split across ranks (n_ranks)                   */
} cd_mode;

/* Kepler elements, structure of arrays.  a > 0 [km], 0 <= e < 1, angles finite [rad]. */
typedef struct {
    const double* a;
    const double* e;
    const double* inc;
    const double* raan;
    const double* argp;
    const double* nu0; /* true anomaly at epoch t = 0 */
} cd_elements;

/* conjunction flags */
#define CD_FLAG_DEGENERATE 2u /* |v_i - v_j| < 1e-9 km/s at t_k: D stationary; tca = t_k, pca = D(t_k) */
#define CD_FLAG_COPLANAR 4u   /* hybrid: pair took the coplanar (grid-refinement) path        */

typedef struct {
    uint32_t i, j;   /* object indices into the element arrays, i < j            */
    uint32_t step;   /* owner step k                                              */
    uint32_t flags;  /* CD_FLAG_*                                                 */
    double tca;      /* time of closest approach [s from epoch]                   */
    double pca;      /* distance at closest approach [km]                        */
} cd_conjunction;    /* 32 B */

typedef struct {
    uint32_t i, j, step;
} cd_candidate;      /* 12 B: the level-1 set (parity hook) */

typedef struct {
    cd_conjunction* data; /* host memory, or device memory if cd_options.outputs_on_device */
    size_t count;
    void* _owner;         /* library bookkeeping; do not touch */
} cd_conjunctions;

/* Per-call statistics (all optional outputs). */
typedef struct {
    uint64_t steps;            /* sampling steps screened by this call (this rank's slice)    */
    uint64_t object_steps;     /* n * steps                                                    */
    uint64_t candidates;       /* |K| for this slice (hybrid: coarse candidates; legacy: pairs
                                  screened by this rank)                                      */
    uint64_t refined;          /* candidates that survived the conservative linear pre-filter
                                  (hybrid: time-window work items + coplanar candidates;
                                  legacy: surviving time-window intervals)                    */
    uint64_t conjunctions;     /* reported rows                                               */
    uint64_t hybrid_ap_rejected, hybrid_coplanar, hybrid_path_rejected, hybrid_time_rejected;
                               /* filter-stage counts (hybrid: per coarse candidate; legacy:
                                  per pair)                                                   */
    uint64_t kernel_launches;  /* CUDA kernels launched by this call                          */
    uint64_t retries;          /* capacity-overflow retries                                   */
    double ms_total;           /* device time of the call (CUDA events on the call's stream)  */
    /* per-phase device time and timed-launch counts, filled only when cd_options.profile_phases
       > 0 (CUDA events on the call's stream around every profile_phases-th launch of a phase;
       no extra syncs): average launch duration = ms_X / launches_X.  The fused step kernel is
       timed as one span per round (ms_scan / launches_scan = its pipelined launch period; its
       launches overlap under programmatic dependent launch), ms_propagate stays 0            */
    double ms_clear, ms_propagate, ms_insert, ms_scan, ms_refine, ms_finalize, ms_precompute;
    uint64_t launches_clear, launches_propagate, launches_insert, launches_scan, launches_refine;
    uint64_t step_launches;    /* all launches of the fused step kernel (timed or not)         */
    double cell_factor;        /* the cell edge L / g_c the call settled on (auto: chosen from the
                                  measured candidate density).  Passing it back as
                                  cd_options.cell_factor to the next call over the same population
                                  (e.g. the next time slice) skips that call's density-probe round */
    int grid_table;            /* the grid structure the call used: 1 open addressing, 2 chained,
                                  3 CSR (sort + segment)                                          */
    uint64_t grids_in_flight;  /* B: sampling steps per in-flight batch (the paper's p grids,
                                  P:236-252): min(batch_object_steps / n, what free memory holds) */
    uint64_t raw_pairs;        /* emit_raw_counts: pairs the scan examined (before the distance
                                  test); with cell_factor = 1 and grid_table = 1 this is the
                                  paper's count of object pairs in the same or neighbouring cells
                                  (each unordered pair once per step)                */
    uint64_t digest;           /* digest_only: sum mod 2^64 over the conjunctions of
                                  i * 0x9E3779B1 + j * 0x85EBCA77 + step * 0xC2B2AE3D (caller ids,
                                  i < j): order-independent, additive over time slices and ranks */
    uint64_t digest_conjunctions; /* digest_only: the number of conjunctions digested          */
    double min_pca;            /* digest_only: the smallest PCA [km] (+inf if none)            */
} cd_stats;

typedef struct {
    double v_margin;          /* Eq. 1 speed [km/s]; default 7.8; 0 => cell = d               */
    double grid_origin[3];    /* grid origin o [km]; default 0; results must not depend on it */
    int device;               /* CUDA device ordinal; -1 = current                            */
    void* stream;             /* cudaStream_t to run on; NULL = the library's own stream      */
    int rank, n_ranks;        /* time slicing: this call screens steps
                                 [floor(rank K / n_ranks), floor((rank+1) K / n_ranks));
                                 default 0, 1                                                 */
    int inputs_on_device;     /* element pointers are device pointers                         */
    int outputs_on_device;    /* cd_conjunctions.data stays in device memory                  */
    int kepler_points;        /* minimum Contour point count N (ref. [43]): 0 = per object
                                 from e (4 for e <= 0.01, 6 <= 0.1, 8 <= 0.3, 12 <= 0.6, 16 above;
                                 DESIGN.md R15); 4, 6, 8, 12 or 16 = at least that many points for
                                 every object (more accuracy, more fp64 work); else CD_EINVAL    */
    double cell_factor;       /* grid cell edge = cell_factor * g_c (>= 1); 1 = the paper's cell
                                 and 27-cell scan; default 0 = auto (chosen from the measured
                                 candidate density; results do not depend on it)               */
    size_t batch_object_steps;/* object-steps per in-flight step batch; 0 = auto              */
    size_t round_steps;       /* steps per refinement round; 0 = auto                         */
    int profile_phases;       /* N > 0: time every N-th launch of each phase into cd_stats     */
    int l2_persist;           /* pin the per-step grid tables in a persisting-L2 window (default
                                 0; raises cudaLimitPersistingL2CacheSize for the device)      */
    int grid_table;           /* per-step grid structure: 1 = the paper's open-addressing hash
                                 map (64-bit keys, linear probing, CAS, per-cell lists);
                                 2 = chained spatial hash (lists per hashed bucket, one atomic
                                 exchange per object); 3 = sort + segment (the open-addressing
                                 slots count each cell's objects, a counting sort by cell makes
                                 each cell one contiguous segment); 0 = default (2; in
                                 half-shell mode 3 once the measured candidate rate reaches 3
                                 per object-step -- crowded cells).
                                 Results are identical; other values CD_EINVAL.                  */
    cd_stats* stats;          /* optional output                                              */
    int propagator;           /* cd_propagator; default CD_PROP_KEPLER                        */
    double shell_lo, shell_hi;/* radial shard [km] (object-space sharding for
                                 populations whose per-step grid exceeds one GPU).  shell_hi = 0:
                                 no shard (default).  Otherwise the call keeps exactly the
                                 candidates whose smaller radius |r| at t_k lies in
                                 [shell_lo, shell_hi) -- positions are bit-identical on every
                                 shard, so the shards of a partition of [0, inf) report disjoint
                                 sets whose union is the unsharded result -- provided the
                                 elements passed are the shard's members (cd_shell_members: own
                                 objects plus the g_c halo above the band).  CD_GRID/CD_HYBRID. */
    /* Device scratch memory of the call (PyTorch supplies memory).  When alloc and
       free are set (both or neither: CD_EINVAL), every device buffer of the call -- orbit
       records, grid arena, queues, sort scratch, results -- comes from alloc(bytes, alloc_ctx)
       (NULL = out of memory -> CD_ENOMEM / CD_ECUDA) and is returned with free(p, alloc_ctx);
       all use is ordered on the call's stream, so a stream-ordered caching allocator on that
       stream (e.g. torch.cuda.caching_allocator_alloc) may reuse a freed block at once.  Device
       results (outputs_on_device) are released with the same free in cd_conjunctions_free, so
       the allocator must outlive them.  NULL (default): the device's stream-ordered pool.     */
    void* (*alloc)(size_t bytes, void* ctx);
    void (*free)(void* p, void* ctx);
    void* alloc_ctx;
    int shards;               /* radial shards screened in turn on this device (CD_GRID and
                                 CD_HYBRID without a shell band): the objects are split into S
                                 radial bands (quantiles of a), each screened with only its
                                 members (the shell_lo/hi rule), so a call's grid memory scales
                                 with n/S plus the halo; the union is exactly the unsharded
                                 result.  0 or 1 = off (default; at 8M objects on one B200 the
                                 bands were measured 1-14 % slower), <= 64                        */
    int resort_steps;         /* spatial slot order: every R sampling steps the objects are
                                 renumbered in Morton order of their current position, so the
                                 grid accesses of neighbouring threads are neighbours in memory
                                 (results do not depend on it).  0 = auto (default: every
                                 max(16, 64 s / dt) steps for >= 4M objects in CD_GRID, else
                                 off), < 0 = off, R > 0 = every R steps                         */
    int emit_raw_counts;      /* also count the pairs the scan examines into cd_stats.raw_pairs
                                 (the paper's raw count with cell_factor = 1, grid_table = 1;
                                 P:95); default 0                                   */
    int digest_only;          /* 1: do not return the conjunctions -- fold each round's records
                                 into cd_stats.digest / digest_conjunctions / min_pca on the
                                 device and reuse the buffer (for screens whose result does not
                                 fit memory, e.g. 8M objects x 7 days: ~4e9 records);
                                 the result is {NULL, 0}.  CD_GRID / CD_HYBRID without in-library
                                 shards; default 0                                               */
} cd_options;

/* Fill *opt with the defaults above. */
void cd_options_init(cd_options* opt);

/* Screen n objects over [t0, t1] at sampling step dt with threshold d.
 * mode = CD_GRID:   g_c = d + v_margin*dt, candidates refined by Brent's method on
 *                   [t_k - t_w, t_k + t_w], t_w = 2 g_c / min(|v_i|, |v_j|).
 * mode = CD_HYBRID: same grid at the (coarse) dt given; candidates pass the apogee/perigee,
 *                   coplanarity, orbit-path and time filters; survivors are refined inside
 *                   their time windows.
 * Validation (CD_EINVAL): elements non-NULL, 2 <= n < 2^32 - 1 (n = 0 or 1 returns an empty
 * result), a > 0, 0 <= e < 1, finite angles, dt > 0, t1 >= t0, d > 0, K < 2^32,
 * cell_factor >= 1, 0 <= rank < n_ranks.  out must be non-NULL. */
cd_status cd_screen(const cd_elements* el, size_t n, double t0, double t1, double dt, double d,
                    cd_mode mode, cd_conjunctions* out);
cd_status cd_screen_ex(const cd_elements* el, size_t n, double t0, double t1, double dt, double d,
                       cd_mode mode, const cd_options* opt /* nullable */, cd_conjunctions* out);

/* The level-1 candidate set K for [t0, t1] at step dt with g_c = d + v_margin*dt
 * (mode is accepted for symmetry; the set does not depend on it).  *out is a library-owned
 * host array of *count entries sorted by (i, j, step); release with cd_candidates_free. */
cd_status cd_candidates(const cd_elements* el, size_t n, double t0, double t1, double dt, double d,
                        cd_mode mode, const cd_options* opt, cd_candidate** out, size_t* count);

/* Positions (and optionally velocities) of all n objects at nt times.  xyz (and vxyz, nullable)
 * are caller-owned host buffers of nt*n*3 doubles, layout [time][object][x,y,z]. */
cd_status cd_propagate(const cd_elements* el, size_t n, const double* t, size_t nt, double* xyz,
                       double* vxyz, const cd_options* opt /* nullable */);

/* Sort n conjunction records that live in device memory by (i, j, step), in place, on `stream`
 * (cudaStream_t; NULL = the legacy default stream).  Used to merge per-rank time slices after
 * an all-gather.  Requires i < j in every record. */
cd_status cd_conjunctions_sort_device(cd_conjunction* data, size_t n, void* stream);

/* Release a result of cd_screen / cd_screen_ex.  Host results are freed immediately.  Device
 * results (outputs_on_device) are released stream-ordered (cudaFreeAsync) on the stream the call
 * ran on (cd_options.stream, or the legacy default stream when the library used its own), so
 * work the caller queued on that stream may still read them; no device-wide synchronisation. */
void cd_conjunctions_free(cd_conjunctions* c);

/* A-priori sizing of a screen (Section IV-B), pure host arithmetic: the
 * paper's Extra-P candidate models and its memory-bounded grid count, evaluated for this
 * library's data structures.  The library uses est_candidates_per_step to size a call's first
 * round (queue capacity, probe length, initial cell edge) before any density is measured. */
typedef struct {
    double samples;                 /* o = K = floor((t1 - t0)/dt) + 1 sampling steps (R4)   */
    double est_candidates;          /* c' over [t0, t1]: Eq. 3 (grid) 2.32e-9 n^2 s^(4/3) t d^(7/4),
                                       Eq. 4 (hybrid) 2.14e-9 n^2 s^(5/3) t d; s = dt [s],
                                       t = t1 - t0 [s] (dt if 0), d [km]                 */
    double est_candidates_per_step; /* c' with t = dt                                                */
    double capacity;                /* c = max(c', 10^4) * 2 * 2                             */
    double capacity_bytes;          /* g_ch = c * 16 B                                       */
    double fixed_bytes;             /* a_s + a_k + a_ch of this library: elements (48 B/object),
                                       orbit records (85 B/object), first-round candidate queue
                                       (12 B/entry) and work items (24 B/entry)                      */
    double bytes_per_grid;          /* a_gh + a_l: one step's grid table + 32 B entries per object   */
    double grids_in_memory;         /* p = (m - a_s - a_k - a_ch) / (a_gh + a_l)             */
    double rounds;                  /* r_c = o / p; +inf if p = 0                            */
    double cell_factor;             /* the auto cell edge L / g_c for the a-priori density           */
} cd_plan_info;

/* Fill *out for screening n objects over [t0, t1] at step dt, threshold d, in mode, with
 * mem_bytes of free device memory m (0 = query the current device: CD_ENODEV without one).
 * Validation as cd_screen (CD_EINVAL); out must be non-NULL. */
cd_status cd_plan(size_t n, double t0, double t1, double dt, double d, cd_mode mode,
                  size_t mem_bytes, cd_plan_info* out);
/* Members of the radial shard [shell_lo, shell_hi) (cd_options.shell_lo/hi): the indices i, in
 * increasing order, whose radius range [a(1-e), a(1+e)] meets [shell_lo, shell_hi + gc) --
 * every object that can be the nearer-to-Earth partner of a pair kept by the shard, or within
 * g_c of one.  Host element pointers; idx is a caller-owned array of n entries; *count is set.
 * Pure host arithmetic.  CD_EINVAL on NULL arguments, shell_hi <= shell_lo, invalid elements. */
cd_status cd_shell_members(const cd_elements* el, size_t n, double shell_lo, double shell_hi,
                           double gc, uint32_t* idx, size_t* count);
void cd_candidates_free(cd_candidate* c);
/* Release the library's cached device memory of `device` (-1: every device used so far): trim
 * its private stream-ordered pool to zero (after a device synchronisation) and free the cached
 * result accumulation buffer.  Results still held by the caller stay valid.  CD_EINVAL for a
 * device out of range; CD_OK without any device. */
cd_status cd_release_caches(int device);
const char* cd_status_str(cd_status s);
const char* cd_last_error(void);
int cd_abi_version(void);
/* Total CUDA kernels launched by this process through the library (diagnostic). */
uint64_t cd_kernel_launches(void);

#ifdef __cplusplus
}
#endif
#endif /* CDSCREEN_H */
