// cd_kernels.cu -- CUDA kernels of the screening hot path (sm_100a, fp64, no tensor cores).
//
//   a1 precompute     k_classify, k_build_records   ("precalculating the reusable
//                                                     parts ... once", P:236 a_k)
//   a2-a4 propagate + cell key + hash insert        k_prop_insert  (Eq. 2)
//   a5-a6 27-cell neighbour scan + candidate queue  k_scan
//   a7 refinement     k_prefilter (conservative linear bound), k_brent
#include <cooperative_groups.h>

#include "cd_internal.h"
#include "cd_refine.cuh"

namespace cg = cooperative_groups;
using namespace cdk;

namespace cdh {

std::atomic<uint64_t> g_launches{0};
thread_local DevAlloc g_dev_alloc;
thread_local cudaMemPool_t g_pool = nullptr;

static inline unsigned blocks_for(int64_t n, int t) { return (unsigned)((n + t - 1) / t); }

// Launch with an optional persisting-L2 access-policy window (per-launch attribute).
// With pdl, the launch may begin while the previous kernel in the stream is still running
// (programmatic dependent launch); the kernel orders its dependent part with griddepcontrol.wait.
template <typename... KArgs, typename... Args>
static cudaError_t launch_ex(void (*kern)(KArgs...), dim3 grid, dim3 block, size_t smem,
                             cudaStream_t st, const L2Win* win, bool pdl, Args... args)
{
    const bool w = win && win->on;
    if (!w && !pdl) {
        kern<<<grid, block, smem, st>>>(args...);
        return cudaGetLastError();
    }
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = grid;
    cfg.blockDim = block;
    cfg.dynamicSmemBytes = smem;
    cfg.stream = st;
    cudaLaunchAttribute at[2];
    unsigned na = 0;
    if (w) {
        at[na].id = cudaLaunchAttributeAccessPolicyWindow;
        at[na++].val.accessPolicyWindow = win->w;
    }
    if (pdl) {
        at[na].id = cudaLaunchAttributeProgrammaticStreamSerialization;
        at[na++].val.programmaticStreamSerializationAllowed = 1;
    }
    cfg.attrs = at;
    cfg.numAttrs = na;
    return cudaLaunchKernelEx(&cfg, kern, args...);
}

__device__ __forceinline__ void pdl_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }
__device__ __forceinline__ void pdl_trigger() { asm volatile("griddepcontrol.launch_dependents;" :::); }

__device__ __forceinline__ void append_count(unsigned long long* cnt)
{
    cg::coalesced_group g = cg::coalesced_threads();
    if (g.thread_rank() == 0) atomicAdd(cnt, (unsigned long long)g.size());
}

// ---------------------------------------------------------------------------------------
// a1: per-object precompute
// ---------------------------------------------------------------------------------------
// min_cls: the class of cd_options.kepler_points (0 = per e only); an object takes the larger of
// its eccentricity class and min_cls, i.e. at least the requested Contour point count
__global__ void k_classify(Elements el, int64_t n, uint32_t* key, uint32_t* idx,
                           unsigned long long* n0, int min_cls)
{
    const int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (i >= n) return;
    const int cl = max(ecc_class(el.e[i]), min_cls);
    key[i] = (uint32_t)cl;
    idx[i] = (uint32_t)i;
    if (cl == 0) append_count(n0);
}

__device__ __forceinline__ void build_record(const Elements& el, const uint32_t* __restrict__ perm, int64_t n,
                                             int64_t r, double* __restrict__ rec, double* trow,
                                             uint8_t* __restrict__ cls, int j2, int min_cls)
{
    const uint32_t i = perm[r];
    const double a = el.a[i], e = el.e[i], inc = el.inc[i];
    const double raan = el.raan[i], argp = el.argp[i], nu0 = el.nu0[i];
    double sO, cO, sw, cw, si, ci;
    sincos(raan, &sO, &cO);
    sincos(argp, &sw, &cw);
    sincos(inc, &si, &ci);
    // perifocal unit vectors (Fig. 8: rotation by Omega, i, omega)
    const double P[3] = {cO * cw - sO * sw * ci, sO * cw + cO * sw * ci, sw * si};
    const double Q[3] = {-cO * sw - sO * cw * ci, -sO * sw + cO * cw * ci, cw * si};
    const double b = a * sqrt((1.0 - e) * (1.0 + e));
    // true anomaly at epoch -> eccentric -> mean anomaly
    double sh, ch;
    sincos(0.5 * nu0, &sh, &ch);
    const double E0 = 2.0 * atan2(sqrt(1.0 - e) * sh, sqrt(1.0 + e) * ch);
    const double M0 = E0 - e * sin(E0);
    // column-major (the per-step build) and object-major (the refinement's gathers)
    auto put = [&](int c, double v) {
        rec[c * n + r] = v;
        trow[c] = v;
    };
    put(kM0, M0);
    const double n0 = sqrt(kMu / (a * a * a));
    if (j2) {
        // J2 secular rates (Vallado & McClain [41] Sec. 9.6):
        //   k = J2 (R_E / p)^2, p = a (1 - e^2)
        //   dM/dt = n0 [1 + 1.5 k sqrt(1 - e^2) (1 - 1.5 sin^2 i)], dOmega/dt = -1.5 n0 k cos i,
        //   domega/dt = 0.75 n0 k (4 - 5 sin^2 i)
        const double sq = sqrt((1.0 - e) * (1.0 + e));
        const double rp = kRe / (a * (1.0 - e) * (1.0 + e));
        const double k = kJ2 * rp * rp;
        put(kNm, n0 * (1.0 + 1.5 * k * sq * (1.0 - 1.5 * si * si)));
        put(kDOm, -1.5 * n0 * k * ci);
        put(kDw, 0.75 * n0 * k * (4.0 - 5.0 * si * si));
        put(kBA, sq);
        put(kAB, 1.0 / sq);
    } else {
        put(kNm, n0);
    }
    put(kE, e);
    put(kAPx, a * P[0]); put(kAPy, a * P[1]); put(kAPz, a * P[2]);
    put(kBQx, b * Q[0]); put(kBQy, b * Q[1]); put(kBQz, b * Q[2]);
    put(kQper, a * (1.0 - e));
    const int cl = max(ecc_class(e), min_cls);
    cls[r] = (uint8_t)cl;
    trow[kAoSCls] = (double)cl;
    trow[kAoS - 1] = 0.0;
    if (!j2)
        for (int c = kDOm; c < kAoSCls; ++c) trow[c] = 0.0;
}


__global__ void k_build_records(Elements el, const uint32_t* __restrict__ perm, int64_t n,
                                double* __restrict__ rec, double* __restrict__ arec,
                                uint8_t* __restrict__ cls, int j2, int min_cls)
{
    // the object-major copy is staged in shared memory and written by the block as one
    // contiguous run (a thread's own 16 doubles at a 128-byte stride had cost 73 us per 1M)
    constexpr int kB = 128;   // threads per block (launch_build_records)
    __shared__ double tile[kB][kAoS + 1];
    const int64_t r0 = blockIdx.x * (int64_t)kB;
    const int64_t r = r0 + threadIdx.x;
    if (r < n) build_record(el, perm, n, r, rec, tile[threadIdx.x], cls, j2, min_cls);
    __syncthreads();
    const int64_t m = n - r0 < kB ? n - r0 : (int64_t)kB;
    for (int k = threadIdx.x; k < m * kAoS; k += kB) arec[r0 * kAoS + k] = tile[k / kAoS][k % kAoS];
}

__global__ void k_propagate_out(Orbits O, const uint32_t* __restrict__ perm,
                                const double* __restrict__ t, int64_t nt, double* xyz, double* vxyz)
{
    const int64_t r = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    const int64_t q = blockIdx.y;
    if (r >= O.n || q >= nt) return;
    double p[3], v[3];
    const int64_t o = (q * O.n + perm[r]) * 3;
    if (vxyz) {
        state<true>(O, r, t[q], p, v);
        vxyz[o] = v[0]; vxyz[o + 1] = v[1]; vxyz[o + 2] = v[2];
    } else {
        state<false>(O, r, t[q], p, v);
    }
    xyz[o] = p[0]; xyz[o + 1] = p[1]; xyz[o + 2] = p[2];
}

cudaError_t launch_classify(const Elements& el, int64_t n, uint32_t* key, uint32_t* idx,
                            unsigned long long* n0, int min_cls, cudaStream_t st, LaunchCount& lc)
{
    k_classify<<<blocks_for(n, 256), 256, 0, st>>>(el, n, key, idx, n0, min_cls);
    lc.bump();
    return cudaGetLastError();
}

cudaError_t launch_build_records(const Elements& el, const uint32_t* perm, int64_t n, double* rec,
                                 double* arec, uint8_t* cls, int j2, int min_cls, cudaStream_t st,
                                 LaunchCount& lc)
{
    k_build_records<<<blocks_for(n, 128), 128, 0, st>>>(el, perm, n, rec, arec, cls, j2, min_cls);
    lc.bump();
    return cudaGetLastError();
}

cudaError_t launch_propagate_out(const Orbits& O, const uint32_t* perm, const double* t, int64_t nt,
                                 double* xyz, double* vxyz, cudaStream_t st, LaunchCount& lc)
{
    for (int64_t q0 = 0; q0 < nt; q0 += 65535) {
        const int64_t m = nt - q0 < 65535 ? nt - q0 : 65535;
        dim3 grid(blocks_for(O.n, 128), (unsigned)m);
        k_propagate_out<<<grid, 128, 0, st>>>(O, perm, t + q0, m, xyz + q0 * O.n * 3,
                                             vxyz ? vxyz + q0 * O.n * 3 : nullptr);
        lc.bump();
    }
    return cudaGetLastError();
}

// ---------------------------------------------------------------------------------------
// radial L2 shards (screen_sharded in cd_api.cu): member gather, id composition, id mapping
// ---------------------------------------------------------------------------------------
__global__ void k_gather_elements(Elements src, const uint32_t* __restrict__ idx, int64_t m,
                                  double* __restrict__ dst)
{
    const int64_t r = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (r >= m) return;
    const uint32_t i = idx[r];
    dst[r] = src.a[i];
    dst[m + r] = src.e[i];
    dst[2 * m + r] = src.inc[i];
    dst[3 * m + r] = src.raan[i];
    dst[4 * m + r] = src.argp[i];
    dst[5 * m + r] = src.nu0[i];
}

__global__ void k_compose_perm(uint32_t* __restrict__ perm, const uint32_t* __restrict__ idx, int64_t m)
{
    const int64_t r = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (r < m) perm[r] = idx[perm[r]];
}

__global__ void k_conj_to_global(const Conj* __restrict__ in, size_t n, const uint32_t* __restrict__ perm,
                                 Conj* __restrict__ out)
{
    const size_t k = blockIdx.x * (size_t)blockDim.x + threadIdx.x;
    if (k >= n) return;
    Conj c = in[k];
    const uint32_t a = perm[c.i], b = perm[c.j];
    c.i = a < b ? a : b;
    c.j = a < b ? b : a;
    out[k] = c;
}

cudaError_t launch_gather_elements(const Elements& src, const uint32_t* idx, int64_t m, double* dst,
                                   cudaStream_t st, LaunchCount& lc)
{
    if (m <= 0) return cudaSuccess;
    k_gather_elements<<<blocks_for(m, 256), 256, 0, st>>>(src, idx, m, dst);
    lc.bump();
    return cudaGetLastError();
}

cudaError_t launch_compose_perm(uint32_t* perm, const uint32_t* idx, int64_t m, cudaStream_t st,
                                LaunchCount& lc)
{
    if (m <= 0) return cudaSuccess;
    k_compose_perm<<<blocks_for(m, 256), 256, 0, st>>>(perm, idx, m);
    lc.bump();
    return cudaGetLastError();
}

cudaError_t launch_conj_to_global(const Conj* in, size_t n, const uint32_t* perm, Conj* out,
                                  cudaStream_t st, LaunchCount& lc)
{
    if (n == 0) return cudaSuccess;
    k_conj_to_global<<<blocks_for((int64_t)n, 256), 256, 0, st>>>(in, n, perm, out);
    lc.bump();
    return cudaGetLastError();
}

// ---------------------------------------------------------------------------------------
// a2-a4: build -- one thread per (object, step) ("one thread per tuple"): Contour Kepler
// solve and Cartesian position, cell key, non-blocking insert into the step's hash grid
// (Eq. 2) and its occupancy bitmap; the entry {x, y, z, next} (Fig. 6) is
// written once, coalesced.  kClass0: objects [0, n0) (e <= 0.01: lean N = 4 Contour path).
// ---------------------------------------------------------------------------------------
// Grid structures (cd_options.grid_table): kOpen = the paper's open-addressing map with per-cell
// lists, kChained = chained spatial hash, kCsr = open-addressing map of per-cell counts plus a
// counting sort of the entries by cell (sort + segment: each cell's objects contiguous).
enum GridKind : int { kOpen = 0, kChained = 1, kCsr = 2, kChainedBall = 3, kChainedLean = 4, kChainedBallLean = 5,
                      kChainedBallLeanSig = 6 };
// kChainedBall: the chained grid compiled for ball-mode scans only (the grid variant's hot
// instance: the half-shell branch's code had cost its ball-mode scan 3 % -- 59.7 vs 61.6 us per
// 1M-object step -- through register allocation)
// kChainedLean / kChainedBallLean / kChainedBallLeanSig: the chained scans without the shard band
// and raw counts (ball mode also without candidate staging; see test_pair's flavours), chosen
// when none of those is active; kChainedLean without the spatial order's slot map
__host__ __device__ constexpr bool is_chained(int k) { return k >= kChained && k != kCsr; }

// CSR grid insert: claim the cell's slot (128-bit CAS from a stale slot to {key, tag | 1}) or
// count the object into it (64-bit atomicAdd on the head word; count in the low 32 bits).
// Returns the slot; *rank = the object's position among its cell's objects.
__device__ __forceinline__ uint32_t grid_count(Slot* slots, uint64_t mask, unsigned long long key,
                                               uint32_t tag, uint32_t* rank)
{
    const unsigned long long th = (unsigned long long)tag << 32;
    uint64_t h = fmix64(key) & mask;
    while (true) {
        unsigned long long w0, w1;
        asm volatile("ld.relaxed.gpu.global.v2.u64 {%0, %1}, [%2];" : "=l"(w0), "=l"(w1) : "l"(slots + h));
        while (true) {
            const bool stale = (uint32_t)(w1 >> 32) != tag;
            if (!stale && w0 != key) break;   // another cell of this pass: next slot (Eq. 2)
            if (!stale) {
                *rank = (uint32_t)atomicAdd(&slots[h].head, 1ull);
                return (uint32_t)h;
            }
            if (cas128(slots + h, w0, w1, key, th | 1ull)) {
                *rank = 0;
                return (uint32_t)h;
            }
        }
        h = (h + 1) & mask;
    }
}

template <bool kClass0, int kGrid, int kJ2>
__device__ __forceinline__ void do_build(const Orbits& O, const GridGeom& g, const GridTab& tab,
                                         Entry* __restrict__ ents, uint64_t mask, int64_t k0, int s,
                                         int64_t r, double t0, double dt, uint32_t tag, Ctrl* ctrl)
{
    const double t = fma((double)(k0 + s), dt, t0);
    double p[3], v[3];
    state<false, kClass0 ? 0 : -1, kJ2>(O, r, t, p, v);
    int c[3];
    uint32_t next = kNil, ctag = 0;
    if (kGrid == kCsr && cell_of(g, p, c)) {
        // counting insert; the entry (slot, rank) is scattered to its cell's segment later
        const uint32_t hb = bit_hash(c[0], c[1], c[2]) & tab.bmask;
        atomicOr(tab.bits + (size_t)s * tab.bwords + (hb >> 5), 1u << (hb & 31));
        next = grid_count(tab.slots + (size_t)s * (mask + 1), mask, pack_key(c[0], c[1], c[2]), tag, &ctag);
    } else if (is_chained(kGrid) && cell_of(g, p, c)) {
        ctag = cell_tag(c[0], c[1], c[2]);
        // chained spatial hash: push onto the list of bucket hash(cell) -- one atomic exchange;
        // heads hold index + 1 (0 = empty bucket)
        const uint32_t b = chain_bucket(c[0], c[1], c[2], tab.bmask);
        const uint32_t prev = atomicExch(tab.bits + (size_t)s * tab.bwords + b,
                                         (tag << kEpochShift) | ((uint32_t)r + 1u));
        next = ((prev >> kEpochShift) == tag && (prev & kIdxMask)) ? (prev & kIdxMask) - 1u : kNil;
    } else if (kGrid == kOpen && cell_of(g, p, c)) {
        const unsigned long long key = pack_key(c[0], c[1], c[2]);
        const uint32_t hb = bit_hash(c[0], c[1], c[2]) & tab.bmask;
        atomicOr(tab.bits + (size_t)s * tab.bwords + (hb >> 5), 1u << (hb & 31));
        next = grid_insert(tab.slots + (size_t)s * (mask + 1), mask, key, tag, (uint32_t)r);
    } else {
        ctrl->err_range = 1;
    }
    Entry en;
    en.x = p[0];
    en.y = p[1];
    en.z = p[2];
    en.next = next;
    en.tag = ctag;
    ents[(size_t)s * O.n + r] = en;
}

// ---------------------------------------------------------------------------------------
// a5-a6: neighbour scan, one thread per (object, step).
//  (1) own cell: walk the object's own list successors -- every same-cell pair is seen exactly
//      once, by the later-inserted object (no probe needed);
//  (2) other cells: half-shell mode (L < 2 g_c, the paper's cell g_c) probes those of
//      the 13 positive half-shell neighbours -- each unordered pair of cells of a 3x3x3 block once
//      -- that lie within reach of the object (halfshell_reach);
//      ball mode (L >= 2 g_c) probes those of the 0-7 other cells overlapping |x - p| < g_c
//      that lie in the positive (lexicographic) half-space of the own cell -- a pair in two
//      cells is seen only from the smaller cell.  Each probe first tests the occupancy bitmap
//      (all bitmap loads of a thread are issued together).
// A pair is a candidate iff |r_i - r_j| < g_c (reading R6); candidates are appended with one
// atomic per group of converged lanes (P:95 saves ids + sampling step).
// ---------------------------------------------------------------------------------------
__constant__ int8_t kHalfShell[14][3] = {
    {0, 0, 0},
    {1, -1, -1}, {1, -1, 0}, {1, -1, 1}, {1, 0, -1}, {1, 0, 0}, {1, 0, 1}, {1, 1, -1}, {1, 1, 0}, {1, 1, 1},
    {0, 1, -1}, {0, 1, 0}, {0, 1, 1},
    {0, 0, 1}};

// Half-shell offsets o = 1..13 whose cell can hold a point within the reach of p: the squared
// distance from p to the cell, per axis 0 (same layer), fr^2 (offset -1) or (1 - fr)^2 (+1) in
// cell units, below rl^2 (rl = reach / L).  Conservative like ball mode: reach = g_c (1 + 1e-9) +
// 1e-9 km exceeds the rounding of fr by orders of magnitude.  (Offsets in kHalfShell's order.)
__device__ __forceinline__ uint32_t halfshell_reach(const double fr[3], double rl)
{
#ifdef CD_NO_HS_PRUNE
    return 0x3FFEu;
#endif
    const double r2 = rl * rl;
    const double x1 = (1.0 - fr[0]) * (1.0 - fr[0]);
    const double ys[3] = {fr[1] * fr[1], 0.0, (1.0 - fr[1]) * (1.0 - fr[1])};
    const double zs[3] = {fr[2] * fr[2], 0.0, (1.0 - fr[2]) * (1.0 - fr[2])};
    uint32_t m = 0;
#pragma unroll
    for (int o = 1; o <= 9; ++o) m |= (x1 + ys[(o - 1) / 3] + zs[(o - 1) % 3] < r2 ? 1u : 0u) << o;
#pragma unroll
    for (int o = 10; o <= 12; ++o) m |= (ys[2] + zs[o - 10] < r2 ? 1u : 0u) << o;
    m |= (zs[2] < r2 ? 1u : 0u) << 13;
    return m;
}

// Warp-level candidate staging (role-C warps of k_step, GridGeom::stage): each warp appends its
// candidates to its own slice of a shared buffer with a shared-memory atomic and flushes them to
// the global queue with one global atomic per warp; a full slice falls back to the
// warp-aggregated global append.  A dense coarse grid (the hybrid's 1.4 candidates per
// object-step) otherwise serialises on the queue counter (hybrid k_step 556 -> 284 us per
// 1M-object step with block-level staging, and a warp-level flush drops the block barrier at the
// end); a sparse one (the grid variant's 0.004) does not need it.
// The buffer is dynamic shared memory, requested only for staged launches: a sparse step keeps
// the whole L1 (static shared memory here cost the grid variant 3 %).
constexpr unsigned kSCand = 1024;              // per block (256 threads)
constexpr unsigned kSWarp = kSCand / 8;        // per warp
extern __shared__ Cand s_cand[];
__shared__ unsigned s_nw[8];
__shared__ unsigned s_rw[8];   // per warp: pairs examined (emit_raw_counts)

// test_pair flavours (bit flags; separate instances so the unused features cost no registers):
// kTpLean = no radial shard band and no raw counts, kTpNoStage = no candidate staging (sparse
// ball-mode grids), kTpSig = the slot -> id map of the spatial order (lean instances only; the
// full one reads it at run time)
constexpr int kTpLean = 1, kTpNoStage = 2, kTpSig = 4;
template <int kLean = 0>
__device__ __forceinline__ void test_pair(const GridGeom& g, uint32_t r, uint32_t j, const double p[3],
                                          const Entry& ej, uint32_t step, Cand* __restrict__ q,
                                          size_t qcap, Ctrl* ctrl)
{
    if (!(kLean & kTpLean) && g.raw) atomicAdd(&s_rw[threadIdx.x >> 5], 1u);
    const double dx = p[0] - ej.x, dy = p[1] - ej.y, dz = p[2] - ej.z;
    if (fma(dx, dx, fma(dy, dy, dz * dz)) < g.gc2) {
        // radial shard: the pair belongs to the shard holding the smaller radius (identical
        // positions on every shard, so exactly one shard keeps it)
        if (!(kLean & kTpLean)) {
            const double ra = fma(p[0], p[0], fma(p[1], p[1], p[2] * p[2]));
            const double rb = fma(ej.x, ej.x, fma(ej.y, ej.y, ej.z * ej.z));
            const double rm = fmin(ra, rb);
            if (!(rm >= g.band_lo2 && rm < g.band_hi2)) return;
        }
        constexpr bool kSigRt = !(kLean & kTpLean) || (kLean & kTpSig);   // slots -> internal ids
        const uint32_t a = kSigRt && g.sig ? g.sig[r] : r, b = kSigRt && g.sig ? g.sig[j] : j;
        Cand cd;
        cd.i = a < b ? a : b;
        cd.j = a < b ? b : a;
        cd.step = step;
        if (!(kLean & kTpNoStage) && g.stage) {
            const unsigned w = threadIdx.x >> 5;
            const unsigned k = atomicAdd(&s_nw[w], 1u);
            if (k < kSWarp) {
                s_cand[w * kSWarp + k] = cd;
                return;
            }
        }
        append(q, qcap, &ctrl->n_cand, cd);
    }
}

template <int kLean = 0>
__device__ __forceinline__ void walk(const GridGeom& g, const Entry* __restrict__ E, uint32_t j,
                                     uint32_t r, const double p[3], bool only_greater, uint32_t step,
                                     Cand* __restrict__ q, size_t qcap, Ctrl* ctrl)
{
    uint32_t guard = g.max_walk;   // a list is never longer than n; a cycle would be a bug
    while (j != kNil) {
        if (guard-- == 0) {
            ctrl->err_internal = 1;
            return;
        }
        const Entry ej = E[j];
        if (!only_greater || j > r) test_pair<kLean>(g, r, j, p, ej, step, q, qcap, ctrl);
        j = ej.next;
    }
}

// Scan one object against the cells listed by (dx, dy, dz) offsets of its own cell: every bitmap
// load is issued before any is resolved; set bits probe the table and walk the cell's list.
// Measured alternatives on the hybrid's dense coarse grid (1M objects, g_c,h = 72.2 km; DESIGN.md
// section 6): a flattened single loop (one entry or one slot probe per iteration, lanes kept
// converged) ran 411 vs 324 us per step -- lockstep iterations wait for the slowest lane's
// dependent load, while these nested loops let a warp's diverged lanes overlap their latencies;
// an apogee/perigee gate in test_pair (the AP filter's rejections, 32 % of the candidates, not
// queued) did not pay: 446 -> 451 us scan, 161 -> 165 us filter per step; 16 lanes per object,
// one half-shell cell each (more loads in flight, 16x the per-lane set-up), 432 vs 282 us; and
// fewer blocks per SM for a spill-free open-map instance (CD_OPEN_MINB 5 / 4 / 3: 48 / 61 / 61
// registers), 301 / 356 / 354 vs 282 us -- occupancy outweighs the spills (and more blocks win:
// 8 per SM, 32 registers, for the half-shell instances, see CD_HALF_MINB / CD_OPEN_MINB).
__device__ __forceinline__ void probe_cell(const GridGeom& g, const Slot* __restrict__ slots,
                                           uint64_t mask, uint32_t tag, int cx, int cy, int cz,
                                           const Entry* __restrict__ E, uint32_t r, const double p[3],
                                           bool only_greater, uint32_t step, Cand* __restrict__ q,
                                           size_t qcap, Ctrl* ctrl)
{
    walk(g, E, grid_find(slots, mask, pack_key(cx, cy, cz), tag), r, p, only_greater, step, q, qcap, ctrl);
}

__device__ __forceinline__ void do_scan(const GridGeom& g, const GridTab& tab,
                                        const Entry* __restrict__ ents, int64_t n, uint64_t mask,
                                        int64_t k0, int s, int64_t r, uint32_t tag,
                                        Cand* __restrict__ q, size_t qcap, Ctrl* ctrl)
{
    const Slot* slots = tab.slots + (size_t)s * (mask + 1);
    const uint32_t* bits = tab.bits + (size_t)s * tab.bwords;
    const uint32_t bmask = tab.bmask;
    const Entry* E = ents + (size_t)s * n;
    const uint32_t step = (uint32_t)(k0 + s);
    const Entry me = E[r];
    const double p[3] = {me.x, me.y, me.z};
    int c[3];
    double fr[3];
    if (!cell_of(g, p, c, fr)) return;
    // (1) own cell: successors in the object's own list
    walk(g, E, me.next, (uint32_t)r, p, false, step, q, qcap, ctrl);
    // (2) other cells
    const uint32_t hx0 = (uint32_t)c[0] * kHX, hy0 = (uint32_t)c[1] * kHY, hz0 = (uint32_t)c[2] * kHZ;
    if (g.halfshell) {
        const uint32_t reach = g.raw ? 0x3FFEu : halfshell_reach(fr, g.reach * g.inv_cell);   // (raw counts: the paper's 27 cells)
        uint32_t hit = 0;
#pragma unroll
        for (int o = 1; o < 14; ++o) {
            const uint32_t hb = bit_mix((hx0 + (uint32_t)kHalfShell[o][0] * kHX) ^
                                        (hy0 + (uint32_t)kHalfShell[o][1] * kHY) ^
                                        (hz0 + (uint32_t)kHalfShell[o][2] * kHZ)) & bmask;
            if ((reach >> o) & 1u) hit |= ((__ldg(bits + (hb >> 5)) >> (hb & 31)) & 1u) << o;
        }
        while (hit) {
            const int o = __ffs(hit) - 1;
            hit &= hit - 1;
            probe_cell(g, slots, mask, tag, c[0] + kHalfShell[o][0], c[1] + kHalfShell[o][1],
                       c[2] + kHalfShell[o][2], E, (uint32_t)r, p, false, step, q, qcap, ctrl);
        }
    } else {
        // ball mode: per axis the other overlapped cell (c - 1 if the ball crosses the lower
        // face, c + 1 if the upper); frac * L is the distance to the lower face
        const double rl = g.reach * g.inv_cell;
        const int d0 = fr[0] < rl ? -1 : (fr[0] > 1.0 - rl ? 1 : 0);
        const int d1 = fr[1] < rl ? -1 : (fr[1] > 1.0 - rl ? 1 : 0);
        const int d2 = fr[2] < rl ? -1 : (fr[2] > 1.0 - rl ? 1 : 0);
        // (c +- 1 stays inside the 21-bit key range because |c| <= kCellMax = 2^20 - 2)
        const uint32_t hx1 = hx0 + (uint32_t)d0 * kHX, hy1 = hy0 + (uint32_t)d1 * kHY,
                       hz1 = hz0 + (uint32_t)d2 * kHZ;
        // cell c + (b0 d0, b1 d1, b2 d2), b = 1..7, exists iff every axis set in b has d != 0;
        // only cells in the positive lexicographic half-space of c are probed, so a pair in two
        // cells is seen from exactly one of them (as in the half-shell scan)
        const uint32_t pos = (d0 > 0 ? 0xAAu : 0u) | (d1 > 0 ? 0x44u : 0u) | (d2 > 0 ? 0x10u : 0u);
        const uint32_t valid = (d0 ? 0xFFu : 0x55u) & (d1 ? 0xFFu : 0x33u) & (d2 ? 0xFFu : 0x0Fu) & pos;
        uint32_t hit = 0;
#pragma unroll
        for (int b = 1; b < 8; ++b) {
            const uint32_t hb = bit_mix(((b & 1) ? hx1 : hx0) ^ ((b & 2) ? hy1 : hy0) ^
                                        ((b & 4) ? hz1 : hz0)) & bmask;
            if ((valid >> b) & 1u) hit |= ((__ldg(bits + (hb >> 5)) >> (hb & 31)) & 1u) << b;
        }
        while (hit) {
            const int b = __ffs(hit) - 1;
            hit &= hit - 1;
            probe_cell(g, slots, mask, tag, c[0] + ((b & 1) ? d0 : 0), c[1] + ((b & 2) ? d1 : 0),
                       c[2] + ((b & 4) ? d2 : 0), E, (uint32_t)r, p, false, step, q, qcap, ctrl);
        }
    }
}

// Chained spatial hash (alternative grid structure): the lists hang off bucket hash(cell), so a
// bucket may also hold objects of other cells -- the exact distance test filters them.
//  * pairs inside the object's own bucket (same cell, or a colliding cell) are found by the
//    later-inserted object walking its own list successors (no probe);
//  * ball mode (L >= 2 g_c): the buckets of the 0-7 ball cells in the positive half-space of
//    the own cell are walked; only entries tagged with the probed cell count (walk_bucket_tag),
//    so a pair in cells A != B is reported once, by the object whose cell is lexicographically
//    smaller (parity hashing keeps these buckets distinct from each other and the own bucket);
//  * half-shell mode (L < 2 g_c): the buckets of the 13 half-shell neighbour cells, again only
//    the probed cell's entries (needs 4x4x4 or larger superblocks, see below).
__device__ __forceinline__ uint32_t head_index(uint32_t h, uint32_t epoch)
{
    return ((h >> kEpochShift) == epoch && (h & kIdxMask)) ? (h & kIdxMask) - 1u : kNil;
}

// ball mode: bucket of the probed cell (tag ctag), which lies in the positive half-space of the
// scanning object's cell -- only the probed cell's own entries count (a colliding neighbour
// cell's entries are found by their own probe, so each pair is reported exactly once)
template <int kLean = 0>
__device__ __forceinline__ void walk_bucket_tag(const GridGeom& g, const Entry* __restrict__ E,
                                                uint32_t h, uint32_t epoch, uint32_t ctag, uint32_t r,
                                                const double p[3], uint32_t step,
                                                Cand* __restrict__ q, size_t qcap, Ctrl* ctrl)
{
    uint32_t j = head_index(h, epoch);
    uint32_t guard = g.max_walk;
    while (j != kNil) {
        if (guard-- == 0) {
            ctrl->err_internal = 1;
            return;
        }
        const Entry ej = E[j];
        if (ej.tag == ctag) test_pair<kLean>(g, r, j, p, ej, step, q, qcap, ctrl);
        j = ej.next;
    }
}

template <bool kBallOnly, int kTP = 0>
__device__ __forceinline__ void do_scan_chained(const GridGeom& g, const GridTab& tab,
                                                const Entry* __restrict__ ents, int64_t n, int64_t k0,
                                                int s, int64_t r, uint32_t epoch, Cand* __restrict__ q,
                                                size_t qcap, Ctrl* ctrl)
{
    const uint32_t* heads = tab.bits + (size_t)s * tab.bwords;
    const uint32_t hmask = tab.bmask;
    const Entry* E = ents + (size_t)s * n;
    // ball-mode instance: E made opaque, so it stays in a register instead of being recomputed from
    // s * n at every walk step (1M step 58.8 -> 57.7 us; the half-shell instance measured +0.5 %)
    if (kBallOnly) asm("" : "+l"(E));
    const uint32_t step = (uint32_t)(k0 + s);
    const Entry me = E[r];
    const double p[3] = {me.x, me.y, me.z};
    int c[3];
    double fr[3];
    if (!cell_of(g, p, c, fr)) return;
    // own bucket: successors only, every pair once (by the later-inserted object)
    walk<kTP>(g, E, me.next, (uint32_t)r, p, false, step, q, qcap, ctrl);
    if (((kTP & kTpLean) && !kBallOnly) || (!kBallOnly && g.halfshell)) {   // (the lean half-shell instance runs half-shell scans only)
        // L < 2 g_c: the 13 half-shell neighbour cells (each unordered pair of cells of a 3x3x3
        // block once, as in do_scan), only the probed cell's entries (tag).  The 27 cells of a
        // 3x3x3 block differ pairwise in (c mod 4) on some axis, so with superblock buckets they
        // never share a bucket: a colliding cell in the own bucket is never a neighbour (its
        // entries fail the distance test), and no pair is seen from two buckets.
        const uint32_t reach = g.raw ? 0x3FFEu : halfshell_reach(fr, g.reach * g.inv_cell);   // (raw counts: the paper's 27 cells)
        uint32_t hit = 0;
#pragma unroll
        for (int o = 1; o < 14; ++o) {
            // (every head loaded, the unreachable ones discarded: branch-free, so the 13 loads are
            // in flight together)
            const uint32_t h = __ldg(heads + chain_bucket(c[0] + kHalfShell[o][0], c[1] + kHalfShell[o][1],
                                                          c[2] + kHalfShell[o][2], hmask));
            hit |= (head_index(h, epoch) != kNil ? 1u : 0u) << o;
        }
        hit &= reach;
        while (hit) {
            const int o = __ffs(hit) - 1;
            hit &= hit - 1;
            const int cx = c[0] + kHalfShell[o][0], cy = c[1] + kHalfShell[o][1], cz = c[2] + kHalfShell[o][2];
            walk_bucket_tag<kTP>(g, E, __ldg(heads + chain_bucket(cx, cy, cz, hmask)), epoch, cell_tag(cx, cy, cz),
                            (uint32_t)r, p, step, q, qcap, ctrl);
        }
        return;
    }
    const double rl = g.reach * g.inv_cell;
    const int d0 = fr[0] < rl ? -1 : (fr[0] > 1.0 - rl ? 1 : 0);
    const int d1 = fr[1] < rl ? -1 : (fr[1] > 1.0 - rl ? 1 : 0);
    const int d2 = fr[2] < rl ? -1 : (fr[2] > 1.0 - rl ? 1 : 0);
    // ball cells (offset o_b = (b&1 ? d0 : 0, b&2 ? d1 : 0, b&4 ? d2 : 0)) in the positive
    // lexicographic half-space o > 0 only: a pair in cells A != B is then probed from exactly
    // one side (B - A > 0 or A - B > 0), and B is in the ball set of the object in A whenever
    // the pair is closer than g_c
    const uint32_t pos = (d0 > 0 ? 0xAAu : 0u) | (d1 > 0 ? 0x44u : 0u) | (d2 > 0 ? 0x10u : 0u);
    const uint32_t valid = (d0 ? 0xFFu : 0x55u) & (d1 ? 0xFFu : 0x33u) & (d2 ? 0xFFu : 0x0Fu) & pos;
    if (!valid) return;
    // the ball's cells differ pairwise in parity -> distinct buckets, no de-duplication
    uint32_t hd[8];
#pragma unroll
    for (int b = 1; b < 8; ++b)
        // every head loaded (branch-free, all in flight together), the invalid ones discarded:
        // 59.4 -> 58.7 us per 1M-object step, 766 -> 759 us per 8M step
        hd[b] = __ldg(heads + chain_bucket(c[0] + ((b & 1) ? d0 : 0), c[1] + ((b & 2) ? d1 : 0),
                                           c[2] + ((b & 4) ? d2 : 0), hmask)) & (((valid >> b) & 1u) ? ~0u : 0u);
#pragma unroll
    for (int b = 1; b < 8; ++b)
        if (hd[b])
            walk_bucket_tag<kTP>(g, E, hd[b], epoch,
                            cell_tag(c[0] + ((b & 1) ? d0 : 0), c[1] + ((b & 2) ? d1 : 0),
                                     c[2] + ((b & 4) ? d2 : 0)),
                            (uint32_t)r, p, step, q, qcap, ctrl);
}

// ---------------------------------------------------------------------------------------
// CSR grid (kCsr, sort + segment): after the build counted every object into its cell's slot,
// k_csr_alloc gives each occupied slot a segment [start, start + count) of the step's entry array
// (warp prefix sums, one atomic per warp) and k_csr_scatter moves each object's entry to
// start + rank: the objects of a cell are contiguous, ordered by cell.  The scan then runs one
// thread per segment position -- the objects of a cell are adjacent lanes probing the same
// neighbour slots -- and reads each neighbour cell as one contiguous range (independent loads
// instead of a linked list's dependent ones).
// ---------------------------------------------------------------------------------------
__global__ void k_csr_alloc(const Slot* __restrict__ slots, uint32_t* __restrict__ start, uint64_t M,
                            int B, uint32_t tag, unsigned long long* __restrict__ total)
{
    const uint64_t gi = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    const int s = (int)(gi / M);
    const uint64_t h = gi - (uint64_t)s * M;
    const bool in = s < B;
    uint32_t cnt = 0;
    if (in) {
        const unsigned long long w1 = slots[(size_t)s * M + h].head;
        cnt = (uint32_t)(w1 >> 32) == tag ? (uint32_t)w1 : 0u;
    }
    // block prefix sum (the block's 256 slots all belong to one step: M is a multiple of 256),
    // one atomic per block on the step's total (one per warp serialised on the single counter)
    __shared__ uint32_t s_w[8];
    __shared__ unsigned long long s_base;
    const unsigned lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    uint32_t inc = cnt;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const uint32_t y = __shfl_up_sync(0xffffffffu, inc, o);
        if (lane >= (unsigned)o) inc += y;
    }
    if (lane == 31) s_w[wid] = inc;
    __syncthreads();
    if (threadIdx.x == 0) {
        uint32_t run = 0;
        for (int w = 0; w < 8; ++w) {
            const uint32_t x = s_w[w];
            s_w[w] = run;
            run += x;
        }
        s_base = (in && run) ? atomicAdd(total + s, (unsigned long long)run) : 0ull;
    }
    __syncthreads();
    if (in) start[(size_t)s * M + h] = (uint32_t)s_base + s_w[wid] + inc - cnt;
}

__global__ void k_csr_scatter(const Entry* __restrict__ tmp, const Slot* __restrict__ slots,
                              const uint32_t* __restrict__ start, uint64_t M, int64_t n, int B,
                              Entry* __restrict__ csr)
{
    const int64_t gi = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    const int s = (int)(gi / n);
    const int64_t r = gi - (int64_t)s * n;
    if (s >= B) return;
    Entry e = tmp[(size_t)s * n + r];
    if (e.next == kNil) return;   // out of the key range (CD_ERANGE already raised)
    const size_t sh = (size_t)s * M + e.next;
    const uint32_t st = start[sh];
    const uint32_t cnt = (uint32_t)slots[sh].head;
    const uint32_t pos = st + e.tag;
    e.next = (uint32_t)r;      // the object
    e.tag = st + cnt;          // end of its cell's segment
    csr[(size_t)s * n + pos] = e;
}

cudaError_t launch_csr_segments(const Slot* slots, uint32_t* start, uint64_t M, const Entry* tmp,
                                Entry* csr, int64_t n, int B, uint32_t tag, unsigned long long* total,
                                cudaStream_t st, LaunchCount& lc)
{
    if (B <= 0) return cudaSuccess;
    cudaError_t e = cudaMemsetAsync(total, 0, sizeof(unsigned long long) * (size_t)B, st);
    if (e != cudaSuccess) return e;
    k_csr_alloc<<<blocks_for((int64_t)(M * (uint64_t)B), 256), 256, 0, st>>>(slots, start, M, B, tag, total);
    lc.bump();
    k_csr_scatter<<<blocks_for(n * B, 256), 256, 0, st>>>(tmp, slots, start, M, n, B, csr);
    lc.bump();
    return cudaGetLastError();
}

// Look a cell up in the CSR slot table: its segment [*st, *st + *cnt), false if empty.
__device__ __forceinline__ bool csr_find(const Slot* __restrict__ slots, const uint32_t* __restrict__ start,
                                         uint64_t mask, unsigned long long key, uint32_t tag,
                                         uint32_t* st, uint32_t* cnt)
{
    uint64_t h = fmix64(key) & mask;
    while (true) {
        const ulonglong2 w = __ldg(reinterpret_cast<const ulonglong2*>(slots + h));
        if ((uint32_t)(w.y >> 32) != tag) return false;
        if (w.x == key) {
            *cnt = (uint32_t)w.y;
            *st = __ldg(start + h);
            return true;
        }
        h = (h + 1) & mask;
    }
}

__device__ __forceinline__ void csr_range(const GridGeom& g, const Entry* __restrict__ C, uint32_t u,
                                          uint32_t end, uint32_t id, const double p[3], uint32_t step,
                                          Cand* __restrict__ q, size_t qcap, Ctrl* ctrl)
{
#pragma unroll 4
    for (; u < end; ++u) {
        const Entry e = C[u];
        test_pair(g, id, e.next, p, e, step, q, qcap, ctrl);
    }
}

__device__ __forceinline__ void do_scan_csr(const GridGeom& g, const GridTab& tab,
                                            const uint32_t* __restrict__ starts, const Entry* __restrict__ csr,
                                            int64_t n, uint64_t mask, int64_t k0, int s, int64_t t,
                                            uint32_t tag, Cand* __restrict__ q, size_t qcap, Ctrl* ctrl)
{
    const Slot* slots = tab.slots + (size_t)s * (mask + 1);
    const uint32_t* start = starts + (size_t)s * (mask + 1);
    const uint32_t* bits = tab.bits + (size_t)s * tab.bwords;
    const uint32_t bmask = tab.bmask;
    const Entry* C = csr + (size_t)s * n;
    const uint32_t step = (uint32_t)(k0 + s);
    const Entry me = C[t];
    const double p[3] = {me.x, me.y, me.z};
    int c[3];
    double fr[3];
    if (!cell_of(g, p, c, fr)) return;
    // (1) own cell: the later positions of the segment, each pair once
    csr_range(g, C, (uint32_t)t + 1, me.tag, me.next, p, step, q, qcap, ctrl);
    // (2) other cells: half-shell (L < 2 g_c) or the positive half-space of the ball (L >= 2 g_c)
    const uint32_t hx0 = (uint32_t)c[0] * kHX, hy0 = (uint32_t)c[1] * kHY, hz0 = (uint32_t)c[2] * kHZ;
    uint32_t st, cnt;
    if (g.halfshell) {
        // the lanes of a crowded cell are adjacent and walk the same neighbour ranges in lockstep:
        // the warp's union of the reach masks keeps them converged (per-lane masks diverged
        // them -- 8M hybrid scan 10.1 -> 15.0 ms per coarse step)
        const uint32_t reach = g.raw ? 0x3FFEu
                                     : __reduce_or_sync(__activemask(), halfshell_reach(fr, g.reach * g.inv_cell));
        uint32_t hit = 0;
#pragma unroll
        for (int o = 1; o < 14; ++o) {
            const uint32_t hb = bit_mix((hx0 + (uint32_t)kHalfShell[o][0] * kHX) ^
                                        (hy0 + (uint32_t)kHalfShell[o][1] * kHY) ^
                                        (hz0 + (uint32_t)kHalfShell[o][2] * kHZ)) & bmask;
            if ((reach >> o) & 1u) hit |= ((__ldg(bits + (hb >> 5)) >> (hb & 31)) & 1u) << o;
        }
        while (hit) {
            const int o = __ffs(hit) - 1;
            hit &= hit - 1;
            if (csr_find(slots, start, mask, pack_key(c[0] + kHalfShell[o][0], c[1] + kHalfShell[o][1],
                                                      c[2] + kHalfShell[o][2]), tag, &st, &cnt))
                csr_range(g, C, st, st + cnt, me.next, p, step, q, qcap, ctrl);
        }
    } else {
        const double rl = g.reach * g.inv_cell;
        const int d0 = fr[0] < rl ? -1 : (fr[0] > 1.0 - rl ? 1 : 0);
        const int d1 = fr[1] < rl ? -1 : (fr[1] > 1.0 - rl ? 1 : 0);
        const int d2 = fr[2] < rl ? -1 : (fr[2] > 1.0 - rl ? 1 : 0);
        const uint32_t hx1 = hx0 + (uint32_t)d0 * kHX, hy1 = hy0 + (uint32_t)d1 * kHY,
                       hz1 = hz0 + (uint32_t)d2 * kHZ;
        const uint32_t pos = (d0 > 0 ? 0xAAu : 0u) | (d1 > 0 ? 0x44u : 0u) | (d2 > 0 ? 0x10u : 0u);
        const uint32_t valid = (d0 ? 0xFFu : 0x55u) & (d1 ? 0xFFu : 0x33u) & (d2 ? 0xFFu : 0x0Fu) & pos;
        uint32_t hit = 0;
#pragma unroll
        for (int b = 1; b < 8; ++b) {
            const uint32_t hb = bit_mix(((b & 1) ? hx1 : hx0) ^ ((b & 2) ? hy1 : hy0) ^
                                        ((b & 4) ? hz1 : hz0)) & bmask;
            if ((valid >> b) & 1u) hit |= ((__ldg(bits + (hb >> 5)) >> (hb & 31)) & 1u) << b;
        }
        while (hit) {
            const int b = __ffs(hit) - 1;
            hit &= hit - 1;
            if (csr_find(slots, start, mask, pack_key(c[0] + ((b & 1) ? d0 : 0), c[1] + ((b & 2) ? d1 : 0),
                                                      c[2] + ((b & 4) ? d2 : 0)), tag, &st, &cnt))
                csr_range(g, C, st, st + cnt, me.next, p, step, q, qcap, ctrl);
        }
    }
}

// ---------------------------------------------------------------------------------------
// One launch per batch (horizontal fusion): blocks of three roles run side by side, so the
// latency-bound build (fp64 Contour + atomics) and scan (probes) hide each other's stalls.
//   role A: build batch b + 1, class-0 objects     (slot set (b+1) % 2, bitmap set (b+1) % 3)
//   role B: build batch b + 1, objects of classes 1-4
//   role C: scan batch b (slot set b % 2, bitmap set b % 3), and zero bitmap set (b+2) % 3
//           (used by batch b - 1, next built by batch b + 2)
// ---------------------------------------------------------------------------------------
#ifndef CD_STEP_MINB
#define CD_STEP_MINB 6
#endif
// blocks per SM of the other instances (measured on the 1M hybrid's half-shell scan: 6 -> 8
// blocks, i.e. 40 -> 32 registers with spills, 222 -> 213 us chained and 256 -> 229 us open
// map; the crowded sort + segment grid at 8M prefers 6: 10.21 vs 10.31 ms)
#ifndef CD_OPEN_MINB
#define CD_OPEN_MINB 8
#endif
#ifndef CD_CSR_MINB
#define CD_CSR_MINB 6
#endif
#ifndef CD_HALF_MINB
#define CD_HALF_MINB 8   // kChained / kChainedLean: the half-shell (and J2 runtime) instances
#endif
// the lean ball instance (the 1M grid's) at 7 blocks per SM: 56.2 -> 53.3 us per step (8: 53.4);
// the lean instance with the slot map (8M, spatial order) stays at 6 (7: 766 vs 738 us)
#ifndef CD_BALL_LEAN_MINB
#define CD_BALL_LEAN_MINB 7
#endif
template <int kGrid, int kJ2>
__global__ void __launch_bounds__(256, kGrid == kChained || kGrid == kChainedLean ? CD_HALF_MINB
                                       : kGrid == kChainedBallLean ? CD_BALL_LEAN_MINB
                                       : is_chained(kGrid) ? CD_STEP_MINB
                                       : kGrid == kCsr     ? CD_CSR_MINB
                                                           : CD_OPEN_MINB) k_step(StepArgs a)
{
    const uint32_t bx = blockIdx.x;
    const uint32_t nbA = (uint32_t)a.nbA, nbB = (uint32_t)a.nbB, nbC = (uint32_t)a.nbC;
    const uint32_t nA = (uint32_t)a.build_B * nbA, nB = (uint32_t)a.build_B * nbB;
    // Programmatic dependent launch (chained grid, StepArgs::pdl): build blocks depend on no
    // earlier launch still running -- the head/entry sets they write were last read two launches
    // ago, and this launch started only after every block of the previous one had triggered,
    // which its scan blocks do after their own wait -- so they trigger at once.  Scan blocks
    // read the previous launch's build output: wait for its completion, then trigger.
    if (bx < nA + nB) pdl_trigger();
    if (bx < nA) {
        const int s = (int)(bx / nbA);
        const int64_t r = (int64_t)(bx % nbA) * 256 + threadIdx.x;
        if (r < a.O.n0)
            do_build<true, kGrid, kJ2>(a.O, a.g, a.build_tab, a.build_ents, a.mask, a.build_k0, s, r, a.t0,
                                     a.dt, a.build_tag, a.ctrl);
    } else if (bx < nA + nB) {
        const uint32_t b2 = bx - nA;
        const int s = (int)(b2 / nbB);
        const int64_t r = a.O.n0 + (int64_t)(b2 % nbB) * 256 + threadIdx.x;
        if (r < a.O.n)
            do_build<false, kGrid, kJ2>(a.O, a.g, a.build_tab, a.build_ents, a.mask, a.build_k0, s, r, a.t0,
                                      a.dt, a.build_tag, a.ctrl);
    } else {
        const uint32_t b3 = bx - nA - nB;
        pdl_wait();
        pdl_trigger();
        // zero the bitmap set of batch b + 2 (all Bmax tables), grid-stride over role-C threads
        const int64_t tid = (int64_t)b3 * 256 + threadIdx.x;
        const int64_t nth = a.nCblocks * 256;
        const int64_t nw4 = (int64_t)a.zero_depth * a.zero_bits_words / 4;
        uint4* zb = reinterpret_cast<uint4*>(a.zero_bits);
        if (!is_chained(kGrid))   // chained heads are epoch-tagged: nothing to clear
            for (int64_t i = tid; i < nw4; i += nth) zb[i] = make_uint4(0u, 0u, 0u, 0u);
        if (a.scan_B == 0) return;
        const int s = (int)(b3 / nbC);
        const int64_t r = (int64_t)(b3 % nbC) * 256 + threadIdx.x;
        constexpr int kTP = kGrid == kChainedLean ? kTpLean
                            : kGrid == kChainedBallLean ? kTpLean | kTpNoStage
                            : kGrid == kChainedBallLeanSig ? kTpLean | kTpNoStage | kTpSig : 0;
        const bool stage = !(kTP & kTpNoStage) && a.g.stage != 0;   // uniform over the launch
        const bool raw = !(kTP & kTpLean) && a.g.raw;
        const unsigned lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
        if (stage || raw) {
            if (lane == 0) {
                s_nw[wid] = 0;
                s_rw[wid] = 0;
            }
            __syncwarp();
        }
        if (r < a.O.n) {
            if (is_chained(kGrid))
                do_scan_chained<kGrid == kChainedBall || kGrid == kChainedBallLean || kGrid == kChainedBallLeanSig, kTP>(a.g, a.scan_tab, a.scan_ents, a.O.n, a.scan_k0, s, r, a.scan_tag, a.q,
                                a.qcap, a.ctrl);
            else if (kGrid == kCsr)
                do_scan_csr(a.g, a.scan_tab, a.scan_start, a.scan_ents, a.O.n, a.mask, a.scan_k0, s, r,
                            a.scan_tag, a.q, a.qcap, a.ctrl);
            else
                do_scan(a.g, a.scan_tab, a.scan_ents, a.O.n, a.mask, a.scan_k0, s, r, a.scan_tag, a.q,
                        a.qcap, a.ctrl);
        }
        if (raw) {
            __syncwarp();
            if (lane == 0 && s_rw[wid]) atomicAdd(&a.ctrl->n_raw, (unsigned long long)s_rw[wid]);
        }
        if (!stage) return;
        // flush the warp's staged candidates: one global atomic, coalesced copy
        __syncwarp();
        const unsigned m = min(s_nw[wid], kSWarp);
        if (m == 0) return;
        unsigned long long base = 0;
        if (lane == 0) base = atomicAdd(&a.ctrl->n_cand, (unsigned long long)m);
        base = __shfl_sync(0xffffffffu, base, 0);
        for (unsigned k = lane; k < m; k += 32) {
            const unsigned long long idx = base + k;
            if (idx < a.qcap) a.q[idx] = s_cand[wid * kSWarp + k];
        }
    }
}

cudaError_t launch_step(StepArgs a, const L2Win* win, cudaStream_t st, LaunchCount& lc)
{
    a.nbA = (int64_t)blocks_for(a.O.n0, 256);
    a.nbB = (int64_t)blocks_for(a.O.n - a.O.n0, 256);
    a.nbC = (int64_t)blocks_for(a.O.n, 256);
    a.nCblocks = a.scan_B * a.nbC;
    if (a.nCblocks == 0 && a.zero_depth > 0) a.nCblocks = 148 * 4;   // zero-only role-C blocks
    const int64_t blocks = a.build_B * (a.nbA + a.nbB) + a.nCblocks;
    if (blocks == 0) return cudaSuccess;
    lc.bump();
    const size_t smem = a.g.stage ? sizeof(Cand) * kSCand : 0;   // candidate staging buffer
    const bool lean = !a.g.raw && a.g.band_lo2 == 0.0 && isinf(a.g.band_hi2);   // (no shard band, no raw counts)
    if (a.O.j2) {   // J2 secular propagator: the rotation is compiled into its own instances
        if (a.chained)
            return launch_ex(a.g.halfshell ? k_step<kChained, 1> : k_step<kChainedBall, 1>, dim3((unsigned)blocks),
                             dim3(256), smem, st, win, a.pdl != 0, a);
        if (a.csr)
            return launch_ex(k_step<kCsr, 1>, dim3((unsigned)blocks), dim3(256), smem, st, win, false, a);
        return launch_ex(k_step<kOpen, 1>, dim3((unsigned)blocks), dim3(256), smem, st, win, false, a);
    }
    if (a.chained)
        return launch_ex(!a.g.halfshell ? (lean && !a.g.stage ? (a.g.sig ? k_step<kChainedBallLeanSig, 0> : k_step<kChainedBallLean, 0>)
                                                               : k_step<kChainedBall, 0>)
                         : lean && !a.g.sig ? k_step<kChainedLean, 0>
                                     : k_step<kChained, 0>,
                         dim3((unsigned)blocks),
                         dim3(256), smem, st, win, a.pdl != 0, a);
    if (a.csr)
        return launch_ex(k_step<kCsr, 0>, dim3((unsigned)blocks), dim3(256), smem, st, win, false, a);
    return launch_ex(k_step<kOpen, 0>, dim3((unsigned)blocks), dim3(256), smem, st, win, false, a);
}

// ---------------------------------------------------------------------------------------
// a7: refinement.
// (1) k_prefilter: state of both objects at t_k.  Degenerate pairs (|dv| < 1e-9 km/s) are
//     reported directly (tca = t_k).  Otherwise a conservative bound discards candidates that
//     cannot have a local minimum below d in the owner cell [t_k - dt/2, t_k + dt/2]:
//         D(t_k + tau) >= |dr + tau dv| - tau^2/2 * (mu/q_i^2 + mu/q_j^2)
//     (Taylor remainder, |acceleration| <= mu / perigee^2).  Survivors become work items with
//     the Brent half-window t_w = 2 g_c / min(|v_i|, |v_j|).
// (2) k_brent: Brent's minimisation (golden section + parabolic interpolation, ref. [44],
//     Boost's implementation in the paper) of D^2(t_k + tau) over
//     tau in [-t_w, t_w] intersected with [t0, t1]; a minimum at an end of the interval is
//     discarded ("the minimum will be found when considering the neighboring
//     interval"); otherwise it is reported iff its owner step is k and D < d.
// ---------------------------------------------------------------------------------------
#ifndef CD_PREFILTER_MINB
#define CD_PREFILTER_MINB 3   // 1 / 3 / 4 blocks per SM: 8M refine 64.8 / 63.3 / 75.3 us per step, 1M 1.47 / 1.32 / 1.29
#endif
__global__ void __launch_bounds__(256, CD_PREFILTER_MINB) k_prefilter(Orbits O, RefineParams P, const Cand* __restrict__ q,
                                                   size_t qcap, Work* __restrict__ w, size_t wcap,
                                                   unsigned long long* n_work, Conj* __restrict__ out,
                                                   size_t ocap, Ctrl* ctrl)
{
    unsigned long long nc = ctrl->n_cand;
    if (nc > qcap) nc = qcap;
    const size_t stride = (size_t)gridDim.x * blockDim.x;
    for (size_t idx = blockIdx.x * (size_t)blockDim.x + threadIdx.x; idx < nc; idx += stride)
        grid_refine_item(O, P, q[idx], 0u, w, wcap, n_work, out, ocap, ctrl);
}

// 4 blocks per SM (<= 128 registers; the evaluations and the Kepler solve are out-of-line calls):
// refine per step 99 -> 61 us at 8M objects, 1.76 -> 1.29 us at 1M, hybrid 102 -> 91 us (1 / 3 / 4 /
// 5 / 6 / 8 blocks measured, profiles/round2_brent_minb.txt)
#ifndef CD_BRENT_MINB
#define CD_BRENT_MINB 4
#endif
__global__ void __launch_bounds__(128, CD_BRENT_MINB) k_brent(Orbits O, RefineParams P, const Work* __restrict__ w,
                                               const unsigned long long* n_work, size_t wcap,
                                               Conj* __restrict__ out, size_t ocap, Ctrl* ctrl)
{
    unsigned long long nw = *n_work;
    if (nw > wcap) nw = wcap;
    const size_t stride = (size_t)gridDim.x * blockDim.x;
    for (size_t idx = blockIdx.x * (size_t)blockDim.x + threadIdx.x; idx < nw; idx += stride) {
        Work it = w[idx];
        if (it.flags & kWorkSetup) {   // hybrid coplanar candidate: grid-variant set-up here
            it.flags &= ~kWorkSetup;
            Cand cd;
            cd.i = it.i; cd.j = it.j; cd.step = it.step;
            if (!grid_refine_setup(O, P, cd, it.flags, it.lo, it.hi, out, ocap, ctrl)) continue;
        }
        const double tk = fma((double)it.step, P.dt, P.t0);
        double x, fx;
        if (!brent_min(O, it.i, it.j, tk, it.lo, it.hi, x, fx)) continue;
        const double tca = tk + x;
        if (tca < P.t0 || tca > P.t1) continue;
        const double kstar = floor((tca - P.t0) / P.dt + 0.5);
        if (kstar != (double)it.step) continue;
        const double pca = sqrt(fx);
        if (!(pca < P.d)) continue;
        Conj cj;
        cj.i = it.i; cj.j = it.j; cj.step = it.step; cj.flags = it.flags;
        cj.tca = tca; cj.pca = pca;
        append(out, ocap, &ctrl->n_conj, cj);
    }
}

// digest_only (cd_options.digest_only): fold the round's conjunction records [0, n_conj) into the
// digest (count, sum of hash(i, j, step) in caller ids, smallest PCA) unless the round overflowed
// (n_conj > ocap: the host redoes it), then empty the buffer for the next round (k_conj_reset)
__global__ void k_conj_digest(const Conj* __restrict__ c, size_t ocap, const uint32_t* __restrict__ perm,
                              Ctrl* ctrl)
{
    const unsigned long long n = ctrl->n_conj;
    if (n > ocap) return;
    const size_t stride = (size_t)gridDim.x * blockDim.x;
    unsigned long long sum = 0, nmin = 0;
    for (size_t k = blockIdx.x * (size_t)blockDim.x + threadIdx.x; k < n; k += stride) {
        const Conj r = c[k];
        uint32_t a = perm[r.i], b = perm[r.j];
        if (a > b) { const uint32_t t = a; a = b; b = t; }
        sum += (unsigned long long)a * 0x9E3779B1ull + (unsigned long long)b * 0x85EBCA77ull +
               (unsigned long long)r.step * 0xC2B2AE3Dull;
        const unsigned long long nb = ~(unsigned long long)__double_as_longlong(r.pca);
        nmin = nb > nmin ? nb : nmin;
    }
    for (int o = 16; o; o >>= 1) {
        sum += __shfl_down_sync(0xffffffffu, sum, o);
        const unsigned long long y = __shfl_down_sync(0xffffffffu, nmin, o);
        nmin = y > nmin ? y : nmin;
    }
    if ((threadIdx.x & 31) == 0) {
        if (sum) atomicAdd(&ctrl->dg_sum, sum);
        if (nmin) atomicMax(&ctrl->dg_notminpca, nmin);
    }
    if (blockIdx.x == 0 && threadIdx.x == 0) atomicAdd(&ctrl->dg_count, n);
}

__global__ void k_conj_reset(size_t ocap, Ctrl* ctrl)
{
    if (ctrl->n_conj <= ocap) ctrl->n_conj = 0;
}

cudaError_t launch_conj_digest(const Conj* c, size_t ocap, const uint32_t* perm, Ctrl* ctrl,
                               cudaStream_t st, LaunchCount& lc)
{
    k_conj_digest<<<148 * 4, 256, 0, st>>>(c, ocap, perm, ctrl);
    k_conj_reset<<<1, 1, 0, st>>>(ocap, ctrl);
    lc.bump(2);
    return cudaGetLastError();
}

cudaError_t launch_prefilter(const Orbits& O, const RefineParams& p, const Cand* q, size_t qcap,
                             Work* w, size_t wcap, unsigned long long* n_work, Conj* out, size_t ocap,
                             Ctrl* ctrl, cudaStream_t st, LaunchCount& lc)
{
    k_prefilter<<<148 * 8, 256, 0, st>>>(O, p, q, qcap, w, wcap, n_work, out, ocap, ctrl);
    lc.bump();
    return cudaGetLastError();
}

cudaError_t launch_brent(const Orbits& O, const RefineParams& p, const Work* w,
                         const unsigned long long* n_work, size_t wcap, Conj* out, size_t ocap,
                         Ctrl* ctrl, cudaStream_t st, LaunchCount& lc)
{
    k_brent<<<148 * 8, 128, 0, st>>>(O, p, w, n_work, wcap, out, ocap, ctrl);
    lc.bump();
    return cudaGetLastError();
}

}  // namespace cdh
