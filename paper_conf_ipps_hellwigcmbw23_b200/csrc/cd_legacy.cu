// cd_legacy.cu -- the legacy full-window filter chain on the device.
//
// The paper's comparison baseline screens every pair with the "classical orbital filters" alone,
// without a grid (PAPER.md:43 apogee/perigee [13], orbit path [13], time filter [15]; legacy
// variant P:189; accuracy comparison P:315-318; "not possible with the legacy variant to
// calculate more than 64,000 satellites").  Here it serves as the recall cross-check of the grid:
// it has no Eq. 1 speed assumption.
//
//   k_legacy_filter  one thread per pair (i < j) of a chunk of the n(n-1)/2 pairs: AP ->
//                    coplanarity -> orbit path -> time windows over the whole [t0, t1] (every
//                    window of A at a surviving node merged with every window of B at the same
//                    node, in time order).  Coplanar pairs search all of [t0, t1].  Each
//                    interval becomes work items of at most kLegacySpan sampling steps.
//   k_legacy_search  one warp per work item: every step t_k whose owner cell
//                    [t_k - dt/2, t_k + dt/2) meets the interval is a sample; with
//                    v_max = v_p,A + v_p,B (perigee speeds, >= |v_A - v_B| always), a minimum
//                    below d within dt/2 of t_k has D(t_k) < d + v_max dt/2, so only such samples
//                    run Brent on [t_k - dt, t_k + dt] n [lo, hi] (cd_refine.cuh), and a sample at
//                    distance D skips the (D - gate)/(v_max dt) steps that cannot reach the gate
//                    (long coplanar searches: pairs far apart are skipped in strides); a minimum is
//                    reported by its owner step (reading R9), with D < d and TCA in [t0, t1].
//                    Degenerate pairs (|v_A - v_B| < 1e-9 km/s: no isolated minimum) are skipped.
#include "cd_filters.cuh"
#include "cd_legacy.h"

using namespace cdk;

namespace cdh {

using namespace filt;

namespace {

constexpr uint32_t kLegacySpan = 2048;   // sampling steps per work item (64 per lane)
constexpr uint32_t kSpanShift = 8;       // Work.flags: bits 0-7 conjunction flags, 8-31 step count

// (i, j), i < j, of linear pair index p (row-major upper triangle of n objects)
__device__ __forceinline__ void pair_of(uint64_t p, int64_t n, uint32_t& i, uint32_t& j)
{
    // row i starts at S(i) = i (2n - i - 1) / 2
    const double nn = (double)n;
    double di = floor(((2.0 * nn - 1.0) - sqrt((2.0 * nn - 1.0) * (2.0 * nn - 1.0) - 8.0 * (double)p)) * 0.5);
    int64_t r = (int64_t)di;
    if (r < 0) r = 0;
    auto start = [&](int64_t x) { return (uint64_t)(x * (2 * n - x - 1) / 2); };
    while (r > 0 && start(r) > p) --r;
    while (start(r + 1) <= p) ++r;
    i = (uint32_t)r;
    j = (uint32_t)(p - start(r) + (uint64_t)r + 1);
}

// Emit the work items of interval [lo, hi] (absolute times): the steps whose owner cells meet it,
// split into spans of at most kLegacySpan steps.
__device__ __forceinline__ void emit_interval(uint32_t i, uint32_t j, uint32_t flags, double lo,
                                              double hi, const LegacyParams& P, Work* w, size_t wcap,
                                              unsigned long long* n_work)
{
    double ka = ceil((lo - P.t0) / P.dt - 0.5), kb = floor((hi - P.t0) / P.dt + 0.5);
    ka = fmax(ka, 0.0);
    kb = fmin(kb, (double)(P.K - 1));
    for (double k = ka; k <= kb; k += (double)kLegacySpan) {
        const double cnt = fmin((double)kLegacySpan, kb - k + 1.0);
        Work it;
        it.i = i;
        it.j = j;
        it.step = (uint32_t)k;
        it.flags = flags | ((uint32_t)cnt << kSpanShift);
        it.lo = lo;
        it.hi = hi;
        append(w, wcap, n_work, it);
    }
}

}  // namespace

__global__ void __launch_bounds__(256) k_legacy_filter(LegacyParams P, const HOrbit* __restrict__ hr,
                                                       int64_t n, uint64_t p0, uint64_t p1,
                                                       Work* __restrict__ w, size_t wcap,
                                                       unsigned long long* n_work, Ctrl* ctrl)
{
    const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
    for (uint64_t p = p0 + blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; p < p1; p += stride) {
        uint32_t i, j;
        pair_of(p, n, i, j);
        const double d = P.d;
        // apogee / perigee first, from 16 bytes of each record
        if (fmax(hr[i].q, hr[j].q) - fmin(hr[i].Q, hr[j].Q) > d) {
            count1(&ctrl->n_ap);
            continue;
        }
        const HOrbit A = hr[i], B = hr[j];
        bool coplanar;
        NodeGeom gA, gB;
        pair_geometry(A, B, d, coplanar, gA, gB);
        if (coplanar) {
            count1(&ctrl->n_coplanar);
            emit_interval(i, j, 4u /* CD_FLAG_COPLANAR */, P.t0, P.t1, P, w, wcap, n_work);
            continue;
        }
        bool any_node = false;
        int nint = 0;
        const double TA = kTwoPiH / A.nm, TB = kTwoPiH / B.nm;
        for (int node = 0; node < 2; ++node) {
            const double sg = node ? -1.0 : 1.0;   // mutual node / opposite node (f + pi)
            if (node_closed(A, B, d, gA, gB, sg)) continue;   // orbit path
            any_node = true;
            double atl, ath, btl, bth;
            node_window(A, gA, sg, atl, ath);
            node_window(B, gB, sg, btl, bth);
            // every window copy k of each object overlapping [t0, t1], merged in time order
            double ka = floor((P.t0 - ath) / TA), kb = floor((P.t0 - bth) / TB);
            for (int guard = 0; guard < (1 << 22); ++guard) {
                const double al = atl + ka * TA, ah = ath + ka * TA;
                const double bl = btl + kb * TB, bh = bth + kb * TB;
                if (al > P.t1 || bl > P.t1) break;
                const double lo = fmax(fmax(al, bl), P.t0), hi = fmin(fmin(ah, bh), P.t1);
                if (hi > lo) {
                    emit_interval(i, j, 0u, lo, hi, P, w, wcap, n_work);
                    ++nint;
                }
                if (ah < bh) ka += 1.0;
                else kb += 1.0;
            }
        }
        if (!any_node) count1(&ctrl->n_path);
        else if (nint == 0) count1(&ctrl->n_time);
        else atomicAdd(&ctrl->n_refined, (unsigned long long)nint);
    }
}

__global__ void __launch_bounds__(128) k_legacy_search(Orbits O, LegacyParams P,
                                                       const HOrbit* __restrict__ hr,
                                                       const Work* __restrict__ w,
                                                       const unsigned long long* n_work, size_t wcap,
                                                       unsigned long long* next_item,
                                                       Conj* __restrict__ out, size_t ocap, Ctrl* ctrl)
{
    unsigned long long nw = *n_work;
    if (nw > wcap) nw = wcap;
    const int lane = threadIdx.x & 31;
    for (;;) {
        unsigned long long idx = 0;
        if (lane == 0) idx = atomicAdd(next_item, 1ull);
        idx = __shfl_sync(0xffffffffu, idx, 0);
        if (idx >= nw) return;
        const Work it = w[idx];
        const uint32_t cnt = it.flags >> kSpanShift, flags = it.flags & 0xffu;
        const HOrbit& A = hr[it.i];
        const HOrbit& B = hr[it.j];
        const double vmax = sqrt(kMu * (1.0 + A.e) / A.q) + sqrt(kMu * (1.0 + B.e) / B.q);
        const double gate = P.d + vmax * 0.5 * P.dt + 1e-9;
        const double gate2 = gate * gate;
        // each lane walks a contiguous sub-span; a sample far outside the gate skips the steps
        // that cannot be gated: |dD/dt| <= v_max, so D >= D_k - v_max m dt >= gate for the next
        // m = floor((D_k - gate) / (v_max dt)) steps
        const uint32_t per = (cnt + 31) / 32;
        const uint32_t s_end = min(cnt, (lane + 1) * per);
        const double inv_step = 1.0 / (vmax * P.dt);
        for (uint32_t s = lane * per; s < s_end; ++s) {
            const uint32_t k = it.step + s;
            const double tk = fma((double)k, P.dt, P.t0);
            const double D2 = dist2_at(O, it.i, it.j, tk);
            if (!(D2 < gate2)) {
                const double m = floor((sqrt(D2) - gate) * inv_step);
                if (m >= 1.0) s += (uint32_t)fmin(m, (double)per);
                continue;
            }
            double ri[3], vi[3], rj[3], vj[3];
            state<true, -1, -1, true>(O, it.i, tk, ri, vi);
            state<true, -1, -1, true>(O, it.j, tk, rj, vj);
            const double dv[3] = {vi[0] - vj[0], vi[1] - vj[1], vi[2] - vj[2]};
            if (dv[0] * dv[0] + dv[1] * dv[1] + dv[2] * dv[2] < 1e-18) continue;   // degenerate
            double x, fx;
            const double lo = fmax(it.lo, tk - P.dt) - tk, hi = fmin(it.hi, tk + P.dt) - tk;
            if (!brent_min(O, it.i, it.j, tk, lo, hi, x, fx)) continue;
            const double tca = tk + x;
            if (tca < P.t0 || tca > P.t1) continue;
            if (floor((tca - P.t0) / P.dt + 0.5) != (double)k) continue;   // owner step
            const double pca = sqrt(fx);
            if (!(pca < P.d)) continue;
            Conj cj;
            cj.i = it.i; cj.j = it.j; cj.step = k; cj.flags = flags;
            cj.tca = tca; cj.pca = pca;
            append(out, ocap, &ctrl->n_conj, cj);
        }
    }
}

cudaError_t launch_legacy_filter(const LegacyParams& p, const void* hrec, int64_t n, uint64_t p0,
                                 uint64_t p1, Work* w, size_t wcap, unsigned long long* n_work,
                                 Ctrl* ctrl, cudaStream_t st, LaunchCount& lc)
{
    if (p1 <= p0) return cudaSuccess;
    const uint64_t blocks = std::min<uint64_t>((p1 - p0 + 255) / 256, 148ull * 16);
    k_legacy_filter<<<(unsigned)blocks, 256, 0, st>>>(p, static_cast<const HOrbit*>(hrec), n, p0, p1,
                                                      w, wcap, n_work, ctrl);
    lc.bump();
    return cudaGetLastError();
}

cudaError_t launch_legacy_search(const Orbits& O, const LegacyParams& p, const void* hrec,
                                 const Work* w, const unsigned long long* n_work, size_t wcap,
                                 unsigned long long* next_item, Conj* out, size_t ocap, Ctrl* ctrl,
                                 cudaStream_t st, LaunchCount& lc)
{
    k_legacy_search<<<148 * 8, 128, 0, st>>>(O, p, static_cast<const HOrbit*>(hrec), w, n_work, wcap,
                                             next_item, out, ocap, ctrl);
    lc.bump();
    return cudaGetLastError();
}

}  // namespace cdh
