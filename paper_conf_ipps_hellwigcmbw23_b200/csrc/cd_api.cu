// cd_api.cu -- C ABI (include/cdscreen.h) and host orchestration of the screening path.
//
// Structure of one call ("four major steps"):
//   1) memory allocation (stream-ordered, pooled)
//   2) per step batch: propagate + insert into the per-step hash grid, neighbour scan P:71
//   3) (hybrid) orbital filter chain
//   4) TCA/PCA refinement
// The sampling steps are processed in rounds (bounded candidate queue, overflow -> retry) and
// within a round in batches of B steps whose grids are in flight together (the paper's p
// parallel grids).
#include <cuda_runtime.h>

#include <algorithm>
#include <chrono>
#include <cmath>
#include <cstdarg>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <mutex>
#include <string>
#include <vector>

#include <sys/mman.h>

#include "../../include/cdscreen.h"
#include "cd_internal.h"
#include "cd_hybrid.h"
#include "cd_legacy.h"

using namespace cdk;
using namespace cdh;

namespace {

thread_local std::string g_err;

// host-side timeline for diagnosis (CD_DEBUG_TIMING=1)
struct DebugClock {
    bool on = getenv("CD_DEBUG_TIMING") != nullptr;
    std::chrono::steady_clock::time_point t0 = std::chrono::steady_clock::now();
    void mark(const char* what, long long a = -1, long long b = -1) const
    {
        if (!on) return;
        const double ms = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
        fprintf(stderr, "[cd %9.3f ms] %s %lld %lld\n", ms, what, a, b);
    }
};
thread_local DebugClock* g_dbg = nullptr;
#define DBG(...) do { if (g_dbg) g_dbg->mark(__VA_ARGS__); } while (0)

cd_status fail(cd_status s, const char* fmt, ...)
{
    char buf[1024];
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(buf, sizeof buf, fmt, ap);
    va_end(ap);
    g_err = buf;
    return s;
}

#define CU(x)                                                                                   \
    do {                                                                                        \
        cudaError_t _e = (x);                                                                   \
        if (_e != cudaSuccess)                                                                  \
            return fail(_e == cudaErrorMemoryAllocation ? CD_ENOMEM : CD_ECUDA, "%s: %s (%s:%d)", \
                        #x, cudaGetErrorString(_e), __FILE__, __LINE__);                         \
    } while (0)

#define TRY(x)                          \
    do {                                \
        cd_status _s = (x);             \
        if (_s != CD_OK) return _s;     \
    } while (0)

// stream-ordered device buffer (dev_malloc: the caller's allocator or the stream-ordered pool)
template <typename T>
struct DBuf {
    T* p = nullptr;
    size_t n = 0;
    cudaStream_t st = nullptr;
    DBuf() = default;
    explicit DBuf(cudaStream_t s) : st(s) {}
    DBuf(const DBuf&) = delete;
    DBuf& operator=(const DBuf&) = delete;
    ~DBuf() { release(); }
    void release()
    {
        if (p) dev_free(p, st);
        p = nullptr;
        n = 0;
    }
    cudaError_t alloc(size_t count)
    {
        release();
        n = count;
        return dev_malloc((void**)&p, sizeof(T) * (count ? count : 1), st);
    }
    T* detach()
    {
        T* q = p;
        p = nullptr;
        n = 0;
        return q;
    }
};

std::mutex g_pool_mu;
cudaMemPool_t g_pools[64] = {};

// Per-host-thread page-locked staging for the per-round counters (4 Ctrl-sized slots), allocated
// once and kept for the thread's lifetime: no call pays cudaMallocHost / cudaFreeHost.
struct PinnedStage {
    Ctrl* p = nullptr;
    ~PinnedStage()
    {
        if (p) cudaFreeHost(p);   // at thread exit (errors after context teardown are ignored)
    }
};
thread_local PinnedStage g_stage;

cd_status pinned_stage(Ctrl** out)
{
    if (!g_stage.p) {
        void* p = nullptr;
        if (cudaMallocHost(&p, 4 * sizeof(Ctrl)) != cudaSuccess || !p)
            return fail(CD_ENOMEM, "page-locked staging allocation failed");
        g_stage.p = static_cast<Ctrl*>(p);
    }
    *out = g_stage.p;
    return CD_OK;
}

// Per-host-thread page-locked bounce buffers for device -> pageable-host result copies: two
// chunks, the DMA of one overlapping the host memcpy of the other (a direct copy into pageable
// memory runs at a fraction of the link rate)
constexpr size_t kBounceBytes = size_t(16) << 20;
struct Bounce {
    unsigned char* p = nullptr;
    cudaEvent_t ev[2] = {nullptr, nullptr};
    ~Bounce()
    {
        if (p) cudaFreeHost(p);
        for (auto e : ev) if (e) cudaEventDestroy(e);
    }
};
thread_local Bounce g_bounce;

cudaError_t copy_to_pageable(void* dst, const void* src, size_t bytes, cudaStream_t st)
{
    if (bytes <= kBounceBytes / 4) {   // small: one direct copy
        cudaError_t e = cudaMemcpyAsync(dst, src, bytes, cudaMemcpyDeviceToHost, st);
        return e != cudaSuccess ? e : cudaStreamSynchronize(st);
    }
    if (!g_bounce.p) {
        cudaError_t e = cudaMallocHost((void**)&g_bounce.p, 2 * kBounceBytes);
        if (e != cudaSuccess) {
            g_bounce.p = nullptr;
            return e;
        }
        for (auto& ev : g_bounce.ev) {
            e = cudaEventCreateWithFlags(&ev, cudaEventDisableTiming);
            if (e != cudaSuccess) return e;
        }
    }
    const size_t nch = (bytes + kBounceBytes - 1) / kBounceBytes;
    auto issue = [&](size_t c) -> cudaError_t {
        const size_t off = c * kBounceBytes, len = std::min(kBounceBytes, bytes - off);
        cudaError_t e = cudaMemcpyAsync(g_bounce.p + (c & 1) * kBounceBytes,
                                        static_cast<const unsigned char*>(src) + off, len,
                                        cudaMemcpyDeviceToHost, st);
        return e != cudaSuccess ? e : cudaEventRecord(g_bounce.ev[c & 1], st);
    };
    cudaError_t e = issue(0);
    for (size_t c = 0; c < nch && e == cudaSuccess; ++c) {
        if (c + 1 < nch) e = issue(c + 1);
        if (e != cudaSuccess) break;
        e = cudaEventSynchronize(g_bounce.ev[c & 1]);
        const size_t off = c * kBounceBytes, len = std::min(kBounceBytes, bytes - off);
        memcpy(static_cast<unsigned char*>(dst) + off, g_bounce.p + (c & 1) * kBounceBytes, len);
    }
    return e;
}

// Per-device cache of the (unsorted) conjunction accumulation buffer (cudaMalloc'd): grow-only up
// to kConjCacheMax bytes, handed from call to call so a repeated or long screen does not regrow it
// (growing a stream-ordered pool by hundreds of MB is a blocking driver call that stalls the round
// pipeline for up to ~1 s).  The event orders the next user after the last use (the finalize sort)
// on the previous call's stream.  cd_release_caches() frees it.
constexpr size_t kConjCacheMax = size_t(1) << 30;
struct ConjCache {
    std::mutex mu;
    Conj* p = nullptr;
    size_t cap = 0;
    cudaEvent_t ready = nullptr;
};
ConjCache g_conj_cache[64];

// Take the cached buffer of device dev (waits on `st` for its last use); false if none / busy.
bool conj_cache_take(int dev, cudaStream_t st, Conj** p, size_t* cap)
{
    if (dev < 0 || dev >= 64) return false;
    ConjCache& c = g_conj_cache[dev];
    std::lock_guard<std::mutex> lk(c.mu);
    if (!c.p) return false;
    if (c.ready) cudaStreamWaitEvent(st, c.ready, 0);
    *p = c.p;
    *cap = c.cap;
    c.p = nullptr;
    c.cap = 0;
    return true;
}

// Return a buffer (its last use already enqueued on `st`); keeps the larger of cached / returned.
void conj_cache_give(int dev, cudaStream_t st, Conj* p, size_t cap)
{
    if (!p) return;
    if (dev < 0 || dev >= 64) {
        cudaFree(p);
        return;
    }
    ConjCache& c = g_conj_cache[dev];
    std::lock_guard<std::mutex> lk(c.mu);
    if ((c.p && c.cap >= cap) || sizeof(Conj) * cap > kConjCacheMax) {
        cudaFree(p);
        return;
    }
    if (c.p) cudaFree(c.p);   // (cudaFree synchronises the device: its last use is done)
    if (!c.ready && cudaEventCreateWithFlags(&c.ready, cudaEventDisableTiming) != cudaSuccess) {
        c.ready = nullptr;
        cudaFree(p);
        c.p = nullptr;
        c.cap = 0;
        return;
    }
    cudaEventRecord(c.ready, st);
    c.p = p;
    c.cap = cap;
}

// Compute capability per device, queried once (cudaGetDeviceProperties costs milliseconds).
int g_cc[64];   // 0 = not yet queried, else major * 10 + minor

// The library's private stream-ordered pool of device dev (see cd_internal.h g_pool).
cudaMemPool_t setup_pool(int dev)
{
    std::lock_guard<std::mutex> lk(g_pool_mu);
    if (dev < 0 || dev >= 64) return nullptr;
    if (!g_pools[dev]) {
        cudaMemPoolProps props = {};
        props.allocType = cudaMemAllocationTypePinned;
        props.handleTypes = cudaMemHandleTypeNone;
        props.location.type = cudaMemLocationTypeDevice;
        props.location.id = dev;
        cudaMemPool_t pool = nullptr;
        if (cudaMemPoolCreate(&pool, &props) != cudaSuccess) {
            cudaGetLastError();
            return nullptr;   // fall back to the device's current pool (cudaMallocAsync)
        }
        uint64_t thr = ~uint64_t(0);
        cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &thr);
        g_pools[dev] = pool;
    }
    return g_pools[dev];
}

struct Owner {
    bool device;
    void* p;
    cudaStream_t st;   // device results: released stream-ordered on the call's stream
    size_t host_bytes; // host results: size of the anonymous mapping (munmap)
    DevAlloc alloc;    // device results from the caller's allocator: released with its free
};

// Optional per-phase device timing (cd_options.profile_phases): CUDA events recorded on the
// call's stream around each launch; elapsed times are harvested after the round's sync.
enum Phase { kPhClear = 0, kPhPropagate, kPhInsert, kPhScan, kPhRefine, kPhFinalize, kPhPrecompute, kNPhase };

struct PhaseTimer {
    bool on = false;
    cudaStream_t st = nullptr;
    std::vector<cudaEvent_t> pool;
    size_t used = 0;
    struct Mark { int ph; size_t a, b; uint64_t nl; };
    std::vector<Mark> marks;
    double ms[kNPhase] = {};
    uint64_t launches[kNPhase] = {};
    int cur = -1;
    size_t cur_a = 0;
    uint64_t every = 1;               // time every `every`-th launch of a phase (sampling)
    uint64_t calls[kNPhase] = {};     // all launches per phase (timed or not)
    ~PhaseTimer()
    {
        for (auto e : pool) cudaEventDestroy(e);
    }
    cudaEvent_t ev()
    {
        if (used == pool.size()) {
            cudaEvent_t e;
            cudaEventCreate(&e);
            pool.push_back(e);
        }
        return pool[used++];
    }
    void start(int ph)
    {
        if (!on) return;
        if (calls[ph]++ % every != 0) return;
        cur = ph;
        cur_a = used;
        cudaEventRecord(ev(), st);
    }
    void stop()
    {
        if (!on || cur < 0) return;
        const size_t b = used;
        cudaEventRecord(ev(), st);
        marks.push_back({cur, cur_a, b, 1});
        cur = -1;
    }
    // unsampled span over nl back-to-back launches of one phase (a round's step loop): the
    // launches keep overlapping each other (programmatic dependent launch) inside the span
    void span_start(int ph)
    {
        if (!on) return;
        cur = ph;
        cur_a = used;
        cudaEventRecord(ev(), st);
    }
    void span_stop(uint64_t nl)
    {
        if (!on || cur < 0) return;
        const size_t b = used;
        cudaEventRecord(ev(), st);
        marks.push_back({cur, cur_a, b, nl});
        calls[cur] += nl;
        cur = -1;
    }
    // call after the stream has been synchronised
    void harvest()
    {
        if (!on) return;
        // marks of a round still in flight (pipelined rounds) stay for a later harvest
        std::vector<Mark> keep;
        for (const Mark& m : marks) {
            if (cudaEventQuery(pool[m.b]) != cudaSuccess) {
                keep.push_back(m);
                continue;
            }
            float x = 0.f;
            if (cudaEventElapsedTime(&x, pool[m.a], pool[m.b]) == cudaSuccess) ms[m.ph] += x;
            launches[m.ph] += m.nl;
        }
        cudaGetLastError();   // clear cudaErrorNotReady
        marks.swap(keep);
        if (marks.empty() && cur < 0) used = 0;
    }
    void to_stats(cd_stats& s) const
    {
        s.ms_clear = ms[kPhClear];
        s.ms_propagate = ms[kPhPropagate];
        s.ms_insert = ms[kPhInsert];
        s.ms_scan = ms[kPhScan];
        s.ms_refine = ms[kPhRefine];
        s.ms_finalize = ms[kPhFinalize];
        s.ms_precompute = ms[kPhPrecompute];
        s.launches_clear = launches[kPhClear];
        s.launches_propagate = launches[kPhPropagate];
        s.launches_insert = launches[kPhInsert];
        s.launches_scan = launches[kPhScan];
        s.launches_refine = launches[kPhRefine];
        s.step_launches = calls[kPhPropagate] + calls[kPhScan];
    }
};

// One library call: device, stream, events, launch count.
struct Call {
    int prev_dev = -1, dev = -1;
    cudaStream_t st = nullptr;
    bool own_stream = false;
    cudaEvent_t ev0 = nullptr, ev1 = nullptr;
    LaunchCount lc;
    PhaseTimer pt;
    ~Call()
    {
        g_dev_alloc = DevAlloc{};
        g_pool = nullptr;
        if (ev0) cudaEventDestroy(ev0);
        if (ev1) cudaEventDestroy(ev1);
        if (own_stream && st) {
            cudaStreamSynchronize(st);
            cudaStreamDestroy(st);
        }
        if (prev_dev >= 0 && prev_dev != dev) cudaSetDevice(prev_dev);
    }
    cd_status begin(const cd_options& o)
    {
        int ndev = 0;
        if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev == 0)
            return fail(CD_ENODEV, "no CUDA device available");
        CU(cudaGetDevice(&prev_dev));
        dev = o.device >= 0 ? o.device : prev_dev;
        if (dev >= ndev) return fail(CD_EINVAL, "device %d out of range (%d devices)", dev, ndev);
        CU(cudaSetDevice(dev));
        int cc = dev < 64 ? g_cc[dev] : 0;
        if (!cc) {
            int major = 0, minor = 0;
            CU(cudaDeviceGetAttribute(&major, cudaDevAttrComputeCapabilityMajor, dev));
            CU(cudaDeviceGetAttribute(&minor, cudaDevAttrComputeCapabilityMinor, dev));
            cc = 10 * major + minor;
            if (dev < 64) g_cc[dev] = cc;
        }
        if (cc != 100)
            return fail(CD_ENODEV, "libcdscreen is built for sm_100a (B200); device %d is sm_%d",
                        dev, cc);
        g_pool = setup_pool(dev);
        g_dev_alloc = DevAlloc{o.alloc, o.free, o.alloc_ctx};
        if (o.stream) {
            st = (cudaStream_t)o.stream;
        } else {
            // a blocking stream: ordered after the work already queued on the legacy default
            // stream (e.g. the copies that produced device-resident inputs), cdscreen.h "Streams"
            CU(cudaStreamCreateWithFlags(&st, cudaStreamDefault));
            own_stream = true;
        }
        CU(cudaEventCreate(&ev0));
        CU(cudaEventCreate(&ev1));
        CU(cudaEventRecord(ev0, st));
        pt.on = o.profile_phases > 0;
        pt.every = o.profile_phases > 0 ? (uint64_t)o.profile_phases : 1;
        pt.st = st;
        return CD_OK;
    }
};

bool is_fin(double x) { return std::isfinite(x); }

cd_status validate_scalars(size_t n, double t0, double t1, double dt, double d, const cd_options& o,
                           int64_t* K)
{
    if (n >= 0xffffffffull) return fail(CD_EINVAL, "n = %zu must be < 2^32 - 1", n);
    if (!is_fin(t0) || !is_fin(t1) || !(t1 >= t0)) return fail(CD_EINVAL, "need finite t1 >= t0");
    if (!is_fin(dt) || !(dt > 0.0)) return fail(CD_EINVAL, "need dt > 0");
    if (!is_fin(d) || !(d > 0.0)) return fail(CD_EINVAL, "need threshold d > 0");
    if (!is_fin(o.v_margin) || o.v_margin < 0.0) return fail(CD_EINVAL, "need v_margin >= 0");
    if (!(o.cell_factor == 0.0 || o.cell_factor >= 1.0) || !is_fin(o.cell_factor))
        return fail(CD_EINVAL, "need cell_factor = 0 (auto) or >= 1");
    if (o.n_ranks < 1 || o.rank < 0 || o.rank >= o.n_ranks)
        return fail(CD_EINVAL, "need 0 <= rank < n_ranks");
    if (o.propagator != CD_PROP_KEPLER && o.propagator != CD_PROP_J2)
        return fail(CD_EINVAL, "unknown propagator %d", o.propagator);
    if (o.shards < 0 || o.shards > 64) return fail(CD_EINVAL, "need 0 <= shards <= 64");
    if (o.grid_table < 0 || o.grid_table > 3) return fail(CD_EINVAL, "grid_table %d: need 0..3", o.grid_table);
    if (kepler_class_of_points(o.kepler_points) < 0)
        return fail(CD_EINVAL, "kepler_points = %d: need 0 (per e) or 4, 6, 8, 12, 16", o.kepler_points);
    if ((o.alloc == nullptr) != (o.free == nullptr))
        return fail(CD_EINVAL, "cd_options.alloc and free must be given together");
    if (!is_fin(o.shell_lo) || !is_fin(o.shell_hi) || o.shell_lo < 0.0 ||
        (o.shell_hi != 0.0 && !(o.shell_hi > o.shell_lo)))
        return fail(CD_EINVAL, "need shell_hi = 0 (no shard) or shell_hi > shell_lo >= 0");
    for (int c = 0; c < 3; ++c)
        if (!is_fin(o.grid_origin[c])) return fail(CD_EINVAL, "grid_origin must be finite");
    const double kk = std::floor((t1 - t0) / dt) + 1.0;
    if (!(kk < 4294967295.0)) return fail(CD_EINVAL, "too many steps: K = %.0f", kk);
    *K = (int64_t)kk;
    return CD_OK;
}

// Validate element values (host copy) -- a > 0, 0 <= e < 1, finite angles.
cd_status validate_elements_host(const double* const v[6], size_t n)
{
    for (size_t i = 0; i < n; ++i) {
        const double a = v[0][i], e = v[1][i];
        if (!(a > 0.0) || !is_fin(a)) return fail(CD_EINVAL, "element %zu: a = %g must be > 0", i, a);
        if (!(e >= 0.0 && e < 1.0)) return fail(CD_EINVAL, "element %zu: e = %g must be in [0, 1)", i, e);
        for (int c = 2; c < 6; ++c)
            if (!is_fin(v[c][i])) return fail(CD_EINVAL, "element %zu: non-finite angle", i);
    }
    return CD_OK;
}

__global__ void k_validate(Elements el, int64_t n, int* bad)
{
    const int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (i >= n) return;
    const double a = el.a[i], e = el.e[i];
    bool ok = a > 0.0 && isfinite(a) && e >= 0.0 && e < 1.0 && isfinite(el.inc[i]) &&
              isfinite(el.raan[i]) && isfinite(el.argp[i]) && isfinite(el.nu0[i]);
    if (!ok) atomicMin(bad, (int)(i < 0x7fffffff ? i : 0x7ffffffe));
}

// Device-resident orbit records of one call (internal order sorted by eccentricity class).
struct OrbitSet {
    DBuf<double> rec;
    DBuf<double> arec;     // refinement records (object-major, kAoS doubles per object)
    DBuf<uint8_t> cls;
    DBuf<uint32_t> perm;   // internal -> caller index
    int64_t n0 = 0;        // class-0 objects (sorted first)
    int j2 = 0;            // CD_PROP_J2 records
    Orbits view() const
    {
        Orbits O;
        O.rec = rec.p;
        O.arec = arec.p;
        O.cls = cls.p;
        O.n = (int64_t)perm.n;
        O.n0 = n0;
        O.j2 = j2;
        return O;
    }
};

cd_status prepare_orbits(Call& C, const cd_elements* el, size_t n, const cd_options& o, OrbitSet& S)
{
    if (!el || !el->a || !el->e || !el->inc || !el->raan || !el->argp || !el->nu0)
        return fail(CD_EINVAL, "elements must be non-NULL");
    cudaStream_t st = C.st;
    S.rec.st = S.arec.st = S.cls.st = S.perm.st = st;
    DBuf<double> up(st);
    Elements E;
    const double* src[6] = {el->a, el->e, el->inc, el->raan, el->argp, el->nu0};
    if (o.inputs_on_device) {
        E = Elements{el->a, el->e, el->inc, el->raan, el->argp, el->nu0};
    } else {
        CU(up.alloc(6 * n));
        for (int c = 0; c < 6; ++c)
            CU(cudaMemcpyAsync(up.p + c * n, src[c], sizeof(double) * n, cudaMemcpyHostToDevice, st));
        E = Elements{up.p, up.p + n, up.p + 2 * n, up.p + 3 * n, up.p + 4 * n, up.p + 5 * n};
    }
    {   // validation on the device (a > 0, 0 <= e < 1, finite angles): first bad index
        DBuf<int> bad(st);
        CU(bad.alloc(1));
        int init = 0x7fffffff;
        CU(cudaMemcpyAsync(bad.p, &init, sizeof(int), cudaMemcpyHostToDevice, st));
        k_validate<<<(unsigned)((n + 255) / 256), 256, 0, st>>>(E, (int64_t)n, bad.p);
        C.lc.bump();
        CU(cudaGetLastError());
        int hb = 0;
        CU(cudaMemcpyAsync(&hb, bad.p, sizeof(int), cudaMemcpyDeviceToHost, st));
        CU(cudaStreamSynchronize(st));
        if (hb != 0x7fffffff) return fail(CD_EINVAL, "element %d: invalid (need a > 0, 0 <= e < 1, finite)", hb);
    }
    C.pt.start(kPhPrecompute);
    DBuf<uint32_t> key(st), idx(st), keyo(st);
    CU(key.alloc(n));
    CU(idx.alloc(n));
    CU(keyo.alloc(n));
    CU(S.perm.alloc(n));
    DBuf<unsigned long long> n0(st);
    CU(n0.alloc(1));
    CU(cudaMemsetAsync(n0.p, 0, sizeof(unsigned long long), st));
    const int min_cls = kepler_class_of_points(o.kepler_points);
    CU(launch_classify(E, (int64_t)n, key.p, idx.p, n0.p, min_cls, st, C.lc));
    unsigned long long hn0 = 0;
    CU(cudaMemcpyAsync(&hn0, n0.p, sizeof hn0, cudaMemcpyDeviceToHost, st));
    CU(sort_pairs_u32(key.p, keyo.p, idx.p, S.perm.p, n, 3, st, C.lc));
    S.j2 = o.propagator == CD_PROP_J2;
    CU(S.rec.alloc((size_t)(S.j2 ? kNCol : kDOm) * n));   // the J2 columns only when used
    CU(S.arec.alloc((size_t)kAoS * n));
    CU(S.cls.alloc(n));
    CU(launch_build_records(E, S.perm.p, (int64_t)n, S.rec.p, S.arec.p, S.cls.p, S.j2, min_cls, st, C.lc));
    C.pt.stop();
    CU(cudaStreamSynchronize(st));   // hn0 is needed on the host
    S.n0 = (int64_t)hn0;
    return CD_OK;
}

uint64_t next_pow2(uint64_t x)
{
    uint64_t p = 1;
    while (p < x) p <<= 1;
    return p;
}

enum class Want { Conj, Cand };

// Cell edge factor m (L = m g_c) from the measured candidate rate c (pairs within g_c per
// object-step): the expected local density is 2c / (4 pi / 3) objects per g_c^3.  Per object
// the scan probes (1 + 2/m)^3 - 1 cells (ball mode, m >= 2) or 13 (half-shell, m = 1) and walks
// the objects of those cells (~ (m + 2)^3 x density, or 27 x density / 2 in half-shell mode);
// a walked object costs about 1.5 probes.  Only performance depends on m (any L >= g_c gives
// the same candidate set).
#ifndef CD_WALK_WEIGHT
#define CD_WALK_WEIGHT 5.0
#endif
double choose_cell_factor(double c)
{
    const double dens = 2.0 * c / 4.18879;
    const double w = CD_WALK_WEIGHT;   // cost of one walked list entry relative to one probe
    double best = 1.0, bestcost = 13.0 + w * 13.5 * dens;
    const double cand[] = {2.0, 3.0, 4.0, 5.0, 6.0, 8.0};
    for (double m : cand) {
        const double probes = std::pow(1.0 + 2.0 / m, 3.0) - 1.0;
        const double cost = probes + w * std::pow(m + 2.0, 3.0) * dens;
        if (cost < bestcost) {
            bestcost = cost;
            best = m;
        }
    }
    return best;
}

// A-priori candidate count, the paper's Extra-P models (Section IV-B):
//   grid   (Eq. 3)  c' = 2.32e-9 n^2 s^(4/3) t d^(7/4)
//   hybrid (Eq. 4)  c' = 2.14e-9 n^2 s^(5/3) t d
// n objects, s seconds per sample, t simulated span [s], d threshold [km].  c' counts the
// (ids, step) entries of the paper's conjunction hash map, i.e. the candidate set; on the
// paper-shaped config-4 population it lands within 2x of the measured count.
double extra_p_candidates(double n, double s, double t, double d, cd_mode mode)
{
    if (mode == CD_HYBRID) return 2.14e-9 * n * n * std::pow(s, 5.0 / 3.0) * t * d;
    return 2.32e-9 * n * n * std::pow(s, 4.0 / 3.0) * t * std::pow(d, 1.75);
}

// Initial candidate-queue capacity (entries) of one call: at least 4M and 4n, grown so that a
// round at the a-priori candidate rate spans >= 64 steps (2^28 cap), like the measured-rate rule
size_t initial_qcap(int64_t n, double est_step)
{
    size_t qcap = std::max<size_t>(size_t(1) << 22, 4 * (size_t)n);
    const double wanted = est_step * 64.0 * 1.25;
    if (wanted > (double)qcap) qcap = (size_t)std::min(wanted, (double)(size_t(1) << 28));
    return qcap;
}

// The conjunction accumulation buffer: plain cudaMalloc (a few ms even for GBs, where growing the
// stream-ordered pool mid-screen was measured at up to ~1 s of blocked host thread), grow-only;
// a replaced buffer is retired and freed after the call's final synchronisation.
struct ConjBuf {
    Conj* p = nullptr;
    size_t n = 0;
    std::vector<Conj*> retired;
    DevAlloc user = g_dev_alloc;   // the caller's allocator, if the call has one
    ConjBuf() = default;
    ConjBuf(const ConjBuf&) = delete;
    ConjBuf& operator=(const ConjBuf&) = delete;
    ~ConjBuf()
    {
        for (Conj* r : retired) release(r);
        if (p) release(p);
    }
    void release(Conj* q)
    {
        if (user.free) user.free(q, user.ctx);
        else cudaFree(q);
    }
    // new buffer of `count` records; the first `keep` records are copied over (stream-ordered)
    cudaError_t grow(size_t count, size_t keep, cudaStream_t st)
    {
        Conj* np = nullptr;
        cudaError_t e = cudaSuccess;
        if (user.alloc) {
            np = static_cast<Conj*>(user.alloc(sizeof(Conj) * (count ? count : 1), user.ctx));
            if (!np) return cudaErrorMemoryAllocation;
        } else {
            e = cudaMalloc((void**)&np, sizeof(Conj) * (count ? count : 1));
        }
        if (e != cudaSuccess) return e;
        if (p && keep) e = cudaMemcpyAsync(np, p, sizeof(Conj) * keep, cudaMemcpyDeviceToDevice, st);
        if (p) retired.push_back(p);
        p = np;
        n = count;
        return e;
    }
    Conj* detach()
    {
        Conj* q = p;
        p = nullptr;
        n = 0;
        return q;
    }
};

struct Result {
    ConjBuf conj;           // unsorted conjunction records (internal ids)
    size_t n_conj = 0;
    DBuf<Cand> cand;        // accumulated candidates (cd_candidates)
    size_t n_cand = 0;
    // host result buffer (outputs on the host): an anonymous mapping advised for transparent
    // huge pages, so the copy-out faults in 2 MB pages instead of 4 KB ones (a 350 MB result
    // otherwise spends hundreds of ms in page faults); released with munmap
    void* host = nullptr;
    size_t host_bytes = 0;
    ~Result() { release_host(host, host_bytes); }
    static void release_host(void* p, size_t bytes)
    {
        if (p) munmap(p, bytes);
    }
    bool alloc_host(size_t count)
    {
        release_host(host, host_bytes);
        host = nullptr;
        const size_t huge = size_t(2) << 20;
        host_bytes = ((sizeof(Conj) * count + huge - 1) / huge) * huge;
        void* p = mmap(nullptr, host_bytes, PROT_READ | PROT_WRITE, MAP_PRIVATE | MAP_ANONYMOUS, -1, 0);
        if (p == MAP_FAILED) {
            host_bytes = 0;
            return false;
        }
        madvise(p, host_bytes, MADV_HUGEPAGE);   // best effort
        host = p;
        return true;
    }
    void* take_host(size_t* bytes)
    {
        void* p = host;
        *bytes = host_bytes;
        host = nullptr;
        host_bytes = 0;
        return p;
    }
};

// The screening loop over this rank's step slice.
cd_status run(Call& C, const OrbitSet& S, double t0, double t1, double dt, double d, cd_mode mode,
              const cd_options& o, int64_t K, Want want, Result& R, cd_stats& stats)
{
    cudaStream_t st = C.st;
    const Orbits O = S.view();
    const int64_t n = O.n;
    const int64_t kb = (int64_t)((__int128)K * o.rank / o.n_ranks);
    const int64_t ke = (int64_t)((__int128)K * (o.rank + 1) / o.n_ranks);
    stats.steps = (uint64_t)(ke - kb);
    stats.object_steps = (uint64_t)(ke - kb) * (uint64_t)n;
    const double gc = d + o.v_margin * dt;   // Eq. 1
    const bool digest = o.digest_only && want == Want::Conj;
    // grid cell edge L = m g_c (m = cell_factor; 0 = auto: start from the a-priori density, then
    // choose from the candidate density measured in the first round, see choose_cell_factor)
    const bool auto_cell = o.cell_factor == 0.0;
    // a-priori candidates per step (Eq. 3 / Eq. 4 with t = one sample): sizes the first round
    // and seeds the auto cell edge before the first round measures the real density
    const double est_step = std::max(1.0, extra_p_candidates((double)n, dt, dt, d, mode));
    double L = gc * (auto_cell ? choose_cell_factor(est_step / std::max<double>(1.0, (double)n)) : o.cell_factor);
    if (L < gc * (1.0 + 1e-12)) L = gc * (1.0 + 1e-12);
    GridGeom g;
    g.ox = o.grid_origin[0];
    g.oy = o.grid_origin[1];
    g.oz = o.grid_origin[2];
    g.inv_cell = 1.0 / L;
    g.gc2 = gc * gc;
    g.reach = gc * (1.0 + 1e-9) + 1e-9;
    g.halfshell = L < 2.0 * gc ? 1 : 0;
    // block-level candidate staging pays at dense candidate rates (>= 0.05 per object-step)
    g.stage = est_step / std::max<double>(1.0, (double)n) >= 0.05 ? 1 : 0;
    g.max_walk = (uint32_t)std::min<int64_t>(n + 1, 0xfffffffe);
    g.band_lo2 = o.shell_hi > 0.0 ? o.shell_lo * o.shell_lo : 0.0;
    g.band_hi2 = o.shell_hi > 0.0 ? o.shell_hi * o.shell_hi : HUGE_VAL;
    g.sig = nullptr;
    g.raw = o.emit_raw_counts ? 1 : 0;
    RefineParams P{t0, t1, dt, d, gc, nullptr};

    R.cand.st = st;
    if (ke <= kb || n < 2) return CD_OK;

    const uint64_t M = next_pow2((uint64_t)std::max<int64_t>(2 * n, 256));   // >= 2n slots (power of 2, >= 256: one CSR allocation block per step)
    const uint64_t mask = M - 1;
    const size_t target = o.batch_object_steps ? o.batch_object_steps : (size_t(1) << 20);
    int64_t Bmax = std::max<int64_t>(1, (int64_t)(target / (size_t)n));
    Bmax = std::min<int64_t>(Bmax, std::min<int64_t>(ke - kb, 65535));

    // per-step grid arena: [slot set 0 | slot set 1 | bitmap set 0 | 1 | 2] x Bmax tables, then
    // two entry buffers.  Launch i of a round builds batch b+1 (slot set (b+1) % 2 with tag
    // (b+1) % 126 + 1, bitmap set (b+1) % 3, entries (b+1) % 2), scans batch b and zeroes bitmap set
    // (b+2) % 3.  Slot sets are zeroed only when their tags wrap.
    // grid structure: 1 = the paper's open-addressing map (slots + occupancy bitmap); 2 = chained
    // spatial hash (bucket heads only); 0 = auto: chained (measured faster than the open map in
    // both scan modes: ball mode at L >= 2 g_c, 13 tagged half-shell buckets at L < 2 g_c), or
    // the CSR grid where the half-shell cells are crowded.  The open-addressing slots are
    // allocated under 0 for the CSR switch after the first round.  3 = CSR grid (sort + segment: the
    // open-addressing slots count each cell's objects, a counting sort makes each cell's entries
    // one contiguous segment).
    // sort + segment pays where the half-shell grid's cells are crowded: measured crossover (hybrid,
    // 1M ... 8M objects at 9 s) at ~2.6 candidates per object-step -- 1M (1.4): open map 421 vs
    // 459 us, 2M (2.6): even, 3M (3.9): -10 %, 4M (5.2): -25 %, 8M (10.4): -27 % per step
    constexpr double kCsrDensity = 3.0;   // candidates per object-step from which grid_table 0 uses it
    bool csr = o.grid_table == 3;
    const bool can_chain = o.grid_table != 1 && o.grid_table != 3, can_open = o.grid_table != 2;
#ifndef CD_CHAIN_FACTOR
#define CD_CHAIN_FACTOR 8
#endif
    const uint64_t chain_words = can_chain ? std::max<uint64_t>(next_pow2((uint64_t)n * CD_CHAIN_FACTOR), 1024) : 0;
    const uint64_t nbits = std::max<uint64_t>(next_pow2((uint64_t)n * 32), 1024);   // open: >= 32 bits/object
    const uint32_t bwords = (uint32_t)std::max<uint64_t>(chain_words, can_open ? nbits / 32 : 0);
    // memory-bounded grids in flight (p = (m - a_s - a_k - a_ch) / (a_gh + a_l)): a
    // batch of B steps holds B grids in each rotating set (2 slot sets, 3 bitmap / head sets, 3
    // entry sets, CSR scratch); B never exceeds what the free device memory holds, keeping an
    // eighth and 256 MB back for queues, sort scratch and results.  (On a 180 GB B200 the default
    // batch, 2^20 object-steps, is the binding limit up to ~10^8 objects.)
    {
        const double per = (can_open ? 2.0 * sizeof(Slot) * (double)M : 0.0) + 3.0 * 4.0 * (double)bwords +
                           3.0 * sizeof(Entry) * (double)n +
                           (csr ? sizeof(Entry) * (double)n + 2.0 * 4.0 * (double)M : 0.0);
        size_t fr = 0, tot = 0;
        // the free-memory query costs a driver call: only when the batch could come near it
        if (per * (double)Bmax > 4e9 && cudaMemGetInfo(&fr, &tot) == cudaSuccess) {
            const double avail = (double)fr * 0.875 - 256e6;
            const int64_t p = avail > 0.0 ? (int64_t)(avail / per) : 0;
            if (p < 1)
                return fail(CD_ENOMEM, "one step's grid (%.3g GB per rotating set) does not fit the free device memory (%.3g GB)",
                            per / 1e9, (double)fr / 1e9);
            Bmax = std::min<int64_t>(Bmax, p);
        }
        cudaGetLastError();
    }
    stats.grids_in_flight = (uint64_t)Bmax;
    const size_t slot_bytes = can_open ? sizeof(Slot) * (size_t)Bmax * M : 0;
    auto pick_chained = [&](const GridGeom& gg) {
        if (n > (int64_t)kMaxChainN) return false;   // 24-bit head indices
        (void)gg;   // chained in both scan modes (half-shell: 13 tagged buckets, measured 280 -> 241 us
                    // per 1M-object hybrid coarse step against the open map)
        return o.grid_table == 2 || o.grid_table == 0;
    };
    bool chained = pick_chained(g);
    const size_t bit_bytes = ((sizeof(uint32_t) * (size_t)Bmax * bwords + 255) / 256) * 256;
    const size_t ent_bytes = sizeof(Entry) * (size_t)Bmax * n;
    const size_t tab_bytes = 2 * slot_bytes + 3 * bit_bytes;
    DBuf<unsigned char> arena(st);
    DBG("run: alloc arena", (long long)(tab_bytes + 3 * ent_bytes));
    CU(arena.alloc(tab_bytes + 3 * ent_bytes));
    DBG("run: arena allocated");
    CU(cudaMemsetAsync(arena.p, 0, tab_bytes, st));
    Slot* slotset[2] = {reinterpret_cast<Slot*>(arena.p), reinterpret_cast<Slot*>(arena.p + slot_bytes)};
    uint32_t* bitset[3];
    for (int h = 0; h < 3; ++h)
        bitset[h] = reinterpret_cast<uint32_t*>(arena.p + 2 * slot_bytes + h * bit_bytes);
    // three entry buffers: with programmatic dependent launch, launch i + 1 builds batch b + 2
    // while launch i may still scan batch b (and build b + 1)
    Entry* entbuf[3];
    for (int h = 0; h < 3; ++h) entbuf[h] = reinterpret_cast<Entry*>(arena.p + tab_bytes + h * ent_bytes);
    // CSR grid: per-object (slot, rank) entries of the batch being built, segment starts per slot
    // (two sets, like the slots), per-step object totals; the segments go to entbuf
    DBuf<Entry> csr_tmp(st);
    DBuf<uint32_t> csr_start(st);
    DBuf<unsigned long long> csr_total(st);
    auto csr_alloc = [&]() -> cd_status {
        if (csr_tmp.p) return CD_OK;
        CU(csr_tmp.alloc((size_t)Bmax * n));
        CU(csr_start.alloc(2 * (size_t)Bmax * M));
        CU(csr_total.alloc((size_t)Bmax));
        return CD_OK;
    };
    if (csr) TRY(csr_alloc());
    static const bool no_pdl = getenv("CD_NO_PDL") != nullptr;   // A/B switch for experiments
    auto tab_of = [&](uint64_t b) {
        return GridTab{slotset[b % 2], bitset[b % 3],
                       chained ? (uint32_t)(chain_words - 1) : (uint32_t)(nbits - 1), bwords};
    };
    // key tags (open map, 7 bits) / head epochs (chained grid, 8 bits): never 0 (= cleared)
    auto tag_of = [&](uint64_t b) {
        return chained ? (uint32_t)(b % 255u) + 1u : (uint32_t)(b % kMaxTag) + 1u;
    };
    uint64_t batch_no = 0;
    // persisting-L2 window over the slot and bitmap sets (they take the random atomics and
    // probes; records, entries and candidate writes stream past them)
    L2Win win;
    if (o.l2_persist) {
        int maxwin = 0, maxpersist = 0;
        cudaDeviceGetAttribute(&maxwin, cudaDevAttrMaxAccessPolicyWindowSize, C.dev);
        cudaDeviceGetAttribute(&maxpersist, cudaDevAttrMaxPersistingL2CacheSize, C.dev);
        if (maxwin > 0 && maxpersist > 0) {
            size_t cur = 0;
            cudaDeviceGetLimit(&cur, cudaLimitPersistingL2CacheSize);
            const size_t setaside = std::min<size_t>((size_t)maxpersist, tab_bytes);
            if (cur < setaside) cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, setaside);
            cudaDeviceGetLimit(&cur, cudaLimitPersistingL2CacheSize);
            win.on = cur > 0;
            win.w.base_ptr = arena.p;
            win.w.num_bytes = std::min<size_t>(tab_bytes, (size_t)maxwin);
            win.w.hitRatio = (float)std::min(1.0, (double)cur / (double)win.w.num_bytes);
            win.w.hitProp = cudaAccessPropertyPersisting;
            win.w.missProp = cudaAccessPropertyStreaming;
        }
        cudaGetLastError();   // persistence is best effort
    }
    size_t qcap = initial_qcap(n, est_step);
    DBuf<Cand> q(st);
    CU(q.alloc(qcap));
    // work items (prefilter / hybrid-filter survivors) are a small fraction of the candidates:
    // start at the base capacity, grow on demand (retry path)
    size_t wcap = want == Want::Conj ? std::min(qcap, std::max<size_t>(size_t(1) << 22, 4 * (size_t)n)) : 0;
    DBuf<Work> w(st);
    if (want == Want::Conj) CU(w.alloc(wcap));
    size_t ocap = size_t(1) << 20;
    if (want == Want::Conj) {
        Conj* cp = nullptr;
        size_t cc = 0;
        if (!g_dev_alloc.alloc && conj_cache_take(C.dev, st, &cp, &cc) && cc >= ocap) {
            R.conj.p = cp;
            R.conj.n = cc;
            ocap = cc;
        } else {
            if (cp) cudaFree(cp);
            CU(R.conj.grow(ocap, 0, st));
        }
    }
    size_t ccap = want == Want::Cand ? (size_t(1) << 20) : 0;
    if (want == Want::Cand) CU(R.cand.alloc(ccap));

    DBuf<unsigned char> hrec(st);
    if (mode == CD_HYBRID && want == Want::Conj) {
        CU(hrec.alloc(hybrid_record_bytes() * (size_t)n));
        CU(launch_build_hybrid_records(O, hrec.p, st, C.lc));
        P.hrec = hrec.p;
    }
    DBuf<Ctrl> ctrl(st);
    CU(ctrl.alloc(1));
    CU(cudaMemsetAsync(ctrl.p, 0, sizeof(Ctrl), st));
    DBuf<unsigned long long> nwork(st);
    CU(nwork.alloc(1));
    // pinned host staging of the per-round counters: two slots (rounds r and r + 1 in flight),
    // cached per host thread so no call pays a page-locked allocation (an RM call that contends
    // with NVML clients such as nvidia-smi)
    Ctrl* hslot[2];
    unsigned long long* hnw[2];
    {
        Ctrl* base = nullptr;
        TRY(pinned_stage(&base));
        for (int s = 0; s < 2; ++s) {
            hslot[s] = base + 2 * s;
            hnw[s] = reinterpret_cast<unsigned long long*>(base + 2 * s + 1);
        }
    }
    DBG("run: staging ready");
    cudaEvent_t rev[2] = {nullptr, nullptr};
    struct EvFree {
        cudaEvent_t* e;
        ~EvFree() { for (int s = 0; s < 2; ++s) if (e[s]) cudaEventDestroy(e[s]); }
    } evf{rev};
    for (int s = 0; s < 2; ++s) CU(cudaEventCreateWithFlags(&rev[s], cudaEventDisableTiming));

    // spatial slot order (cd_options.resort_steps): build and scan run over
    // slots; every R steps the slots are renumbered in Morton order of the positions of the last
    // built step.  Hot build records / class bytes / slot -> internal id map, double-buffered:
    // a launch builds batch b + 1 in the new order while it scans batch b in the old one.
    const int rs_opt = o.resort_steps;
    // auto: on for populations whose per-step grid is far beyond L2 (>= 4M objects, grid variant;
    // measured at 8M: 894 -> 785 us per step with R = 64 at dt = 1 s), off below (at 1M the
    // re-sort costs more than the locality returns: 60.3 vs 61.4 us per step)
    const int64_t resort_auto = (n >= 4000000 && mode == CD_GRID)
                                    ? std::max<int64_t>(16, (int64_t)std::llround(64.0 / dt)) : 0;
    const int64_t resort_R = rs_opt < 0 ? 0 : rs_opt > 0 ? rs_opt : resort_auto;
    const bool spatial = resort_R > 0 && n >= 4096 && !csr;   // (CSR segments are cell-ordered)
    // auto sort + segment (grid_table 0, half-shell map, no spatial order): from the a-priori
    // density now, from the measured one once the first round has settled the cell edge
    auto pick_csr = [&](double per_object_step) {
        return o.grid_table == 3 ||
               (o.grid_table == 0 && !spatial && g.halfshell && per_object_step >= kCsrDensity);
    };
    csr = pick_csr(est_step / std::max<double>(1.0, (double)n));
    if (csr) {
        chained = false;
        TRY(csr_alloc());
    }
    const int ncolH = S.j2 ? kNCol : kDOm;
    DBuf<double> Hrec[2] = {DBuf<double>(st), DBuf<double>(st)};
    DBuf<uint8_t> Hcls[2] = {DBuf<uint8_t>(st), DBuf<uint8_t>(st)};
    DBuf<uint32_t> Hsig[2] = {DBuf<uint32_t>(st), DBuf<uint32_t>(st)};
    DBuf<unsigned long long> rkey(st), rkey2(st);
    DBuf<uint32_t> rval(st), rval2(st);
    DBuf<unsigned char> rtmp(st);
    SpaceSort SS{};
    if (spatial) {
        for (int h = 0; h < 2; ++h) {
            CU(Hrec[h].alloc((size_t)ncolH * (size_t)n));
            CU(Hcls[h].alloc((size_t)n));
            CU(Hsig[h].alloc((size_t)n));
        }
        CU(rkey.alloc((size_t)n));
        CU(rkey2.alloc((size_t)n));
        CU(rval.alloc((size_t)n));
        CU(rval2.alloc((size_t)n));
        CU(space_sort_temp_bytes(n, &SS.tmp_bytes));
        CU(rtmp.alloc(SS.tmp_bytes));
        SS = SpaceSort{rkey.p, rkey2.p, rval.p, rval2.p, rtmp.p, SS.tmp_bytes};
    }
    int order_ver = -1;                       // -1: slots are internal ids (no order yet)
    int batch_ver[3] = {-1, -1, -1};          // order version each entry buffer was built with
    int64_t since_resort = resort_R;          // steps built since the last re-sort
    auto hot_view = [&](int v) {
        if (v < 0) return O;
        Orbits h = O;
        h.rec = Hrec[v & 1].p;
        h.cls = Hcls[v & 1].p;
        return h;
    };
    auto sig_of = [&](int v) -> const uint32_t* { return v < 0 ? nullptr : Hsig[v & 1].p; };

    // first round: half the queue at the a-priori rate; in auto-cell mode it is also the density
    // probe, kept short (enough candidates for a density estimate, <= 41 steps)
    int64_t Rsteps = o.round_steps ? (int64_t)o.round_steps
                                   : std::max<int64_t>(1, std::min<int64_t>(1 << 16, (int64_t)(0.5 * (double)qcap / est_step)));
    if (!o.round_steps && auto_cell)
        Rsteps = std::max<int64_t>(1, std::min<int64_t>(Rsteps, std::min<int64_t>(41, (int64_t)std::ceil(2e5 / est_step))));
    // cumulative device counters as of the last accepted round (the rollback state of a redo)
    unsigned long long conj_before = 0;
    unsigned long long hyb_before[4] = {0, 0, 0, 0};
    // the cell edge is settled once the first round has measured the candidate density
    bool settled = !auto_cell;
    // rounds are software-pipelined one deep: round r + 1 is enqueued before the host waits for
    // round r's counters, so the GPU never idles while the host checks capacities and enqueues
    // the next ~500 launches.  Capacity overflows are rare: the later round is drained and both
    // are redone.  The candidate hook (Want::Cand) copies each accepted round's queue out, so it
    // runs unpipelined.
    const int depth = want == Want::Cand ? 1 : 2;
    struct Round { int64_t k, Rk; int slot; size_t qcap, wcap, ocap; };   // capacities it ran with
    Round inflight[2];
    int nin = 0, next_slot = 0;
    auto enqueue_round = [&](int64_t kr, int64_t Rk, int slot) -> cd_status {
        CU(cudaMemsetAsync(&ctrl.p->n_cand, 0, sizeof(unsigned long long), st));
        CU(cudaMemsetAsync(&ctrl.p->n_raw, 0, sizeof(unsigned long long), st));
        CU(cudaMemsetAsync(nwork.p, 0, sizeof(unsigned long long), st));
        // software pipeline over the round's batches: launch i builds batch i and scans i - 1
        const int64_t J = (Rk + Bmax - 1) / Bmax;
        for (int64_t i = 0; i <= J; ++i) {
            StepArgs sa{};
            if (spatial && i < J && since_resort >= resort_R && batch_no + (uint64_t)i >= 1) {
                // re-sort from the positions of the last built batch (its step 0)
                const uint64_t prev = batch_no + (uint64_t)i - 1;
                const int v = order_ver;
                const int nv = v + 1;
                const Orbits hv = hot_view(v);
                CU(space_resort(SS, entbuf[prev % 3], hv.rec, hv.cls, sig_of(v), n, ncolH, S.j2,
                                Hrec[nv & 1].p, Hcls[nv & 1].p, Hsig[nv & 1].p, st, C.lc));
                order_ver = nv;
                since_resort = 0;
            }
            sa.O = hot_view(order_ver);
            sa.g = g;
            sa.mask = mask;
            sa.t0 = t0;
            sa.dt = dt;
            sa.q = q.p;
            sa.qcap = qcap;
            sa.ctrl = ctrl.p;
            const uint64_t bb = batch_no + (uint64_t)i;   // batch built in this launch
            if (i < J) {
                if (chained && bb % 255u < 3 && bb >= 3) {
                    // head set bb % 3 is used by batches of one residue mod 3; its epochs
                    // (bb % 255 + 1) would repeat within the next 255 batches: zero it (its
                    // last scan, of batch bb - 3, finished two launches ago)
                    CU(cudaMemsetAsync(bitset[bb % 3], 0, bit_bytes, st));
                }
                if (can_open && bb % kMaxTag < 2 && bb >= 2) {
                    // this slot set's tags wrap with this batch: zero it (its last scan, of
                    // batch bb - 2, finished in the previous launch)
                    CU(cudaMemsetAsync(slotset[bb % 2], 0, slot_bytes, st));
                }
                sa.build_k0 = kr + i * Bmax;
                sa.build_B = std::min<int64_t>(Bmax, kr + Rk - sa.build_k0);
                sa.build_tab = tab_of(bb);
                sa.build_ents = csr ? csr_tmp.p : entbuf[bb % 3];
                sa.build_tag = tag_of(bb);
                batch_ver[bb % 3] = order_ver;
                since_resort += sa.build_B;
            }
            if (i > 0) {
                sa.scan_k0 = kr + (i - 1) * Bmax;
                sa.scan_B = std::min<int64_t>(Bmax, kr + Rk - sa.scan_k0);
                sa.scan_tab = tab_of(bb - 1);
                sa.scan_ents = entbuf[(bb - 1) % 3];
                sa.scan_tag = tag_of(bb - 1);
                sa.g.sig = sig_of(batch_ver[(bb - 1) % 3]);
                if (csr) sa.scan_start = csr_start.p + ((bb - 1) % 2) * (size_t)Bmax * M;
            }
            sa.csr = csr ? 1 : 0;
            sa.zero_bits = bitset[(bb + 1) % 3];   // batch bb - 2's bitmaps, next built by bb + 1
            sa.zero_bits_words = bwords;
            sa.zero_depth = chained ? 0 : Bmax;   // chained heads are epoch-tagged
            sa.chained = chained ? 1 : 0;
            sa.pdl = chained && !no_pdl ? 1 : 0;
            if (i == 0) C.pt.span_start(kPhScan);
            CU(launch_step(sa, &win, st, C.lc));
            if (csr && i < J)   // segments of the batch just built, for the next launch's scan
                CU(launch_csr_segments(slotset[bb % 2], csr_start.p + (bb % 2) * (size_t)Bmax * M, M,
                                       csr_tmp.p, entbuf[bb % 3], n, (int)sa.build_B, tag_of(bb),
                                       csr_total.p, st, C.lc));
        }
        C.pt.span_stop((uint64_t)J + 1);
        batch_no += (uint64_t)J;
        if (want == Want::Conj) {
            C.pt.start(kPhRefine);
            if (mode == CD_HYBRID) {
                CU(launch_hybrid_filter(O, P, q.p, qcap, w.p, wcap, nwork.p, R.conj.p, ocap, ctrl.p,
                                        st, C.lc));
                CU(launch_brent(O, P, w.p, nwork.p, wcap, R.conj.p, ocap, ctrl.p, st, C.lc));
            } else {
                CU(launch_prefilter(O, P, q.p, qcap, w.p, wcap, nwork.p, R.conj.p, ocap, ctrl.p, st,
                                    C.lc));
                CU(launch_brent(O, P, w.p, nwork.p, wcap, R.conj.p, ocap, ctrl.p, st, C.lc));
            }
            C.pt.stop();
        }
        CU(cudaMemcpyAsync(hslot[slot], ctrl.p, sizeof(Ctrl), cudaMemcpyDeviceToHost, st));
        CU(cudaMemcpyAsync(hnw[slot], nwork.p, sizeof(unsigned long long), cudaMemcpyDeviceToHost, st));
        if (digest)   // after the snapshot: the snapshot's digest is that of the rounds before
            CU(launch_conj_digest(R.conj.p, ocap, S.perm.p, ctrl.p, st, C.lc));
        CU(cudaEventRecord(rev[slot], st));
        DBG("round: enqueued", (long long)kr, (long long)Rk);
        return CD_OK;
    };

    int64_t k = kb;
    while (k < ke || nin > 0) {
        if (k < ke && nin < depth && (settled || nin == 0)) {
            const int64_t Rk = std::min<int64_t>(Rsteps, ke - k);
            const int slot = next_slot;
            next_slot ^= 1;
            TRY(enqueue_round(k, Rk, slot));
            inflight[nin++] = Round{k, Rk, slot, qcap, wcap, ocap};
            k += Rk;
            continue;
        }
        // wait for the oldest round in flight
        const Round rd = inflight[0];
        if (nin == 2) inflight[0] = inflight[1];
        --nin;
        CU(cudaEventSynchronize(rev[rd.slot]));
        DBG("round: synced", (long long)rd.k, (long long)rd.Rk);
        C.pt.harvest();
        const Ctrl* hctrl = hslot[rd.slot];
        const unsigned long long hnwork = *hnw[rd.slot];
        if (hctrl->err_internal)
            return fail(CD_EINTERNAL, "internal: a grid cell list did not terminate");
        if (hctrl->err_range)
            return fail(CD_ERANGE, "a position fell outside the cell-key range (+-%lld cells of edge %g km)",
                        (long long)kCellMax, L);
        bool redo = false;
        if (hctrl->n_cand > rd.qcap) {
            ++stats.retries;
            if (rd.Rk > 1) {
                const double rate = (double)hctrl->n_cand / (double)rd.Rk;
                Rsteps = std::max<int64_t>(1, std::min<int64_t>(rd.Rk / 2, (int64_t)(0.5 * rd.qcap / rate)));
            } else {
                qcap = (size_t)(hctrl->n_cand * 1.25) + 1024;
                CU(q.alloc(qcap));
                if (want == Want::Conj) {
                    wcap = qcap;
                    CU(w.alloc(wcap));
                }
            }
            redo = true;
        } else if (want == Want::Conj && hnwork > rd.wcap) {
            ++stats.retries;
            wcap = std::max(wcap, (size_t)(hnwork * 1.25) + 1024);
            CU(w.alloc(wcap));
            redo = true;
        } else if (want == Want::Conj && hctrl->n_conj > rd.ocap) {
            ++stats.retries;
            const size_t ncap = std::max<size_t>(2 * ocap, (size_t)(hctrl->n_conj * 1.25) + 1024);
            CU(R.conj.grow(ncap, conj_before, st));
            ocap = ncap;
            redo = true;
        }
        if (redo) {
            // drain the later round (if any), roll the cumulative counters back to the last
            // accepted round and restart from this round's first step
            CU(cudaStreamSynchronize(st));
            C.pt.harvest();
            nin = 0;
            Ctrl back = *hctrl;
            back.n_conj = conj_before;
            back.n_ap = hyb_before[0];
            back.n_coplanar = hyb_before[1];
            back.n_path = hyb_before[2];
            back.n_time = hyb_before[3];
            back.n_cand = 0;
            back.n_raw = 0;
            back.err_range = 0;
            back.err_internal = 0;
            Ctrl* stage = hslot[rd.slot];
            *stage = back;
            CU(cudaMemcpyAsync(ctrl.p, stage, sizeof(Ctrl), cudaMemcpyHostToDevice, st));
            CU(cudaStreamSynchronize(st));
            k = rd.k;
            continue;
        }
        // round accepted
        stats.candidates += hctrl->n_cand;
        stats.raw_pairs += hctrl->n_raw;
        stats.refined += hnwork;
        if (want == Want::Cand && hctrl->n_cand) {
            if (R.n_cand + hctrl->n_cand > ccap) {
                const size_t ncap = std::max<size_t>(2 * ccap, R.n_cand + hctrl->n_cand + 1024);
                DBuf<Cand> nb(st);
                CU(nb.alloc(ncap));
                if (R.n_cand)
                    CU(cudaMemcpyAsync(nb.p, R.cand.p, sizeof(Cand) * R.n_cand, cudaMemcpyDeviceToDevice, st));
                std::swap(R.cand.p, nb.p);
                std::swap(R.cand.n, nb.n);
                ccap = ncap;
            }
            CU(cudaMemcpyAsync(R.cand.p + R.n_cand, q.p, sizeof(Cand) * hctrl->n_cand,
                               cudaMemcpyDeviceToDevice, st));
            R.n_cand += hctrl->n_cand;
        }
        conj_before = digest ? 0 : hctrl->n_conj;   // (digest_only: the buffer was emptied)
        hyb_before[0] = hctrl->n_ap;
        hyb_before[1] = hctrl->n_coplanar;
        hyb_before[2] = hctrl->n_path;
        hyb_before[3] = hctrl->n_time;
        // grow the work and output buffers ahead of need (a round that overflows is redone).
        // Both reallocations are stream-ordered behind the round still in flight: the output
        // copy moves the whole old buffer, including what that round appends; it is checked
        // against the capacities it ran with (Round).
        if (want == Want::Conj && hnwork > wcap / 2) {
            wcap = std::max<size_t>(2 * wcap, 2 * hnwork);
            CU(w.alloc(wcap));
        }
        // output: grown once the projected total (x 1.25) would not fit, to 1.5x the projection,
        // so a long screen grows it early (little to copy) and rarely
        const double done_steps = (double)(rd.k + rd.Rk - kb);
        const double proj_conj = (double)conj_before * (double)(ke - kb) / std::max(1.0, done_steps);
        // (from the first round on: it runs alone, so growing after it leaves no round in flight
        // with the old capacity -- measured: a first growth one round later made the round then in
        // flight overflow and be redone, 118 of 200 steps at 8M objects)
        if (want == Want::Conj && (1.25 * proj_conj > (double)ocap || conj_before > ocap * 9 / 10)) {
            const size_t ncap = std::max<size_t>(2 * ocap, (size_t)(1.5 * proj_conj));
            DBG("grow: output", (long long)ocap, (long long)ncap);
            CU(R.conj.grow(ncap, ocap, st));
            DBG("grow: allocated");
            ocap = ncap;
        }
        if (!settled) {   // first round done: pick the cell edge from the measured density
            const double dens = (double)hctrl->n_cand / ((double)rd.Rk * (double)n);
            const double m = choose_cell_factor(dens);
            g.stage = dens >= 0.05 ? 1 : 0;
            L = gc * m;
            if (L < gc * (1.0 + 1e-12)) L = gc * (1.0 + 1e-12);
            g.inv_cell = 1.0 / L;
            g.halfshell = L < 2.0 * gc ? 1 : 0;
            const bool was_chained = chained;
            chained = pick_chained(g);
            csr = pick_csr(dens);
            if (csr) {
                chained = false;
                TRY(csr_alloc());
            }
            if (chained != was_chained) {
                // the bitmap / head sets change meaning (occupancy bits <-> epoch-tagged list
                // heads): clear all three, stream-ordered after the round already in flight
                CU(cudaMemsetAsync(bitset[0], 0, 3 * bit_bytes, st));
            }
            settled = true;
        }
        if (!o.round_steps) {
            const double rate = std::max(1.0, (double)hctrl->n_cand / (double)rd.Rk);
            // dense candidate rates (hybrid): grow the queue so a round spans >= 64 steps, within
            // a 2^28-entry (3 GB) cap.  The queue is reallocated stream-ordered: a round still
            // in flight keeps the old buffer until it finishes.
            const double wanted = rate * 64.0 * 1.25;
            if (wanted > (double)qcap && qcap < (size_t(1) << 28)) {
                qcap = (size_t)std::min(wanted, (double)(size_t(1) << 28));
                CU(q.alloc(qcap));   // (the work-item buffer grows on demand via the retry path)
            }
            Rsteps = std::max<int64_t>(1, std::min<int64_t>(1 << 16, (int64_t)(0.5 * qcap / rate)));
        }
    }
    R.n_conj = (size_t)conj_before;
    if (digest) {   // the last round's digest ran after its snapshot: read the final counters
        Ctrl fin;
        CU(cudaMemcpyAsync(&fin, ctrl.p, sizeof(Ctrl), cudaMemcpyDeviceToHost, st));
        CU(cudaStreamSynchronize(st));
        stats.digest = fin.dg_sum;
        stats.digest_conjunctions = fin.dg_count;
        const unsigned long long bits = ~fin.dg_notminpca;
        double mp;
        memcpy(&mp, &bits, sizeof mp);
        stats.min_pca = fin.dg_count ? mp : INFINITY;
        R.n_conj = 0;
    }
    stats.cell_factor = L / gc;
    stats.grid_table = csr ? 3 : chained ? 2 : 1;
    stats.hybrid_ap_rejected = hyb_before[0];
    stats.hybrid_coplanar = hyb_before[1];
    stats.hybrid_path_rejected = hyb_before[2];
    stats.hybrid_time_rejected = hyb_before[3];
    return CD_OK;
}

// Legacy full-window filter chain (mode CD_LEGACY, cd_legacy.cu): the
// n(n-1)/2 pairs are filtered in chunks; each chunk's intervals are searched before the next
// chunk is filtered.  A chunk whose work items or records overflow is redone with larger
// buffers (device counters restored first).  Ranks share the pairs by contiguous ranges.
cd_status run_legacy(Call& C, const OrbitSet& S, double t0, double t1, double dt, double d,
                     const cd_options& o, int64_t K, Result& R, cd_stats& stats)
{
    cudaStream_t st = C.st;
    const Orbits O = S.view();
    const int64_t n = O.n;
    const unsigned __int128 total = n >= 2 ? (unsigned __int128)n * (unsigned __int128)(n - 1) / 2 : 0;
    const uint64_t pb = (uint64_t)(total * (unsigned)o.rank / (unsigned)o.n_ranks);
    const uint64_t pe = (uint64_t)(total * (unsigned)(o.rank + 1) / (unsigned)o.n_ranks);
    stats.steps = (uint64_t)K;
    stats.object_steps = (uint64_t)K * (uint64_t)n;
    stats.candidates = pe - pb;   // pairs screened by this rank
    if (pe <= pb) return CD_OK;
    LegacyParams P{t0, t1, dt, d, K};
    DBuf<unsigned char> hrec(st);
    CU(hrec.alloc(hybrid_record_bytes() * (size_t)n));
    CU(launch_build_hybrid_records(O, hrec.p, st, C.lc));
    DBuf<Ctrl> ctrl(st);
    CU(ctrl.alloc(1));
    CU(cudaMemsetAsync(ctrl.p, 0, sizeof(Ctrl), st));
    DBuf<unsigned long long> cnt(st);   // [0] work items, [1] next item of the search
    CU(cnt.alloc(2));
    size_t wcap = size_t(1) << 22;
    DBuf<Work> w(st);
    CU(w.alloc(wcap));
    size_t ocap = size_t(1) << 20;
    CU(R.conj.grow(ocap, 0, st));
    Ctrl before{}, after{};
    unsigned long long hw[2];
    uint64_t chunk = uint64_t(1) << 26;
    C.pt.start(kPhRefine);
    for (uint64_t p0 = pb; p0 < pe;) {
        const uint64_t p1 = std::min<uint64_t>(pe, p0 + chunk);
        CU(cudaMemcpyAsync(&before, ctrl.p, sizeof(Ctrl), cudaMemcpyDeviceToHost, st));
        CU(cudaMemsetAsync(cnt.p, 0, 2 * sizeof(unsigned long long), st));
        CU(launch_legacy_filter(P, hrec.p, n, p0, p1, w.p, wcap, cnt.p, ctrl.p, st, C.lc));
        CU(launch_legacy_search(O, P, hrec.p, w.p, cnt.p, wcap, cnt.p + 1, R.conj.p, ocap, ctrl.p, st,
                                C.lc));
        CU(cudaMemcpyAsync(hw, cnt.p, sizeof hw, cudaMemcpyDeviceToHost, st));
        CU(cudaMemcpyAsync(&after, ctrl.p, sizeof(Ctrl), cudaMemcpyDeviceToHost, st));
        CU(cudaStreamSynchronize(st));
        const bool wover = hw[0] > wcap, oover = after.n_conj > ocap;
        if (wover || oover) {   // redo the chunk with room for it
            ++stats.retries;
            if (wover) {
                wcap = (size_t)(hw[0] * 1.25) + 1024;
                CU(w.alloc(wcap));
            }
            if (oover) {
                const size_t ncap = std::max<size_t>(2 * ocap, (size_t)(after.n_conj * 1.25) + 1024);
                CU(R.conj.grow(ncap, before.n_conj, st));
                ocap = ncap;
            }
            CU(cudaMemcpyAsync(ctrl.p, &before, sizeof(Ctrl), cudaMemcpyHostToDevice, st));
            continue;
        }
        p0 = p1;
        // keep a chunk's work items within the buffer: grow the chunk while they fill < 1/4
        if (hw[0] < wcap / 4 && chunk < (uint64_t(1) << 34)) chunk *= 2;
        else if (hw[0] > wcap / 2 && chunk > (uint64_t(1) << 16)) chunk /= 2;
    }
    C.pt.stop();
    R.n_conj = (size_t)after.n_conj;
    stats.refined = after.n_refined;
    stats.hybrid_ap_rejected = after.n_ap;
    stats.hybrid_coplanar = after.n_coplanar;
    stats.hybrid_path_rejected = after.n_path;
    stats.hybrid_time_rejected = after.n_time;
    return CD_OK;
}

// Radial shards screened in turn on one device (cd_options.shards; SURVEY 8(f) row 2 applied
// on one device): a large population's per-step grid (~64 B per object) overflows the 126 MB L2
// and the scan turns into DRAM-latency-bound random access, and a population beyond HBM needs
// its grid split.  The objects are split into S radial bands (quantiles of a);
// each band is screened in turn with only its members (cd_shell_members' rule: own band + g_c
// halo above it) and keeps the candidates whose smaller radius lies in the band, so the union of
// the bands' results is exactly the unsharded result (tests/test_gpu_shards.py).  Measured on
// one B200 at 8M objects (tools/shard_sweep.py, device-resident inputs, tuned cell edge): 1407
// us per step unsharded, 1456 / 1427 / 1608 with 2 / 3 / 4 bands -- the halo and the eccentric
// objects replicated into every band cost what the smaller grid saves -- so the default is off;
// the option bounds the per-call grid memory (a band holds ~n/S objects plus its halo).
int shard_count(const cd_options& o, size_t n, cd_mode mode)
{
    (void)n;
    if (mode == CD_LEGACY || o.shell_hi != 0.0) return 1;
    return o.shards > 0 ? o.shards : 1;
}

cd_status screen_sharded(Call& C, const cd_elements* el, size_t n, double t0, double t1, double dt,
                         double d, cd_mode mode, const cd_options& o, int64_t K, int S,
                         DBuf<Conj>& sorted, size_t& nconj, cd_stats& stats)
{
    cudaStream_t st = C.st;
    if (!el || !el->a || !el->e || !el->inc || !el->raan || !el->argp || !el->nu0)
        return fail(CD_EINVAL, "elements must be non-NULL");
    // the full element set on the device once (validated), a and e on the host for the bands
    DBuf<double> up(st);
    Elements E;
    std::vector<double> ha(n), he(n);
    if (o.inputs_on_device) {
        E = Elements{el->a, el->e, el->inc, el->raan, el->argp, el->nu0};
        CU(cudaMemcpyAsync(ha.data(), el->a, sizeof(double) * n, cudaMemcpyDeviceToHost, st));
        CU(cudaMemcpyAsync(he.data(), el->e, sizeof(double) * n, cudaMemcpyDeviceToHost, st));
        CU(cudaStreamSynchronize(st));
    } else {
        const double* src[6] = {el->a, el->e, el->inc, el->raan, el->argp, el->nu0};
        TRY(validate_elements_host(src, n));
        CU(up.alloc(6 * n));
        for (int c = 0; c < 6; ++c)
            CU(cudaMemcpyAsync(up.p + c * n, src[c], sizeof(double) * n, cudaMemcpyHostToDevice, st));
        E = Elements{up.p, up.p + n, up.p + 2 * n, up.p + 3 * n, up.p + 4 * n, up.p + 5 * n};
        memcpy(ha.data(), el->a, sizeof(double) * n);
        memcpy(he.data(), el->e, sizeof(double) * n);
    }
    // band edges: quantiles of a (strictly increasing; duplicates merge bands)
    std::vector<double> edges{0.0};
    {
        std::vector<double> tmp = ha;
        for (int s = 1; s < S; ++s) {
            const size_t k = n * (size_t)s / (size_t)S;
            std::nth_element(tmp.begin(), tmp.begin() + k, tmp.end());
            if (tmp[k] > edges.back()) edges.push_back(tmp[k]);
        }
        edges.push_back(1.0e9);
    }
    const double gc = d + o.v_margin * dt;
    DBuf<Conj> all(st);
    size_t nall = 0;
    std::vector<uint32_t> idx;
    idx.reserve(n);
    for (size_t s = 0; s + 1 < edges.size(); ++s) {
        const double lo = edges[s], hi = edges[s + 1];
        idx.clear();
        for (size_t i = 0; i < n; ++i)
            if (ha[i] * (1.0 + he[i]) >= lo && ha[i] * (1.0 - he[i]) < hi + gc) idx.push_back((uint32_t)i);
        const int64_t m = (int64_t)idx.size();
        if (m < 2) continue;
        DBuf<uint32_t> didx(st);
        CU(didx.alloc((size_t)m));
        CU(cudaMemcpyAsync(didx.p, idx.data(), sizeof(uint32_t) * (size_t)m, cudaMemcpyHostToDevice, st));
        DBuf<double> sub(st);
        CU(sub.alloc(6 * (size_t)m));
        CU(launch_gather_elements(E, didx.p, m, sub.p, st, C.lc));
        const cd_elements sel{sub.p, sub.p + m, sub.p + 2 * m, sub.p + 3 * m, sub.p + 4 * m, sub.p + 5 * m};
        cd_options os = o;
        os.inputs_on_device = 1;
        os.shell_lo = lo;
        os.shell_hi = hi;
        OrbitSet Ss;
        TRY(prepare_orbits(C, &sel, (size_t)m, os, Ss));
        CU(launch_compose_perm(Ss.perm.p, didx.p, m, st, C.lc));   // internal -> global ids
        Result Rs;
        cd_stats ss;
        memset(&ss, 0, sizeof ss);
        TRY(run(C, Ss, t0, t1, dt, d, mode, os, K, Want::Conj, Rs, ss));
        stats.candidates += ss.candidates;
        stats.raw_pairs += ss.raw_pairs;
        stats.refined += ss.refined;
        stats.retries += ss.retries;
        stats.hybrid_ap_rejected += ss.hybrid_ap_rejected;
        stats.hybrid_coplanar += ss.hybrid_coplanar;
        stats.hybrid_path_rejected += ss.hybrid_path_rejected;
        stats.hybrid_time_rejected += ss.hybrid_time_rejected;
        stats.steps = ss.steps;
        if (Rs.n_conj) {
            if (nall + Rs.n_conj > all.n) {
                DBuf<Conj> grown(st);
                CU(grown.alloc(std::max(2 * all.n, nall + Rs.n_conj)));
                if (nall) CU(cudaMemcpyAsync(grown.p, all.p, sizeof(Conj) * nall, cudaMemcpyDeviceToDevice, st));
                const size_t cap = grown.n;
                all.release();
                all.p = grown.detach();
                all.n = cap;
            }
            CU(launch_conj_to_global(Rs.conj.p, Rs.n_conj, Ss.perm.p, all.p + nall, st, C.lc));
            nall += Rs.n_conj;
        }
        const size_t cap = Rs.conj.n;
        if (!Rs.conj.user.alloc) conj_cache_give(C.dev, st, Rs.conj.detach(), cap);
    }
    stats.object_steps = stats.steps * (uint64_t)n;
    nconj = nall;
    if (nall) {
        C.pt.start(kPhFinalize);
        CU(sorted.alloc(nall));
        CU(finalize_conj(all.p, nall, nullptr, sorted.p, st, C.lc));
        C.pt.stop();
    }
    return CD_OK;
}

cd_options defaults()
{
    cd_options o;
    cd_options_init(&o);
    return o;
}

cd_status screen_impl(const cd_elements* el, size_t n, double t0, double t1, double dt, double d,
                      cd_mode mode, const cd_options* opt, cd_conjunctions* out)
{
    if (!out) return fail(CD_EINVAL, "out must be non-NULL");
    out->data = nullptr;
    out->count = 0;
    out->_owner = nullptr;
    const cd_options o = opt ? *opt : defaults();
    if (mode != CD_GRID && mode != CD_HYBRID && mode != CD_LEGACY)
        return fail(CD_EINVAL, "unknown mode %d", (int)mode);
    if (mode != CD_GRID && o.propagator != CD_PROP_KEPLER)
        return fail(CD_EINVAL, "CD_HYBRID and CD_LEGACY need CD_PROP_KEPLER (the filters assume fixed orbit planes)");
    if (mode == CD_LEGACY && o.shell_hi != 0.0)
        return fail(CD_EINVAL, "CD_LEGACY splits pairs by rank; radial shards apply to the grid");
    if (o.digest_only && (mode == CD_LEGACY || o.shards > 1))
        return fail(CD_EINVAL, "digest_only needs CD_GRID or CD_HYBRID without in-library shards");
    int64_t K = 0;
    TRY(validate_scalars(n, t0, t1, dt, d, o, &K));
    cd_stats stats;
    memset(&stats, 0, sizeof stats);
    DebugClock dbg;
    g_dbg = &dbg;
    struct Reset { ~Reset() { g_dbg = nullptr; } } reset_dbg;
    Call C;
    TRY(C.begin(o));
    DBG("screen: begin");
    Result R;
    DBuf<Conj> sorted(C.st);
    const int n_shards = n > 1 ? shard_count(o, n, mode) : 1;
    if (n_shards > 1) {
        size_t nc = 0;
        TRY(screen_sharded(C, el, n, t0, t1, dt, d, mode, o, K, n_shards, sorted, nc, stats));
        R.n_conj = nc;
    } else {
        OrbitSet S;
        if (n > 0) TRY(prepare_orbits(C, el, n, o, S));
        else if (!el) return fail(CD_EINVAL, "elements must be non-NULL");
        DBG("screen: orbits ready");
        if (mode == CD_LEGACY) TRY(run_legacy(C, S, t0, t1, dt, d, o, K, R, stats));
        else TRY(run(C, S, t0, t1, dt, d, mode, o, K, Want::Conj, R, stats));
        DBG("screen: run done");
        if (R.n_conj) {
            C.pt.start(kPhFinalize);
            CU(sorted.alloc(R.n_conj));
            CU(finalize_conj(R.conj.p, R.n_conj, S.perm.p, sorted.p, C.st, C.lc));
            C.pt.stop();
        }
        // the accumulation buffer goes back to the per-device cache (its last use, the sort,
        // is enqueued on C.st)
        // (with the caller's allocator it is simply released by R's destructor)
        const size_t cap = R.conj.n;
        if (!R.conj.user.alloc) conj_cache_give(C.dev, C.st, R.conj.detach(), cap);
    }
    Owner* own = new Owner{o.outputs_on_device != 0, nullptr, C.own_stream ? nullptr : C.st, 0,
                           g_dev_alloc};
    if (R.n_conj) {
        if (o.outputs_on_device) {
            own->p = sorted.detach();
        } else {
            size_t hb = 0;
            void* h = R.alloc_host(R.n_conj) ? R.take_host(&hb) : nullptr;
            if (!h) {
                delete own;
                return fail(CD_ENOMEM, "host allocation of %zu records failed", R.n_conj);
            }
            own->p = h;
            own->host_bytes = hb;
            const cudaError_t e = copy_to_pageable(h, sorted.p, sizeof(cd_conjunction) * R.n_conj, C.st);
            if (e != cudaSuccess) {
                Result::release_host(h, hb);
                delete own;
                return fail(CD_ECUDA, "copy-out: %s", cudaGetErrorString(e));
            }
        }
    }
    DBG("screen: finalized");
    CU(cudaEventRecord(C.ev1, C.st));
    CU(cudaEventSynchronize(C.ev1));
    DBG("screen: end synced");
    float ms = 0.f;
    cudaEventElapsedTime(&ms, C.ev0, C.ev1);
    stats.ms_total = ms;
    stats.conjunctions = o.digest_only ? stats.digest_conjunctions : R.n_conj;
    stats.kernel_launches = C.lc.n;
    C.pt.harvest();
    C.pt.to_stats(stats);
    if (o.stats) *o.stats = stats;
    out->data = static_cast<cd_conjunction*>(own->p);
    out->count = R.n_conj;
    out->_owner = own;
    return CD_OK;
}

}  // namespace

extern "C" {

cd_status cd_shell_members(const cd_elements* el, size_t n, double shell_lo, double shell_hi,
                           double gc, uint32_t* idx, size_t* count)
{
    try {
        if (!el || !el->a || !el->e || !idx || !count) return fail(CD_EINVAL, "NULL argument");
        *count = 0;
        if (!is_fin(shell_lo) || !is_fin(shell_hi) || !is_fin(gc) || shell_lo < 0.0 ||
            !(shell_hi > shell_lo) || gc < 0.0)
            return fail(CD_EINVAL, "need shell_hi > shell_lo >= 0 and g_c >= 0");
        if (n >= 0xffffffffull) return fail(CD_EINVAL, "n too large");
        size_t c = 0;
        for (size_t i = 0; i < n; ++i) {
            const double a = el->a[i], e = el->e[i];
            if (!(a > 0.0) || !(e >= 0.0 && e < 1.0)) return fail(CD_EINVAL, "element %zu invalid", i);
            // radius range [q, Q] meets [shell_lo, shell_hi + g_c)
            if (a * (1.0 + e) >= shell_lo && a * (1.0 - e) < shell_hi + gc) idx[c++] = (uint32_t)i;
        }
        *count = c;
        return CD_OK;
    } catch (...) {
        return fail(CD_EINTERNAL, "unexpected C++ exception");
    }
}

void cd_options_init(cd_options* o)
{
    if (!o) return;
    memset(o, 0, sizeof *o);
    o->v_margin = 7.8;   // Eq. 1: typical LEO speed
    o->device = -1;
    o->rank = 0;
    o->n_ranks = 1;
    o->cell_factor = 0.0;   // auto (1.0 = the paper's cell edge g_c, 27-cell neighbourhood)
    o->l2_persist = 0;
    o->grid_table = 0;
    o->propagator = CD_PROP_KEPLER;
}

cd_status cd_screen(const cd_elements* el, size_t n, double t0, double t1, double dt, double d,
                    cd_mode mode, cd_conjunctions* out)
{
    return cd_screen_ex(el, n, t0, t1, dt, d, mode, nullptr, out);
}

cd_status cd_screen_ex(const cd_elements* el, size_t n, double t0, double t1, double dt, double d,
                       cd_mode mode, const cd_options* opt, cd_conjunctions* out)
{
    try {
        return screen_impl(el, n, t0, t1, dt, d, mode, opt, out);
    } catch (...) {
        return fail(CD_EINTERNAL, "unexpected C++ exception");
    }
}

cd_status cd_candidates(const cd_elements* el, size_t n, double t0, double t1, double dt, double d,
                        cd_mode mode, const cd_options* opt, cd_candidate** out, size_t* count)
{
    try {
        if (!out || !count) return fail(CD_EINVAL, "out and count must be non-NULL");
        *out = nullptr;
        *count = 0;
        if (mode != CD_GRID && mode != CD_HYBRID) return fail(CD_EINVAL, "unknown mode %d", (int)mode);
        const cd_options o = opt ? *opt : defaults();
        int64_t K = 0;
        TRY(validate_scalars(n, t0, t1, dt, d, o, &K));
        cd_stats stats;
        memset(&stats, 0, sizeof stats);
        Call C;
        TRY(C.begin(o));
        Result R;
        DBuf<Cand> sorted(C.st);
        OrbitSet S;
        if (n > 0) TRY(prepare_orbits(C, el, n, o, S));
        TRY(run(C, S, t0, t1, dt, d, mode, o, K, Want::Cand, R, stats));
        cd_candidate* h = nullptr;
        if (R.n_cand) {
            CU(sorted.alloc(R.n_cand));
            CU(finalize_cand(R.cand.p, R.n_cand, S.perm.p, sorted.p, C.st, C.lc));
            h = (cd_candidate*)malloc(sizeof(cd_candidate) * R.n_cand);
            if (!h) return fail(CD_ENOMEM, "host allocation failed");
            cudaError_t e = cudaMemcpyAsync(h, sorted.p, sizeof(cd_candidate) * R.n_cand,
                                            cudaMemcpyDeviceToHost, C.st);
            if (e == cudaSuccess) e = cudaStreamSynchronize(C.st);
            if (e != cudaSuccess) {
                free(h);
                return fail(CD_ECUDA, "copy-out: %s", cudaGetErrorString(e));
            }
        }
        CU(cudaEventRecord(C.ev1, C.st));
        CU(cudaEventSynchronize(C.ev1));
        float ms = 0.f;
        cudaEventElapsedTime(&ms, C.ev0, C.ev1);
        stats.ms_total = ms;
        stats.kernel_launches = C.lc.n;
        if (o.stats) *o.stats = stats;
        *out = h;
        *count = R.n_cand;
        return CD_OK;
    } catch (...) {
        return fail(CD_EINTERNAL, "unexpected C++ exception");
    }
}

cd_status cd_propagate(const cd_elements* el, size_t n, const double* t, size_t nt, double* xyz,
                       double* vxyz, const cd_options* opt)
{
    try {
        if (!xyz || (!t && nt)) return fail(CD_EINVAL, "t and xyz must be non-NULL");
        if (n == 0 || nt == 0) return CD_OK;
        if (n >= 0xffffffffull) return fail(CD_EINVAL, "n too large");
        for (size_t q = 0; q < nt; ++q)
            if (!is_fin(t[q])) return fail(CD_EINVAL, "non-finite time");
        const cd_options o = opt ? *opt : defaults();
        if (kepler_class_of_points(o.kepler_points) < 0)
            return fail(CD_EINVAL, "kepler_points = %d: need 0 (per e) or 4, 6, 8, 12, 16", o.kepler_points);
        if (o.propagator != CD_PROP_KEPLER && o.propagator != CD_PROP_J2)
            return fail(CD_EINVAL, "unknown propagator %d", o.propagator);
        Call C;
        TRY(C.begin(o));
        OrbitSet S;
        TRY(prepare_orbits(C, el, n, o, S));
        DBuf<double> dt_(C.st), dx(C.st), dv(C.st);
        CU(dt_.alloc(nt));
        CU(dx.alloc(nt * n * 3));
        if (vxyz) CU(dv.alloc(nt * n * 3));
        CU(cudaMemcpyAsync(dt_.p, t, sizeof(double) * nt, cudaMemcpyHostToDevice, C.st));
        CU(launch_propagate_out(S.view(), S.perm.p, dt_.p, (int64_t)nt, dx.p, vxyz ? dv.p : nullptr,
                                C.st, C.lc));
        CU(cudaMemcpyAsync(xyz, dx.p, sizeof(double) * nt * n * 3, cudaMemcpyDeviceToHost, C.st));
        if (vxyz) CU(cudaMemcpyAsync(vxyz, dv.p, sizeof(double) * nt * n * 3, cudaMemcpyDeviceToHost, C.st));
        CU(cudaStreamSynchronize(C.st));
        if (o.stats) {
            cd_stats s;
            memset(&s, 0, sizeof s);
            s.kernel_launches = C.lc.n;
            *o.stats = s;
        }
        return CD_OK;
    } catch (...) {
        return fail(CD_EINTERNAL, "unexpected C++ exception");
    }
}

cd_status cd_conjunctions_sort_device(cd_conjunction* data, size_t n, void* stream)
{
    try {
        if (n == 0) return CD_OK;
        if (!data) return fail(CD_EINVAL, "data must be non-NULL");
        cudaStream_t st = (cudaStream_t)stream;
        // scratch from the library's private pool of the current device (which keeps its memory:
        // the device's default pool would unmap and remap it on every merge)
        int dev = 0;
        CU(cudaGetDevice(&dev));
        struct PoolScope {
            explicit PoolScope(cudaMemPool_t p) { g_pool = p; }
            ~PoolScope() { g_pool = nullptr; }
        } scope(setup_pool(dev));
        LaunchCount lc;
        DBuf<Conj> tmp(st);
        CU(tmp.alloc(n));
        CU(finalize_conj(reinterpret_cast<const Conj*>(data), n, nullptr, tmp.p, st, lc));
        CU(cudaMemcpyAsync(data, tmp.p, sizeof(Conj) * n, cudaMemcpyDeviceToDevice, st));
        return CD_OK;
    } catch (...) {
        return fail(CD_EINTERNAL, "unexpected C++ exception");
    }
}

void cd_conjunctions_free(cd_conjunctions* c)
{
    if (!c) return;
    Owner* own = static_cast<Owner*>(c->_owner);
    if (own) {
        if (own->p) {
            // stream-ordered release (no device-wide synchronisation): after the work the
            // caller queued on the call's stream (the legacy default stream if the library
            // created its own)
            if (own->device && own->alloc.free) own->alloc.free(own->p, own->alloc.ctx);
            else if (own->device) cudaFreeAsync(own->p, own->st);
            else munmap(own->p, own->host_bytes);
        }
        delete own;
    }
    c->data = nullptr;
    c->count = 0;
    c->_owner = nullptr;
}

cd_status cd_plan(size_t n, double t0, double t1, double dt, double d, cd_mode mode,
                  size_t mem_bytes, cd_plan_info* out)
{
    try {
        if (!out) return fail(CD_EINVAL, "out must be non-NULL");
        memset(out, 0, sizeof *out);
        if (mode != CD_GRID && mode != CD_HYBRID) return fail(CD_EINVAL, "unknown mode %d", (int)mode);
        cd_options o;
        cd_options_init(&o);
        int64_t K = 0;
        TRY(validate_scalars(n, t0, t1, dt, d, o, &K));
        if (mem_bytes == 0) {
            int ndev = 0;
            if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev == 0)
                return fail(CD_ENODEV, "mem_bytes = 0 needs a CUDA device (free memory query)");
            size_t fr = 0, tot = 0;
            CU(cudaMemGetInfo(&fr, &tot));
            mem_bytes = fr;
        }
        const double nn = (double)n;
        const double span = t1 - t0 > 0.0 ? t1 - t0 : dt;
        out->samples = (double)K;
        out->est_candidates = extra_p_candidates(nn, dt, span, d, mode);
        out->est_candidates_per_step = extra_p_candidates(nn, dt, dt, d, mode);
        out->capacity = std::max(out->est_candidates, 1e4) * 2.0 * 2.0;
        out->capacity_bytes = out->capacity * 16.0;
        // this library's structures: a_s elements, a_k orbit records (column- and
        // object-major) + class + permutation, a_ch the round's candidate queue (12 B) and work items (24 B)
        const double qcap = (double)initial_qcap((int64_t)n, std::max(1.0, out->est_candidates_per_step));
        const double wcap = std::min(qcap, std::max(4194304.0, 4.0 * nn));
        out->fixed_bytes = 48.0 * nn + (8.0 * kDOm + 8.0 * kAoS + 1.0 + 4.0) * nn + 12.0 * qcap + 24.0 * wcap;
        // a_gh + a_l of one step's grid, in the structure the auto cell edge selects for the
        // a-priori density: chained heads (4 B x next_pow2(8n)) in ball mode, the open map
        // (16 B x next_pow2(2n) slots + next_pow2(32n)-bit occupancy) in half-shell mode, plus the
        // 32-byte entries {x, y, z, next}
        const double m = choose_cell_factor(std::max(1.0, out->est_candidates_per_step) / std::max(1.0, nn));
        const double n_u = std::max(1.0, nn);
        const double chained = 4.0 * (double)next_pow2((uint64_t)(CD_CHAIN_FACTOR * n_u));
        const double open = 16.0 * (double)next_pow2((uint64_t)(2.0 * n_u)) +
                            (double)next_pow2((uint64_t)(32.0 * n_u)) / 8.0;
        out->bytes_per_grid = (m < 2.0 ? open : chained) + 32.0 * nn;
        out->grids_in_memory = std::max(0.0, ((double)mem_bytes - out->fixed_bytes) / out->bytes_per_grid);
        out->rounds = out->grids_in_memory > 0.0 ? out->samples / out->grids_in_memory : INFINITY;
        out->cell_factor = m;
        return CD_OK;
    } catch (...) {
        return fail(CD_EINTERNAL, "unexpected C++ exception");
    }
}

void cd_candidates_free(cd_candidate* c) { free(c); }

cd_status cd_release_caches(int device)
{
    try {
        int ndev = 0;
        if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev == 0) {
            cudaGetLastError();
            return CD_OK;   // nothing was ever cached
        }
        int prev = 0;
        CU(cudaGetDevice(&prev));
        const int lo = device >= 0 ? device : 0, hi = device >= 0 ? device + 1 : std::min(ndev, 64);
        if (device >= ndev) return fail(CD_EINVAL, "device %d out of range (%d devices)", device, ndev);
        for (int dv = lo; dv < hi; ++dv) {
            CU(cudaSetDevice(dv));
            {
                ConjCache& c = g_conj_cache[dv];
                std::lock_guard<std::mutex> lk(c.mu);
                if (c.p) {
                    if (c.ready) cudaEventSynchronize(c.ready);
                    cudaFree(c.p);
                }
                c.p = nullptr;
                c.cap = 0;
            }
            std::lock_guard<std::mutex> lk(g_pool_mu);
            if (g_pools[dv]) {
                CU(cudaDeviceSynchronize());   // blocks freed stream-ordered are back in the pool
                CU(cudaMemPoolTrimTo(g_pools[dv], 0));
            }
        }
        CU(cudaSetDevice(prev));
        return CD_OK;
    } catch (...) {
        return fail(CD_EINTERNAL, "unexpected C++ exception");
    }
}

const char* cd_status_str(cd_status s)
{
    switch (s) {
    case CD_OK: return "CD_OK";
    case CD_EINVAL: return "CD_EINVAL";
    case CD_ENOMEM: return "CD_ENOMEM";
    case CD_ECUDA: return "CD_ECUDA";
    case CD_ENCCL: return "CD_ENCCL";
    case CD_ERANGE: return "CD_ERANGE";
    case CD_EINTERNAL: return "CD_EINTERNAL";
    case CD_ENODEV: return "CD_ENODEV";
    }
    return "CD_UNKNOWN";
}

const char* cd_last_error(void) { return g_err.c_str(); }

int cd_abi_version(void) { return CD_ABI_VERSION; }

uint64_t cd_kernel_launches(void) { return cdh::g_launches.load(); }

}  // extern "C"
