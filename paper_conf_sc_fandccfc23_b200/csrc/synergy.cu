// synergy.cu — C-ABI implementation (include/synergy.h): validation, model packing, launch
// configuration, library-owned scratch and the host-buffer end-to-end path.  All compute runs in
// the kernels: kernels_tm.cuh (default tree-major path), kernels_gen.cuh (general exact path),
// kernels_svr.cuh (SVR member), kernels.cuh (finish, selection, Pareto, choice error, plan).
#include <cuda_runtime.h>

#include <algorithm>
#include <atomic>
#include <cmath>
#include <cstdarg>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <list>
#include <mutex>
#include <new>
#include <string>
#include <vector>

#include "internal.h"
#include "kernels.cuh"
#include "kernels_gen.cuh"
#include "kernels_svr.cuh"
#include "kernels_svr_tc.cuh"
#include "kernels_tm.cuh"
#include "synergy.h"

using namespace syn;

namespace {
constexpr int kMaxDevices = 64;
}

struct CutCopy {                 // clock-cut copy of a model's blocks for one clock table
    long long uid;               // syn_clocks uid
    uint4* p;
    cudaStream_t built_on;       // stream the k_cut_blocks build was enqueued on
    cudaEvent_t ready;           // recorded after the build; null once known complete
};

struct syn_model {
    int device;
    int n_inputs;
    int n_trees;
    int max_depth;
    long long n_nodes;
    long long bytes;
    void* alloc;
    DevModel dm;
    long long n_blocks;                                   // 2-level blocks (2 x uint4 each)
    std::vector<CutCopy> cuts;                            // per clock table
};

struct syn_clocks {
    int device;
    int n_f;
    float* d_freqs;
    long long uid;            // unique per created table (keys the models' clock-cut copies)
};

struct syn_workspace {
    int device;
    float* d_features;
    size_t cap_features;      // bytes
    int* d_choice;
    size_t cap_choice;        // bytes
};

namespace {

thread_local std::string g_err;
struct LaunchInfo {
    int kernels;
    long long evals;
    long long grid;
    int block;
    int variant;
};
thread_local LaunchInfo g_last = {0, 0, 0, 0, 0};

// Variant codes reported by synergy_last_launch (tests / bench read which path ran).
constexpr int kVarTm = 4000;      // k_tm_walk + k_tm_finish
constexpr int kVarGen = 5000;     // k_gen_forest + k_gen_finish

// Optional per-kernel device timing (synergy_timing_enable): CUDA events recorded on the launch
// stream around every library kernel launch; read back (summed per kernel) by synergy_timing_read.
struct TimedLaunch {
    const char* name;
    cudaEvent_t a, b;
};
std::mutex g_tmu;
bool g_timing = false;
std::vector<TimedLaunch> g_tl;
std::vector<cudaEvent_t> g_evpool;

cudaEvent_t take_event() {
    if (!g_evpool.empty()) {
        cudaEvent_t e = g_evpool.back();
        g_evpool.pop_back();
        return e;
    }
    cudaEvent_t e = nullptr;
    if (cudaEventCreate(&e) != cudaSuccess) {
        cudaGetLastError();
        return nullptr;
    }
    return e;
}

struct KernelTimer {   // records around one launch when timing is enabled
    const char* name;
    cudaStream_t st;
    cudaEvent_t a = nullptr;
    KernelTimer(const char* n, cudaStream_t s) : name(n), st(s) {
        std::lock_guard<std::mutex> lock(g_tmu);
        if (!g_timing) return;
        a = take_event();
        if (a) cudaEventRecord(a, st);
    }
    ~KernelTimer() {
        if (!a) return;
        std::lock_guard<std::mutex> lock(g_tmu);
        cudaEvent_t b = take_event();
        if (!b) {
            g_evpool.push_back(a);
            return;
        }
        cudaEventRecord(b, st);
        g_tl.push_back({name, a, b});
    }
};

syn_status fail(syn_status st, const char* fmt, ...) {
    char buf[512];
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(buf, sizeof buf, fmt, ap);
    va_end(ap);
    g_err = buf;
    return st;
}

syn_status cuda_fail(cudaError_t e, const char* what) {
    return fail(e == cudaErrorMemoryAllocation ? SYN_ERR_OOM : SYN_ERR_CUDA, "%s: %s", what,
                cudaGetErrorString(e));
}

syn_status ok() {
    g_err.clear();
    return SYN_OK;
}

struct DeviceGuard {   // switch to `dev` for the scope, restore afterwards
    int prev = -1;
    bool okay = false;
    explicit DeviceGuard(int dev) {
        if (cudaGetDevice(&prev) == cudaSuccess && cudaSetDevice(dev) == cudaSuccess) okay = true;
    }
    ~DeviceGuard() {
        if (prev >= 0) cudaSetDevice(prev);
    }
};

bool current_device_is(int dev) {
    int cur = -1;
    return cudaGetDevice(&cur) == cudaSuccess && cur == dev;
}

// ------------------------------------------------------------------------ tuning knobs
// Read once from the environment (SYNERGY_<NAME>) at first use; synergy_config_set changes them
// at run time (tests use it to force launch-configuration variants).  0 / -1 = automatic.
struct Knobs {
    std::atomic<long long> algo{0};       // 0 auto, 1 force k_gen (general exact path)
    std::atomic<long long> tm_kb{0};      // k_tm_walk kernels per feature block (32..1024)
    std::atomic<long long> tm_ctas{0};    // k_tm_walk CTAs (default one wave: 1024 / threads-per-CTA per SM)
    std::atomic<long long> tm_nsub{0};    // clock sub-ranges per (kernel, tree) task
    std::atomic<long long> tm_split{-1};  // per-tree sub-range split: -1 auto (small batches), 0 off, 1 on
    std::atomic<long long> tm_nt{0};      // k_tm_walk threads per CTA: 0 automatic, 512 or 1024
    std::atomic<long long> split_piece{4};// model create: sub-range target cost, in quarters of the mean
    std::atomic<long long> tm_dyn{-1};    // dynamic task fetch: -1 auto, 0 off, 1 on
    std::atomic<long long> tm_pdl{1};     // programmatic dependent launch of k_tm_finish
    std::atomic<long long> tm_slab{0};    // kernels per slab (0: D of one slab <= 48 MB)
    std::atomic<long long> tm_lpt{-1};    // expected-cost tree order for ~1 task per lane: -1 auto, 0 off, 1 on
    std::atomic<long long> tm_pipe{2};    // slab pipeline: 1 finish on a side stream, 2 + two walk streams
    std::atomic<long long> tm_kt{0};      // k_tm_finish kernels per CTA
    std::atomic<long long> gen_kt{0};     // k_gen_finish kernels per CTA
    std::atomic<long long> svr_splits{0}; // k_svr / k_svr_tc SV-range splits (0: fill the SMs)
    std::atomic<long long> svr_tc{1};     // SVR contraction on tcgen05 (int8 digit products); 0: fp64 k_svr
    std::atomic<long long> tm_small{-1};  // single-launch k_tm_small: -1 auto (small batches), 0 off, 1 on
};
Knobs g_knobs;
struct KnobName {
    const char* name;
    std::atomic<long long>* v;
};
const KnobName kKnobs[] = {{"algo", &g_knobs.algo},       {"tm_kb", &g_knobs.tm_kb},   {"tm_ctas", &g_knobs.tm_ctas},
                           {"tm_nsub", &g_knobs.tm_nsub}, {"tm_split", &g_knobs.tm_split}, {"tm_nt", &g_knobs.tm_nt}, {"split_piece", &g_knobs.split_piece}, {"tm_dyn", &g_knobs.tm_dyn}, {"tm_pdl", &g_knobs.tm_pdl},
                           {"tm_slab", &g_knobs.tm_slab}, {"tm_pipe", &g_knobs.tm_pipe}, {"tm_lpt", &g_knobs.tm_lpt}, {"tm_kt", &g_knobs.tm_kt},
                           {"gen_kt", &g_knobs.gen_kt}, {"svr_splits", &g_knobs.svr_splits},
                           {"svr_tc", &g_knobs.svr_tc}, {"tm_small", &g_knobs.tm_small}};
std::once_flag g_knobs_once;

const Knobs& knobs() {
    std::call_once(g_knobs_once, [] {
        for (const KnobName& k : kKnobs) {
            char env[64] = "SYNERGY_";
            for (int i = 0; k.name[i] && i < 40; ++i) env[8 + i] = (char)toupper(k.name[i]), env[9 + i] = 0;
            const char* v = getenv(env);
            if (v && *v) k.v->store(atoll(v));
        }
    });
    return g_knobs;
}

// -------------------------------------------------------------------- per-device state
struct DevState {
    std::once_flag once;
    int sms = 148;
    int optin = 227 * 1024;               // max shared memory per CTA (opt-in)
    int walk_dyn_max = 0;                 // dynamic shared memory k_tm_walk / k_tm_finish may take
    int finish_dyn_max = 0;
    int small_dyn_max = 0;                // k_tm_small
    cudaError_t init_err = cudaSuccess;
    cudaMemPool_t pool = nullptr;         // library-owned stream-ordered pool (release threshold max)
    std::mutex occ_mu;
    std::vector<std::pair<size_t, int>> finish_occ;   // k_tm_finish: (smem bytes, CTAs per SM)
};
DevState g_dev[kMaxDevices];

// Opt a kernel in to the largest dynamic shared memory the device allows next to its static
// shared memory.
template <typename K>
cudaError_t allow_smem(K kernel, int optin) {
    cudaFuncAttributes fa;
    cudaError_t e = cudaFuncGetAttributes(&fa, kernel);
    if (e != cudaSuccess) return e;
    return cudaFuncSetAttribute(kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, optin - (int)fa.sharedSizeBytes);
}

// Once per device (the attribute is per device): query limits, opt every kernel with dynamic
// shared memory in to the device maximum, create the library pool.
DevState* dev_state(int dev) {
    if (dev < 0 || dev >= kMaxDevices) return nullptr;
    DevState& d = g_dev[dev];
    std::call_once(d.once, [&d, dev] {
        DeviceGuard g(dev);
        int v = 0;
        if (cudaDeviceGetAttribute(&v, cudaDevAttrMultiProcessorCount, dev) == cudaSuccess && v > 0) d.sms = v;
        if (cudaDeviceGetAttribute(&v, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev) == cudaSuccess && v > 0) d.optin = v;
        cudaError_t e = cudaSuccess;
        auto chk = [&e](cudaError_t x) { if (e == cudaSuccess) e = x; };
        chk(allow_smem(k_tm_walk<512, true, false>, d.optin));
        chk(allow_smem(k_tm_walk<512, false, false>, d.optin));
        chk(allow_smem(k_tm_walk<512, true, true>, d.optin));
        chk(allow_smem(k_tm_walk<512, false, true>, d.optin));
        chk(allow_smem(k_tm_walk<1024, true, false>, d.optin));
        chk(allow_smem(k_tm_walk<1024, false, false>, d.optin));
        chk(allow_smem(k_tm_walk<1024, true, true>, d.optin));
        chk(allow_smem(k_tm_walk<1024, false, true>, d.optin));
        chk(allow_smem(k_tm_walk<512, true, false, true>, d.optin));
        chk(allow_smem(k_tm_walk<512, false, false, true>, d.optin));
        chk(allow_smem(k_tm_finish, d.optin));
        chk(allow_smem(k_tm_small<true, false>, d.optin));
        chk(allow_smem(k_tm_small<false, false>, d.optin));
        chk(allow_smem(k_tm_small<true, true>, d.optin));
        chk(allow_smem(k_tm_small<false, true>, d.optin));
        chk(allow_smem(k_svr<1>, d.optin));
        chk(allow_smem(k_svr<2>, d.optin));
        chk(allow_smem(k_svr<3>, d.optin));
        chk(allow_smem(k_svr<4>, d.optin));
        chk(allow_smem(k_svr<5>, d.optin));
        chk(allow_smem(k_svr<6>, d.optin));
        chk(allow_smem(k_svr<7>, d.optin));
        chk(allow_smem(k_svr<8>, d.optin));
        chk(allow_smem(k_svr_u, d.optin));
        chk(allow_smem(k_svr_tc, d.optin));
        chk(allow_smem(k_svr_udig, d.optin));
        cudaFuncAttributes fa;
        if (e == cudaSuccess) chk(cudaFuncGetAttributes(&fa, k_tm_walk<1024, false, true>));
        d.walk_dyn_max = d.optin - (int)fa.sharedSizeBytes;
        if (e == cudaSuccess) chk(cudaFuncGetAttributes(&fa, k_tm_finish));
        d.finish_dyn_max = d.optin - (int)fa.sharedSizeBytes;
        if (e == cudaSuccess) chk(cudaFuncGetAttributes(&fa, k_tm_small<false, true>));
        d.small_dyn_max = d.optin - (int)fa.sharedSizeBytes;
        cudaMemPoolProps props;
        memset(&props, 0, sizeof props);
        props.allocType = cudaMemAllocationTypePinned;
        props.handleTypes = cudaMemHandleTypeNone;
        props.location.type = cudaMemLocationTypeDevice;
        props.location.id = dev;
        if (e == cudaSuccess) {
            chk(cudaMemPoolCreate(&d.pool, &props));
            if (e == cudaSuccess) {
                unsigned long long thr = ~0ULL;
                chk(cudaMemPoolSetAttribute(d.pool, cudaMemPoolAttrReleaseThreshold, &thr));
            }
        }
        if (e != cudaSuccess) cudaGetLastError();
        d.init_err = e;
    });
    return &d;
}

syn_status need_dev(int dev, DevState** out) {
    DevState* d = dev_state(dev);
    if (!d) return fail(SYN_ERR_INVALID_ARG, "device %d out of range", dev);
    if (d->init_err != cudaSuccess) return cuda_fail(d->init_err, "device setup");
    *out = d;
    return SYN_OK;
}

bool capturing(cudaStream_t st) {
    cudaStreamCaptureStatus cs = cudaStreamCaptureStatusNone;
    if (cudaStreamIsCapturing(st, &cs) != cudaSuccess) {
        cudaGetLastError();
        return false;
    }
    return cs != cudaStreamCaptureStatusNone;
}

syn_status pool_alloc(DevState* d, size_t bytes, cudaStream_t st, void** out, const char* what) {
    cudaError_t e = cudaMallocFromPoolAsync(out, std::max<size_t>(bytes, 256), d->pool, st);
    if (e != cudaSuccess) {
        cudaGetLastError();
        *out = nullptr;
        return e == cudaErrorMemoryAllocation ? fail(SYN_ERR_OOM, "%s: %zu bytes", what, bytes) : cuda_fail(e, what);
    }
    return SYN_OK;
}

syn_status check_targets(const syn_target* t, int32_t n_t) {
    if (n_t < 1 || n_t > SYNERGY_MAX_TARGETS) return fail(SYN_ERR_INVALID_ARG, "n_targets=%d outside [1, %d]", n_t, SYNERGY_MAX_TARGETS);
    if (!t) return fail(SYN_ERR_INVALID_ARG, "h_targets is NULL");
    for (int i = 0; i < n_t; ++i) {
        if (t[i].kind < SYN_MAX_PERF || t[i].kind > SYN_PL_ABS) return fail(SYN_ERR_INVALID_ARG, "target %d: unknown kind %d", i, t[i].kind);
        if (t[i].kind >= SYN_ES && !(t[i].x >= 0.0f && t[i].x <= 100.0f))
            return fail(SYN_ERR_INVALID_ARG, "target %d: x=%g outside [0, 100]", i, (double)t[i].x);
    }
    return SYN_OK;
}

// ------------------------------------------------------------------ tree-major path (kernels_tm.cuh)
// D difference arrays live in a library-owned buffer per (device, stream).  k_tm_finish zeroes
// every entry it reads, so a buffer is all-zero between calls on its stream; a call that fails
// after enqueuing k_tm_walk marks it dirty and the next call clears it with a memset.  Growing a
// buffer is stream-ordered (pool free + alloc + memset on the caller's stream, no host sync).
struct TmBuf {
    int dev;
    cudaStream_t st;
    int kind;                        // 0 / 1: D and its second slab buffer
    long long* p;
    size_t bytes;
    bool dirty;
};
std::mutex g_tm_mu;
std::list<TmBuf> g_tm_bufs;          // list: entries never move

syn_status tm_buffer(DevState* ds, int dev, cudaStream_t st, size_t bytes, TmBuf** out, int kind) {
    std::lock_guard<std::mutex> lock(g_tm_mu);
    TmBuf* b = nullptr;
    for (TmBuf& x : g_tm_bufs)
        if (x.dev == dev && x.st == st && x.kind == kind) b = &x;
    if (!b) {
        g_tm_bufs.push_back({dev, st, kind, nullptr, 0, false});
        b = &g_tm_bufs.back();
    }
    cudaError_t e = cudaSuccess;
    if (b->bytes < bytes) {
        if (capturing(st))
            return fail(SYN_ERR_UNSUPPORTED, "the sweep's scratch must grow inside a stream capture: call "
                                             "synergy_prepare (or run one call of this shape) before capturing");
        if (b->p) cudaFreeAsync(b->p, st);             // after the queued work on this stream
        b->p = nullptr;
        b->bytes = 0;
        void* p = nullptr;
        syn_status s = pool_alloc(ds, bytes, st, &p, "tree-major difference arrays");
        if (s != SYN_OK) return s;
        b->p = static_cast<long long*>(p);
        b->bytes = bytes;
        b->dirty = true;
    }
    if (b->dirty) {
        if ((e = cudaMemsetAsync(b->p, 0, b->bytes, st)) != cudaSuccess) return cuda_fail(e, "cudaMemsetAsync(D)");
        b->dirty = false;
    }
    *out = b;
    return ok();
}

// Slab pipeline (several kernel slabs per call): the finish of slab i runs on a library-owned
// side stream while the walk of slab i + 1 runs (on the caller's stream, or with tm_pipe 2 on the
// caller's stream for even slabs and a second library stream for odd ones), D double-buffered.
// Two library streams (finishes; odd slabs' walks with tm_pipe 2) and six events per (device,
// caller stream).
struct TmAux {
    int dev;
    cudaStream_t st;
    cudaStream_t st2;
    cudaStream_t stw;                     // second walk stream (tm_pipe 2: odd slabs' walks)
    cudaEvent_t walked[2], finished[2];
    cudaEvent_t fork, joinw;              // st -> stw before the first slab; stw -> st on failure
};
std::list<TmAux> g_tm_aux;

syn_status tm_aux(int dev, cudaStream_t st, TmAux** out) {
    std::lock_guard<std::mutex> lock(g_tm_mu);
    for (TmAux& x : g_tm_aux)
        if (x.dev == dev && x.st == st) {
            *out = &x;
            return ok();
        }
    if (capturing(st))
        return fail(SYN_ERR_UNSUPPORTED, "slab-pipeline stream must be created before a stream capture: call "
                                         "synergy_prepare (or run one call of this shape) first");
    TmAux x;
    x.dev = dev;
    x.st = st;
    cudaError_t e = cudaStreamCreateWithFlags(&x.st2, cudaStreamNonBlocking);
    if (e == cudaSuccess) e = cudaStreamCreateWithFlags(&x.stw, cudaStreamNonBlocking);
    if (e == cudaSuccess) e = cudaEventCreateWithFlags(&x.fork, cudaEventDisableTiming);
    if (e == cudaSuccess) e = cudaEventCreateWithFlags(&x.joinw, cudaEventDisableTiming);
    for (int i = 0; i < 2 && e == cudaSuccess; ++i) {
        if ((e = cudaEventCreateWithFlags(&x.walked[i], cudaEventDisableTiming)) == cudaSuccess)
            e = cudaEventCreateWithFlags(&x.finished[i], cudaEventDisableTiming);
    }
    if (e != cudaSuccess) return cuda_fail(e, "slab pipeline stream/events");
    g_tm_aux.push_back(x);
    *out = &g_tm_aux.back();
    return ok();
}

// Clock-cut copy of a model's blocks for one clock table (kernels_tm.cuh, k_cut_blocks), built on
// first use on the caller's stream and cached in the model.  Later calls on another stream wait
// for the build's event (until it is known complete); nothing synchronises the host.
std::mutex g_cut_mu;
syn_status cut_blocks(DevState* ds, syn_model* m, const syn_clocks* c, cudaStream_t st, const uint4** out) {
    std::lock_guard<std::mutex> lock(g_cut_mu);
    for (CutCopy& cb : m->cuts) {
        if (cb.uid != c->uid) continue;
        if (cb.ready && !capturing(st)) {
            const cudaError_t q = cudaEventQuery(cb.ready);
            if (q == cudaSuccess) {
                cudaEventDestroy(cb.ready);
                cb.ready = nullptr;
            } else if (q != cudaErrorNotReady) {
                cudaGetLastError();
            }
        }
        if (cb.ready && cb.built_on != st) {
            const cudaError_t e = cudaStreamWaitEvent(st, cb.ready, 0);
            if (e != cudaSuccess) return cuda_fail(e, "wait for the clock-cut copy");
        }
        *out = cb.p;
        return ok();
    }
    if (capturing(st))
        return fail(SYN_ERR_UNSUPPORTED, "the clock-cut copy of a (model, clock table) pair must be built before a "
                                         "stream capture: call synergy_prepare (or run one call) first");
    void* p = nullptr;
    const long long nb = std::max<long long>(m->n_blocks, 1);
    syn_status s = pool_alloc(ds, (size_t)nb * 2 * sizeof(uint4), st, &p, "clock-cut blocks");
    if (s != SYN_OK) return s;
    cudaError_t e = cudaSuccess;
    if (m->n_blocks > 0) {
        KernelTimer kt("k_cut_blocks", st);
        k_cut_blocks<<<(unsigned)((m->n_blocks + 255) / 256), 256, 0, st>>>(
            m->dm.blocks, m->n_blocks, m->n_inputs - 1, c->d_freqs, c->n_f, m->dm.fx32 ? m->dm.fx_scale : 0.0,
            static_cast<uint4*>(p));
        e = cudaGetLastError();
    }
    cudaEvent_t ev = nullptr;
    if (e == cudaSuccess && (e = cudaEventCreateWithFlags(&ev, cudaEventDisableTiming)) == cudaSuccess)
        e = cudaEventRecord(ev, st);
    if (e != cudaSuccess) {
        cudaFreeAsync(p, st);
        if (ev) cudaEventDestroy(ev);
        return cuda_fail(e, "k_cut_blocks");
    }
    m->cuts.push_back({c->uid, static_cast<uint4*>(p), st, ev});
    *out = static_cast<const uint4*>(p);
    return ok();
}

constexpr size_t kTmSlabBytes = 48u << 20;   // D bytes per slab (stays L2-resident with the model)

const DevModel& dm_of(const SweepArgs& a, int m) { return m == 0 ? a.ms : m == 1 ? a.me : a.mx[m - 2]; }
bool present(const SweepArgs& a, int m) { return m < 2 || a.has_x[m - 2]; }

// k_tm_walk kernels per feature block: a power of two in [32, 1024] whose [F + 2][kb] fp32 feature
// table fits the budget (64 KB for large batches, 32 KB otherwise), and no more than the batch
// needs.  Large batches take 1024: a 1024-thread CTA's lanes then cover one tree at a time (the
// task pools walk unit-major), so the SM's L1 holds one tree (measured: c3 walk 2.54 -> 2.29 ms
// per slab, c4 0.94 -> 0.89 ms, from 256).
int tm_kb(int F, long long n_k, long long knob, bool large) {
    const size_t xs = (size_t)(F + 2) * 4;
    const int kmax = large ? 1024 : n_k >= 2048 ? 512 : 256;   // c5 walk 182 -> 173 us with 512; c2 (1000
                                                                // kernels, a partial block) 72 -> 87 us
    const size_t budget = large ? 65536 : 32768;
    int kb = kmax;
    while (kb > 32 && (xs * kb > budget || kb / 2 >= n_k)) kb /= 2;
    if (knob > 0) {
        while (kb > 32 && kb > knob) kb /= 2;
        while (kb < 1024 && kb * 2 <= knob && xs * kb * 2 <= 65536) kb *= 2;
    }
    return kb;
}
// k_tm_walk threads per CTA: 1024 (one CTA per SM: one tree window and one feature table per SM
// instead of two; measured c3 walk 2.62 -> 2.51 ms per slab) for large batches, 512 (two CTAs per
// SM) when a lane has only a few tasks (c2 72 -> 92 us and c5 181 -> 198 us with 1024)
int tm_nt(long long tasks, int sms) {
    const long long k = knobs().tm_nt.load();
    if (k == 512 || k == 1024) return (int)k;
    return tasks >= 8LL * 1024 * sms ? 1024 : 512;
}
size_t tm_walk_smem(int F, int kb, int tt, int units, int nt = 1024) {
    return (size_t)tt * sizeof(TmTree) + (size_t)kTmS * nt * 8 + (size_t)kb * (F + 2) * 4 + (size_t)units * 8 +
           (size_t)tt + 16;
}
size_t tm_finish_smem(int nm, int k, int n_f, int xs, int nslot) {
    return (size_t)nm * k * n_f * 12 + (size_t)n_f * 4 + (size_t)k * xs * 4 + 32 + (size_t)k * nslot * n_f * 8;
}

// Tree-major path: needs every forest within the exact int64 leaf range (fx_ok), at least one
// tree, and k_tm_walk / k_tm_finish within the device's shared memory.  Else the general path.
bool tm_eligible(const SweepArgs& a, int nm, const DevState* ds) {
    int tt = 0, nslot = 0;
    for (int m = 0; m < nm; ++m) {
        if (!present(a, m)) continue;
        const DevModel& d = dm_of(a, m);
        if (d.forest_weight == 0.0 || d.n_trees == 0) continue;
        if (!d.fx_ok) return false;
        tt += d.n_trees;
        ++nslot;
    }
    if (tt == 0) return false;
    if (tm_walk_smem(a.F, 32, tt, 0, 512) > (size_t)ds->walk_dyn_max) return false;   // the smallest launch
    return tm_finish_smem(nm, 1, a.n_f, (a.F + 2) | 1, nslot) <= (size_t)ds->finish_dyn_max;
}

int finish_ctas_per_sm(DevState* ds, int fnt, size_t smem) {
    std::lock_guard<std::mutex> lock(ds->occ_mu);
    for (auto& e : ds->finish_occ)
        if (e.first == smem) return e.second;
    int nb = 0;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, k_tm_finish, fnt, smem) != cudaSuccess) {
        cudaGetLastError();
        nb = 0;
    }
    ds->finish_occ.push_back({smem, nb});
    return nb;
}

syn_status run_tm(SweepArgs a, int nm, syn_model* const* models, const syn_clocks* clocks, cudaStream_t st,
                  DevState* ds, bool prepare_only, int* launches) {
    const Knobs& K = knobs();
    const int device = clocks->device;
    DevModel* dms[4] = {&a.ms, &a.me, &a.mx[0], &a.mx[1]};
    for (int m = 0; m < nm; ++m) {
        if (!models[m] || dms[m]->forest_weight == 0.0 || dms[m]->n_trees == 0) continue;
        const uint4* cb = nullptr;
        syn_status cs = cut_blocks(ds, models[m], clocks, st, &cb);
        if (cs != SYN_OK) return cs;
        dms[m]->blocks = cb;
    }
    TmArgs t;
    memset(&t, 0, sizeof t);
    const int n_f = a.n_f, F = a.F;
    const long long n_k = a.n_k;
    int tt = 0;
    t.nslot = 0;
    for (int m = 0; m < 4; ++m) {
        t.slot_of[m] = -1;
        if (m >= nm || !present(a, m)) continue;
        const DevModel& d = dm_of(a, m);
        if (d.forest_weight == 0.0 || d.n_trees == 0) continue;
        t.slot_of[m] = t.nslot++;
        tt += d.n_trees;
    }
    t.nm = nm;
    bool fxall = true;                            // every forest has int32 fixed-point leaves
    for (int m = 0; m < nm; ++m)
        if (t.slot_of[m] >= 0 && !dms[m]->fx32) fxall = false;
    a.xs = (F + 2) | 1;
    // small batches (at most one kernel per SM, at most 4096 (tree, clock) walks per kernel): one
    // launch, k_tm_small, one CTA per kernel with direct walks and the finish; the clock-cut
    // blocks are staged in shared memory when they fit in 96 KB (c1: 23 -> ? us)
    {
        const long long ks = K.tm_small.load();
        const size_t ssmem = tm_finish_smem(nm, 1, n_f, a.xs, t.nslot) + (size_t)(F + 2) * 4 + 16;
        size_t sblk = 0;
        for (int m = 0; m < nm; ++m)
            if (t.slot_of[m] >= 0) sblk += (size_t)dms[m]->nblk * 32;
        const bool stage = sblk <= 96 * 1024 && ssmem + sblk <= (size_t)ds->small_dyn_max;
        if (ks != 0 && n_k <= INT_MAX && ssmem <= (size_t)ds->small_dyn_max &&
            (ks > 0 || (n_k <= ds->sms && (long long)tt * n_f <= 4096))) {
            *launches = 0;
            if (prepare_only) return ok();
            a.tile_k = 1;
            t.s = a;
            t.slab0 = 0;
            t.nks = (int)n_k;
            const size_t sm = ssmem + (stage ? sblk : 0);
            cudaError_t e;
            {
                KernelTimer ktm("k_tm_small", st);
                const unsigned g = (unsigned)n_k;
                switch ((fxall ? 1 : 0) + (stage ? 2 : 0)) {
                    case 0: k_tm_small<false, false><<<g, 512, sm, st>>>(t); break;
                    case 1: k_tm_small<true, false><<<g, 512, sm, st>>>(t); break;
                    case 2: k_tm_small<false, true><<<g, 512, sm, st>>>(t); break;
                    default: k_tm_small<true, true><<<g, 512, sm, st>>>(t); break;
                }
                e = cudaGetLastError();
            }
            if (e != cudaSuccess) return cuda_fail(e, "k_tm_small launch");
            *launches = 1;
            return ok();
        }
    }
    // large batches (>= 8 tasks per lane): 1024-thread CTAs and 1024-kernel feature blocks
    int NTW = tm_nt(std::min<long long>(n_k, 1LL << 40) * tt, ds->sms);
    if (tm_walk_smem(F, 32, tt, 0, NTW) > (size_t)ds->walk_dyn_max) NTW = 512;
    int kb = tm_kb(F, n_k, K.tm_kb.load(), NTW == 1024);
    while (kb > 32 && tm_walk_smem(F, kb, tt, 0, NTW) > (size_t)ds->walk_dyn_max) kb /= 2;
    t.kb = kb;
    t.kb_log2 = 0;
    while ((1 << t.kb_log2) < kb) ++t.kb_log2;
    const size_t row = (size_t)t.nslot * n_f * sizeof(long long);
    // kernels per slab: a multiple of the feature block, D of one slab <= kTmSlabBytes (L2-resident)
    long long nks = std::max<long long>(kb, (long long)(kTmSlabBytes / row) / kb * kb);
    if (K.tm_slab.load() > 0) nks = std::max<long long>(kb, K.tm_slab.load() / kb * kb);
    nks = std::min<long long>(nks, n_k);
    TmBuf* buf = nullptr;
    syn_status s = tm_buffer(ds, device, st, (size_t)nks * row, &buf, 0);
    if (s != SYN_OK) return s;
    t.D = buf->p;
    // several slabs: finish(i) on a side stream overlaps walk(i + 1); D alternates between two
    // buffers and walk(i + 2) waits for finish(i), which zeroes its buffer (tm_pipe 2, default:
    // the walks alternate between two streams too, see below)
    const bool pipe = n_k > nks && K.tm_pipe.load() != 0;
    TmBuf* buf2 = nullptr;
    TmAux* aux = nullptr;
    if (pipe) {
        if ((s = tm_buffer(ds, device, st, (size_t)nks * row, &buf2, 1)) != SYN_OK) return s;
        if ((s = tm_aux(device, st, &aux)) != SYN_OK) return s;
    }
    // finish tile: KT kernels per CTA, fp64 + fp32 per (model, kernel, clock) in shared memory
    // (small: the finish is a latency chain per CTA, so small batches want many CTAs)
    const int fnt = 256;
    auto fsmem_of = [&](int k) { return tm_finish_smem(nm, k, n_f, a.xs, t.nslot); };
    int kt_cap = 1;
    while (kt_cap < 8 && fsmem_of(kt_cap + 1) <= std::min<size_t>((size_t)ds->finish_dyn_max, 150 * 1024)) ++kt_cap;
    // the smallest tile whose finish grid fits in one wave of resident CTAs (a partial second wave
    // doubles the finish's latency chain: c5 KT 3 -> 7 = 1195 -> 512 CTAs, 46 -> 37 us); when no
    // tile fits, the largest (kt_cap)
    int kt = 0;
    for (int k = 1; k <= kt_cap && !kt; ++k) {
        const int nb = finish_ctas_per_sm(ds, fnt, fsmem_of(k));
        if (nb > 0 && (nks + k - 1) / k <= (long long)nb * ds->sms) kt = k;
    }
    if (!kt) kt = kt_cap;
    if (K.tm_kt.load() > 0) kt = (int)std::min<long long>(K.tm_kt.load(), kt_cap);
    a.tile_k = kt;
    if (prepare_only) {                           // scratch, copies and the occupancy cache exist now
        *launches = 0;
        return ok();
    }
    const size_t fsmem = fsmem_of(kt);
    int usplit = 0;                               // units of the per-tree split (smode 2)
    for (int m = 0; m < nm; ++m)
        if (t.slot_of[m] >= 0) usplit += dms[m]->units_split;
    const int ctas = (int)std::max<long long>(1, K.tm_ctas.load() > 0 ? K.tm_ctas.load() : (1024LL / NTW) * ds->sms);
    t.s = a;
    int n = 0;
    int slab = 0;
    cudaError_t e = cudaSuccess;
    // tm_pipe 2: walks alternate between the caller's stream and a second walk stream, so walk(i + 1)
    // does not wait for walk(i) (it needs only its D buffer, zeroed by finish(i - 1)) and its CTAs
    // take the SMs that walk(i)'s last CTAs leave (a slab's tail left ~8 % of the SM cycles idle:
    // ncu sm__cycles_active / elapsed on c3; measured c3 16.0 -> 15.2 ms per step, c4 -0.5 %)
    const bool pipe2 = pipe && K.tm_pipe.load() == 2;
    if (pipe2 && ((e = cudaEventRecord(aux->fork, st)) != cudaSuccess ||
                  (e = cudaStreamWaitEvent(aux->stw, aux->fork, 0)) != cudaSuccess))
        return cuda_fail(e, "slab pipeline fork");
    auto fail_launch = [&](const char* what) {
        buf->dirty = true;
        if (buf2) buf2->dirty = true;
        if (pipe && slab > 0) cudaStreamWaitEvent(st, aux->finished[(slab - 1) & 1], 0);
        if (pipe2 && cudaEventRecord(aux->joinw, aux->stw) == cudaSuccess) cudaStreamWaitEvent(st, aux->joinw, 0);
        return cuda_fail(e, what);
    };
    for (long long s0 = 0; s0 < n_k; s0 += nks, ++slab) {
        t.slab0 = s0;
        t.nks = (int)std::min<long long>(nks, n_k - s0);
        const int pb = slab & 1;
        const cudaStream_t wst = pipe2 && pb ? aux->stw : st;                 // this slab's walk stream
        if (pipe) {
            t.D = pb ? buf2->p : buf->p;
            if (slab >= 2 && (e = cudaStreamWaitEvent(wst, aux->finished[pb], 0)) != cudaSuccess)
                return fail_launch("slab pipeline wait");
        }
        // tiny batches: split every (kernel, tree) task into clock sub-ranges while there are fewer
        // tasks than resident lanes (at most 8 sub-ranges of at least 8 clocks; each sub-range
        // adds a root descent, so batches with a task per lane keep whole tasks)
        t.nsub = 1;
        const long long lanes = (long long)ctas * NTW;
        while (t.nsub < 8 && (long long)t.nks * tt * t.nsub < lanes && n_f / (2 * t.nsub) >= 8 &&
               tm_walk_smem(F, kb, tt, 2 * tt * t.nsub, NTW) <= (size_t)ds->walk_dyn_max)
            t.nsub *= 2;
        if (K.tm_nsub.load() >= 1 && K.tm_nsub.load() <= std::min(n_f, 64) &&
            tm_walk_smem(F, kb, tt, tt * (int)K.tm_nsub.load(), NTW) <= (size_t)ds->walk_dyn_max)
            t.nsub = (int)K.tm_nsub.load();
        // small batches (2-8 tasks per lane): the longest walks bound the launch's tail, so trees
        // whose expected run count exceeds the model's mean are split into clock sub-ranges
        // (smode 2; measured: c5 walk 194 -> 182 us; at ~1 task per lane (c2) every lane is on its
        // critical path and the extra root descents cost more: 72 -> 76 us, so it stays off there)
        t.smode = t.nsub > 1 ? 1 : 0;
        t.units = tt * t.nsub;
        const long long ksplit = K.tm_split.load();
        const long long per_lane = (long long)t.nks * tt / std::max<long long>(lanes, 1);   // tasks per lane
        if (t.smode == 0 && usplit > tt && (ksplit > 0 || (ksplit < 0 && per_lane >= 2 && per_lane < 8)) &&
            tm_walk_smem(F, kb, tt, usplit, NTW) <= (size_t)ds->walk_dyn_max) {
            t.smode = 2;
            t.units = usplit;
        }
        t.n_tasks = (long long)((t.nks + kb - 1) / kb) * t.units * kb;
        // about one task per lane (c2): the trees in expected-cost order, alternating the costliest
        // and the cheapest remaining (broot_lpt), so each CTA's range starts with a costly tree and
        // the lanes that finish first take the cheap ones (measured c2 walk 70 -> 66.5 us; with
        // more tasks per lane the order cost c5 11 % and c3 2 %, so it stays off there)
        {
            const long long kl = K.tm_lpt.load();
            t.lpt = (t.smode == 0 && NTW == 512 && (kl > 0 || (kl < 0 && !pipe && per_lane < 2 && (long long)t.nks * tt >= lanes)))
                        ? 1 : 0;
            DevModel* tm[4] = {&t.s.ms, &t.s.me, &t.s.mx[0], &t.s.mx[1]};
            for (int m = 0; m < nm; ++m)
                if (t.slot_of[m] >= 0) tm[m]->broot = t.lpt ? dms[m]->broot_lpt : dms[m]->broot;
        }
        const size_t wsmem = tm_walk_smem(F, kb, tt, t.smode ? t.units : 0, NTW);
        // a few tasks per lane: dynamic task fetch balances walks of different lengths
        // per-lane-index task pools by default (L1-resident tree window, balanced, conflict-free);
        // static lane streams on request (tm_dyn = 0)
        t.dyn = K.tm_dyn.load() >= 0 ? (K.tm_dyn.load() ? 1 : 0) : 1;
        {
            const long long g = std::max<long long>(1, std::min<long long>(ctas, (t.n_tasks + 255) / 256));
            KernelTimer ktm("k_tm_walk", wst);
            const int cls = (fxall ? 1 : 0) + (t.smode ? 2 : 0) + (NTW == 1024 ? 4 : 0);
            switch (cls) {
                case 0: if (t.lpt) k_tm_walk<512, false, false, true><<<(unsigned)g, 512, wsmem, wst>>>(t);
                        else k_tm_walk<512, false, false><<<(unsigned)g, 512, wsmem, wst>>>(t);
                        break;
                case 1: if (t.lpt) k_tm_walk<512, true, false, true><<<(unsigned)g, 512, wsmem, wst>>>(t);
                        else k_tm_walk<512, true, false><<<(unsigned)g, 512, wsmem, wst>>>(t);
                        break;
                case 2: k_tm_walk<512, false, true><<<(unsigned)g, 512, wsmem, wst>>>(t); break;
                case 3: k_tm_walk<512, true, true><<<(unsigned)g, 512, wsmem, wst>>>(t); break;
                case 4: k_tm_walk<1024, false, false><<<(unsigned)g, 1024, wsmem, wst>>>(t); break;
                case 5: k_tm_walk<1024, true, false><<<(unsigned)g, 1024, wsmem, wst>>>(t); break;
                case 6: k_tm_walk<1024, false, true><<<(unsigned)g, 1024, wsmem, wst>>>(t); break;
                default: k_tm_walk<1024, true, true><<<(unsigned)g, 1024, wsmem, wst>>>(t); break;
            }
            e = cudaGetLastError();
        }
        if (e != cudaSuccess) return fail_launch("k_tm_walk launch");
        cudaStream_t fst = st;
        if (pipe) {
            if ((e = cudaEventRecord(aux->walked[pb], wst)) != cudaSuccess ||
                (e = cudaStreamWaitEvent(aux->st2, aux->walked[pb], 0)) != cudaSuccess)
                return fail_launch("slab pipeline fork");
            fst = aux->st2;
        }
        {
            KernelTimer ktm("k_tm_finish", fst);
            const dim3 fgrid((unsigned)((t.nks + kt - 1) / kt));
            if (!pipe && K.tm_pdl.load() != 0) {
                // programmatic dependent launch: the finish grid is scheduled while the walk runs
                // and waits (griddepcontrol.wait) for it before reading D
                cudaLaunchConfig_t lc;
                memset(&lc, 0, sizeof lc);
                lc.gridDim = fgrid;
                lc.blockDim = dim3((unsigned)fnt);
                lc.dynamicSmemBytes = fsmem;
                lc.stream = fst;
                cudaLaunchAttribute at[1];
                at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
                at[0].val.programmaticStreamSerializationAllowed = 1;
                lc.attrs = at;
                lc.numAttrs = 1;
                e = cudaLaunchKernelEx(&lc, k_tm_finish, t);
            } else {
                k_tm_finish<<<fgrid, fnt, fsmem, fst>>>(t);
                e = cudaGetLastError();
            }
        }
        if (e == cudaSuccess && pipe) e = cudaEventRecord(aux->finished[pb], aux->st2);
        if (e != cudaSuccess) return fail_launch("k_tm_finish launch");
        n += 2;
    }
    if (pipe && (e = cudaStreamWaitEvent(st, aux->finished[(slab - 1) & 1], 0)) != cudaSuccess)   // join
        return cuda_fail(e, "slab pipeline join");
    *launches = n;
    return ok();
}

// ---------------------------------------------------------- general exact path (kernels_gen.cuh)
constexpr size_t kGenSlabBytes = 64u << 20;   // fp64 + fp32 scratch per kernel slab

syn_status run_gen(SweepArgs a, int nm, cudaStream_t st, DevState* ds, int* launches) {
    const Knobs& K = knobs();
    const int n_f = a.n_f;
    const long long n_k = a.n_k;
    const size_t per_kernel = (size_t)nm * n_f * 12;
    long long nks = std::max<long long>(1, (long long)(kGenSlabBytes / per_kernel));
    nks = std::min<long long>(nks, n_k);
    int kt = (int)std::max<long long>(1, std::min<long long>(8, nks / (2LL * ds->sms)));
    if (K.gen_kt.load() > 0) kt = (int)std::min<long long>(K.gen_kt.load(), 64);
    a.tile_k = kt;
    void* scr = nullptr;
    const size_t mvb = (size_t)nks * per_kernel / 12 * 8;
    syn_status s = pool_alloc(ds, (size_t)nks * per_kernel + 256, st, &scr, "general-path scratch");
    if (s != SYN_OK) return s;
    GenArgs g;
    memset(&g, 0, sizeof g);
    g.s = a;
    g.mv = static_cast<double*>(scr);
    g.sv = reinterpret_cast<float*>(static_cast<char*>(scr) + (mvb + 255) / 256 * 256);
    g.nm = nm;
    int n = 0;
    cudaError_t e = cudaSuccess;
    for (long long s0 = 0; s0 < n_k && e == cudaSuccess; s0 += nks) {
        g.slab0 = s0;
        g.nks = (int)std::min<long long>(nks, n_k - s0);
        const long long units = (long long)g.nks * n_f;
        {
            KernelTimer kt1("k_gen_forest", st);
            k_gen_forest<<<(unsigned)((units + 255) / 256), 256, 0, st>>>(g);
            e = cudaGetLastError();
        }
        if (e != cudaSuccess) break;
        {
            KernelTimer kt2("k_gen_finish", st);
            k_gen_finish<<<(unsigned)((g.nks + kt - 1) / kt), 256, 0, st>>>(g);
            e = cudaGetLastError();
        }
        n += 2;
    }
    cudaFreeAsync(scr, st);
    if (e != cudaSuccess) return cuda_fail(e, "general-path launch");
    *launches = n;
    return ok();
}

// ------------------------------------------------------------------------ SVR member
// SVR members (kernels_svr.cuh): per model, V = clock factors and the split contractions P into
// stream-ordered scratch from the library pool; dm.svr_p / svr_splits point the finish step at
// them.  Released (cudaFreeAsync) after the sweep's kernels are enqueued.
struct SvrScratch {
    std::vector<void*> bufs;
    cudaStream_t st = nullptr;
    int launches = 0;
    void release() {
        for (void* b : bufs) cudaFreeAsync(b, st);
        bufs.clear();
    }
    ~SvrScratch() { release(); }
};

template <int CPT>
cudaError_t launch_svr_t(const SvrArgs& sa, dim3 grid, cudaStream_t st) {
    const size_t smem = (size_t)kSvrStages * kSvrJC * (kSvrTK + 32 * CPT) * sizeof(double) + kSvrStages * 8;
    k_svr<CPT><<<grid, 256, smem, st>>>(sa);
    return cudaGetLastError();
}

constexpr size_t kSvrSlabBytes = 256u << 20;   // U scratch per kernel slab

// Tensor-core SVR contraction (kernels_svr_tc.cuh): the V digit planes once per call, then per
// kernel slab the U digit planes and k_svr_tc over (128-kernel tile, 64-clock tile, SV split).
syn_status prepare_svr_tc(DevModel& dm, DevState* ds, const float* d_features, long long n_k, int F,
                          const syn_clocks* clocks, cudaStream_t st, SvrScratch& scr) {
    scr.st = st;
    const int n_f = clocks->n_f;
    const int tiles_n = (n_f + kTcN - 1) / kTcN;
    const int n_svp = (dm.n_sv + kTcKC - 1) / kTcKC * kTcKC;
    const int n_chunks = n_svp / kTcKC;
    // kernel slabs (multiples of the 128-kernel tile) bound the U digit planes to kSvrSlabBytes
    long long nks = std::max<long long>(kTcM, (long long)(kSvrSlabBytes / ((size_t)n_svp * kTcDig)) / kTcM * kTcM);
    nks = std::min<long long>(nks, (n_k + kTcM - 1) / kTcM * kTcM);
    const long long tiles = (std::min(nks, n_k) + kTcM - 1) / kTcM * tiles_n;
    // split the SV range until the grid covers the resident CTA slots (kTcCtasPerSm per SM)
    int splits = (int)std::max<long long>(1, (long long)kTcCtasPerSm * ds->sms / std::max<long long>(tiles, 1));
    splits = std::min(splits, kSvrMaxSplits);
    if (knobs().svr_splits.load() > 0) splits = (int)std::min<long long>(knobs().svr_splits.load(), kSvrMaxSplits);
    splits = std::max(1, std::min(splits, n_chunks));
    const int cps = (n_chunks + splits - 1) / splits;
    splits = (n_chunks + cps - 1) / cps;
    auto al = [](size_t b) { return (b + 255) / 256 * 256; };
    const size_t pb = (size_t)splits * (size_t)n_k * n_f * sizeof(double);
    const size_t vqb = (size_t)tiles_n * n_chunks * kTcBBytes;
    const size_t uqb = (size_t)((nks + kTcM - 1) / kTcM) * n_chunks * kTcABytes;
    const size_t o_vq = al(pb), o_uq = o_vq + al(vqb), total = o_uq + uqb;
    void* buf = nullptr;
    syn_status ps = pool_alloc(ds, total, st, &buf, "SVR scratch");
    if (ps != SYN_OK) return ps;
    scr.bufs.push_back(buf);
    char* b = static_cast<char*>(buf);
    SvrTcArgs ta;
    memset(&ta, 0, sizeof ta);
    SvrArgs& sa = ta.s;
    sa.features = d_features;
    sa.n_k = n_k;
    sa.F = F;
    sa.freqs = clocks->d_freqs;
    sa.n_f = n_f;
    sa.sv = dm.sv;
    sa.dual = dm.dual;
    sa.in_mean = dm.in_mean;
    sa.in_scale = dm.in_scale;
    sa.gamma = dm.svr_gamma;
    sa.n_sv = dm.n_sv;
    sa.n_svp = n_svp;
    sa.P = reinterpret_cast<double*>(b);
    ta.Vq = reinterpret_cast<unsigned char*>(b + o_vq);
    ta.Uq = reinterpret_cast<unsigned char*>(b + o_uq);
    ta.eU = dm.svr_eU;
    ta.chunks_per_split = cps;
    cudaError_t e = cudaSuccess;
    {
        KernelTimer kt("k_svr_vdig", st);
        k_svr_vdig<<<dim3((unsigned)tiles_n, (unsigned)n_chunks), 2 * kTcN, 0, st>>>(ta);
        e = cudaGetLastError();
    }
    if (e != cudaSuccess) return cuda_fail(e, "k_svr_vdig launch");
    scr.launches += 1;
    const size_t usmem = (size_t)kTcM * (F + 1) * sizeof(double) + (size_t)kTcKC * F * sizeof(float);
    if (usmem > (size_t)ds->optin) return fail(SYN_ERR_UNSUPPORTED, "SVR member with %d inputs exceeds shared memory", F + 1);
    for (long long s0 = 0; s0 < n_k; s0 += nks) {
        sa.slab0 = s0;
        sa.nks = (int)std::min<long long>(nks, n_k - s0);
        const int mts = (sa.nks + kTcM - 1) / kTcM;
        {
            KernelTimer kt("k_svr_udig", st);
            k_svr_udig<<<dim3((unsigned)mts, (unsigned)n_chunks), 256, usmem, st>>>(ta);
            e = cudaGetLastError();
        }
        if (e == cudaSuccess) {
            KernelTimer kt("k_svr_tc", st);
            k_svr_tc<<<dim3((unsigned)tiles_n, (unsigned)mts, (unsigned)splits), kTcThreads, kTcSmem, st>>>(ta);
            e = cudaGetLastError();
        }
        if (e != cudaSuccess) return cuda_fail(e, "SVR tensor-core contraction");
        scr.launches += 2;
    }
    dm.svr_p = sa.P;
    dm.svr_splits = splits;
    return ok();
}

syn_status prepare_svr(DevModel& dm, DevState* ds, const float* d_features, long long n_k, int F, const syn_clocks* clocks,
                       cudaStream_t st, SvrScratch& scr) {
    if (dm.svr_weight == 0.0) return ok();
    // the tensor-core path keeps every level accumulator exact in int32 for n_sv <= 16384
    if (knobs().svr_tc.load() != 0 && dm.n_sv <= 16384) return prepare_svr_tc(dm, ds, d_features, n_k, F, clocks, st, scr);
    scr.st = st;
    const int n_f = clocks->n_f;
    const int cpt = std::min(8, (n_f + 31) / 32);
    const int tn = 32 * cpt;
    const int tiles_n = (n_f + tn - 1) / tn;
    const int n_svp = (dm.n_sv + kSvrJC - 1) / kSvrJC * kSvrJC;
    const int n_chunks = n_svp / kSvrJC;
    // kernel slabs bound the U scratch; each slab is one k_svr_u + one k_svr launch
    long long nks = std::max<long long>(kSvrTK, (long long)(kSvrSlabBytes / ((size_t)n_svp * 8)) / kSvrTK * kSvrTK);
    nks = std::min<long long>(nks, (n_k + kSvrTK - 1) / kSvrTK * kSvrTK);
    const long long tiles = (std::min(nks, n_k) + kSvrTK - 1) / kSvrTK * tiles_n;
    if ((nks + kSvrTK - 1) / kSvrTK > 0x7fffffffLL) return fail(SYN_ERR_UNSUPPORTED, "n_kernels too large for k_svr");
    // split the SV range across CTAs until the grid covers the SMs (at most kSvrMaxSplits)
    int splits = (int)std::max<long long>(1, ds->sms / std::max<long long>(tiles, 1));
    splits = std::min(splits, kSvrMaxSplits);
    if (knobs().svr_splits.load() > 0) splits = (int)std::min<long long>(knobs().svr_splits.load(), kSvrMaxSplits);
    splits = std::max(1, std::min(splits, n_chunks));
    const int cps = (n_chunks + splits - 1) / splits;
    splits = (n_chunks + cps - 1) / cps;
    const size_t pb = (size_t)splits * (size_t)n_k * n_f * sizeof(double);
    const size_t vb = (size_t)tiles_n * n_svp * tn * sizeof(double);
    const size_t ub = (size_t)((nks + kSvrTK - 1) / kSvrTK) * n_svp * kSvrTK * sizeof(double);
    const size_t voff = (pb + 255) / 256 * 256, uoff = voff + (vb + 255) / 256 * 256;
    const size_t total = uoff + ub;
    void* buf = nullptr;
    syn_status ps = pool_alloc(ds, total, st, &buf, "SVR scratch");
    if (ps != SYN_OK) return ps;
    scr.bufs.push_back(buf);
    SvrArgs sa;
    memset(&sa, 0, sizeof sa);
    sa.features = d_features;
    sa.n_k = n_k;
    sa.F = F;
    sa.freqs = clocks->d_freqs;
    sa.n_f = n_f;
    sa.sv = dm.sv;
    sa.dual = dm.dual;
    sa.in_mean = dm.in_mean;
    sa.in_scale = dm.in_scale;
    sa.gamma = dm.svr_gamma;
    sa.n_sv = dm.n_sv;
    sa.n_svp = n_svp;
    sa.tn = tn;
    sa.chunks_per_split = cps;
    sa.P = static_cast<double*>(buf);
    sa.Vt = reinterpret_cast<double*>(static_cast<char*>(buf) + voff);
    sa.Ut = reinterpret_cast<double*>(static_cast<char*>(buf) + uoff);
    const long long nv = (long long)tiles_n * n_svp * tn;
    cudaError_t e;
    {
        KernelTimer kt("k_svr_v", st);
        k_svr_v<<<(unsigned)((nv + 255) / 256), 256, 0, st>>>(sa);
        e = cudaGetLastError();
    }
    if (e != cudaSuccess) return cuda_fail(e, "k_svr_v launch");
    scr.launches += 1;
    const size_t usmem = (size_t)F * (64 * sizeof(double) + kSvrJC * sizeof(float));
    if (usmem > (size_t)ds->optin) return fail(SYN_ERR_UNSUPPORTED, "SVR member with %d inputs exceeds shared memory", F + 1);
    for (long long s0 = 0; s0 < n_k; s0 += nks) {
        sa.slab0 = s0;
        sa.nks = (int)std::min<long long>(nks, n_k - s0);
        const unsigned kts = (unsigned)((sa.nks + kSvrTK - 1) / kSvrTK);
        {
            KernelTimer kt("k_svr_u", st);
            k_svr_u<<<dim3(kts, (unsigned)(n_svp / kSvrJC)), 256, usmem, st>>>(sa);
            e = cudaGetLastError();
        }
        if (e != cudaSuccess) return cuda_fail(e, "k_svr_u launch");
        const dim3 grid(kts, (unsigned)tiles_n, (unsigned)splits);
        KernelTimer kt("k_svr", st);
        switch (cpt) {
            case 1: e = launch_svr_t<1>(sa, grid, st); break;
            case 2: e = launch_svr_t<2>(sa, grid, st); break;
            case 3: e = launch_svr_t<3>(sa, grid, st); break;
            case 4: e = launch_svr_t<4>(sa, grid, st); break;
            case 5: e = launch_svr_t<5>(sa, grid, st); break;
            case 6: e = launch_svr_t<6>(sa, grid, st); break;
            case 7: e = launch_svr_t<7>(sa, grid, st); break;
            default: e = launch_svr_t<8>(sa, grid, st); break;
        }
        if (e != cudaSuccess) return cuda_fail(e, "k_svr launch");
        scr.launches += 2;
    }
    dm.svr_p = sa.P;
    dm.svr_splits = splits;
    return ok();
}

// --------------------------------------------------------------------- sweep driver

syn_status validate_models(const syn_model* const* models, int nm, int32_t F, const syn_clocks* clocks) {
    if (!models[0] || !models[1]) return fail(SYN_ERR_INVALID_ARG, "model is NULL");
    if (!clocks) return fail(SYN_ERR_INVALID_ARG, "clocks is NULL");
    for (int m = 0; m < nm; ++m) {
        const syn_model* x = models[m];
        if (!x) continue;
        if (F + 1 != x->n_inputs)
            return fail(SYN_ERR_INVALID_ARG, "n_features+1=%d does not match model %d n_inputs=%d", F + 1, m, x->n_inputs);
        if (x->device != clocks->device) return fail(SYN_ERR_INVALID_ARG, "model %d / clocks on different devices", m);
    }
    if (!current_device_is(clocks->device)) return fail(SYN_ERR_INVALID_ARG, "clocks device differs from the current device");
    return SYN_OK;
}

// One predict / sweep / sweep4 call.  models[0..1] speedup, energy; models[2..3] (nm == 4) direct
// EDP / ED2P or NULL.  pred[m] = output planes or NULL.
syn_status run_sweep(const syn_model* const* models, int nm, const float* d_features, int64_t n_k, int32_t F,
                     const syn_clocks* clocks, int32_t def, const syn_target* targets, int32_t n_t,
                     int32_t* d_choice, float* const* pred, int mode, cudaStream_t st, bool prepare_only = false) {
    syn_status vs = validate_models(models, nm, F, clocks);
    if (vs != SYN_OK) return vs;
    if (n_k < 0) return fail(SYN_ERR_INVALID_ARG, "n_kernels=%lld < 0", (long long)n_k);
    const int n_f = clocks->n_f;
    if (mode == kModeSweep) {
        if (def < 0 || def >= n_f) return fail(SYN_ERR_INVALID_ARG, "default_idx=%d outside [0, %d)", def, n_f);
        if (!prepare_only) {
            vs = check_targets(targets, n_t);
            if (vs != SYN_OK) return vs;
        }
    } else if (def < -1 || def >= n_f) {
        return fail(SYN_ERR_INVALID_ARG, "default_idx=%d outside [-1, %d)", def, n_f);
    }
    if (n_k == 0) {
        g_last = {0, 0, 0, 0, 0};
        return ok();
    }
    if (!prepare_only) {
        if (!d_features) return fail(SYN_ERR_INVALID_ARG, "d_features is NULL");
        if (mode == kModeSweep && !d_choice) return fail(SYN_ERR_INVALID_ARG, "d_choice is NULL");
        if (mode == kModePredict && (!pred[0] || !pred[1])) return fail(SYN_ERR_INVALID_ARG, "d_speedup/d_energy is NULL");
    }
    if ((n_k + 7) / 8 > 0x7fffffffLL) return fail(SYN_ERR_UNSUPPORTED, "n_kernels too large for one call");
    DevState* ds = nullptr;
    if ((vs = need_dev(clocks->device, &ds)) != SYN_OK) return vs;

    SweepArgs a;
    memset(&a, 0, sizeof a);
    a.ms = models[0]->dm;
    a.me = models[1]->dm;
    for (int x = 0; x < 2; ++x)
        if (nm > 2 + x && models[2 + x]) {
            a.mx[x] = models[2 + x]->dm;
            a.has_x[x] = 1;
        }
    a.features = d_features;
    a.n_k = n_k;
    a.F = F;
    a.freqs = clocks->d_freqs;
    a.n_f = n_f;
    a.def = def;
    a.n_t = mode == kModeSweep && !prepare_only ? n_t : 0;
    for (int t = 0; t < a.n_t; ++t) {
        a.kind[t] = targets[t].kind;
        a.frac[t] = (double)targets[t].x / 100.0;   // the oracle's frac (oracle.c select)
    }
    a.choice = d_choice;
    a.S_out = pred[0];
    a.E_out = pred[1];
    a.X_out[0] = nm > 2 ? pred[2] : nullptr;
    a.X_out[1] = nm > 3 ? pred[3] : nullptr;
    a.mode = mode;
    a.xs = (F + 2) | 1;
    const bool tm = knobs().algo.load() == 0 && tm_eligible(a, nm, ds);
    if (prepare_only) {
        if (!tm) return ok();
        int nl = 0;
        return run_tm(a, nm, const_cast<syn_model* const*>(models), clocks, st, ds, true, &nl);
    }
    SvrScratch scr;
    DevModel* dms[4] = {&a.ms, &a.me, &a.mx[0], &a.mx[1]};
    syn_status ss = SYN_OK;
    for (int m = 0; m < nm && ss == SYN_OK; ++m)
        if (present(a, m)) ss = prepare_svr(*dms[m], ds, d_features, n_k, F, clocks, st, scr);
    if (ss != SYN_OK) return ss;
    int nl = 0;
    if (tm) {
        ss = run_tm(a, nm, const_cast<syn_model* const*>(models), clocks, st, ds, false, &nl);
        if (ss != SYN_OK) return ss;
        g_last = {nl + scr.launches, n_k * (long long)n_f, 0, 0, kVarTm};
        return ok();
    }
    ss = run_gen(a, nm, st, ds, &nl);
    if (ss != SYN_OK) return ss;
    g_last = {nl + scr.launches, n_k * (long long)n_f, ((long long)n_k * n_f + 255) / 256, 256, kVarGen};
    return ok();
}

}  // namespace

// =============================================================================== C ABI

extern "C" {

const char* synergy_last_error(void) { return g_err.c_str(); }

int32_t synergy_version(void) { return SYNERGY_VERSION; }

syn_status synergy_config_set(const char* key, int64_t value) {
    if (!key) return fail(SYN_ERR_INVALID_ARG, "key is NULL");
    knobs();
    for (const KnobName& k : kKnobs)
        if (!strcmp(k.name, key)) {
            k.v->store(value);
            return ok();
        }
    return fail(SYN_ERR_INVALID_ARG, "unknown tuning key '%s'", key);
}

syn_status synergy_config_get(const char* key, int64_t* value) {
    if (!key || !value) return fail(SYN_ERR_INVALID_ARG, "key/value is NULL");
    knobs();
    for (const KnobName& k : kKnobs)
        if (!strcmp(k.name, key)) {
            *value = k.v->load();
            return ok();
        }
    return fail(SYN_ERR_INVALID_ARG, "unknown tuning key '%s'", key);
}

syn_status synergy_model_create(const syn_model_desc* d, int32_t device, syn_model** out) {
    if (!out) return fail(SYN_ERR_INVALID_ARG, "out is NULL");
    *out = nullptr;
    if (!d) return fail(SYN_ERR_INVALID_ARG, "desc is NULL");
    if (d->n_inputs < 1 || d->n_inputs > SYNERGY_MAX_INPUTS)
        return fail(SYN_ERR_INVALID_ARG, "n_inputs=%d outside [1, %d]", d->n_inputs, SYNERGY_MAX_INPUTS);
    if (!std::isfinite(d->linear_weight) || !std::isfinite(d->forest_weight) || !std::isfinite(d->svr_weight))
        return fail(SYN_ERR_INVALID_ARG, "member weights must be finite");
    if (d->linear_weight == 0.0 && d->forest_weight == 0.0 && d->svr_weight == 0.0)
        return fail(SYN_ERR_INVALID_ARG, "all member weights are 0");
    if (d->linear_weight != 0.0 && !d->lin_w) return fail(SYN_ERR_INVALID_ARG, "lin_w is NULL");
    const int F = d->n_inputs - 1;
    const bool has_svr = d->svr_weight != 0.0;
    if (has_svr) {
        if (d->n_sv < 1 || d->n_sv > (1 << 24)) return fail(SYN_ERR_INVALID_ARG, "n_sv=%d outside [1, 2^24]", d->n_sv);
        if (!d->sv || !d->dual_coef || !d->in_mean || !d->in_scale)
            return fail(SYN_ERR_INVALID_ARG, "SVR arrays must be non-NULL");
        if (!std::isfinite(d->svr_gamma) || d->svr_gamma < 0.0 || !std::isfinite(d->svr_intercept))
            return fail(SYN_ERR_INVALID_ARG, "svr_gamma must be finite and >= 0, svr_intercept finite");
        for (int64_t q = 0; q < (int64_t)d->n_sv * d->n_inputs; ++q)
            if (!std::isfinite(d->sv[q])) return fail(SYN_ERR_INVALID_ARG, "sv[%lld] is not finite", (long long)q);
        for (int j = 0; j < d->n_sv; ++j)
            if (!std::isfinite(d->dual_coef[j])) return fail(SYN_ERR_INVALID_ARG, "dual_coef[%d] is not finite", j);
        for (int q = 0; q < d->n_inputs; ++q)
            if (!std::isfinite(d->in_mean[q]) || !std::isfinite(d->in_scale[q]) || d->in_scale[q] == 0.0)
                return fail(SYN_ERR_INVALID_ARG, "in_mean/in_scale[%d] not finite or scale 0", q);
    }
    const uint32_t leaf_code = (uint32_t)(F + 1);
    std::vector<uint2> nodes;
    std::vector<int2> trees;
    int max_depth = 0;
    if (d->forest_weight != 0.0) {
        if (d->n_trees < 1) return fail(SYN_ERR_INVALID_ARG, "n_trees=%d < 1", d->n_trees);
        if (!d->tree_offset || !d->feature || !d->left || !d->right || !d->value)
            return fail(SYN_ERR_INVALID_ARG, "forest arrays must be non-NULL");
        std::vector<int64_t> queue;
        std::vector<int> qdepth;
        std::vector<char> seen;
        trees.resize(d->n_trees);
        for (int t = 0; t < d->n_trees; ++t) {
            const int64_t b = d->tree_offset[t], e = d->tree_offset[t + 1];
            if (b < 0 || e <= b) return fail(SYN_ERR_INVALID_ARG, "tree %d: bad node range [%lld, %lld)", t, (long long)b, (long long)e);
            const int64_t n = e - b;
            if (n > kMaxDelta) return fail(SYN_ERR_UNSUPPORTED, "tree %d: %lld nodes > %d", t, (long long)n, kMaxDelta);
            seen.assign((size_t)n, 0);
            queue.assign(1, 0);
            qdepth.assign(1, 0);
            seen[0] = 1;
            const int64_t base = (int64_t)nodes.size();
            if (base + n > 0x7ffffff0LL) return fail(SYN_ERR_UNSUPPORTED, "more than 2^31 nodes");
            int depth = 0;
            // breadth-first re-layout: children pushed together, so right = left + 1
            for (size_t p = 0; p < queue.size(); ++p) {
                const int64_t id = queue[p];
                const int32_t f = d->feature[b + id];
                const float v = d->value[b + id];
                uint32_t vb;
                memcpy(&vb, &v, 4);
                depth = std::max(depth, qdepth[p]);
                if (f < 0) {
                    // leaves must be finite: the exact sums (Q8) are defined on reals
                    if (!std::isfinite(v))
                        return fail(SYN_ERR_INVALID_ARG, "tree %d node %lld: leaf value is not finite", t, (long long)id);
                    nodes.push_back(make_uint2(vb, 0xFFFFFF00u | leaf_code));
                    continue;
                }
                if (f >= d->n_inputs) return fail(SYN_ERR_INVALID_ARG, "tree %d node %lld: feature %d >= n_inputs", t, (long long)id, f);
                const int32_t l = d->left[b + id], r = d->right[b + id];
                if (l < 0 || l >= n || r < 0 || r >= n)
                    return fail(SYN_ERR_INVALID_ARG, "tree %d node %lld: child id outside the tree", t, (long long)id);
                if (seen[l] || seen[r] || l == r)
                    return fail(SYN_ERR_INVALID_ARG, "tree %d node %lld: a node is reached twice (not a tree)", t, (long long)id);
                seen[l] = seen[r] = 1;
                if (qdepth[p] + 1 > SYNERGY_MAX_DEPTH)
                    return fail(SYN_ERR_UNSUPPORTED, "tree %d deeper than %d", t, SYNERGY_MAX_DEPTH);
                const int32_t delta = (int32_t)(queue.size() - p);
                queue.push_back(l);
                qdepth.push_back(qdepth[p] + 1);
                queue.push_back(r);
                qdepth.push_back(qdepth[p] + 1);
                nodes.push_back(make_uint2(vb, ((uint32_t)delta << kCodeBits) | (uint32_t)f));
            }
            trees[t] = make_int2((int)base, depth);
            max_depth = std::max(max_depth, depth);
        }
    }
    // exact fixed-point scale for the leaf sums: s = -(smallest leaf ulp exponent); fx_ok when
    // T * max|v| * 2^s < 2^62 (one int64), fx32 when every |v| * 2^s < 2^31
    int fx_ok = 0, fx_s = 0, fx32 = 0;
    if (d->forest_weight != 0.0) {
        int min_lsb = 1 << 30, max_e = -(1 << 30);
        for (const uint2& nd : nodes) {
            if ((nd.y & 0xffu) != leaf_code) continue;
            float v;
            memcpy(&v, &nd.x, 4);
            if (v == 0.0f) continue;
            int e2 = 0;
            std::frexp(v, &e2);                       // |v| in [2^(e2-1), 2^e2)
            min_lsb = std::min(min_lsb, std::max(e2 - 24, -149));
            max_e = std::max(max_e, e2);
        }
        if (max_e == -(1 << 30)) { fx_ok = 1; fx_s = 0; fx32 = 1; }   // all leaves zero
        else {
            fx_s = -min_lsb;
            int lg = 0;
            while ((1LL << lg) < (long long)d->n_trees + 1) ++lg;
            fx_ok = (max_e + fx_s + lg <= 61) ? 1 : 0;
            fx32 = (fx_ok && max_e + fx_s <= 31) ? 1 : 0;
        }
    }

    // Per-tree clock sub-range split for small batches (k_tm_walk unit tables): the expected number
    // of runs (clock intervals sharing a leaf) of a walk over all clocks, with every static split
    // taken as 50/50: sum over the leaves of 2^-(static splits on the path), counting only leaves
    // whose clock interval (from the clock-split thresholds on the path) is not empty.  A tree gets
    // ceil(runs / the model's mean runs) sub-ranges, at most 8.
    std::vector<int2> tsplit;
    std::vector<int> lpt;                                  // expected-cost order (broot_lpt)
    int units_split = 0;
    if (d->forest_weight != 0.0) {
        std::vector<double> cost((size_t)d->n_trees, 0.0);
        struct Item { int64_t id; double w; float clo, chi; };
        std::vector<Item> st;
        double mean = 0.0;
        for (int t = 0; t < d->n_trees; ++t) {
            const int64_t b = d->tree_offset[t];
            st.assign(1, Item{0, 1.0, -INFINITY, INFINITY});
            double c = 0.0;
            while (!st.empty()) {
                const Item it = st.back();
                st.pop_back();
                const int32_t f = d->feature[b + it.id];
                if (f < 0) { c += it.w; continue; }
                const float thr = d->value[b + it.id];
                const int32_t l = d->left[b + it.id], r = d->right[b + it.id];
                if (f == F) {
                    if (std::min(it.chi, thr) > it.clo) st.push_back({l, it.w, it.clo, std::min(it.chi, thr)});
                    if (it.chi > std::max(it.clo, thr)) st.push_back({r, it.w, std::max(it.clo, thr), it.chi});
                } else {
                    st.push_back({l, 0.5 * it.w, it.clo, it.chi});
                    st.push_back({r, 0.5 * it.w, it.clo, it.chi});
                }
            }
            cost[t] = std::max(c, 1e-9);
            mean += cost[t];
        }
        mean /= d->n_trees;
        std::vector<int> by(d->n_trees);
        for (int t = 0; t < d->n_trees; ++t) by[t] = t;
        std::stable_sort(by.begin(), by.end(), [&](int x, int y) { return cost[x] > cost[y]; });
        lpt.resize(d->n_trees);
        for (int i = 0, lo = 0, hi = d->n_trees - 1; lo <= hi; ++i) lpt[i] = (i & 1) ? by[hi--] : by[lo++];
        tsplit.resize(d->n_trees);
        for (int t = 0; t < d->n_trees; ++t) {
            const double piece = mean * (double)std::max<long long>(1, knobs().split_piece.load()) / 4.0;
            const int ns = std::max(1, std::min(8, (int)std::ceil(cost[t] / piece - 1e-9)));
            tsplit[t] = make_int2(units_split, ns);
            units_split += ns;
        }
    }

    // 2-level blocks (see internal.h): built from the validated description, breadth-first
    std::vector<uint4> blocks;
    std::vector<int> broot;
    if (d->forest_weight != 0.0) {
        broot.resize(d->n_trees);
        std::vector<int64_t> q;
        std::vector<int64_t> qb;
        for (int t = 0; t < d->n_trees; ++t) {
            const int64_t b = d->tree_offset[t];
            auto is_leaf = [&](int64_t id) { return d->feature[b + id] < 0; };
            auto fbits = [&](int64_t id) { uint32_t u; memcpy(&u, &d->value[b + id], 4); return u; };
            if ((blocks.size() >> 1) + 1 > 0x7ffffff0ULL) return fail(SYN_ERR_UNSUPPORTED, "too many blocks");
            broot[t] = (int)(blocks.size() >> 1);
            blocks.resize(blocks.size() + 2);
            q.assign(1, 0);
            qb.assign(1, broot[t]);
            for (size_t p = 0; p < q.size(); ++p) {
                const int64_t id = q[p];
                uint32_t w[8] = {0, 0, 0, 0, 0, 0, 0, 0};
                w[0] = fbits(id);
                if (is_leaf(id)) {
                    w[3] = leaf_code | (leaf_code << 8) | (leaf_code << 16);
                } else {
                    uint32_t codes = (uint32_t)d->feature[b + id];
                    // the grandchild blocks of a block (a "family", allocated consecutively) never
                    // straddle a 128-byte line: lanes of a warp that leave the same block for
                    // different grandchildren then share one L1 line (one wavefront)
                    int fam = 0;
                    for (int dd = 0; dd < 2; ++dd) {
                        const int64_t c = dd ? d->right[b + id] : d->left[b + id];
                        if (is_leaf(c)) continue;
                        fam += !is_leaf(d->left[b + c]) + !is_leaf(d->right[b + c]);
                    }
                    if (fam >= 2 && (int)((blocks.size() >> 1) & 3) + fam > 4)
                        blocks.resize(((blocks.size() >> 1) + 3) / 4 * 4 * 2, make_uint4(0, 0, 0, 0));
                    for (int dd = 0; dd < 2; ++dd) {
                        const int64_t c = dd ? d->right[b + id] : d->left[b + id];
                        w[1 + dd] = fbits(c);
                        if (is_leaf(c)) {
                            codes |= leaf_code << (8 + 8 * dd);
                            continue;
                        }
                        codes |= (uint32_t)d->feature[b + c] << (8 + 8 * dd);
                        for (int ee = 0; ee < 2; ++ee) {
                            const int64_t g2 = ee ? d->right[b + c] : d->left[b + c];
                            const int slot = 2 * dd + ee;
                            if (is_leaf(g2)) {
                                w[4 + slot] = fbits(g2);
                                codes |= 1u << (24 + slot);
                            } else {
                                const int64_t gi = (int64_t)(blocks.size() >> 1);
                                blocks.resize(blocks.size() + 2);
                                w[4 + slot] = (uint32_t)gi;
                                q.push_back(g2);
                                qb.push_back(gi);
                            }
                        }
                    }
                    w[3] = codes;
                }
                blocks[2 * qb[p]] = make_uint4(w[0], w[1], w[2], w[3]);
                blocks[2 * qb[p] + 1] = make_uint4(w[4], w[5], w[6], w[7]);
            }
        }
    }

    DeviceGuard g(device);
    if (!g.okay) return fail(SYN_ERR_INVALID_ARG, "cannot select device %d", device);
    const size_t nb = std::max<size_t>(nodes.size(), 1) * sizeof(uint2);
    const size_t tb = std::max<size_t>(trees.size(), 1) * sizeof(int2);
    const size_t lb = (size_t)d->n_inputs * sizeof(double);
    const size_t bb = std::max<size_t>(blocks.size(), 2) * sizeof(uint4);
    const size_t rb = std::max<size_t>(broot.size(), 1) * sizeof(int);
    const size_t off_t = (nb + 255) / 256 * 256, off_l = off_t + (tb + 255) / 256 * 256;
    const size_t off_b = off_l + (lb + 255) / 256 * 256, off_r = off_b + (bb + 255) / 256 * 256;
    const size_t n_sv = has_svr ? (size_t)d->n_sv : 0;
    const size_t svb = n_sv * d->n_inputs * sizeof(float), dcb = n_sv * sizeof(double);
    const size_t off_sv = off_r + (rb + 255) / 256 * 256, off_dc = off_sv + (svb + 255) / 256 * 256;
    const size_t off_mn = off_dc + (dcb + 255) / 256 * 256, off_sc = off_mn + (lb + 255) / 256 * 256;
    const size_t off_ts = ((has_svr ? off_sc + lb : off_r + rb) + 255) / 256 * 256;
    const size_t tsb = std::max<size_t>(tsplit.size(), 1) * sizeof(int2);
    const size_t off_lp = (off_ts + tsb + 255) / 256 * 256;
    std::vector<int> broot_lpt(lpt.size());
    for (size_t i = 0; i < lpt.size(); ++i) broot_lpt[i] = broot[lpt[i]];
    const size_t total = off_lp + rb;
    void* mem = nullptr;
    cudaError_t e = cudaMalloc(&mem, total);
    if (e != cudaSuccess) return cuda_fail(e, "cudaMalloc(model)");
    char* base = static_cast<char*>(mem);
    std::vector<double> lw((size_t)d->n_inputs, 0.0);
    if (d->linear_weight != 0.0) std::copy(d->lin_w, d->lin_w + d->n_inputs, lw.begin());
    if ((!nodes.empty() && (e = cudaMemcpy(base, nodes.data(), nodes.size() * sizeof(uint2), cudaMemcpyHostToDevice)) != cudaSuccess) ||
        (!trees.empty() && (e = cudaMemcpy(base + off_t, trees.data(), trees.size() * sizeof(int2), cudaMemcpyHostToDevice)) != cudaSuccess) ||
        (e = cudaMemcpy(base + off_l, lw.data(), lb, cudaMemcpyHostToDevice)) != cudaSuccess ||
        (!blocks.empty() && (e = cudaMemcpy(base + off_b, blocks.data(), blocks.size() * sizeof(uint4), cudaMemcpyHostToDevice)) != cudaSuccess) ||
        (!broot.empty() && (e = cudaMemcpy(base + off_r, broot.data(), broot.size() * sizeof(int), cudaMemcpyHostToDevice)) != cudaSuccess) ||
        (!tsplit.empty() && (e = cudaMemcpy(base + off_ts, tsplit.data(), tsplit.size() * sizeof(int2), cudaMemcpyHostToDevice)) != cudaSuccess) ||
        (!broot_lpt.empty() && (e = cudaMemcpy(base + off_lp, broot_lpt.data(), broot_lpt.size() * sizeof(int), cudaMemcpyHostToDevice)) != cudaSuccess) ||
        (has_svr && ((e = cudaMemcpy(base + off_sv, d->sv, svb, cudaMemcpyHostToDevice)) != cudaSuccess ||
                     (e = cudaMemcpy(base + off_dc, d->dual_coef, dcb, cudaMemcpyHostToDevice)) != cudaSuccess ||
                     (e = cudaMemcpy(base + off_mn, d->in_mean, lb, cudaMemcpyHostToDevice)) != cudaSuccess ||
                     (e = cudaMemcpy(base + off_sc, d->in_scale, lb, cudaMemcpyHostToDevice)) != cudaSuccess))) {
        cudaFree(mem);
        return cuda_fail(e, "cudaMemcpy(model)");
    }
    syn_model* m = new (std::nothrow) syn_model;
    if (!m) {
        cudaFree(mem);
        return fail(SYN_ERR_OOM, "host allocation failed");
    }
    memset(&m->dm, 0, sizeof m->dm);
    m->device = device;
    m->n_inputs = d->n_inputs;
    m->n_trees = d->forest_weight != 0.0 ? d->n_trees : 0;
    m->max_depth = max_depth;
    m->n_nodes = (long long)nodes.size();
    m->bytes = (long long)total;
    m->alloc = mem;
    m->dm.nodes = reinterpret_cast<const uint2*>(base);
    m->dm.trees = reinterpret_cast<const int2*>(base + off_t);
    m->dm.lin_w = reinterpret_cast<const double*>(base + off_l);
    m->dm.lin_b = d->linear_weight != 0.0 ? d->lin_b : 0.0;
    m->dm.lin_weight = d->linear_weight;
    m->dm.forest_weight = d->forest_weight;
    m->dm.n_trees = m->n_trees;
    m->dm.depth = max_depth;
    m->dm.blocks = reinterpret_cast<const uint4*>(base + off_b);
    m->dm.broot = reinterpret_cast<const int*>(base + off_r);
    m->dm.broot_lpt = reinterpret_cast<const int*>(base + off_lp);
    m->dm.tsplit = reinterpret_cast<const int2*>(base + off_ts);
    m->dm.units_split = units_split;
    m->n_blocks = (long long)(blocks.size() >> 1);
    m->dm.nblk = (int)m->n_blocks;
    m->dm.fx_ok = fx_ok;
    m->dm.fx32 = fx32;
    m->dm.fx_s = fx_s;
    m->dm.fx_scale = std::ldexp(1.0, fx_s);
    m->dm.fx_inv = std::ldexp(1.0, -fx_s);
    m->dm.svr_weight = d->svr_weight;
    m->dm.n_sv = (int)n_sv;
    if (has_svr) {
        m->dm.sv = reinterpret_cast<const float*>(base + off_sv);
        m->dm.dual = reinterpret_cast<const double*>(base + off_dc);
        m->dm.in_mean = reinterpret_cast<const double*>(base + off_mn);
        m->dm.in_scale = reinterpret_cast<const double*>(base + off_sc);
        m->dm.svr_gamma = d->svr_gamma;
        m->dm.svr_b = d->svr_intercept;
        double mx = 0.0;
        for (int j = 0; j < d->n_sv; ++j) mx = std::max(mx, std::fabs(d->dual_coef[j]));
        int e = 0;
        if (mx > 0.0) std::frexp(mx, &e);                  // mx in [2^(e-1), 2^e)
        m->dm.svr_eU = e;
    }
    m->dm.svr_p = nullptr;
    m->dm.svr_splits = 0;
    *out = m;
    return ok();
}

syn_status synergy_model_destroy(syn_model* m) {
    if (!m) return ok();
    {
        DeviceGuard g(m->device);
        cudaDeviceSynchronize();           // no queued work may still read the model's copies
        cudaFree(m->alloc);
        for (CutCopy& cb : m->cuts) {
            cudaFreeAsync(cb.p, nullptr);
            if (cb.ready) cudaEventDestroy(cb.ready);
        }
        cudaStreamSynchronize(nullptr);
        cudaGetLastError();
    }
    delete m;
    return ok();
}

syn_status synergy_model_info(const syn_model* m, int32_t* n_inputs, int32_t* n_trees, int64_t* n_nodes,
                              int32_t* max_depth, int64_t* device_bytes) {
    if (!m) return fail(SYN_ERR_INVALID_ARG, "model is NULL");
    if (n_inputs) *n_inputs = m->n_inputs;
    if (n_trees) *n_trees = m->n_trees;
    if (n_nodes) *n_nodes = m->n_nodes;
    if (max_depth) *max_depth = m->max_depth;
    if (device_bytes) *device_bytes = m->bytes;
    return ok();
}

syn_status synergy_clocks_create(const float* h, int32_t n_f, int32_t device, syn_clocks** out) {
    if (!out) return fail(SYN_ERR_INVALID_ARG, "out is NULL");
    *out = nullptr;
    if (!h) return fail(SYN_ERR_INVALID_ARG, "h_freqs is NULL");
    if (n_f < 1 || n_f > SYNERGY_MAX_FREQS) return fail(SYN_ERR_INVALID_ARG, "n_freqs=%d outside [1, %d]", n_f, SYNERGY_MAX_FREQS);
    for (int i = 0; i < n_f; ++i)
        if (!std::isfinite(h[i])) return fail(SYN_ERR_INVALID_ARG, "freqs[%d] is not finite", i);
    for (int i = 1; i < n_f; ++i)
        if (!(h[i - 1] < h[i])) return fail(SYN_ERR_INVALID_ARG, "freqs not strictly ascending at %d", i);
    DeviceGuard g(device);
    if (!g.okay) return fail(SYN_ERR_INVALID_ARG, "cannot select device %d", device);
    float* d = nullptr;
    cudaError_t e = cudaMalloc(&d, (size_t)n_f * sizeof(float));
    if (e != cudaSuccess) return cuda_fail(e, "cudaMalloc(clocks)");
    if ((e = cudaMemcpy(d, h, (size_t)n_f * sizeof(float), cudaMemcpyHostToDevice)) != cudaSuccess) {
        cudaFree(d);
        return cuda_fail(e, "cudaMemcpy(clocks)");
    }
    syn_clocks* c = new (std::nothrow) syn_clocks;
    if (!c) {
        cudaFree(d);
        return fail(SYN_ERR_OOM, "host allocation failed");
    }
    c->device = device;
    c->n_f = n_f;
    c->d_freqs = d;
    static std::atomic<long long> next_uid{1};
    c->uid = next_uid++;
    *out = c;
    return ok();
}

syn_status synergy_clocks_destroy(syn_clocks* c) {
    if (!c) return ok();
    {
        DeviceGuard g(c->device);
        cudaFree(c->d_freqs);
    }
    delete c;
    return ok();
}

syn_status synergy_clocks_info(const syn_clocks* c, int32_t* n_freqs) {
    if (!c) return fail(SYN_ERR_INVALID_ARG, "clocks is NULL");
    if (n_freqs) *n_freqs = c->n_f;
    return ok();
}

syn_status synergy_prepare(const syn_model* const* models, int32_t n_models, int64_t n_kernels, int32_t n_features,
                           const syn_clocks* clocks, syn_stream stream) {
    if (!models) return fail(SYN_ERR_INVALID_ARG, "models is NULL");
    if (n_models != 2 && n_models != 4) return fail(SYN_ERR_INVALID_ARG, "n_models=%d (2 or 4)", n_models);
    float* pred[4] = {nullptr, nullptr, nullptr, nullptr};
    return run_sweep(models, n_models, nullptr, n_kernels, n_features, clocks, 0, nullptr, 0, nullptr, pred,
                     kModeSweep, static_cast<cudaStream_t>(stream), true);
}

syn_status synergy_predict(const syn_model* sp, const syn_model* en, const float* d_features, int64_t n_k,
                           int32_t F, const syn_clocks* clocks, int32_t def, float* d_S, float* d_E,
                           syn_stream stream) {
    const syn_model* models[2] = {sp, en};
    float* pred[4] = {d_S, d_E, nullptr, nullptr};
    return run_sweep(models, 2, d_features, n_k, F, clocks, def, nullptr, 0, nullptr, pred, kModePredict,
                     static_cast<cudaStream_t>(stream));
}

syn_status synergy_sweep(const syn_model* sp, const syn_model* en, const float* d_features, int64_t n_k,
                         int32_t F, const syn_clocks* clocks, int32_t def, const syn_target* targets,
                         int32_t n_t, int32_t* d_choice, float* d_S, float* d_E, syn_stream stream) {
    const syn_model* models[2] = {sp, en};
    float* pred[4] = {d_S, d_E, nullptr, nullptr};
    return run_sweep(models, 2, d_features, n_k, F, clocks, def, targets, n_t, d_choice, pred, kModeSweep,
                     static_cast<cudaStream_t>(stream));
}

syn_status synergy_sweep4(const syn_model* const* models, const float* d_features, int64_t n_k, int32_t F,
                          const syn_clocks* clocks, int32_t def, const syn_target* targets, int32_t n_t,
                          int32_t* d_choice, float* d_pred, syn_stream stream) {
    if (!models) return fail(SYN_ERR_INVALID_ARG, "models is NULL");
    float* pred[4] = {nullptr, nullptr, nullptr, nullptr};
    if (d_pred && n_k > 0 && clocks) {
        const size_t plane = (size_t)n_k * clocks->n_f;
        pred[0] = d_pred;
        pred[1] = d_pred + plane;
        pred[2] = models[2] ? d_pred + 2 * plane : nullptr;
        pred[3] = models[3] ? d_pred + 3 * plane : nullptr;
    }
    return run_sweep(models, 4, d_features, n_k, F, clocks, def, targets, n_t, d_choice, pred, kModeSweep,
                     static_cast<cudaStream_t>(stream));
}

syn_status synergy_select(const float* d_S, const float* d_E, int64_t n_k, int32_t n_f, int32_t def,
                          const syn_target* targets, int32_t n_t, int32_t* d_choice, syn_stream stream) {
    if (n_k < 0) return fail(SYN_ERR_INVALID_ARG, "n_kernels=%lld < 0", (long long)n_k);
    if (n_f < 1 || n_f > SYNERGY_MAX_FREQS) return fail(SYN_ERR_INVALID_ARG, "n_freqs=%d outside [1, %d]", n_f, SYNERGY_MAX_FREQS);
    if (def < 0 || def >= n_f) return fail(SYN_ERR_INVALID_ARG, "default_idx=%d outside [0, %d)", def, n_f);
    syn_status s = check_targets(targets, n_t);
    if (s != SYN_OK) return s;
    if (n_k == 0) {
        g_last = {0, 0, 0, 0, 0};
        return ok();
    }
    if (!d_S || !d_E || !d_choice) return fail(SYN_ERR_INVALID_ARG, "device buffer is NULL");
    SelectArgs a;
    memset(&a, 0, sizeof a);
    a.S = d_S;
    a.E = d_E;
    a.n_k = n_k;
    a.n_f = n_f;
    a.def = def;
    a.n_t = n_t;
    for (int t = 0; t < n_t; ++t) {
        a.kind[t] = targets[t].kind;
        a.frac[t] = (double)targets[t].x / 100.0;   // the oracle's frac (oracle.c select)
    }
    a.choice = d_choice;
    int dev = 0;
    cudaGetDevice(&dev);
    DevState* ds = nullptr;
    if ((s = need_dev(dev, &ds)) != SYN_OK) return s;
    const int block = 256;
    const long long need = (n_k + 7) / 8;
    const long long grid = std::min<long long>(need, (long long)ds->sms * 8);
    {
        KernelTimer kt("k_select", static_cast<cudaStream_t>(stream));
        k_select<<<(unsigned)grid, block, 0, static_cast<cudaStream_t>(stream)>>>(a);
    }
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return cuda_fail(e, "k_select launch");
    g_last = {1, n_k * (long long)n_f, grid, block, 0};
    return ok();
}

syn_status synergy_pareto(const float* d_S, const float* d_E, int64_t n_k, int32_t n_f, uint8_t* d_front,
                          syn_stream stream) {
    if (n_k < 0) return fail(SYN_ERR_INVALID_ARG, "n_kernels=%lld < 0", (long long)n_k);
    if (n_f < 1 || n_f > SYNERGY_MAX_FREQS) return fail(SYN_ERR_INVALID_ARG, "n_freqs=%d outside [1, %d]", n_f, SYNERGY_MAX_FREQS);
    if (n_k == 0) return ok();
    if (!d_S || !d_E || !d_front) return fail(SYN_ERR_INVALID_ARG, "device buffer is NULL");
    int dev = 0;
    cudaGetDevice(&dev);
    DevState* ds = nullptr;
    syn_status s = need_dev(dev, &ds);
    if (s != SYN_OK) return s;
    const long long grid = std::min<long long>((n_k + 7) / 8, (long long)ds->sms * 8);
    {
        KernelTimer kt("k_pareto", static_cast<cudaStream_t>(stream));
        k_pareto<<<(unsigned)grid, 256, 0, static_cast<cudaStream_t>(stream)>>>(d_S, d_E, n_k, n_f, d_front);
    }
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return cuda_fail(e, "k_pareto launch");
    g_last = {1, n_k * (long long)n_f, grid, 256, 0};
    return ok();
}

syn_status synergy_choice_error(const float* d_S, const float* d_E, int64_t n_k, int32_t n_f, int32_t def,
                                const syn_target* targets, int32_t n_t, const int32_t* d_pred, double* d_err,
                                double* d_summary, syn_stream stream) {
    if (n_k < 0) return fail(SYN_ERR_INVALID_ARG, "n_kernels=%lld < 0", (long long)n_k);
    if (n_f < 1 || n_f > SYNERGY_MAX_FREQS) return fail(SYN_ERR_INVALID_ARG, "n_freqs=%d outside [1, %d]", n_f, SYNERGY_MAX_FREQS);
    if (def < 0 || def >= n_f) return fail(SYN_ERR_INVALID_ARG, "default_idx=%d outside [0, %d)", def, n_f);
    syn_status vs = check_targets(targets, n_t);
    if (vs != SYN_OK) return vs;
    if (!d_summary) return fail(SYN_ERR_INVALID_ARG, "d_summary is NULL");
    if (n_k > 0 && (!d_S || !d_E || !d_pred || !d_err)) return fail(SYN_ERR_INVALID_ARG, "device buffer is NULL");
    SelectArgs a;
    memset(&a, 0, sizeof a);
    a.S = d_S;
    a.E = d_E;
    a.n_k = n_k;
    a.n_f = n_f;
    a.def = def;
    a.n_t = n_t;
    for (int t = 0; t < n_t; ++t) {
        a.kind[t] = targets[t].kind;
        a.frac[t] = (double)targets[t].x / 100.0;   // the oracle's frac (oracle.c select)
    }
    int dev = 0;
    cudaGetDevice(&dev);
    DevState* ds = nullptr;
    if ((vs = need_dev(dev, &ds)) != SYN_OK) return vs;
    cudaStream_t st = static_cast<cudaStream_t>(stream);
    if (n_k > 0) {
        const long long grid = std::min<long long>((n_k + 7) / 8, (long long)ds->sms * 8);
        KernelTimer kt("k_choice_error", st);
        k_choice_error<<<(unsigned)grid, 256, 0, st>>>(a, d_pred, d_err);
    }
    {
        KernelTimer kt("k_error_reduce", st);
        k_error_reduce<<<n_t, 256, 0, st>>>(d_err, n_k, n_t, d_summary);
    }
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return cuda_fail(e, "k_choice_error launch");
    g_last = {n_k > 0 ? 2 : 1, n_k * (long long)n_f, 0, 256, 0};
    return ok();
}

syn_status synergy_plan(const int32_t* d_choice, int64_t n_k, int32_t n_t, const syn_clocks* clocks, float* d_mhz,
                        syn_stream stream) {
    if (!clocks) return fail(SYN_ERR_INVALID_ARG, "clocks is NULL");
    if (n_k < 0) return fail(SYN_ERR_INVALID_ARG, "n_kernels=%lld < 0", (long long)n_k);
    if (n_t < 1 || n_t > SYNERGY_MAX_TARGETS) return fail(SYN_ERR_INVALID_ARG, "n_targets=%d outside [1, %d]", n_t, SYNERGY_MAX_TARGETS);
    if (!current_device_is(clocks->device)) return fail(SYN_ERR_INVALID_ARG, "clocks device differs from the current device");
    if (n_k == 0) return ok();
    if (!d_choice || !d_mhz) return fail(SYN_ERR_INVALID_ARG, "device buffer is NULL");
    DevState* ds = nullptr;
    syn_status s = need_dev(clocks->device, &ds);
    if (s != SYN_OK) return s;
    const long long n = n_k * (long long)n_t;
    const long long grid = std::min<long long>((n + 255) / 256, (long long)ds->sms * 16);
    {
        KernelTimer kt("k_plan", static_cast<cudaStream_t>(stream));
        k_plan<<<(unsigned)grid, 256, 0, static_cast<cudaStream_t>(stream)>>>(d_choice, n, clocks->d_freqs, clocks->n_f, d_mhz);
    }
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return cuda_fail(e, "k_plan launch");
    g_last = {1, n, grid, 256, 0};
    return ok();
}

syn_status synergy_workspace_create(int32_t device, syn_workspace** out) {
    if (!out) return fail(SYN_ERR_INVALID_ARG, "out is NULL");
    syn_workspace* w = new (std::nothrow) syn_workspace;
    if (!w) return fail(SYN_ERR_OOM, "host allocation failed");
    w->device = device;
    w->d_features = nullptr;
    w->cap_features = 0;
    w->d_choice = nullptr;
    w->cap_choice = 0;
    *out = w;
    return ok();
}

syn_status synergy_workspace_destroy(syn_workspace* w) {
    if (!w) return ok();
    {
        DeviceGuard g(w->device);
        cudaFree(w->d_features);
        cudaFree(w->d_choice);
    }
    delete w;
    return ok();
}

syn_status synergy_sweep_host(syn_workspace* w, const syn_model* sp, const syn_model* en, const float* h_features,
                              int64_t n_k, int32_t F, const syn_clocks* clocks, int32_t def,
                              const syn_target* targets, int32_t n_t, int32_t* h_choice, syn_stream stream) {
    if (!w) return fail(SYN_ERR_INVALID_ARG, "workspace is NULL");
    if (!clocks || !current_device_is(w->device) || clocks->device != w->device)
        return fail(SYN_ERR_INVALID_ARG, "workspace/clocks device differs from the current device");
    if (n_k > 0 && (!h_features || !h_choice)) return fail(SYN_ERR_INVALID_ARG, "host buffer is NULL");
    const syn_model* models[2] = {sp, en};
    syn_status vs = validate_models(models, 2, F, clocks);
    if (vs != SYN_OK) return vs;
    if (n_k < 0) return fail(SYN_ERR_INVALID_ARG, "n_kernels=%lld < 0", (long long)n_k);
    const int n_f = clocks->n_f;
    if (def < 0 || def >= n_f) return fail(SYN_ERR_INVALID_ARG, "default_idx=%d outside [0, %d)", def, n_f);
    if ((vs = check_targets(targets, n_t)) != SYN_OK) return vs;
    const size_t fb = (size_t)n_k * (size_t)F * sizeof(float);
    const size_t cb = (size_t)n_k * (size_t)n_t * sizeof(int32_t);
    cudaStream_t st = static_cast<cudaStream_t>(stream);
    cudaError_t e;
    if (fb > w->cap_features) {
        cudaFree(w->d_features);
        w->d_features = nullptr;
        w->cap_features = 0;
        if ((e = cudaMalloc(&w->d_features, fb)) != cudaSuccess) return cuda_fail(e, "cudaMalloc(workspace)");
        w->cap_features = fb;
    }
    if (cb > w->cap_choice) {
        cudaFree(w->d_choice);
        w->d_choice = nullptr;
        w->cap_choice = 0;
        if ((e = cudaMalloc(&w->d_choice, cb)) != cudaSuccess) return cuda_fail(e, "cudaMalloc(workspace)");
        w->cap_choice = cb;
    }
    if (n_k > 0 && (e = cudaMemcpyAsync(w->d_features, h_features, fb, cudaMemcpyHostToDevice, st)) != cudaSuccess)
        return cuda_fail(e, "cudaMemcpyAsync H2D");
    float* pred[4] = {nullptr, nullptr, nullptr, nullptr};
    syn_status s = run_sweep(models, 2, w->d_features, n_k, F, clocks, def, targets, n_t, w->d_choice, pred,
                             kModeSweep, st);
    if (s != SYN_OK) return s;
    if (n_k > 0 && (e = cudaMemcpyAsync(h_choice, w->d_choice, cb, cudaMemcpyDeviceToHost, st)) != cudaSuccess)
        return cuda_fail(e, "cudaMemcpyAsync D2H");
    return ok();
}

syn_status synergy_timing_enable(int32_t on) {
    std::lock_guard<std::mutex> lock(g_tmu);
    g_timing = on != 0;
    return ok();
}

syn_status synergy_timing_read(int32_t cap, const char** names, double* total_ms, double* busy_ms,
                               int64_t* launches, int32_t* n_kernels) {
    if (cap < 0 || (cap > 0 && (!names || !total_ms || !launches)) || !n_kernels)
        return fail(SYN_ERR_INVALID_ARG, "bad timing_read buffers");
    std::lock_guard<std::mutex> lock(g_tmu);
    std::vector<const char*> nm;
    std::vector<double> ms;
    std::vector<int64_t> cnt;
    std::vector<std::vector<std::pair<double, double>>> iv;       // per kernel: launch intervals
    syn_status st = SYN_OK;
    const cudaEvent_t ref = g_tl.empty() ? nullptr : g_tl.front().a;
    double far = 0.0;                                            // incomparable launches (see below)
    for (const TimedLaunch& t : g_tl) {
        float x = 0.0f, xa = 0.0f, xb = 0.0f;
        cudaError_t e = cudaEventSynchronize(t.b);
        if (e == cudaSuccess) e = cudaEventSynchronize(t.a);
        if (e == cudaSuccess) e = cudaEventElapsedTime(&x, t.a, t.b);
        if (e != cudaSuccess && st == SYN_OK) st = cuda_fail(e, "timing events");
        // on a common time axis (the first event's); events of another device cannot be compared:
        // such a launch counts as an interval of its own, placed after everything else
        double ia, ib;
        if (cudaEventElapsedTime(&xa, ref, t.a) == cudaSuccess && cudaEventElapsedTime(&xb, ref, t.b) == cudaSuccess) {
            ia = xa;
            ib = xb;
        } else {
            cudaGetLastError();
            ia = 1e9 + far;
            ib = ia + x;
            far += (double)x + 1.0;
        }
        size_t k = 0;
        while (k < nm.size() && strcmp(nm[k], t.name)) ++k;
        if (k == nm.size()) { nm.push_back(t.name); ms.push_back(0.0); cnt.push_back(0); iv.emplace_back(); }
        ms[k] += x;
        cnt[k] += 1;
        iv[k].push_back({ia, ib});
    }
    for (const TimedLaunch& t : g_tl) {
        g_evpool.push_back(t.a);
        g_evpool.push_back(t.b);
    }
    g_tl.clear();
    *n_kernels = (int32_t)nm.size();
    for (int32_t k = 0; k < (int32_t)nm.size() && k < cap; ++k) {
        names[k] = nm[k];
        total_ms[k] = ms[k];
        launches[k] = cnt[k];
        if (busy_ms) {                                          // union of the launch intervals
            std::sort(iv[k].begin(), iv[k].end());
            double busy = 0.0, a0 = 0.0, b0 = 0.0;
            bool open = false;
            for (const auto& q : iv[k]) {
                if (open && q.first <= b0) {
                    b0 = std::max(b0, q.second);
                } else {
                    if (open) busy += b0 - a0;
                    a0 = q.first;
                    b0 = q.second;
                    open = true;
                }
            }
            if (open) busy += b0 - a0;
            busy_ms[k] = busy;
        }
    }
    return st == SYN_OK ? ok() : st;
}

syn_status synergy_last_launch(int32_t* kernels, int64_t* evals, int64_t* grid, int32_t* block, int32_t* variant) {
    if (kernels) *kernels = g_last.kernels;
    if (evals) *evals = g_last.evals;
    if (grid) *grid = g_last.grid;
    if (block) *block = g_last.block;
    if (variant) *variant = g_last.variant;
    return ok();
}

}  // extern "C"
