// synergy.cu — C-ABI implementation (include/synergy.h): validation, model packing, launch
// configuration and the host-buffer end-to-end path.  All compute runs in kernels.cuh.
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
#include "kernels_iv.cuh"
#include "kernels_ws.cuh"
#include "kernels_da.cuh"
#include "kernels_svr.cuh"
#include "kernels_tm.cuh"
#include "kernels_tr.cuh"
#include "synergy.h"

using namespace syn;

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
    std::vector<std::pair<long long, uint4*>> cut_blocks;  // per clock table (uid): k_cut_blocks copy
    std::vector<std::pair<long long, uint4*>> tr_blocks;   // per clock table (uid): k_tr_layout copy
    long long max_tree_blocks;                            // blocks of the largest tree
};

struct syn_clocks {
    int device;
    int n_f;
    float* d_freqs;
    unsigned short* d_grid;   // clock-cut hint table, kGrid + 1 entries
    float f0, inv_step;
    long long uid;            // unique per created table (keys the models' clock-cut block copies)
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

int sm_count(int dev) {
    static int cached[64] = {0};
    if (dev < 0 || dev >= 64) return 148;
    if (!cached[dev]) {
        int v = 0;
        if (cudaDeviceGetAttribute(&v, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess || v <= 0) v = 148;
        cached[dev] = v;
    }
    return cached[dev];
}

syn_status check_targets(const syn_target* t, int32_t n_t) {
    if (n_t < 1 || n_t > SYNERGY_MAX_TARGETS) return fail(SYN_ERR_INVALID_ARG, "n_targets=%d outside [1, %d]", n_t, SYNERGY_MAX_TARGETS);
    if (!t) return fail(SYN_ERR_INVALID_ARG, "h_targets is NULL");
    for (int i = 0; i < n_t; ++i) {
        if (t[i].kind < SYN_MAX_PERF || t[i].kind > SYN_PL) return fail(SYN_ERR_INVALID_ARG, "target %d: unknown kind %d", i, t[i].kind);
        if ((t[i].kind == SYN_ES || t[i].kind == SYN_PL) && !(t[i].x >= 0.0f && t[i].x <= 100.0f))
            return fail(SYN_ERR_INVALID_ARG, "target %d: x=%g outside [0, 100]", i, (double)t[i].x);
    }
    return SYN_OK;
}

// ---------------------------------------------------------------- launch configuration

struct Config {
    int algo;                 // 0 = direct traversal (k_sweep), 1 = clock-interval (k_sweep_iv)
    int slots, tilp, tile_k, nt, xs;
    int tc, words, vcap, vs, region;
    int win, slot_bytes, head_bytes;
    size_t smem;
};

int env_int(const char* name, int dflt) {
    const char* v = getenv(name);
    return (v && *v) ? atoi(v) : dflt;
}

size_t sweep_smem(int tile_k, int n_f, int xs) {
    return (size_t)tile_k * ((size_t)n_f * 24 + (size_t)xs * 4) + (size_t)n_f * 4;
}

// Choose per-thread slots (units in flight) and trees-in-flight so that the grid keeps every
// SM busy for small batches (slots=1, 4 trees in flight) and amortises staging for large ones.
Config choose_config(long long n_k, int n_f, int F, int dev) {
    Config c;
    c.algo = 0;
    c.tc = c.words = c.vcap = c.vs = c.region = 0;
    c.win = c.slot_bytes = c.head_bytes = 0;
    const long long resident = (long long)sm_count(dev) * 2048;
    const long long evals = n_k * (long long)n_f;
    c.slots = evals >= 16 * resident ? 8 : evals >= 8 * resident ? 4 : evals >= 4 * resident ? 2 : 1;
    c.tilp = c.slots <= 2 ? 4 : c.slots == 4 ? 2 : 1;
    c.xs = (F + 2) | 1;   // odd stride: rows of different kernels land in different banks
    long long tk = std::max(1, (256 * c.slots) / n_f);
    tk = std::min<long long>(tk, std::max<long long>(n_k, 1));
    while (tk > 1 && sweep_smem((int)tk, n_f, c.xs) > 200 * 1024) --tk;
    c.tile_k = (int)tk;
    long long thr = (c.tile_k * (long long)n_f + c.slots - 1) / c.slots;
    thr = (thr + 31) / 32 * 32;
    c.nt = (int)std::min<long long>(std::max<long long>(thr, 32), 512);
    c.smem = sweep_smem(c.tile_k, n_f, c.xs);
    return c;
}

// Clock-interval kernel: NT threads, TK kernels per CTA, TC = NT / TK trees per chunk (one
// (kernel, tree) task per thread), accumulators for the TK x n_f units in shared memory.
// Small batches use TK = 1 so the grid spans the SMs; large ones TK = 4 so a chunk's trees are
// shared by more kernels (L1 reuse of the upper levels).
size_t iv_smem(int nt, int tk, int n_f, int xs, int words, int vs, int* region) {
    const int tc = std::max(1, nt / tk);
    size_t tasks = (size_t)tc * tk * ((size_t)words * 8 + (size_t)vs * 8);
    tasks = std::max(tasks, (size_t)tk * n_f * 8);            // finish-phase float scratch
    tasks = (tasks + 15) & ~(size_t)15;
    *region = (int)tasks;
    return (size_t)tk * n_f * 16 + tasks + (size_t)n_f * 4 + (size_t)tk * xs * 4 + (kGrid + 1) * 2 + 16;
}

bool choose_iv(long long n_k, int n_f, int F, int dev, Config& c) {
    if (n_f > 1024) return false;
    const int sms = sm_count(dev);
    c.nt = env_int("SYNERGY_NT", 128) >= 256 ? 256 : 128;
    int tk = (int)std::min<long long>(4, std::max<long long>(1, n_k / (8LL * sms)));
    tk = env_int("SYNERGY_TK", tk);
    tk = (int)std::max<long long>(1, std::min<long long>(std::min(tk, c.nt), std::max<long long>(n_k, 1)));
    c.algo = 1;
    c.slots = 0;
    c.tilp = 0;
    c.tile_k = tk;
    c.xs = (F + 2) | 1;
    c.tc = std::max(1, c.nt / tk);
    c.words = (n_f + 31) / 32;
    c.vcap = std::max(1, env_int("SYNERGY_VCAP", 24));
    c.vs = c.vcap | 1;
    c.smem = iv_smem(c.nt, tk, n_f, c.xs, c.words, c.vs, &c.region);
    return c.smem <= 220 * 1024;
}

template <int NT, int MINB>
cudaError_t launch_iv_t(const SweepArgs& a, const Config& c, long long grid, cudaStream_t st) {
    static size_t smem_set = 48 * 1024;
    if (c.smem > smem_set) {
        cudaError_t e = cudaFuncSetAttribute(k_sweep_iv<NT, MINB>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)c.smem);
        if (e != cudaSuccess) return e;
        smem_set = c.smem;
    }
    k_sweep_iv<NT, MINB><<<(unsigned)grid, NT, c.smem, st>>>(a);
    return cudaGetLastError();
}

cudaError_t launch_iv(const SweepArgs& a, const Config& c, long long grid, cudaStream_t st) {
    return c.nt == 256 ? launch_iv_t<256, 4>(a, c, grid, st) : launch_iv_t<128, 8>(a, c, grid, st);
}

// Warp-streaming kernel: KPC kernels per CTA, one warp per (kernel, model), WIN-slot ring
// window of finished trees per warp, accumulators in registers (n_f <= 256).
bool choose_ws(long long n_k, int n_f, int F, int dev, Config& c) {
    if (n_f > 256) return false;
    int kpc = env_int("SYNERGY_KPC", 2);
    kpc = std::max(1, std::min(kpc, 4));
    kpc = (int)std::min<long long>(kpc, std::max<long long>(n_k, 1));
    c.algo = 2;
    c.slots = 0;
    c.tilp = 0;
    c.tile_k = kpc;
    c.nt = 64 * kpc;
    c.xs = (F + 2) | 1;
    c.words = (n_f + 31) / 32;
    c.vcap = std::max(1, env_int("SYNERGY_VCAP", 32));
    c.vs = c.vcap;
    int win = std::max(32, std::min(1024, env_int("SYNERGY_WIN", 64)));
    c.win = 32;
    while (c.win * 2 <= win) c.win *= 2;                 // power of two: slot = tree & (WIN-1)
    int sb = c.vs * 4 + c.words * 4 + 8;
    c.slot_bytes = (sb + 7) & ~7;
    c.head_bytes = (int)((((size_t)(n_f + kpc * c.xs) * 4 + (kGrid + 1) * 2) + 15) & ~(size_t)15);
    const size_t slots = (size_t)2 * kpc * c.win * c.slot_bytes;
    const size_t fin = (size_t)kpc * n_f * 24;
    c.smem = c.head_bytes + std::max(slots, fin);
    c.tc = c.region = 0;
    return c.smem <= 220 * 1024;
}

template <int CL>
cudaError_t launch_ws_t(const SweepArgs& a, const Config& c, long long grid, cudaStream_t st) {
    static size_t smem_set = 48 * 1024;
    if (c.smem > smem_set) {
        cudaError_t e = cudaFuncSetAttribute(k_sweep_ws<CL>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)c.smem);
        if (e != cudaSuccess) return e;
        smem_set = c.smem;
    }
    k_sweep_ws<CL><<<(unsigned)grid, c.nt, c.smem, st>>>(a);
    return cudaGetLastError();
}

cudaError_t launch_ws(const SweepArgs& a, const Config& c, long long grid, cudaStream_t st) {
    if (c.words <= 2) return launch_ws_t<2>(a, c, grid, st);
    if (c.words <= 4) return launch_ws_t<4>(a, c, grid, st);
    return launch_ws_t<8>(a, c, grid, st);
}

// Difference-array kernel: KPC kernels per CTA, exact int64 leaf sums (needs fx_ok forests).
// KPC grows when a kernel has fewer trees than the CTA has threads, so lanes keep walking and
// the per-CTA staging / finish is amortised.
size_t da_head(int nt, int kpc, int n_f, int xs, int nm) {
    const size_t h = (size_t)kpc * nm * (n_f + 1) * 8 + (size_t)nt * kpc * nm * 8 + (size_t)nm * kpc * n_f * 12 +
                     (size_t)n_f * 4 + (size_t)kpc * xs * 4 + (size_t)(kGrid + 2) * 2 + 16;
    return (h + 15) & ~(size_t)15;
}

// The per-thread top-block cache (TOPC) is only allocated when enabled: shared memory comes out of
// the same 256 KB as L1, and this kernel lives on L1 hits of the upper tree blocks.
bool da_topc() { return env_int("SYNERGY_TOPC", 0) != 0; }

size_t da_smem(int nt, int kpc, int n_f, int xs, int nm) {
    return da_head(nt, kpc, n_f, xs, nm) + (da_topc() ? (size_t)nt * 160 : 0);
}

bool choose_da(const syn_model* sp, const syn_model* en, long long n_k, int n_f, int F, Config& c,
               const syn_model* x2 = nullptr, const syn_model* x3 = nullptr) {
    if (n_f > 2048) return false;
    if ((sp->n_trees && !sp->dm.fx_ok) || (en->n_trees && !en->dm.fx_ok)) return false;
    if ((x2 && x2->n_trees && !x2->dm.fx_ok) || (x3 && x3->n_trees && !x3->dm.fx_ok)) return false;
    const int nm = (x2 || x3) ? 4 : 2;
    const int tt = std::max(1, sp->n_trees + en->n_trees + (x2 ? x2->n_trees : 0) + (x3 ? x3->n_trees : 0));
    int nt = env_int("SYNERGY_NT", 128);
    nt = nt >= 256 ? 256 : (nt >= 128 ? 128 : 64);
    int kpc = tt >= nt ? 1 : (3 * nt + 2 * tt - 1) / (2 * tt);      // ~1.5 tasks per thread
    kpc = (int)std::min<long long>(kpc, std::max<long long>(1, n_k / (2LL * sm_count(0))));   // fill the SMs
    kpc = env_int("SYNERGY_KPC", kpc);
    kpc = (int)std::max<long long>(1, std::min<long long>(std::min(kpc, 16), std::max<long long>(n_k, 1)));
    c.algo = 3;
    c.tilp = 0;
    c.tile_k = kpc;
    c.nt = nt;
    c.xs = (F + 2) | 1;
    c.tc = c.words = c.vcap = c.vs = c.region = 0;
    c.win = c.slot_bytes = c.head_bytes = 0;
    // small batches: split each (kernel, tree) task into R clock sub-ranges so that there are at
    // least ~4 tasks per resident lane (R = 1 for large batches: every split costs an extra walk)
    const long long lanes = (long long)sm_count(0) * 1024, tasks = std::max<long long>(1, n_k * tt);
    int nsub = (int)std::min<long long>(2, std::max<long long>(1, (4 * lanes + tasks - 1) / tasks));
    nsub = std::max(1, std::min(env_int("SYNERGY_NSUB", nsub), std::max(1, n_f)));
    c.slots = nsub;                                        // carried to SweepArgs.nsub
    c.smem = da_smem(nt, kpc, n_f, c.xs, nm);
    while (c.smem > 200 * 1024 && c.tile_k > 1) c.smem = da_smem(nt, --c.tile_k, n_f, c.xs, nm);
    c.head_bytes = (int)da_head(nt, c.tile_k, n_f, c.xs, nm);
    return c.smem <= 200 * 1024;
}

template <int NT, bool TOPC>
cudaError_t launch_da_t(const SweepArgs& a, const Config& c, long long grid, cudaStream_t st) {
    static size_t smem_set = 48 * 1024;
    if (c.smem > smem_set) {
        cudaError_t e = cudaFuncSetAttribute(k_sweep_da<NT, TOPC>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)c.smem);
        if (e != cudaSuccess) return e;
        smem_set = c.smem;
    }
    k_sweep_da<NT, TOPC><<<(unsigned)grid, NT, c.smem, st>>>(a);
    return cudaGetLastError();
}

cudaError_t launch_da(const SweepArgs& a, const Config& c, long long grid, cudaStream_t st) {
    const bool topc = da_topc();
    if (c.nt == 256) return topc ? launch_da_t<256, true>(a, c, grid, st) : launch_da_t<256, false>(a, c, grid, st);
    if (c.nt == 128) return topc ? launch_da_t<128, true>(a, c, grid, st) : launch_da_t<128, false>(a, c, grid, st);
    return topc ? launch_da_t<64, true>(a, c, grid, st) : launch_da_t<64, false>(a, c, grid, st);
}

// ------------------------------------------------------------------ tree-major path (kernels_tm.cuh)
// D difference arrays live in a library-owned buffer per (device, stream).  k_tm_finish zeroes
// every entry it reads, so a buffer is all-zero between calls on its stream; a call that fails
// after enqueuing k_tm_walk marks it dirty and the next call clears it with a memset.
struct TmBuf {
    int dev;
    cudaStream_t st;
    int kind;                        // 0/2: D and its second slab buffer (all-zero between calls), 1: k_tr_walk features
    long long* p;
    size_t bytes;
    bool dirty;
};
std::mutex g_tm_mu;
std::list<TmBuf> g_tm_bufs;          // list: entries never move

syn_status tm_buffer(int dev, cudaStream_t st, size_t bytes, TmBuf** out, int kind = 0) {
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
        if (b->p) {
            cudaStreamSynchronize(st);          // the old buffer may still be read by queued work
            cudaFree(b->p);
            b->p = nullptr;
            b->bytes = 0;
        }
        if ((e = cudaMalloc(&b->p, bytes)) != cudaSuccess) {
            cudaGetLastError();
            b->p = nullptr;
            return e == cudaErrorMemoryAllocation ? fail(SYN_ERR_OOM, "tree-major D buffer of %zu bytes", bytes)
                                                  : cuda_fail(e, "cudaMalloc(D)");
        }
        b->bytes = bytes;
        b->dirty = true;
    }
    if (b->dirty && kind != 1) {
        if ((e = cudaMemsetAsync(b->p, 0, b->bytes, st)) != cudaSuccess) return cuda_fail(e, "cudaMemsetAsync(D)");
        b->dirty = false;
    }
    *out = b;
    return ok();
}

// Slab pipeline (several kernel slabs per call): the finish of slab i runs on a library-owned
// second stream while the walk of slab i + 1 runs on the caller's stream, with D double-buffered.
// One side stream and three events per (device, caller stream).
struct TmAux {
    int dev;
    cudaStream_t st;
    cudaStream_t st2;
    cudaEvent_t walked[2], finished[2];
};
std::list<TmAux> g_tm_aux;

syn_status tm_aux(int dev, cudaStream_t st, TmAux** out) {
    std::lock_guard<std::mutex> lock(g_tm_mu);
    for (TmAux& x : g_tm_aux)
        if (x.dev == dev && x.st == st) {
            *out = &x;
            return ok();
        }
    TmAux x;
    x.dev = dev;
    x.st = st;
    cudaError_t e = cudaStreamCreateWithFlags(&x.st2, cudaStreamNonBlocking);
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
// first use and cached in the model.  The build is synchronous (once per model and table) so any
// stream may use the copy afterwards.
std::mutex g_cut_mu;
syn_status cut_blocks(syn_model* m, const syn_clocks* c, const uint4** out) {
    std::lock_guard<std::mutex> lock(g_cut_mu);
    for (auto& cb : m->cut_blocks)
        if (cb.first == c->uid) {
            *out = cb.second;
            return ok();
        }
    uint4* p = nullptr;
    const long long nb = std::max<long long>(m->n_blocks, 1);
    cudaError_t e = cudaMalloc(&p, (size_t)nb * 2 * sizeof(uint4));
    if (e != cudaSuccess) {
        cudaGetLastError();
        return cuda_fail(e, "cudaMalloc(clock-cut blocks)");
    }
    if (m->n_blocks > 0)
        k_cut_blocks<<<(unsigned)((m->n_blocks + 255) / 256), 256>>>(m->dm.blocks, m->n_blocks, m->n_inputs - 1,
                                                                   c->d_freqs, c->n_f, m->dm.fx32 ? m->dm.fx_scale : 0.0, p);
    if ((e = cudaGetLastError()) != cudaSuccess || (e = cudaDeviceSynchronize()) != cudaSuccess) {
        cudaFree(p);
        return cuda_fail(e, "k_cut_blocks");
    }
    m->cut_blocks.push_back({c->uid, p});
    *out = p;
    return ok();
}

// Tree-resident copy (kernels_tr.cuh, k_tr_layout) of a model's clock-cut blocks, cached like them.
syn_status tr_blocks(syn_model* m, const syn_clocks* c, const uint4* cut, const uint4** out) {
    std::lock_guard<std::mutex> lock(g_cut_mu);
    for (auto& cb : m->tr_blocks)
        if (cb.first == c->uid) {
            *out = cb.second;
            return ok();
        }
    uint4* p = nullptr;
    const long long nb = std::max<long long>(m->n_blocks, 1);
    cudaError_t e = cudaMalloc(&p, (size_t)nb * 2 * sizeof(uint4));
    if (e != cudaSuccess) {
        cudaGetLastError();
        return cuda_fail(e, "cudaMalloc(tree-resident blocks)");
    }
    if (m->n_trees > 0)
        k_tr_layout<<<(unsigned)m->n_trees, 256>>>(cut, m->dm.broot, m->n_trees, m->n_blocks, p);
    if ((e = cudaGetLastError()) != cudaSuccess || (e = cudaDeviceSynchronize()) != cudaSuccess) {
        cudaFree(p);
        return cuda_fail(e, "k_tr_layout");
    }
    m->tr_blocks.push_back({c->uid, p});
    *out = p;
    return ok();
}

constexpr size_t kTmSlabBytes = 48u << 20;
constexpr size_t kTrTreeMax = 64u << 10;     // largest tree (bytes of 2-level blocks) k_tr_walk stages   // D bytes per slab (stays L2-resident with the model)

// Tree-major path (k_tm_walk + k_tm_finish per kernel slab).  Needs every forest within the exact
// int64 leaf range (fx_ok) and at least one tree; returns false (nothing enqueued) otherwise.
bool tm_eligible(const SweepArgs& a, int nm) {
    int tt = 0;
    for (int m = 0; m < nm; ++m) {
        if (m >= 2 && !a.has_x[m - 2]) continue;
        const DevModel& d = m == 0 ? a.ms : m == 1 ? a.me : a.mx[m - 2];
        if (d.forest_weight == 0.0 || d.n_trees == 0) continue;
        if (!d.fx_ok) return false;
        tt += d.n_trees;
    }
    return tt > 0;
}

syn_status run_tm(SweepArgs a, int nm, syn_model* const* models, const syn_clocks* clocks, cudaStream_t st,
                  int* launches, int* variant) {
    const int device = clocks->device;
    DevModel* dms[4] = {&a.ms, &a.me, &a.mx[0], &a.mx[1]};
    // k_tm_walk (trees read through L1) by default; SYNERGY_TM_MODE=tr selects the tree-resident
    // k_tr_walk when every tree fits its shared tree buffer (measured slower on the bench
    // forests: with two 44-KB tree buffers per SM the lanes wait for stragglers)
    const char* mode_env = getenv("SYNERGY_TM_MODE");
    bool use_tr = mode_env && !strcmp(mode_env, "tr");
    long long max_tb = 1;
    for (int m = 0; m < nm; ++m)
        if (models[m] && dms[m]->forest_weight != 0.0 && dms[m]->n_trees > 0)
            max_tb = std::max(max_tb, models[m]->max_tree_blocks);
    if ((size_t)max_tb * 32 > kTrTreeMax) use_tr = false;
    for (int m = 0; m < nm; ++m)                  // k_tr_walk decodes int32 fixed-point leaves only
        if (models[m] && dms[m]->forest_weight != 0.0 && dms[m]->n_trees > 0 && !dms[m]->fx32) use_tr = false;
    TrArgs r;
    memset(&r, 0, sizeof r);
    for (int m = 0; m < nm; ++m) {
        if (!models[m] || dms[m]->forest_weight == 0.0 || dms[m]->n_trees == 0) continue;
        const uint4* cb = nullptr;
        syn_status cs = cut_blocks(models[m], clocks, &cb);
        if (cs != SYN_OK) return cs;
        dms[m]->blocks = cb;
        if (use_tr && (cs = tr_blocks(models[m], clocks, cb, &r.trb[m])) != SYN_OK) return cs;
    }
    TmArgs t;
    memset(&t, 0, sizeof t);
    const int n_f = a.n_f, F = a.F;
    const long long n_k = a.n_k;
    int tt = 0;
    t.nslot = 0;
    for (int m = 0; m < 4; ++m) {
        t.slot_of[m] = -1;
        if (m >= nm || (m >= 2 && !a.has_x[m - 2])) continue;
        const DevModel& d = m == 0 ? a.ms : m == 1 ? a.me : a.mx[m - 2];
        if (d.forest_weight == 0.0 || d.n_trees == 0) continue;
        t.slot_of[m] = t.nslot++;
        tt += d.n_trees;
    }
    t.nm = nm;
    bool fxall = true;                            // every forest has int32 fixed-point leaves
    for (int m = 0; m < nm; ++m)
        if (t.slot_of[m] >= 0 && !dms[m]->fx32) fxall = false;
    // kernels per feature block: a power of two in [32, 256], F * kb floats of shared memory
    int kb = 256;
    while (kb > 32 && ((size_t)F * kb * 4 > 32768 || kb / 2 >= n_k)) kb /= 2;
    const int kb_env = env_int("SYNERGY_TM_KB", kb);
    while (kb > 32 && kb > kb_env) kb /= 2;
    while (kb < 256 && kb * 2 <= kb_env) kb *= 2;
    t.kb = kb;
    t.kb_log2 = 0;
    while ((1 << t.kb_log2) < kb) ++t.kb_log2;
    const size_t row = (size_t)t.nslot * n_f * sizeof(long long);
    // kernels per slab: a multiple of the feature block, D of one slab <= kTmSlabBytes (L2-resident)
    long long nks = std::max<long long>(kb, (long long)(kTmSlabBytes / row) / kb * kb);
    const int slab_env = env_int("SYNERGY_TM_SLAB", 0);
    if (slab_env > 0) nks = std::max<long long>(kb, slab_env / kb * kb);
    nks = std::min<long long>(nks, n_k);
    // k_tr_walk chunk size P (kernels per unit): 1024, halved down to 512 while that leaves fewer
    // than 4 units per SM; the slab's transposed features ride in the same scratch as D
    const int sms_tr = sm_count(device);
    int P = 1024;
    while (P > 512 && (long long)tt * ((std::min<long long>(nks, n_k) + P - 1) / P) < 4LL * sms_tr) P /= 2;
    const int p_env = env_int("SYNERGY_TR_P", P);
    if (p_env >= 32 && p_env <= 2048 && p_env % 32 == 0) P = p_env;
    TmBuf* buf = nullptr;
    syn_status s = tm_buffer(device, st, (size_t)nks * row, &buf);
    if (s != SYN_OK) return s;
    t.D = buf->p;
    // several slabs: finish(i) on a side stream overlaps walk(i + 1); D alternates between two
    // buffers and walk(i + 2) waits for finish(i), which zeroes its buffer
    const bool pipe = n_k > nks && env_int("SYNERGY_TM_PIPE", 1) != 0;
    TmBuf* buf2 = nullptr;
    TmAux* aux = nullptr;
    if (pipe) {
        if ((s = tm_buffer(device, st, (size_t)nks * row, &buf2, 2)) != SYN_OK) return s;
        if ((s = tm_aux(device, st, &aux)) != SYN_OK) return s;
    }
    if (use_tr && F > 0) {
        TmBuf* fb = nullptr;
        if ((s = tm_buffer(device, st, (size_t)((nks + P - 1) / P) * F * P * 4, &fb, 1)) != SYN_OK) return s;
        r.featT = reinterpret_cast<const float*>(fb->p);
    }
    // finish tile: KT kernels per CTA, fp64 + fp32 per (model, kernel, clock) in shared memory
    // (small: the finish is a latency chain per CTA, so small batches want many CTAs)
    int kt = std::max(1, std::min(8, (int)((150 * 1024) / ((size_t)nm * n_f * 12 + (size_t)t.nslot * n_f * 8))));
    const int kt_cap = kt;                                         // shared-memory bound
    a.xs = (F + 2) | 1;
    int fnt = env_int("SYNERGY_TM_FNT", 256);                     // finish CTA size
    if (fnt != 128 && fnt != 256) fnt = 256;
    auto fsmem_of = [&](int k) {
        return (size_t)nm * k * n_f * 12 + (size_t)n_f * 4 + (size_t)k * a.xs * 4 + 32 + (size_t)k * t.nslot * n_f * 8;
    };
    static size_t fset = 48 * 1024, wset = 48 * 1024;
    cudaError_t e = cudaSuccess;
    if (fsmem_of(kt_cap) > fset) {
        if ((e = cudaFuncSetAttribute(k_tm_finish, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)fsmem_of(kt_cap))) != cudaSuccess)
            return cuda_fail(e, "k_tm_finish attribute");
        fset = fsmem_of(kt_cap);
    }
    // the smallest tile whose finish grid fits in one wave of resident CTAs (a partial second wave
    // doubles the finish's latency chain: c5 KT 3 -> 7 = 1195 -> 512 CTAs, 46 -> 37 us); when no
    // tile fits, the largest (kt_cap)
    {
        const int sms = sm_count(device);
        int fit = 0;
        for (int k = 1; k <= kt_cap && !fit; ++k) {
            int nb = 0;
            if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, k_tm_finish, fnt, fsmem_of(k)) != cudaSuccess) {
                cudaGetLastError();
                break;
            }
            if (nb > 0 && (nks + k - 1) / k <= (long long)nb * sms) fit = k;
        }
        kt = fit ? fit : kt_cap;
    }
    kt = std::max(1, std::min(env_int("SYNERGY_TM_KT", kt), 8));
    a.tile_k = kt;
    const size_t fsmem = fsmem_of(kt);
    const size_t wsmem = (size_t)kTmS * kTmNT * 8 + (size_t)(F + 2) * kTmNT * 4 + 16 + (size_t)tt * 8;
    if (fsmem > fset) {
        if ((e = cudaFuncSetAttribute(k_tm_finish, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)fsmem)) != cudaSuccess)
            return cuda_fail(e, "k_tm_finish attribute");
        fset = fsmem;
    }
    if (wsmem > wset) {
        if ((e = cudaFuncSetAttribute(k_tm_walk<kTmNT, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)wsmem)) != cudaSuccess ||
            (e = cudaFuncSetAttribute(k_tm_walk<kTmNT, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)wsmem)) != cudaSuccess)
            return cuda_fail(e, "k_tm_walk attribute");
        wset = wsmem;
    }
    static int carve_set = -1;                 // same shared-memory carveout for both kernels
    const int carve = env_int("SYNERGY_TM_CARVE", -1);
    if (carve != carve_set && carve >= 0) {
        cudaFuncSetAttribute(k_tm_walk<kTmNT, true>, cudaFuncAttributePreferredSharedMemoryCarveout, carve);
        cudaFuncSetAttribute(k_tm_walk<kTmNT, false>, cudaFuncAttributePreferredSharedMemoryCarveout, carve);
        cudaFuncSetAttribute(k_tm_finish, cudaFuncAttributePreferredSharedMemoryCarveout, carve);
        cudaGetLastError();
        carve_set = carve;
    }
    const int ctas = std::max(1, env_int("SYNERGY_TM_CTAS", 2 * sm_count(device)));
    // k_tr_walk: kTrNB tree buffers + the chunk's [F][P] features + record stacks
    r.tree_smem = (int)(((size_t)max_tb * 32 + 127) / 128 * 128);
    r.P = P;
    const size_t rsmem = (size_t)kTrNB * r.tree_smem + (size_t)F * P * 4 + (size_t)kTmS * kTrNT * 8;
    if (use_tr) {
        static size_t rset = 48 * 1024;
        if (rsmem > rset) {
            if ((e = cudaFuncSetAttribute(k_tr_walk<kTrNT>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)rsmem)) != cudaSuccess)
                return cuda_fail(e, "k_tr_walk attribute");
            rset = rsmem;
        }
    }
    t.s = a;
    int n = 0;
    int slab = 0;
    for (long long s0 = 0; s0 < n_k; s0 += nks, ++slab) {
        t.slab0 = s0;
        t.nks = (int)std::min<long long>(nks, n_k - s0);
        const int pb = slab & 1;
        if (pipe) {
            t.D = pb ? buf2->p : buf->p;
            if (slab >= 2 && (e = cudaStreamWaitEvent(st, aux->finished[pb], 0)) != cudaSuccess)
                return cuda_fail(e, "slab pipeline wait");
        }
        // tiny batches: split every (kernel, tree) task into clock sub-ranges while there are fewer
        // tasks than resident lanes (at most 8 sub-ranges of at least 8 clocks; each sub-range
        // adds a root descent, so batches with a task per lane keep whole tasks)
        t.nsub = 1;
        const long long lanes = (long long)ctas * kTmNT;
        while (t.nsub < 8 && (long long)t.nks * tt * t.nsub < lanes && n_f / (2 * t.nsub) >= 8) t.nsub *= 2;
        const int ns_env = env_int("SYNERGY_TM_NSUB", t.nsub);
        if (ns_env >= 1 && ns_env <= n_f && ns_env <= 64) t.nsub = ns_env;
        t.n_tasks = (long long)((t.nks + kb - 1) / kb) * tt * t.nsub * kb;
        // a few tasks per lane: dynamic task fetch balances walks of different lengths
        t.dyn = env_int("SYNERGY_TM_DYN", t.n_tasks < 4 * lanes ? 1 : 0) ? 1 : 0;
        if (use_tr) {
            // unit = (tree, chunk of P kernels), one CTA per SM over contiguous unit ranges
            r.nchunks = (t.nks + P - 1) / P;
            r.tm = t;
            {
                const long long nf = (long long)r.nchunks * F * P;
                KernelTimer ktf("k_tr_feat", st);
                if (nf > 0) k_tr_feat<<<(unsigned)((nf + 255) / 256), 256, 0, st>>>(a.features, t.slab0, t.nks, F, P, r.nchunks, const_cast<float*>(r.featT));
                e = cudaGetLastError();
            }
            const long long units = (long long)r.nchunks * tt;
            const long long g = std::max<long long>(1, std::min<long long>(env_int("SYNERGY_TR_CTAS", sms_tr), units));
            if (e == cudaSuccess) {
                KernelTimer ktm("k_tr_walk", st);
                k_tr_walk<kTrNT><<<(unsigned)g, kTrNT, rsmem, st>>>(r);
                e = cudaGetLastError();
            }
            if (e != cudaSuccess) {
                buf->dirty = true;
                if (buf2) buf2->dirty = true;
                if (pipe && slab > 0) cudaStreamWaitEvent(st, aux->finished[(slab - 1) & 1], 0);
                return cuda_fail(e, "k_tr_walk launch");
            }
            ++n;
        } else {
            const long long g = std::max<long long>(1, std::min<long long>(ctas, (t.n_tasks + 255) / 256));
            {
                KernelTimer ktm("k_tm_walk", st);
                if (fxall)
                    k_tm_walk<kTmNT, true><<<(unsigned)g, kTmNT, wsmem, st>>>(t);
                else
                    k_tm_walk<kTmNT, false><<<(unsigned)g, kTmNT, wsmem, st>>>(t);
                e = cudaGetLastError();
            }
            if (e != cudaSuccess) {
                buf->dirty = true;
                if (buf2) buf2->dirty = true;
                if (pipe && slab > 0) cudaStreamWaitEvent(st, aux->finished[(slab - 1) & 1], 0);
                return cuda_fail(e, "k_tm_walk launch");
            }
        }
        cudaStream_t fst = st;
        if (pipe) {
            if ((e = cudaEventRecord(aux->walked[pb], st)) != cudaSuccess ||
                (e = cudaStreamWaitEvent(aux->st2, aux->walked[pb], 0)) != cudaSuccess) {
                buf->dirty = buf2->dirty = true;
                return cuda_fail(e, "slab pipeline fork");
            }
            fst = aux->st2;
        }
        {
            KernelTimer ktm("k_tm_finish", fst);
            if (!pipe && env_int("SYNERGY_TM_PDL", 1) != 0) {
                // programmatic dependent launch: the finish grid is scheduled while the walk runs
                // and waits (griddepcontrol.wait) for it before reading D
                cudaLaunchConfig_t lc;
                memset(&lc, 0, sizeof lc);
                lc.gridDim = dim3((unsigned)((t.nks + kt - 1) / kt));
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
                k_tm_finish<<<(unsigned)((t.nks + kt - 1) / kt), fnt, fsmem, fst>>>(t);
                e = cudaGetLastError();
            }
        }
        if (e == cudaSuccess && pipe) e = cudaEventRecord(aux->finished[pb], aux->st2);
        if (e != cudaSuccess) {
            buf->dirty = true;
            if (buf2) buf2->dirty = true;
            if (pipe && slab > 0) cudaStreamWaitEvent(st, aux->finished[(slab - 1) & 1], 0);
            return cuda_fail(e, "k_tm_finish launch");
        }
        n += 2;
    }
    if (pipe && (e = cudaStreamWaitEvent(st, aux->finished[(slab - 1) & 1], 0)) != cudaSuccess)   // join
        return cuda_fail(e, "slab pipeline join");
    *launches = n;
    *variant = use_tr ? 4001 : 4000;
    return ok();
}

template <int S, int T>
cudaError_t launch_sweep_t(const SweepArgs& a, const Config& c, long long grid, cudaStream_t st) {
    static size_t smem_set = 48 * 1024;   // per-instantiation opt-in high-water mark
    if (c.smem > smem_set) {
        cudaError_t e = cudaFuncSetAttribute(k_sweep<S, T>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)c.smem);
        if (e != cudaSuccess) return e;
        smem_set = c.smem;
    }
    k_sweep<S, T><<<(unsigned)grid, c.nt, c.smem, st>>>(a);
    return cudaGetLastError();
}

cudaError_t launch_sweep(const SweepArgs& a, const Config& c, long long grid, cudaStream_t st) {
    switch (c.slots) {
        case 1: return launch_sweep_t<1, 4>(a, c, grid, st);
        case 2: return launch_sweep_t<2, 4>(a, c, grid, st);
        case 4: return launch_sweep_t<4, 2>(a, c, grid, st);
        default: return launch_sweep_t<8, 1>(a, c, grid, st);
    }
}

syn_status validate_sweep(const syn_model* sp, const syn_model* en, int64_t n_k, int32_t F,
                          const syn_clocks* clocks, int32_t def, const syn_target* targets, int32_t n_t, int mode) {
    if (!sp || !en) return fail(SYN_ERR_INVALID_ARG, "model is NULL");
    if (!clocks) return fail(SYN_ERR_INVALID_ARG, "clocks is NULL");
    if (n_k < 0) return fail(SYN_ERR_INVALID_ARG, "n_kernels=%lld < 0", (long long)n_k);
    if (F + 1 != sp->n_inputs || F + 1 != en->n_inputs)
        return fail(SYN_ERR_INVALID_ARG, "n_features+1=%d does not match model n_inputs (%d, %d)", F + 1, sp->n_inputs, en->n_inputs);
    const int n_f = clocks->n_f;
    if (mode == kModeSweep) {
        if (def < 0 || def >= n_f) return fail(SYN_ERR_INVALID_ARG, "default_idx=%d outside [0, %d)", def, n_f);
        syn_status s = check_targets(targets, n_t);
        if (s != SYN_OK) return s;
    } else if (def < -1 || def >= n_f) {
        return fail(SYN_ERR_INVALID_ARG, "default_idx=%d outside [-1, %d)", def, n_f);
    }
    if (sp->device != clocks->device || en->device != clocks->device || !current_device_is(clocks->device))
        return fail(SYN_ERR_INVALID_ARG, "model/clocks device differs from the current device");
    return SYN_OK;
}

// Library-owned stream-ordered pool per device for the SVR scratch: memory freed with
// cudaFreeAsync stays mapped (release threshold = max), so steady-state calls reuse it instead
// of remapping; the process's default pool and its settings are left alone.
cudaMemPool_t svr_pool(int dev) {
    static std::mutex mu;
    static cudaMemPool_t pools[64] = {};
    if (dev < 0 || dev >= 64) return nullptr;
    std::lock_guard<std::mutex> lock(mu);
    if (!pools[dev]) {
        cudaMemPoolProps props;
        memset(&props, 0, sizeof props);
        props.allocType = cudaMemAllocationTypePinned;
        props.handleTypes = cudaMemHandleTypeNone;
        props.location.type = cudaMemLocationTypeDevice;
        props.location.id = dev;
        cudaMemPool_t p = nullptr;
        if (cudaMemPoolCreate(&p, &props) != cudaSuccess) {
            cudaGetLastError();
            return nullptr;
        }
        unsigned long long thr = ~0ULL;
        cudaMemPoolSetAttribute(p, cudaMemPoolAttrReleaseThreshold, &thr);
        pools[dev] = p;
    }
    return pools[dev];
}

// SVR members (kernels_svr.cuh): per model, V = clock factors and the split contractions P into
// stream-ordered scratch; dm.svr_p / svr_splits point the finish step at them.  Released with
// release() after the sweep kernel is enqueued (cudaFreeAsync keeps it alive until then).
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
    static bool smem_set = false;
    const size_t smem = (size_t)kSvrStages * kSvrJC * (kSvrTK + 32 * CPT) * sizeof(double) + kSvrStages * 8;
    if (!smem_set) {
        cudaError_t e = cudaFuncSetAttribute(k_svr<CPT>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        if (e != cudaSuccess) return e;
        smem_set = true;
    }
    k_svr<CPT><<<grid, 256, smem, st>>>(sa);
    return cudaGetLastError();
}

constexpr size_t kSvrSlabBytes = 256u << 20;   // U scratch per kernel slab

syn_status prepare_svr(DevModel& dm, int device, const float* d_features, long long n_k, int F, const syn_clocks* clocks,
                       cudaStream_t st, SvrScratch& scr) {
    if (dm.svr_weight == 0.0) return ok();
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
    int splits = (int)std::max<long long>(1, sm_count(device) / std::max<long long>(tiles, 1));
    splits = std::min(splits, kSvrMaxSplits);
    splits = env_int("SYNERGY_SVR_SPLITS", splits);
    splits = std::max(1, std::min(splits, n_chunks));
    const int cps = (n_chunks + splits - 1) / splits;
    splits = (n_chunks + cps - 1) / cps;
    const size_t pb = (size_t)splits * (size_t)n_k * n_f * sizeof(double);
    const size_t vb = (size_t)tiles_n * n_svp * tn * sizeof(double);
    const size_t ub = (size_t)((nks + kSvrTK - 1) / kSvrTK) * n_svp * kSvrTK * sizeof(double);
    const size_t voff = (pb + 255) / 256 * 256, uoff = voff + (vb + 255) / 256 * 256;
    const size_t total = uoff + ub;
    void* buf = nullptr;
    cudaMemPool_t pool = svr_pool(device);
    if (!pool) return fail(SYN_ERR_CUDA, "cannot create the SVR scratch pool on device %d", device);
    cudaError_t e = cudaMallocFromPoolAsync(&buf, total, pool, st);
    if (e != cudaSuccess) {
        cudaGetLastError();
        return e == cudaErrorMemoryAllocation ? fail(SYN_ERR_OOM, "SVR scratch of %zu bytes", total)
                                              : cuda_fail(e, "cudaMallocFromPoolAsync(SVR scratch)");
    }
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
    {
        KernelTimer kt("k_svr_v", st);
        k_svr_v<<<(unsigned)((nv + 255) / 256), 256, 0, st>>>(sa);
        e = cudaGetLastError();
    }
    if (e != cudaSuccess) return cuda_fail(e, "k_svr_v launch");
    scr.launches += 1;
    static bool u_smem_set = false;
    const size_t usmem = (size_t)F * (64 * sizeof(double) + kSvrJC * sizeof(float));
    if (usmem > 48 * 1024 && !u_smem_set) {
        if ((e = cudaFuncSetAttribute(k_svr_u, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024)) != cudaSuccess)
            return cuda_fail(e, "k_svr_u attribute");
        u_smem_set = true;
    }
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

syn_status run_sweep(const syn_model* sp, const syn_model* en, const float* d_features, int64_t n_k,
                     int32_t F, const syn_clocks* clocks, int32_t def, const syn_target* targets, int32_t n_t,
                     int32_t* d_choice, float* d_S, float* d_E, int mode, cudaStream_t st) {
    syn_status vs = validate_sweep(sp, en, n_k, F, clocks, def, targets, n_t, mode);
    if (vs != SYN_OK) return vs;
    const int n_f = clocks->n_f;
    if (n_k == 0) {
        g_last = {0, 0, 0, 0, 0};
        return ok();
    }
    if (!d_features) return fail(SYN_ERR_INVALID_ARG, "d_features is NULL");
    if (mode == kModeSweep && !d_choice) return fail(SYN_ERR_INVALID_ARG, "d_choice is NULL");
    if (mode == kModePredict && (!d_S || !d_E)) return fail(SYN_ERR_INVALID_ARG, "d_speedup/d_energy is NULL");

    SweepArgs a;
    memset(&a, 0, sizeof a);
    a.ms = sp->dm;
    a.me = en->dm;
    a.features = d_features;
    a.n_k = n_k;
    a.F = F;
    a.freqs = clocks->d_freqs;
    a.n_f = n_f;
    a.def = def;
    a.n_t = mode == kModeSweep ? n_t : 0;
    for (int t = 0; t < a.n_t; ++t) {
        a.kind[t] = targets[t].kind;
        a.x[t] = targets[t].x;
    }
    a.choice = d_choice;
    a.S_out = d_S;
    a.E_out = d_E;
    a.mode = mode;
    // default: clock-interval traversal when forests are present and n_f <= 1024;
    // SYNERGY_ALGO=direct forces the per-clock root-to-leaf kernel (A/B and fallback)
    const char* algo_env = getenv("SYNERGY_ALGO");
    const bool force_direct = algo_env && !strcmp(algo_env, "direct");
    const bool force_iv = algo_env && !strcmp(algo_env, "iv");
    const bool force_ws = algo_env && !strcmp(algo_env, "ws");
    Config c;
    const bool forests = sp->n_trees > 0 || en->n_trees > 0;
    // default: order-free difference-array kernel (exact int64 leaf sums; n_f <= 2048), else the
    // in-order warp-streaming kernel (n_f <= 256), else the chunked interval kernel
    // (n_f <= 1024), else per-clock direct traversal; SYNERGY_ALGO=ws|iv|direct forces one
    bool chosen = false;
    if (!force_direct && forests) {
        if (!force_iv && !force_ws) chosen = choose_da(sp, en, n_k, n_f, F, c);
        if (!chosen && !force_iv) chosen = choose_ws(n_k, n_f, F, clocks->device, c);
        if (!chosen) chosen = choose_iv(n_k, n_f, F, clocks->device, c);
    }
    if (!chosen) c = choose_config(n_k, n_f, F, clocks->device);
    a.tile_k = c.tile_k;
    a.xs = c.xs;
    a.tc = c.tc;
    a.words = c.words;
    a.vcap = c.vcap;
    a.vs = c.vs;
    a.region = c.region;
    a.win = c.win;
    a.slot_bytes = c.slot_bytes;
    a.head_bytes = c.head_bytes;
    a.grid = clocks->d_grid;
    a.f0 = clocks->f0;
    a.inv_step = clocks->inv_step;
    a.nsub = c.algo == 3 ? c.slots : 1;
    const long long grid = (n_k + c.tile_k - 1) / c.tile_k;
    if (grid > 0x7fffffffLL) return fail(SYN_ERR_UNSUPPORTED, "n_kernels too large for one launch");
    SvrScratch scr;
    syn_status ss = prepare_svr(a.ms, clocks->device, d_features, n_k, F, clocks, st, scr);
    if (ss == SYN_OK) ss = prepare_svr(a.me, clocks->device, d_features, n_k, F, clocks, st, scr);
    if (ss != SYN_OK) return ss;
    // default: tree-major resume walks (kernels_tm.cuh) whenever the exact int64 leaf sums apply;
    // SYNERGY_ALGO=da|ws|iv|direct selects one of the single-launch kernels instead
    if (!algo_env && tm_eligible(a, 2)) {
        int nl = 0;
        syn_model* ms[2] = {const_cast<syn_model*>(sp), const_cast<syn_model*>(en)};
        int var = 4000;
        ss = run_tm(a, 2, ms, clocks, st, &nl, &var);
        if (ss != SYN_OK) return ss;
        g_last = {nl + scr.launches, n_k * (long long)n_f, (long long)std::min<long long>(2LL * sm_count(clocks->device), n_k),
                  var == 4001 ? kTrNT : kTmNT, var};
        return ok();
    }
    static const char* knames[4] = {"k_sweep", "k_sweep_iv", "k_sweep_ws", "k_sweep_da"};
    cudaError_t e;
    {
        KernelTimer kt(knames[c.algo], st);
        e = c.algo == 3 ? launch_da(a, c, grid, st)
                  : c.algo == 2 ? launch_ws(a, c, grid, st)
                  : c.algo == 1 ? launch_iv(a, c, grid, st)
                                : launch_sweep(a, c, grid, st);
    }
    static const char* names[4] = {"k_sweep launch", "k_sweep_iv launch", "k_sweep_ws launch", "k_sweep_da launch"};
    if (e != cudaSuccess) return cuda_fail(e, names[c.algo]);
    g_last = {1 + scr.launches, n_k * (long long)n_f, grid, c.nt, c.algo ? c.algo * 1000 + c.tile_k : c.slots * 10 + c.tilp};
    return ok();
}

}  // namespace

// =============================================================================== C ABI

extern "C" {

const char* synergy_last_error(void) { return g_err.c_str(); }

int32_t synergy_version(void) { return SYNERGY_VERSION; }

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
    // exact fixed-point scale for the leaf sums (k_sweep_da): s = -(smallest leaf ulp exponent)
    int fx_ok = 0, fx_s = 0, fx32 = 0;
    if (d->forest_weight != 0.0) {
        int min_lsb = 1 << 30, max_e = -(1 << 30);
        bool finite = true;
        for (int t = 0; t < d->n_trees && finite; ++t)
            for (int64_t id = d->tree_offset[t]; id < d->tree_offset[t + 1]; ++id) {
                if (d->feature[id] >= 0) continue;
                const float v = d->value[id];
                if (!std::isfinite(v)) { finite = false; break; }
                if (v == 0.0f) continue;
                int e2 = 0;
                std::frexp(v, &e2);                       // |v| in [2^(e2-1), 2^e2)
                min_lsb = std::min(min_lsb, std::max(e2 - 24, -149));
                max_e = std::max(max_e, e2);
            }
        if (finite) {
            if (max_e == -(1 << 30)) { fx_ok = 1; fx_s = 0; fx32 = 1; }   // all leaves zero
            else {
                fx_s = -min_lsb;
                int lg = 0;
                while ((1LL << lg) < (long long)d->n_trees + 1) ++lg;
                fx_ok = (max_e + fx_s + lg <= 61) ? 1 : 0;
                fx32 = (fx_ok && max_e + fx_s <= 31) ? 1 : 0;
            }
        }
    }
    const int pad_leaf = (int)nodes.size();
    nodes.push_back(make_uint2(0u, 0xFFFFFF00u | leaf_code));

    // 2-level blocks (see internal.h): built from the validated description, breadth-first
    std::vector<uint4> blocks;
    std::vector<int> broot;
    int bdepth = 1;
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
            bdepth = std::max(bdepth, (trees[t].y + 1) / 2);
        }
    }

    DeviceGuard g(device);
    if (!g.okay) return fail(SYN_ERR_INVALID_ARG, "cannot select device %d", device);
    const size_t nb = nodes.size() * sizeof(uint2);
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
    const size_t total = has_svr ? off_sc + lb : off_r + rb;
    void* mem = nullptr;
    cudaError_t e = cudaMalloc(&mem, total);
    if (e != cudaSuccess) return cuda_fail(e, "cudaMalloc(model)");
    char* base = static_cast<char*>(mem);
    std::vector<double> lw((size_t)d->n_inputs, 0.0);
    if (d->linear_weight != 0.0) std::copy(d->lin_w, d->lin_w + d->n_inputs, lw.begin());
    if ((e = cudaMemcpy(base, nodes.data(), nb, cudaMemcpyHostToDevice)) != cudaSuccess ||
        (!trees.empty() && (e = cudaMemcpy(base + off_t, trees.data(), trees.size() * sizeof(int2), cudaMemcpyHostToDevice)) != cudaSuccess) ||
        (e = cudaMemcpy(base + off_l, lw.data(), lb, cudaMemcpyHostToDevice)) != cudaSuccess ||
        (!blocks.empty() && (e = cudaMemcpy(base + off_b, blocks.data(), blocks.size() * sizeof(uint4), cudaMemcpyHostToDevice)) != cudaSuccess) ||
        (!broot.empty() && (e = cudaMemcpy(base + off_r, broot.data(), broot.size() * sizeof(int), cudaMemcpyHostToDevice)) != cudaSuccess) ||
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
    m->n_nodes = (long long)nodes.size() - 1;
    m->bytes = (long long)total;
    m->alloc = mem;
    m->dm.nodes = reinterpret_cast<const uint2*>(base);
    m->dm.trees = reinterpret_cast<const int2*>(base + off_t);
    m->dm.lin_w = reinterpret_cast<const double*>(base + off_l);
    m->dm.lin_b = d->linear_weight != 0.0 ? d->lin_b : 0.0;
    m->dm.lin_weight = d->linear_weight;
    m->dm.forest_weight = d->forest_weight;
    m->dm.n_trees = m->n_trees;
    m->dm.pad_leaf = pad_leaf;
    m->dm.depth = max_depth;
    m->dm.blocks = reinterpret_cast<const uint4*>(base + off_b);
    m->dm.broot = reinterpret_cast<const int*>(base + off_r);
    m->dm.bdepth = bdepth;
    m->n_blocks = (long long)(blocks.size() >> 1);
    m->dm.nblk = (int)m->n_blocks;
    m->max_tree_blocks = 0;
    for (size_t t = 0; t < broot.size(); ++t)
        m->max_tree_blocks = std::max<long long>(m->max_tree_blocks,
                                                 (t + 1 < broot.size() ? broot[t + 1] : m->n_blocks) - broot[t]);
    m->dm.fx_ok = fx_ok;
    m->dm.fx32 = fx32;
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
        cudaFree(m->alloc);
        for (auto& cb : m->cut_blocks) cudaFree(cb.second);
        for (auto& cb : m->tr_blocks) cudaFree(cb.second);
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
    // clock-cut hint grid: grid[b] = #{i : f_i < f_0 + b * step}, b = 0..kGrid (any rounding is
    // fine: the kernels finish every cut with exact comparisons against the table)
    const float f0 = h[0], span = h[n_f - 1] - h[0];
    const float step = span > 0.0f ? span / (float)kGrid : 1.0f;
    std::vector<unsigned short> grid(kGrid + 1);
    for (int b = 0; b <= kGrid; ++b) {
        const float edge = f0 + (float)b * step;
        grid[b] = (unsigned short)(std::lower_bound(h, h + n_f, edge) - h);
    }
    float* d = nullptr;
    const size_t gbytes = (size_t)(kGrid + 1) * sizeof(unsigned short);
    const size_t goff = ((size_t)n_f * sizeof(float) + 255) / 256 * 256;
    cudaError_t e = cudaMalloc(&d, goff + gbytes);
    if (e != cudaSuccess) return cuda_fail(e, "cudaMalloc(clocks)");
    if ((e = cudaMemcpy(d, h, (size_t)n_f * sizeof(float), cudaMemcpyHostToDevice)) != cudaSuccess ||
        (e = cudaMemcpy(reinterpret_cast<char*>(d) + goff, grid.data(), gbytes, cudaMemcpyHostToDevice)) != cudaSuccess) {
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
    c->d_grid = reinterpret_cast<unsigned short*>(reinterpret_cast<char*>(d) + goff);
    c->f0 = f0;
    c->inv_step = 1.0f / step;
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

syn_status synergy_predict(const syn_model* sp, const syn_model* en, const float* d_features, int64_t n_k,
                           int32_t F, const syn_clocks* clocks, int32_t def, float* d_S, float* d_E,
                           syn_stream stream) {
    return run_sweep(sp, en, d_features, n_k, F, clocks, def, nullptr, 0, nullptr, d_S, d_E, kModePredict,
                     static_cast<cudaStream_t>(stream));
}

syn_status synergy_sweep(const syn_model* sp, const syn_model* en, const float* d_features, int64_t n_k,
                         int32_t F, const syn_clocks* clocks, int32_t def, const syn_target* targets,
                         int32_t n_t, int32_t* d_choice, float* d_S, float* d_E, syn_stream stream) {
    return run_sweep(sp, en, d_features, n_k, F, clocks, def, targets, n_t, d_choice, d_S, d_E, kModeSweep,
                     static_cast<cudaStream_t>(stream));
}

syn_status synergy_sweep4(const syn_model* const* models, const float* d_features, int64_t n_k, int32_t F,
                          const syn_clocks* clocks, int32_t def, const syn_target* targets, int32_t n_t,
                          int32_t* d_choice, float* d_pred, syn_stream stream) {
    if (!models) return fail(SYN_ERR_INVALID_ARG, "models is NULL");
    const syn_model* sp = models[0];
    const syn_model* en = models[1];
    const syn_model* x2 = models[2];
    const syn_model* x3 = models[3];
    syn_status vs = validate_sweep(sp, en, n_k, F, clocks, def, targets, n_t, kModeSweep);
    if (vs != SYN_OK) return vs;
    for (const syn_model* xm : {x2, x3}) {
        if (!xm) continue;
        if (xm->n_inputs != F + 1) return fail(SYN_ERR_INVALID_ARG, "direct EDP/ED2P model n_inputs mismatch");
        if (xm->device != clocks->device) return fail(SYN_ERR_INVALID_ARG, "model device differs from clocks");
    }
    if (n_k == 0) {
        g_last = {0, 0, 0, 0, 0};
        return ok();
    }
    if (!d_features || !d_choice) return fail(SYN_ERR_INVALID_ARG, "device buffer is NULL");
    const int n_f = clocks->n_f;
    Config c;
    if (!choose_da(sp, en, n_k, n_f, F, c, x2, x3))
        return fail(SYN_ERR_UNSUPPORTED, "four-model sweep needs forests within the exact int64 leaf range and n_freqs <= 2048");
    SweepArgs a;
    memset(&a, 0, sizeof a);
    a.ms = sp->dm;
    a.me = en->dm;
    if (x2) { a.mx[0] = x2->dm; a.has_x[0] = 1; }
    if (x3) { a.mx[1] = x3->dm; a.has_x[1] = 1; }
    if (!x2 && !x3) a.has_x[0] = 0;
    a.features = d_features;
    a.n_k = n_k;
    a.F = F;
    a.freqs = clocks->d_freqs;
    a.n_f = n_f;
    a.def = def;
    a.n_t = n_t;
    for (int t = 0; t < n_t; ++t) {
        a.kind[t] = targets[t].kind;
        a.x[t] = targets[t].x;
    }
    a.choice = d_choice;
    if (d_pred) {
        const size_t plane = (size_t)n_k * n_f;
        a.S_out = d_pred;
        a.E_out = d_pred + plane;
        a.X_out[0] = x2 ? d_pred + 2 * plane : nullptr;
        a.X_out[1] = x3 ? d_pred + 3 * plane : nullptr;
    }
    a.mode = kModeSweep;
    a.tile_k = c.tile_k;
    a.xs = c.xs;
    a.head_bytes = c.head_bytes;
    a.grid = clocks->d_grid;
    a.f0 = clocks->f0;
    a.inv_step = clocks->inv_step;
    a.nsub = c.slots;
    const long long grid = (n_k + c.tile_k - 1) / c.tile_k;
    if (grid > 0x7fffffffLL) return fail(SYN_ERR_UNSUPPORTED, "n_kernels too large for one launch");
    const cudaStream_t st = static_cast<cudaStream_t>(stream);
    SvrScratch scr;
    syn_status ss = SYN_OK;
    DevModel* dms[4] = {&a.ms, &a.me, &a.mx[0], &a.mx[1]};
    for (int m = 0; m < 4 && ss == SYN_OK; ++m)
        if (m < 2 || a.has_x[m - 2]) ss = prepare_svr(*dms[m], clocks->device, d_features, n_k, F, clocks, st, scr);
    if (ss != SYN_OK) return ss;
    const char* algo_env = getenv("SYNERGY_ALGO");
    if (!algo_env && tm_eligible(a, 4)) {
        int nl = 0;
        syn_model* ms[4] = {const_cast<syn_model*>(sp), const_cast<syn_model*>(en), const_cast<syn_model*>(x2),
                            const_cast<syn_model*>(x3)};
        int var = 4000;
        ss = run_tm(a, 4, ms, clocks, st, &nl, &var);
        if (ss != SYN_OK) return ss;
        g_last = {nl + scr.launches, n_k * (long long)n_f, (long long)std::min<long long>(2LL * sm_count(clocks->device), n_k),
                  var == 4001 ? kTrNT : kTmNT, var};
        return ok();
    }
    cudaError_t e;
    {
        KernelTimer kt("k_sweep_da", st);
        e = launch_da(a, c, grid, st);
    }
    if (e != cudaSuccess) return cuda_fail(e, "k_sweep_da launch");
    g_last = {1 + scr.launches, n_k * (long long)n_f, grid, c.nt, 3000 + c.tile_k};
    return ok();
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
        a.x[t] = targets[t].x;
    }
    a.choice = d_choice;
    int dev = 0;
    cudaGetDevice(&dev);
    const int block = 256;
    const long long need = (n_k + 7) / 8;
    const long long grid = std::min<long long>(need, (long long)sm_count(dev) * 8);
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
    const long long grid = std::min<long long>((n_k + 7) / 8, (long long)sm_count(dev) * 8);
    k_pareto<<<(unsigned)grid, 256, 0, static_cast<cudaStream_t>(stream)>>>(d_S, d_E, n_k, n_f, d_front);
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
        a.x[t] = targets[t].x;
    }
    int dev = 0;
    cudaGetDevice(&dev);
    cudaStream_t st = static_cast<cudaStream_t>(stream);
    if (n_k > 0) {
        const long long grid = std::min<long long>((n_k + 7) / 8, (long long)sm_count(dev) * 8);
        k_choice_error<<<(unsigned)grid, 256, 0, st>>>(a, d_pred, d_err);
    }
    k_error_reduce<<<n_t, 256, 0, st>>>(d_err, n_k, n_t, d_summary);
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return cuda_fail(e, "k_choice_error launch");
    g_last = {2, n_k * (long long)n_f, 0, 256, 0};
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
    const long long n = n_k * (long long)n_t;
    const long long grid = std::min<long long>((n + 255) / 256, (long long)sm_count(clocks->device) * 16);
    k_plan<<<(unsigned)grid, 256, 0, static_cast<cudaStream_t>(stream)>>>(d_choice, n, clocks->d_freqs, clocks->n_f, d_mhz);
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
    syn_status vs = validate_sweep(sp, en, n_k, F, clocks, def, targets, n_t, kModeSweep);
    if (vs != SYN_OK) return vs;
    const size_t fb = (size_t)n_k * (size_t)F * sizeof(float);
    const size_t cb = (size_t)n_k * (size_t)std::max(n_t, 0) * sizeof(int32_t);
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
    syn_status s = run_sweep(sp, en, w->d_features, n_k, F, clocks, def, targets, n_t, w->d_choice, nullptr,
                             nullptr, kModeSweep, st);
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

syn_status synergy_timing_read(int32_t cap, const char** names, double* total_ms, int64_t* launches,
                               int32_t* n_kernels) {
    if (cap < 0 || (cap > 0 && (!names || !total_ms || !launches)) || !n_kernels)
        return fail(SYN_ERR_INVALID_ARG, "bad timing_read buffers");
    std::lock_guard<std::mutex> lock(g_tmu);
    std::vector<const char*> nm;
    std::vector<double> ms;
    std::vector<int64_t> cnt;
    syn_status st = SYN_OK;
    for (const TimedLaunch& t : g_tl) {
        float x = 0.0f;
        cudaError_t e = cudaEventSynchronize(t.b);
        if (e == cudaSuccess) e = cudaEventElapsedTime(&x, t.a, t.b);
        if (e != cudaSuccess && st == SYN_OK) st = cuda_fail(e, "timing events");
        size_t k = 0;
        while (k < nm.size() && strcmp(nm[k], t.name)) ++k;
        if (k == nm.size()) { nm.push_back(t.name); ms.push_back(0.0); cnt.push_back(0); }
        ms[k] += x;
        cnt[k] += 1;
        g_evpool.push_back(t.a);
        g_evpool.push_back(t.b);
    }
    g_tl.clear();
    *n_kernels = (int32_t)nm.size();
    for (int32_t k = 0; k < (int32_t)nm.size() && k < cap; ++k) {
        names[k] = nm[k];
        total_ms[k] = ms[k];
        launches[k] = cnt[k];
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
