// ts_host.cu -- host side of libtriosim: the C ABI of include/triosim.h.
//
// load_trace   host validation + H2D + K1a ingest kernel
// build_sweep  topology validation, BFS routes (S5), PP auto-partition,
//              per-point status (R3), structural classes, device pools, work lists
// simulate     K1b rescale + K2 expansion (all classes) + K3 timeline (requested points),
//              stream-ordered on the caller's stream
// results      D2H (synchronising) or stream-ordered D2D
#include <cuda_runtime.h>
#include <algorithm>
#include <cmath>
#include <cstdarg>
#include <cstdio>
#include <cstring>
#include <map>
#include <mutex>
#include <chrono>
#include <cstdlib>
#include <memory>
#include <string>
#include <tuple>
#include <vector>
#include "ts_internal.h"

using namespace ts;

namespace {

// Device block cache: load_trace / build_sweep / release run every step of a user's loop (bench.py's
// e2e), and each of them would otherwise pay ~50 cudaMalloc / cudaFree (cudaFree synchronises the
// device).  Freed blocks are kept per (device, capacity) and reused for a request of at least half
// their size.  A block is only returned to the cache where no launch can still use it: release() and
// set_breakdown() synchronise the device first, and a reallocated buffer synchronises before it gives
// its old block back (what cudaFree did implicitly).  TS_NO_BLOCK_CACHE=1 turns the cache off.
struct BlockCache {
    std::mutex mu;
    std::multimap<std::pair<int, size_t>, void *> blocks;
    size_t bytes = 0;
    // at most TS_BLOCK_CACHE_MB (default 512) MiB of idle blocks are kept; a failing cudaMalloc of ours
    // empties the cache of that device first, and triosim_destroy empties it
    const size_t kMaxBytes = size_t(getenv("TS_BLOCK_CACHE_MB") ? atol(getenv("TS_BLOCK_CACHE_MB")) : 512) << 20;
    bool on = getenv("TS_NO_BLOCK_CACHE") == nullptr || atoi(getenv("TS_NO_BLOCK_CACHE")) == 0;
    cudaError_t get(void **p, size_t want, size_t *cap, int *dev) {
        cudaError_t e = cudaGetDevice(dev);
        if (e != cudaSuccess) return e;
        want = (want + 511) & ~size_t(511);
        if (on) {
            std::lock_guard<std::mutex> g(mu);
            auto it = blocks.lower_bound({*dev, want});
            if (it != blocks.end() && it->first.first == *dev && it->first.second <= 2 * want) {
                *p = it->second;
                *cap = it->first.second;
                bytes -= *cap;
                blocks.erase(it);
                return cudaSuccess;
            }
        }
        *cap = want;
        e = cudaMalloc(p, want);
        if (e == cudaErrorMemoryAllocation && on) {   // give the cached blocks of this device back, retry
            cudaGetLastError();
            trim(*dev);
            e = cudaMalloc(p, want);
        }
        return e;
    }
    void put(void *p, size_t cap, int dev) {
        if (on) {
            std::lock_guard<std::mutex> g(mu);
            if (bytes + cap <= kMaxBytes) {
                blocks.insert({{dev, cap}, p});
                bytes += cap;
                return;
            }
        }
        cudaFree(p);
    }
    void trim(int dev) {
        std::lock_guard<std::mutex> g(mu);
        for (auto it = blocks.begin(); it != blocks.end();) {
            if (it->first.first == dev) { cudaFree(it->second); bytes -= it->first.second; it = blocks.erase(it); }
            else ++it;
        }
    }
};
// TS_HOST_TIMING=1: wall time of build_sweep's host phases on stderr (diagnostics only)
struct PhaseTimer {
    bool on = getenv("TS_HOST_TIMING") != nullptr;
    std::chrono::steady_clock::time_point t = std::chrono::steady_clock::now();
    void mark(const char *what) {
        if (!on) return;
        auto n = std::chrono::steady_clock::now();
        fprintf(stderr, "[ts_host] %-14s %8.3f ms\n", what, std::chrono::duration<double, std::milli>(n - t).count());
        t = n;
    }
};

BlockCache &block_cache() {
    static BlockCache *c = new BlockCache();   // never destroyed: no CUDA calls during static teardown
    return *c;
}

template <class T>
struct DevBuf {
    T *p = nullptr;
    size_t n = 0, cap = 0;
    int dev = 0;
    ~DevBuf() { if (p) block_cache().put(p, cap, dev); }
    cudaError_t alloc(size_t count) {
        if (p) {
            cudaDeviceSynchronize();   // a launch may still use the old block (cudaFree synchronised too)
            block_cache().put(p, cap, dev);
            p = nullptr;
        }
        n = count;
        if (count == 0) count = 1;
        void *q = nullptr;
        cudaError_t e = block_cache().get(&q, count * sizeof(T), &cap, &dev);
        p = e == cudaSuccess ? (T *)q : nullptr;
        return e;
    }
    cudaError_t upload(const std::vector<T> &v) {
        cudaError_t e = alloc(v.size());
        if (e != cudaSuccess || v.empty()) return e;
        return cudaMemcpy(p, v.data(), v.size() * sizeof(T), cudaMemcpyHostToDevice);
    }
};

struct Trace {
    ~Trace() { cudaDeviceSynchronize(); }   // before the members' blocks go back to the cache
    std::vector<triosim_op> ops;
    std::vector<triosim_tensor> ts;
    std::vector<uint32_t> io;
    uint32_t b0 = 0, n_layers = 0;
    int32_t first_opt = -1;   // first OPT-phase op (R28 needs one to apply updates)
    std::vector<int32_t> prod;
    // trace-level facts the host needs (route needs, cost estimates, partitions)
    uint32_t n_wgrad = 0;
    uint64_t wgrad_bytes = 0;
    uint32_t n_out_total = 0, n_in_total = 0;
    std::map<int, std::vector<uint32_t>> auto_plans;   // pp -> first layers
    DevBuf<triosim_op> d_ops;
    DevBuf<triosim_tensor> d_ts;
    DevBuf<uint32_t> d_io;
    DevBuf<double> d_time;
    DevBuf<uint32_t> d_info, d_layer, d_wgrad;
    DevBuf<int32_t> d_prod, d_scal;
    TraceDev dev;
    int n_sweeps = 0;
};

struct Sweep {
    ~Sweep() {
        cudaDeviceSynchronize();   // before the members' blocks go back to the cache
        if (ev_done) cudaEventDestroy(ev_done);
    }
    int trace_handle = -1;
    uint64_t n_pts = 0;
    std::vector<int32_t> status;            // host-side status per point (-1 = simulate)
    std::vector<int> width;                 // W per point
    std::vector<double> cost;
    std::vector<ClassDesc> classes;
    std::vector<uint32_t> coll_list, pipe_list;
    DevBuf<ClassDesc> d_cls;
    DevBuf<uint32_t> d_coll_list, d_pipe_list;
    DevBuf<double> d_dur;
    DevBuf<OpHook> d_hooks;
    DevBuf<CollEnt> d_colls;
    DevBuf<int32_t> d_scr_i32;
    DevBuf<unsigned long long> d_scr_u64;
    DevBuf<uint32_t> d_plans;
    DevBuf<StageInfo> d_stages;
    DevBuf<StageEnt> d_ents;
    DevBuf<SendEnt> d_sends;
    DevBuf<RecvEnt> d_recvs;
    DevBuf<HStage> d_hst;
    DevBuf<HEnt> d_hents;
    DevBuf<HSend> d_hsends;
    std::vector<uint32_t> hyb_list;
    DevBuf<uint32_t> d_hyb_list;
    DevBuf<TopoDev> d_topo;
    DevBuf<double> d_bw, d_lat;
    DevBuf<uint32_t> d_rt_off, d_ro;
    DevBuf<uint8_t> d_rt_len;
    DevBuf<uint16_t> d_rt_links;
    DevBuf<PointDesc> d_pts;
    DevBuf<triosim_result> d_res;
    std::vector<uint32_t> work[N_GROUPS];    // per (W index, mode)
    DevBuf<uint32_t> d_work[N_GROUPS];
    std::vector<int> mode;                   // per point
    uint32_t lmax[N_GROUPS] = {};            // hybrid CTA groups: largest topology (links) among their points
    uint32_t pmax[N_GROUPS] = {};            // hybrid groups: most photonic ports among their points (R20)
    int occ[N_GROUPS] = {};                  // hybrid CTA groups: resident CTAs per SM at that smem
    DevBuf<unsigned int> d_counter;
    DevBuf<unsigned long long> d_alg;
    cudaStream_t last_stream = nullptr;
    cudaEvent_t ev_done = nullptr;           // recorded on last_stream after the last simulate_batch's K3 joins
    // R22 per-layer breakdown (triosim_set_breakdown): per-class layer compute, per-point [3][L]
    // communication accumulators, staging for host-bound copies
    bool bd = false;
    DevBuf<double> d_lcomp, d_bd_acc, d_bd_stage;
    // R23 timeline of one point (triosim_timeline)
    DevBuf<triosim_task_rec> d_tl_tasks;
    DevBuf<triosim_flow_rec> d_tl_flows;
    DevBuf<unsigned long long> d_tl_cnt;
    DevBuf<uint32_t> d_one;
};

int w_index(int W) { int i = 0; while ((2 << i) < W) i++; return i; }
const int W_OF[N_WIDTHS] = {2, 4, 8, 16, 32, 64, 128, 256, 512, 1024};

}  // namespace

struct triosim_ctx {
    int device = 0;
    int n_sms = 148;
    std::string err;
    std::map<int, std::unique_ptr<Trace>> traces;
    std::map<int, std::unique_ptr<Sweep>> sweeps;
    int next_handle = 1;
    cudaStream_t side[N_GROUPS] = {};
    cudaEvent_t ev_fork = nullptr, ev_join[N_GROUPS] = {};
    uint64_t n_k1 = 0, n_k2 = 0, n_k3 = 0;
    int occ[N_GROUPS] = {};
    // optional CUDA-event timing of each simulate_batch (recorded on the caller's stream)
    static constexpr int NT = 512;
    bool timing = false;
    int n_timed = 0;
    cudaEvent_t t_begin[NT] = {}, t_mid[NT] = {}, t_end[NT] = {};
};

static triosim_status fail(triosim_ctx *c, triosim_status st, const char *fmt, ...) {
    char buf[512];
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(buf, sizeof buf, fmt, ap);
    va_end(ap);
    if (c) c->err = buf;
    return st;
}
#define CK(call)                                                                                    \
    do {                                                                                            \
        cudaError_t _e = (call);                                                                    \
        if (_e != cudaSuccess)                                                                      \
            return fail(ctx, _e == cudaErrorMemoryAllocation ? TRIOSIM_ENOMEM : TRIOSIM_ECUDA,      \
                        "%s: %s (%s:%d)", #call, cudaGetErrorString(_e), __FILE__, __LINE__);       \
    } while (0)

extern "C" {

static std::vector<uint32_t> stage_partition(const triosim_op *ops, uint32_t n_ops, uint32_t L, uint32_t S);

triosim_status triosim_create(int cuda_device, triosim_ctx **out) {
    if (!out) return TRIOSIM_EINVAL;
    *out = nullptr;
    int n = 0;
    if (cudaGetDeviceCount(&n) != cudaSuccess || cuda_device < 0 || cuda_device >= n) return TRIOSIM_EUNSUPPORTED;
    cudaDeviceProp prop;
    if (cudaGetDeviceProperties(&prop, cuda_device) != cudaSuccess) return TRIOSIM_ECUDA;
    if (prop.major != 10 || prop.minor != 0) return TRIOSIM_EUNSUPPORTED;  // built for sm_100a only
    if (cudaSetDevice(cuda_device) != cudaSuccess) return TRIOSIM_ECUDA;
    auto *ctx = new (std::nothrow) triosim_ctx();
    if (!ctx) return TRIOSIM_ENOMEM;
    ctx->device = cuda_device;
    ctx->n_sms = prop.multiProcessorCount;
    for (int i = 0; i < N_GROUPS; i++) {
        if (cudaStreamCreateWithFlags(&ctx->side[i], cudaStreamNonBlocking) != cudaSuccess ||
            cudaEventCreateWithFlags(&ctx->ev_join[i], cudaEventDisableTiming) != cudaSuccess) {
            triosim_destroy(ctx);
            return TRIOSIM_ECUDA;
        }
        const int Wi = W_OF[i / N_MODES], md = i % N_MODES;
        ctx->occ[i] = md == MODE_HYBRID ? (Wi <= 32 ? k3h_max_blocks_per_sm(Wi, 0, 0) : 1)
                                        : Wi <= 32 ? k3_max_blocks_per_sm(Wi, md) : 1;
    }
    if (cudaEventCreateWithFlags(&ctx->ev_fork, cudaEventDisableTiming) != cudaSuccess) {
        triosim_destroy(ctx);
        return TRIOSIM_ECUDA;
    }
    *out = ctx;
    return TRIOSIM_OK;
}

void triosim_destroy(triosim_ctx *ctx) {
    if (!ctx) return;
    cudaSetDevice(ctx->device);
    cudaDeviceSynchronize();
    ctx->sweeps.clear();
    ctx->traces.clear();
    for (int i = 0; i < N_GROUPS; i++) {
        if (ctx->side[i]) cudaStreamDestroy(ctx->side[i]);
        if (ctx->ev_join[i]) cudaEventDestroy(ctx->ev_join[i]);
    }
    if (ctx->ev_fork) cudaEventDestroy(ctx->ev_fork);
    for (int i = 0; i < triosim_ctx::NT; i++) {
        if (ctx->t_begin[i]) cudaEventDestroy(ctx->t_begin[i]);
        if (ctx->t_mid[i]) cudaEventDestroy(ctx->t_mid[i]);
        if (ctx->t_end[i]) cudaEventDestroy(ctx->t_end[i]);
    }
    const int dev = ctx->device;
    delete ctx;
    block_cache().trim(dev);   // destroy gives the device memory back
}

const char *triosim_last_error(const triosim_ctx *ctx) { return ctx ? ctx->err.c_str() : "null context"; }

triosim_status triosim_stage_partition(const triosim_trace_desc *t, uint32_t n_stages, uint32_t *first_layer) {
    if (!t || !first_layer || !t->ops || t->n_ops == 0 || n_stages == 0) return TRIOSIM_EINVAL;
    uint32_t L = 0;
    for (uint32_t o = 0; o < t->n_ops; o++)
        if (t->ops[o].phase == TRIOSIM_PHASE_FWD) L = std::max(L, t->ops[o].layer + 1);
    if (n_stages > L) return TRIOSIM_EINVAL;
    for (uint32_t o = 0; o < t->n_ops; o++)
        if (t->ops[o].layer >= L || !(t->ops[o].time_s >= 0.0) || std::isinf(t->ops[o].time_s)) return TRIOSIM_EINVAL;
    const std::vector<uint32_t> fl = stage_partition(t->ops, t->n_ops, L, n_stages);
    std::copy(fl.begin(), fl.end(), first_layer);
    return TRIOSIM_OK;
}

triosim_status triosim_launch_counts(const triosim_ctx *ctx, uint64_t *k1, uint64_t *k2, uint64_t *k3) {
    if (!ctx) return TRIOSIM_EINVAL;
    if (k1) *k1 = ctx->n_k1;
    if (k2) *k2 = ctx->n_k2;
    if (k3) *k3 = ctx->n_k3;
    return TRIOSIM_OK;
}

// ------------------------------------------------------------------------------------------
// load_trace
// ------------------------------------------------------------------------------------------
triosim_status triosim_load_trace(triosim_ctx *ctx, const triosim_trace_desc *t, int32_t *trace_id) {
    if (!ctx || !t || !trace_id) return fail(ctx, TRIOSIM_EINVAL, "null argument");
    CK(cudaSetDevice(ctx->device));
    if (t->n_ops == 0 || t->trace_batch == 0 || !t->ops || (t->n_tensors && !t->tensors) || (t->n_io && !t->io))
        return fail(ctx, TRIOSIM_EINVAL, "empty trace or trace_batch == 0");
    auto tr = std::make_unique<Trace>();
    tr->ops.assign(t->ops, t->ops + t->n_ops);
    tr->ts.assign(t->tensors, t->tensors + t->n_tensors);
    tr->io.assign(t->io, t->io + t->n_io);
    tr->b0 = t->trace_batch;
    tr->prod.assign(t->n_tensors, -1);
    for (uint32_t x = 0; x < t->n_tensors; x++)
        if (tr->ts[x].category > TRIOSIM_CAT_OTHER) return fail(ctx, TRIOSIM_EINVAL, "tensor %u: bad category", x);
    int last_phase = 0;
    uint32_t next_layer = 0;
    for (uint32_t o = 0; o < t->n_ops; o++) {
        const triosim_op &op = tr->ops[o];
        if (op.phase > 2 || op.phase < last_phase) return fail(ctx, TRIOSIM_EINVAL, "op %u: phases not FWD* BWD* OPT*", o);
        last_phase = op.phase;
        if (op.phase == 2 && tr->first_opt < 0) tr->first_opt = (int32_t)o;
        if (!(op.time_s >= 0.0) || std::isinf(op.time_s)) return fail(ctx, TRIOSIM_EINVAL, "op %u: bad time", o);
        if ((uint64_t)op.io_off + op.n_in + op.n_out > t->n_io) return fail(ctx, TRIOSIM_EINVAL, "op %u: io out of range", o);
        if (op.tp_role > 7) return fail(ctx, TRIOSIM_EINVAL, "op %u: bad tp_role", o);
        if (op.phase == 0) {
            if (op.layer == next_layer) next_layer++;
            else if (op.layer > next_layer) return fail(ctx, TRIOSIM_EINVAL, "op %u: layers not numbered by first FWD use", o);
        } else if (op.layer >= next_layer) {
            return fail(ctx, TRIOSIM_EINVAL, "op %u: layer without FWD op", o);
        }
        for (uint32_t k = 0; k < op.n_in; k++)
            if (tr->io[op.io_off + k] >= t->n_tensors) return fail(ctx, TRIOSIM_EINVAL, "op %u: input id out of range", o);
        for (uint32_t k = 0; k < op.n_out; k++) {
            uint32_t x = tr->io[op.io_off + op.n_in + k];
            if (x >= t->n_tensors) return fail(ctx, TRIOSIM_EINVAL, "op %u: output id out of range", o);
            if (tr->prod[x] != -1) return fail(ctx, TRIOSIM_EINVAL, "tensor %u produced twice", x);
            tr->prod[x] = (int32_t)o;
        }
        tr->n_out_total += op.n_out;
        tr->n_in_total += op.n_in;
    }
    for (uint32_t o = 0; o < t->n_ops; o++) {
        const triosim_op &op = tr->ops[o];
        for (uint32_t k = 0; k < op.n_in; k++)
            if (tr->prod[tr->io[op.io_off + k]] >= (int32_t)o) return fail(ctx, TRIOSIM_EINVAL, "op %u reads a tensor before it is produced", o);
    }
    tr->n_layers = next_layer;
    if (tr->n_layers == 0) return fail(ctx, TRIOSIM_EINVAL, "no FWD op");
    for (uint32_t x = 0; x < t->n_tensors; x++)
        if (tr->ts[x].category == TRIOSIM_CAT_WGRAD && tr->prod[x] >= 0 && tr->ops[tr->prod[x]].phase != 2) {
            tr->n_wgrad++;
            tr->wgrad_bytes += tr->ts[x].bytes_b0;
        }
    // stage to the device and run the ingest kernel
    CK(tr->d_ops.upload(tr->ops));
    CK(tr->d_ts.upload(tr->ts));
    CK(tr->d_io.upload(tr->io));
    CK(tr->d_time.alloc(t->n_ops));
    CK(tr->d_info.alloc(t->n_ops));
    CK(tr->d_layer.alloc(t->n_ops));
    CK(tr->d_wgrad.alloc(std::max<uint32_t>(tr->n_wgrad, 1)));
    CK(tr->d_prod.alloc(std::max<uint32_t>(t->n_tensors, 1)));
    CK(tr->d_scal.alloc(4));
    CK(cudaMemset(tr->d_prod.p, 0xff, sizeof(int32_t) * std::max<uint32_t>(t->n_tensors, 1)));
    int32_t scal0[4] = {0, INT32_MAX, -1, 0};
    CK(cudaMemcpy(tr->d_scal.p, scal0, sizeof scal0, cudaMemcpyHostToDevice));
    TraceDev &D = tr->dev;
    D.ops = tr->d_ops.p; D.ts = tr->d_ts.p; D.io = tr->d_io.p;
    D.time = tr->d_time.p; D.info = tr->d_info.p; D.layer = tr->d_layer.p; D.prod = tr->d_prod.p;
    D.wgrad = tr->d_wgrad.p; D.scal = tr->d_scal.p;
    D.n_ops = t->n_ops; D.n_ts = t->n_tensors; D.n_io = t->n_io; D.b0 = t->trace_batch; D.n_layers = tr->n_layers;
    D.pad = 0;
    CK(launch_k1_ingest(D, 0));
    ctx->n_k1++;
    CK(cudaDeviceSynchronize());
    int h = ctx->next_handle++;
    ctx->traces[h] = std::move(tr);
    *trace_id = h;
    return TRIOSIM_OK;
}

// ------------------------------------------------------------------------------------------
// host helpers: routing (BFS, ascending neighbours, first discovery) and the PP partition
// ------------------------------------------------------------------------------------------
// R8 automatic stage plan ("automatically assigns layers to GPUs to balance workloads"): the
// contiguous partition of the L layers into S stages that minimises the largest stage cost -- the
// left fold, in layer order, of the per-layer sums of trace times -- with ties broken towards the
// lexicographically smallest vector of first layers.  Computed here as (1) a binary search of the
// optimum V over the sorted candidate stage costs, with feasibility "the suffix from layer i splits
// into s stages of cost <= V" decided per V by interval reachability (a stage starting at i may end
// anywhere up to the last layer whose fold from i stays <= V, because adding non-negative times
// never decreases a fold), then (2) a left-to-right pass taking each stage's end as early as the
// rest stays feasible.  O(S L log L) per plan; pinned by exhaustive search (tests/test_abi_cpu.py).
static std::vector<uint32_t> stage_partition(const triosim_op *ops, uint32_t n_ops, uint32_t L, uint32_t S) {
    std::vector<double> lc(L, 0.0);
    for (uint32_t o = 0; o < n_ops; o++) lc[ops[o].layer] = lc[ops[o].layer] + ops[o].time_s;
    // fold[a][b - a]: left fold of lc[a..b]; end[a] (per V): last b with fold(a, b) <= V
    std::vector<std::vector<double>> fold(L);
    std::vector<double> cand;
    cand.reserve((size_t)L * (L + 1) / 2);
    for (uint32_t a = 0; a < L; a++) {
        fold[a].resize(L - a);
        double s = 0.0;
        for (uint32_t b = a; b < L; b++) { s = s + lc[b]; fold[a][b - a] = s; cand.push_back(s); }
    }
    std::sort(cand.begin(), cand.end());
    cand.erase(std::unique(cand.begin(), cand.end()), cand.end());
    // ok[s][i] (s = 1..S, i = 0..L): layers i..L-1 split into exactly s non-empty stages of cost <= V
    std::vector<std::vector<char>> ok(S + 1, std::vector<char>(L + 1, 0));
    std::vector<uint32_t> last(L);
    std::vector<uint32_t> pre(L + 2);
    auto feasible = [&](double V) -> bool {
        for (uint32_t a = 0; a < L; a++) {
            // fold(a, .) is non-decreasing: binary search the last end that fits
            const auto &f = fold[a];
            last[a] = (uint32_t)(std::upper_bound(f.begin(), f.end(), V) - f.begin());   // stages a..a+last-1 fit
        }
        for (uint32_t i = 0; i <= L; i++) ok[1][i] = (i < L && last[i] == L - i);
        for (uint32_t s = 2; s <= S; s++) {
            // ok[s][i] = any ok[s-1][j] for j in [i+1, i+last[i]]: prefix counts of ok[s-1]
            pre[0] = 0;
            for (uint32_t j = 0; j <= L; j++) pre[j + 1] = pre[j] + (ok[s - 1][j] ? 1u : 0u);
            for (uint32_t i = 0; i <= L; i++) {
                ok[s][i] = 0;
                if (i < L && last[i] >= 1) {
                    const uint32_t lo = i + 1, hi = i + last[i];   // inclusive
                    ok[s][i] = pre[hi + 1] - pre[lo] > 0;
                }
            }
        }
        return ok[S][0] != 0;
    };
    size_t lo = 0, hi = cand.size() - 1;   // cand[hi] (the whole fold's max) is always feasible for S <= L
    while (lo < hi) {
        const size_t mid = lo + (hi - lo) / 2;
        if (feasible(cand[mid])) hi = mid; else lo = mid + 1;
    }
    feasible(cand[lo]);
    std::vector<uint32_t> fl(S, 0);
    uint32_t i = 0;
    for (uint32_t k = 1; k < S; k++) {
        const uint32_t rest = S - k;   // stages still to place after this one
        uint32_t j = i + 1;
        while (j < L && !(j <= i + last[i] && ok[rest][j])) j++;
        fl[k] = j;
        i = j;
    }
    return fl;
}
static std::vector<uint32_t> auto_partition(const Trace &T, int S) {
    return stage_partition(T.ops.data(), (uint32_t)T.ops.size(), T.n_layers, (uint32_t)S);
}

struct HostTopo {
    uint32_t n_nodes, n_gpus, n_links, max_hops;
    bool photonic = false;
    triosim_photonic ph = {};
    std::vector<uint32_t> ro;
    std::vector<uint32_t> rt_off;   // n_gpus^2
    std::vector<uint8_t> rt_len;
    std::vector<uint16_t> links;    // route pool (local)
};

static triosim_status prep_topology(triosim_ctx *ctx, const triosim_topology &tp, uint32_t idx, HostTopo &H) {
    if (tp.n_gpus == 0 || tp.n_gpus > tp.n_nodes || (tp.n_links && !tp.links))
        return fail(ctx, TRIOSIM_EINVAL, "topology %u: bad sizes", idx);
    H.n_nodes = tp.n_nodes; H.n_gpus = tp.n_gpus; H.n_links = tp.n_links; H.max_hops = 0;
    if (tp.net_model > TRIOSIM_NET_PHOTONIC) return fail(ctx, TRIOSIM_EINVAL, "topology %u: unknown net_model", idx);
    H.photonic = tp.net_model == TRIOSIM_NET_PHOTONIC;
    if (H.photonic) {
        if (!tp.photonic) return fail(ctx, TRIOSIM_EINVAL, "topology %u: photonic parameters missing", idx);
        H.ph = *tp.photonic;
        const triosim_photonic &P = H.ph;
        if (P.ports == 0 || P.ports > (uint32_t)MAX_PORTS || !(P.link_bw_Bps > 0.0) || std::isinf(P.link_bw_Bps) ||
            !(P.setup_s >= 0.0) || std::isinf(P.setup_s) || !(P.lat_s >= 0.0) || std::isinf(P.lat_s))
            return fail(ctx, TRIOSIM_EINVAL, "topology %u: photonic ports must be 1..%d, bw > 0, setup/lat >= 0",
                        idx, MAX_PORTS);
    }
    std::vector<std::vector<std::pair<uint32_t, uint32_t>>> adj(tp.n_nodes);
    std::vector<std::vector<uint32_t>> seen(tp.n_nodes);
    for (uint32_t e = 0; e < tp.n_links; e++) {
        const triosim_link &l = tp.links[e];
        if (l.src >= tp.n_nodes || l.dst >= tp.n_nodes || l.src == l.dst)
            return fail(ctx, TRIOSIM_EINVAL, "topology %u link %u: bad endpoints", idx, e);
        if (!(l.bw_Bps > 0.0) || std::isinf(l.bw_Bps) || !(l.lat_s >= 0.0) || std::isinf(l.lat_s))
            return fail(ctx, TRIOSIM_EINVAL, "topology %u link %u: bw must be > 0, lat >= 0", idx, e);
        for (uint32_t d : seen[l.src])
            if (d == l.dst) return fail(ctx, TRIOSIM_EINVAL, "topology %u: duplicate link %u->%u", idx, l.src, l.dst);
        seen[l.src].push_back(l.dst);
        adj[l.src].push_back({l.dst, e});
    }
    for (auto &v : adj) std::sort(v.begin(), v.end());
    H.ro.resize(tp.n_gpus);
    std::vector<char> used(tp.n_gpus, 0);
    for (uint32_t i = 0; i < tp.n_gpus; i++) {
        uint32_t g = tp.ring_order ? tp.ring_order[i] : i;
        if (g >= tp.n_gpus || used[g]) return fail(ctx, TRIOSIM_EINVAL, "topology %u: ring_order not a permutation", idx);
        used[g] = 1;
        H.ro[i] = g;
    }
    const uint32_t G = tp.n_gpus;
    H.rt_off.assign((size_t)G * G, 0);
    H.rt_len.assign((size_t)G * G, NO_ROUTE);
    std::vector<int32_t> par(tp.n_nodes);
    std::vector<uint32_t> q(tp.n_nodes);
    for (uint32_t s = 0; s < G; s++) {
        std::fill(par.begin(), par.end(), -2);
        par[s] = -1;
        uint32_t qh = 0, qt = 0;
        q[qt++] = s;
        while (qh < qt) {
            uint32_t u = q[qh++];
            for (auto &pe : adj[u])
                if (par[pe.first] == -2) { par[pe.first] = (int32_t)pe.second; q[qt++] = pe.first; }
        }
        for (uint32_t d = 0; d < G; d++) {
            size_t k = (size_t)s * G + d;
            if (d == s) { H.rt_len[k] = 0; H.rt_off[k] = 0; continue; }
            if (par[d] == -2) continue;
            std::vector<uint16_t> path;
            for (uint32_t v = d; v != s; v = tp.links[par[v]].src) path.push_back((uint16_t)par[v]);
            std::reverse(path.begin(), path.end());
            if (path.size() > 250) continue;
            H.rt_off[k] = (uint32_t)H.links.size();
            H.rt_len[k] = (uint8_t)path.size();
            H.max_hops = std::max<uint32_t>(H.max_hops, (uint32_t)path.size());
            H.links.insert(H.links.end(), path.begin(), path.end());
        }
    }
    return TRIOSIM_OK;
}

// ------------------------------------------------------------------------------------------
// build_sweep
// ------------------------------------------------------------------------------------------
triosim_status triosim_build_sweep(triosim_ctx *ctx, int32_t trace_id, const triosim_topology *topos, uint32_t n_topos,
                                   const triosim_stage_plans *plans, const triosim_point *pts, uint64_t n_pts,
                                   int32_t *sweep_id) {
    if (!ctx || !sweep_id || (n_topos && !topos) || (n_pts && !pts)) return fail(ctx, TRIOSIM_EINVAL, "null argument");
    CK(cudaSetDevice(ctx->device));
    auto it = ctx->traces.find(trace_id);
    if (it == ctx->traces.end()) return fail(ctx, TRIOSIM_ENOTFOUND, "unknown trace %d", trace_id);
    Trace &T = *it->second;
    if (n_pts > (1ull << 31)) return fail(ctx, TRIOSIM_EINVAL, "too many points");
    if (plans && plans->n_plans && (!plans->off || !plans->first_layer)) return fail(ctx, TRIOSIM_EINVAL, "bad plans");
    if (plans && plans->n_plans && plans->off[0] != 0) return fail(ctx, TRIOSIM_EINVAL, "bad plans");
    if (plans)
        for (uint32_t k = 0; k < plans->n_plans; k++)
            if (plans->off[k + 1] < plans->off[k]) return fail(ctx, TRIOSIM_EINVAL, "bad plan offsets");

    PhaseTimer PT;
    static const int widen_from = getenv("TS_WIDEN_FROM") ? atoi(getenv("TS_WIDEN_FROM")) : 16;
    std::vector<HostTopo> HT(n_topos);
    for (uint32_t i = 0; i < n_topos; i++) {
        triosim_status st = prep_topology(ctx, topos[i], i, HT[i]);
        if (st != TRIOSIM_OK) return st;
    }
    PT.mark("topologies");
    auto S = std::make_unique<Sweep>();
    S->trace_handle = trace_id;
    S->n_pts = n_pts;
    S->status.assign(n_pts, -1);
    S->width.assign(n_pts, 0);
    S->cost.assign(n_pts, 0.0);
    S->mode.assign(n_pts, 0);
    std::vector<PointDesc> pdesc(n_pts);
    std::map<std::tuple<int, int, int, int, int, int, int, uint64_t, uint32_t, int, int>, uint32_t> cls_of;
    std::vector<uint32_t> plan_pool;
    const uint32_t N = (uint32_t)T.ops.size(), NT = (uint32_t)T.ts.size();

    // trace-level counts used for cost estimates
    uint32_t n_tp_coll[2] = {0, 0};
    for (const auto &op : T.ops) {
        for (uint32_t k = 0; k < op.n_out; k++) {
            uint8_t cat = T.ts[T.io[op.io_off + op.n_in + k]].category;
            if ((op.tp_role & 4) && (op.phase == 0 || (op.phase == 1 && cat == TRIOSIM_CAT_AGRAD))) n_tp_coll[0]++;
            if (((op.tp_role & 3) == 2 && op.phase == 0) || ((op.tp_role & 3) == 1 && op.phase == 1 && cat == TRIOSIM_CAT_AGRAD))
                n_tp_coll[1]++;
        }
    }

    decltype(cls_of)::key_type last_key{};
    uint32_t last_c = 0;
    bool have_last = false;
    for (uint64_t i = 0; i < n_pts; i++) {
        triosim_point pt = pts[i];
        auto setst = [&](int st) { S->status[i] = st; };
        // R3, in order
        if (pt.topo >= n_topos) { setst(TRIOSIM_PT_BAD_CONFIG); continue; }
        if (pt.strategy > TRIOSIM_HOP || (pt.strategy != TRIOSIM_HOP && pt.tp_mode > 1) ||
            pt.coll_algo > TRIOSIM_ALGO_RSAG || pt.ring_chunks > 16) {
            setst(TRIOSIM_PT_BAD_CONFIG);
            continue;
        }
        if (!(pt.bw_scale > 0.0) || std::isinf(pt.bw_scale) || !(pt.lat_scale >= 0.0) || std::isinf(pt.lat_scale)) {
            setst(TRIOSIM_PT_BAD_CONFIG);
            continue;
        }
        const HostTopo &tp = HT[pt.topo];
        const uint32_t dp = pt.dp, tpd = pt.tp, pp = pt.pp, mb = pt.microbatches;
        bool bad = dp == 0 || tpd == 0 || pp == 0;
        if (!bad && pt.strategy == TRIOSIM_HOP) {
            // R28: graph, an OPT op to apply updates, n even (double ring: n % 4 == 0), one iteration at least
            if (pt.tp_mode > TRIOSIM_HOP_DOUBLE_RING || T.first_opt < 0) { setst(TRIOSIM_PT_BAD_CONFIG); continue; }
            if (tpd != 1 || pp != 1 || mb == 0 || dp < 2 || dp % 2 || (pt.tp_mode == TRIOSIM_HOP_DOUBLE_RING && dp % 4) ||
                dp > tp.n_gpus) { setst(TRIOSIM_PT_BAD_DEGREES); continue; }
            if (pt.global_batch == 0 || pt.global_batch % dp != 0) { setst(TRIOSIM_PT_BAD_BATCH); continue; }
            // warp-segment kernel only: <= 32 workers on a flow-network topology that fits a segment's links
            int W = 0, W0 = 2;
            while (W0 < (int)dp) W0 <<= 1;
            if (!tp.photonic && tp.max_hops <= MAX_ROUTE_K3)
                for (int w = W0; w <= 32; w <<= 1)
                    if ((int)tp.n_links <= lmax_warp(w)) { W = w; break; }
            if (W == 0) { setst(TRIOSIM_PT_TOO_LARGE); continue; }
            const uint32_t b_loc = pt.global_batch / dp;
            auto key = std::make_tuple((int)TRIOSIM_HOP, (int)dp, (int)b_loc, (int)pt.tp_mode, 0, 0, 1, (uint64_t)0,
                                       (uint32_t)pt.hop, (int)mb, -2);
            uint32_t c;
            auto ci = cls_of.find(key);
            if (ci == cls_of.end()) {
                ClassDesc cd;
                std::memset(&cd, 0, sizeof cd);
                cd.mode = MODE_HOP;
                cd.strategy = TRIOSIM_HOP;
                cd.tp_mode = pt.tp_mode;   // the communication graph
                cd.p = dp;
                cd.m = mb;
                cd.tpdeg = 1;
                cd.dp = 1;
                cd.b_loc = b_loc;
                cd.nch = 1;
                cd.hop = pt.hop;
                cd.r_b = (double)b_loc / (double)T.b0;
                c = (uint32_t)S->classes.size();
                S->classes.push_back(cd);
                cls_of[key] = c;
            } else {
                c = ci->second;
            }
            PointDesc &pd = pdesc[i];
            pd.bw_scale = pt.bw_scale;
            pd.lat_scale = pt.lat_scale;
            pd.cls = c;
            pd.topo = pt.topo;
            pd.idx = (uint32_t)i;
            pd.pad = 0;
            S->width[i] = W;
            S->mode[i] = MODE_HOP;
            S->cost[i] = (double)mb * N * 2.0 + (double)mb * 4.0 * 16.0 * dp;
            continue;
        }
        if (!bad) {
            if ((pt.strategy == TRIOSIM_DP || pt.strategy == TRIOSIM_DDP) && (tpd != 1 || pp != 1)) bad = true;
            if (pt.strategy == TRIOSIM_TP && (dp != 1 || pp != 1)) bad = true;
            if (pt.strategy == TRIOSIM_PP && (dp != 1 || tpd != 1)) bad = true;
        }
        const bool piped = pt.strategy == TRIOSIM_PP || pt.strategy == TRIOSIM_HYBRID;
        if (!bad && piped && mb == 0) bad = true;
        if (!bad && (uint64_t)dp * tpd * pp > tp.n_gpus) bad = true;
        if (!bad && (pp > T.n_layers || pp > 64)) bad = true;
        if (bad) { setst(TRIOSIM_PT_BAD_DEGREES); continue; }
        const uint64_t mm = piped ? mb : 1;
        if (pt.global_batch == 0 || pt.global_batch % ((uint64_t)dp * mm) != 0) { setst(TRIOSIM_PT_BAD_BATCH); continue; }
        std::vector<uint32_t> plan;
        int plan_key = -1;
        if (piped && pt.stage_plan >= 0) {
            if (!plans || (uint32_t)pt.stage_plan >= plans->n_plans) { setst(TRIOSIM_PT_BAD_PLAN); continue; }
            uint32_t a0 = plans->off[pt.stage_plan], a1 = plans->off[pt.stage_plan + 1];
            plan.assign(plans->first_layer + a0, plans->first_layer + a1);
            bool ok = plan.size() == pp && plan[0] == 0;
            for (size_t s = 1; ok && s < plan.size(); s++) ok = plan[s] > plan[s - 1] && plan[s] < T.n_layers;
            if (!ok) { setst(TRIOSIM_PT_BAD_PLAN); continue; }
            plan_key = pt.stage_plan;
        }
        // GPU kernel limits: warp segments (<= 32 lanes, lmax_warp links) for DP / DDP / TP / PP; the
        // HYBRID kernel (warp segments up to 32 ranks, one point per CTA up to 1024 ranks, LMAX_CTA links)
        // for HYBRID and for DDP / TP / PP points beyond the warp kernels -- DDP = (dp,1,1,1),
        // TP = (1,tp,1,1), PP = (1,1,pp,m) reproduce those strategies bit for bit (R9, pinned)
        const uint32_t lanes = pt.strategy == TRIOSIM_TP ? tpd : pt.strategy == TRIOSIM_PP ? pp
                             : pt.strategy == TRIOSIM_HYBRID ? dp * tpd * pp : dp;
        auto lm = [&](bool h, int w) { return !h ? lmax_warp(w) : w <= 32 ? lmax_hybrid(w) : LMAX_CTA; };
        int W0 = 2;
        while (W0 < (int)lanes) W0 <<= 1;
        // DP / DDP / TP points of 9-16 GPUs run on twice their segment width (one point per warp): the
        // segments of a warp diverge on every event, and the spare lanes hash half of the ring
        // fast-forward's events (R19).  Widening 5-8-GPU points too was measured equal on C2 (3.59 vs 3.55 ms
        // per step) and 37 % slower on C3 (75.7 vs 55.3 ms: its TP = 8 points run the general path, where
        // the halved number of resident points costs a second wave) -- profiles/r2_ab_widen_minb.txt.
        // Results are identical for any W >= lanes.  TS_WIDEN_FROM=8 widens from 5 GPUs, 0 turns it off.
        if (widen_from > 0 && W0 >= widen_from && W0 < 32 && pt.strategy != TRIOSIM_PP && pt.strategy != TRIOSIM_HYBRID)
            W0 <<= 1;
        // photonic points (R20) always run in the HYBRID kernel, whose lanes own their logical links;
        // DataParallel maps to HYBRID with its buckets triggered after the backward pass
        int W = 0;
        bool dp_after = false;
        // R27's double binary tree runs in the hybrid kernel (its lanes hold tree B on a spare flow slot)
        // a warp kernel keeps owner bits for <= MAX_ROUTE_K3 hops: longer routes also go to the hybrid kernel
        if (pt.strategy != TRIOSIM_HYBRID && !tp.photonic && pt.coll_algo != TRIOSIM_ALGO_DBTREE && tp.max_hops <= MAX_ROUTE_K3)
            for (int w = W0; w <= 32; w <<= 1)
                if ((int)tp.n_links <= lm(false, w)) { W = w; break; }
        if (W == 0) {
            if (pt.strategy != TRIOSIM_HYBRID) {
                dp_after = pt.strategy == TRIOSIM_DP;
                if (pt.strategy != TRIOSIM_PP) pt.microbatches = 1;
                pt.strategy = TRIOSIM_HYBRID;
            }
            for (int w = W0; w <= 1024; w <<= 1)
                if (tp.photonic || (int)tp.n_links <= lm(true, w)) { W = w; break; }
        }
        // photonic tree collectives: a broadcast flow parent -> child lives in the child's lane but needs the
        // parent's logical links (ports are the sender's, R20); not supported by this kernel
        // (a class without collective groups -- dp = tp = 1 -- has no tree to run)
        if (tp.photonic && (pt.coll_algo == TRIOSIM_ALGO_TREE || pt.coll_algo == TRIOSIM_ALGO_DBTREE) && (dp > 1 || tpd > 1)) W = 0;
        // R27: tree B needs the other group's flow slot -- not with both a TP and a DP group
        if (pt.coll_algo == TRIOSIM_ALGO_DBTREE && dp > 1 && tpd > 1) W = 0;
        // K2's pipeline / hybrid expansion keeps the layer -> stage map in shared memory (K2P_MAX_LAYERS)
        if ((pt.strategy == TRIOSIM_PP || pt.strategy == TRIOSIM_HYBRID) && T.n_layers > K2P_MAX_LAYERS) W = 0;
        if (W == 0) { setst(TRIOSIM_PT_TOO_LARGE); continue; }
        const uint32_t mbe = pt.microbatches;   // after a DDP / TP -> HYBRID mapping this is 1
        // structural class
        const bool hyb = pt.strategy == TRIOSIM_HYBRID;
        const int mode = hyb ? MODE_HYBRID : pt.strategy == TRIOSIM_PP ? MODE_PIPE : MODE_COLL;
        uint32_t b_loc = pt.strategy == TRIOSIM_TP ? pt.global_batch
                       : pt.strategy == TRIOSIM_PP ? pt.global_batch / mbe
                       : hyb ? pt.global_batch / (dp * mbe) : pt.global_batch / dp;
        int key_mode = (pt.strategy == TRIOSIM_TP || hyb) ? pt.tp_mode : 0;
        int key_algo = mode != MODE_PIPE ? pt.coll_algo : 0;
        uint64_t key_bucket = (pt.strategy == TRIOSIM_DP || pt.strategy == TRIOSIM_DDP || hyb) ? pt.bucket_bytes : 0;
        uint32_t key_first = key_bucket ? pt.first_bucket_bytes : 0;   // R24
        int key_m = (mode == MODE_PIPE || hyb) ? (int)mbe : 0;
        int key_nch = mode != MODE_PIPE && pt.ring_chunks > 1 ? (int)pt.ring_chunks : 1;   // R25
        auto key = std::make_tuple((int)pt.strategy + (dp_after ? 100 : 0), (int)lanes, (int)b_loc, key_mode, hyb ? (int)dp : 0,
                                   hyb ? (int)tpd : 0, key_algo * 32 + key_nch, key_bucket, key_first, key_m,
                                   (mode == MODE_PIPE || hyb) ? plan_key : -2);
        // consecutive points of a sweep usually share their class (bandwidth / latency scales are not part
        // of it): reuse the previous lookup
        uint32_t c;
        auto ci = (have_last && key == last_key) ? cls_of.end() : cls_of.find(key);
        if (have_last && key == last_key) {
            c = last_c;
        } else if (ci == cls_of.end()) {
            ClassDesc cd;
            std::memset(&cd, 0, sizeof cd);
            cd.mode = mode;
            cd.strategy = pt.strategy;
            cd.dp_after_bwd = dp_after ? 1u : 0u;
            cd.tp_mode = key_mode;
            cd.algo = key_algo;
            cd.p = hyb ? pp : lanes;
            cd.m = (mode == MODE_PIPE || hyb) ? mbe : 1;
            cd.tpdeg = (pt.strategy == TRIOSIM_TP || hyb) ? tpd : 1;
            cd.dp = hyb ? dp : 1;
            cd.b_loc = b_loc;
            cd.bucket_bytes = key_bucket;
            cd.first_bucket = key_first;
            cd.nch = (uint32_t)key_nch;
            cd.r_b = (double)b_loc / (double)T.b0;
            if (mode == MODE_PIPE || hyb) {
                if (plan_key < 0) {
                    auto ap = T.auto_plans.find((int)pp);
                    if (ap == T.auto_plans.end()) ap = T.auto_plans.emplace((int)pp, auto_partition(T, (int)pp)).first;
                    plan = ap->second;
                }
                cd.plan_off = (uint32_t)plan_pool.size();
                plan_pool.insert(plan_pool.end(), plan.begin(), plan.end());
            }
            c = (uint32_t)S->classes.size();
            S->classes.push_back(cd);
            cls_of[key] = c;
        } else {
            c = ci->second;
        }
        last_key = key;
        last_c = c;
        have_last = true;
        PointDesc &pd = pdesc[i];
        pd.bw_scale = pt.bw_scale;
        pd.lat_scale = pt.lat_scale;
        pd.cls = c;
        pd.topo = pt.topo;
        pd.idx = (uint32_t)i;
        pd.pad = 0;
        S->width[i] = W;
        // K3 variant: tree-capable collectives only for classes that use the tree algorithm
        S->mode[i] = (mode == MODE_COLL && pt.coll_algo == TRIOSIM_ALGO_TREE) ? MODE_TREE : mode;
        if (hyb) S->mode[i] = MODE_HYBRID;
        double cost;
        if (mode == MODE_COLL) {
            double ncol = pt.strategy == TRIOSIM_TP ? n_tp_coll[pt.tp_mode == TRIOSIM_TP_PAPER ? 0 : 1]
                        : (key_bucket == 0 ? T.n_wgrad : std::ceil((double)T.wgrad_bytes / (double)key_bucket));
            cost = (double)N * 2 + ncol * 2.0 * lanes * 8.0;
        } else if (hyb) {
            cost = (double)mbe * N * 2.0 / pp + (double)mbe * 16.0 * lanes;
        } else {
            cost = (double)mbe * N * 2.0 / lanes + (double)mbe * 2.0 * 8.0 * lanes;
        }
        S->cost[i] = cost;
    }

    PT.mark("points");
    // per-class pools
    uint32_t dur_n = 0, hook_n = 0, coll_n = 0, scr_i = 0, scr_u = 0, stage_n = 0, ent_n = 0, send_n = 0, recv_n = 0;
    uint32_t hst_n = 0, hent_n = 0, hsend_n = 0;
    for (uint32_t c = 0; c < S->classes.size(); c++) {
        ClassDesc &cd = S->classes[c];
        cd.dur_off = dur_n; dur_n += N;
        if (cd.mode == MODE_COLL || cd.mode == MODE_HOP) {
            S->coll_list.push_back(c);
            cd.hook_off = hook_n; hook_n += N;
            cd.coll_cap = cd.mode == MODE_HOP ? 0 : (cd.strategy == TRIOSIM_TP) ? T.n_out_total : T.n_wgrad;
            if (cd.algo == TRIOSIM_ALGO_RSAG) cd.coll_cap *= 2;   // R29: ReduceScatter + AllGather per AllReduce
            cd.coll_off = coll_n; coll_n += cd.coll_cap;
            if (cd.strategy == TRIOSIM_TP) { cd.scratch_off = scr_i; scr_i += NT; }
        } else if (cd.mode == MODE_HYBRID) {
            S->hyb_list.push_back(c);
            cd.stage_off = stage_n; stage_n += cd.p;
            cd.hst_off = hst_n; hst_n += cd.p;
            cd.ent_off = hent_n; cd.ent_cap = N; hent_n += N;
            cd.send_cap = T.n_out_total * (cd.p > 1 ? cd.p - 1 : 1);
            cd.send_off = hsend_n; hsend_n += cd.send_cap;
            cd.recv_cap = T.n_in_total;
            cd.recv_off = recv_n; recv_n += cd.recv_cap;
            cd.tcol_cap = T.n_out_total * (cd.algo == TRIOSIM_ALGO_RSAG ? 2 : 1);
            cd.tcol_off = coll_n; coll_n += cd.tcol_cap;
            cd.dcol_cap = T.n_wgrad * (cd.algo == TRIOSIM_ALGO_RSAG ? 2 : 1);
            cd.dcol_off = coll_n; coll_n += cd.dcol_cap;
            cd.scratch_off = scr_u; scr_u += NT;
        } else {
            S->pipe_list.push_back(c);
            cd.stage_off = stage_n; stage_n += cd.p;
            cd.ent_off = ent_n; cd.ent_cap = N; ent_n += N;
            cd.send_cap = T.n_out_total * (cd.p > 1 ? cd.p - 1 : 1);
            cd.send_off = send_n; send_n += cd.send_cap;
            cd.recv_cap = T.n_in_total;
            cd.recv_off = recv_n; recv_n += cd.recv_cap;
            cd.scratch_off = scr_u; scr_u += NT;
        }
    }
    PT.mark("class pools");
    // topologies to the device
    std::vector<TopoDev> td(n_topos);
    std::vector<double> bw, lat;
    std::vector<uint32_t> rt_off, ro;
    std::vector<uint8_t> rt_len;
    std::vector<uint16_t> rt_links;
    for (uint32_t i = 0; i < n_topos; i++) {
        TopoDev &d = td[i];
        d.n_nodes = HT[i].n_nodes; d.n_gpus = HT[i].n_gpus; d.n_links = HT[i].n_links;
        d.link_off = (uint32_t)bw.size();
        for (uint32_t e = 0; e < topos[i].n_links; e++) { bw.push_back(topos[i].links[e].bw_Bps); lat.push_back(topos[i].links[e].lat_s); }
        d.rt_off = (uint32_t)rt_off.size();
        uint32_t base = (uint32_t)rt_links.size();
        for (size_t k = 0; k < HT[i].rt_off.size(); k++) { rt_off.push_back(HT[i].rt_off[k] + base); rt_len.push_back(HT[i].rt_len[k]); }
        rt_links.insert(rt_links.end(), HT[i].links.begin(), HT[i].links.end());
        d.ro_off = (uint32_t)ro.size();
        ro.insert(ro.end(), HT[i].ro.begin(), HT[i].ro.end());
        d.ring_disjoint_lo = d.ring_disjoint_hi = 0;
        d.net = HT[i].photonic ? TRIOSIM_NET_PHOTONIC : TRIOSIM_NET_FLOW;
        d.ports = HT[i].ph.ports; d.buf_slots = HT[i].ph.buf_slots; d.pad = 0;
        d.ph_bw = HT[i].ph.link_bw_Bps; d.ph_setup = HT[i].ph.setup_s; d.ph_lat = HT[i].ph.lat_s;
        if (!HT[i].photonic) {
            const HostTopo &Ht = HT[i];
            const uint32_t G = Ht.n_gpus;
            for (uint32_t pp = 2; pp <= std::min<uint32_t>(G, 32); pp++) {
                std::vector<char> seen(Ht.n_links, 0);
                bool ok = true;
                for (uint32_t r = 0; r < pp && ok; r++) {
                    const size_t k = (size_t)Ht.ro[r] * G + Ht.ro[(r + 1) % pp];
                    if (Ht.rt_len[k] == NO_ROUTE) { ok = false; break; }
                    for (uint32_t h = 0; h < Ht.rt_len[k]; h++) {
                        const uint16_t e = Ht.links[Ht.rt_off[k] + h];
                        if (seen[e]) { ok = false; break; }
                        seen[e] = 1;
                    }
                }
                if (ok) {
                    if (pp < 32) d.ring_disjoint_lo |= 1u << pp;
                    else d.ring_disjoint_hi |= 1u << (pp - 32);
                }
            }
        }
    }
    PT.mark("routes");
    CK(S->d_topo.upload(td));
    CK(S->d_bw.upload(bw));
    CK(S->d_lat.upload(lat));
    CK(S->d_rt_off.upload(rt_off));
    CK(S->d_rt_len.upload(rt_len));
    CK(S->d_rt_links.upload(rt_links));
    CK(S->d_ro.upload(ro));
    CK(S->d_cls.upload(S->classes));
    CK(S->d_coll_list.upload(S->coll_list));
    CK(S->d_pipe_list.upload(S->pipe_list));
    CK(S->d_hyb_list.upload(S->hyb_list));
    CK(S->d_hst.alloc(hst_n));
    CK(S->d_hents.alloc(hent_n));
    CK(S->d_hsends.alloc(hsend_n));
    CK(S->d_dur.alloc(dur_n));
    CK(S->d_hooks.alloc(hook_n));
    CK(S->d_colls.alloc(coll_n));
    CK(S->d_scr_i32.alloc(scr_i));
    CK(S->d_scr_u64.alloc(scr_u));
    CK(S->d_plans.upload(plan_pool));
    CK(S->d_stages.alloc(stage_n));
    CK(S->d_ents.alloc(ent_n));
    CK(S->d_sends.alloc(send_n));
    CK(S->d_recvs.alloc(recv_n));
    CK(S->d_pts.upload(pdesc));
    // result records: host-decided statuses now, simulated points overwritten by K3
    std::vector<triosim_result> res0(n_pts);
    std::memset(res0.data(), 0, sizeof(triosim_result) * n_pts);
    for (uint64_t i = 0; i < n_pts; i++) res0[i].status = S->status[i] < 0 ? TRIOSIM_PT_OK : S->status[i];
    CK(S->d_res.upload(res0));
    PT.mark("uploads");
    // work lists per width, most expensive first (LPT)
    // The cost estimate is a function of the structural class, so the order (cost desc, class, index)
    // is a counting sort by class followed by a sort of the classes (was a 10k-point stable_sort, 0.6 ms).
    // The order only schedules work; results do not depend on it.
    const size_t ncls = S->classes.size();
    std::vector<double> ccost(ncls, -1.0);
    std::vector<uint64_t> cstart(ncls + 1, 0);
    for (uint64_t i = 0; i < n_pts; i++)
        if (S->status[i] < 0) {
            const uint32_t c = pdesc[i].cls;
            cstart[c + 1]++;
            if (S->cost[i] > ccost[c]) ccost[c] = S->cost[i];
        }
    std::vector<uint32_t> corder(ncls);
    for (uint32_t c = 0; c < ncls; c++) corder[c] = c;
    std::sort(corder.begin(), corder.end(), [&](uint32_t a, uint32_t b) {
        if (ccost[a] != ccost[b]) return ccost[a] > ccost[b];
        return a < b;
    });
    std::vector<uint64_t> cpos(ncls, 0);
    {
        uint64_t off = 0;
        for (uint32_t c : corder) { cpos[c] = off; off += cstart[c + 1]; }
        cstart.back() = off;   // total simulated points
    }
    std::vector<uint64_t> order(cstart.back());
    for (uint64_t i = 0; i < n_pts; i++)
        if (S->status[i] < 0) order[cpos[pdesc[i].cls]++] = i;
    PT.mark("wl sort");
    for (uint64_t i : order) {
        const int g = N_MODES * w_index(S->width[i]) + S->mode[i];
        S->work[g].push_back((uint32_t)i);
        const HostTopo &ht = HT[pts[i].topo];
        if (S->width[i] > 32 && !ht.photonic) {
            const uint32_t r = (ht.n_links + 63) / 64 * 64;
            if (r > S->lmax[g]) S->lmax[g] = r;
        }
        if (ht.photonic && ht.ph.ports > S->pmax[g]) S->pmax[g] = ht.ph.ports;
    }
    for (int g = 0; g < N_GROUPS; g++)
        if (S->lmax[g] || S->pmax[g]) S->occ[g] = k3h_max_blocks_per_sm(W_OF[g / N_MODES], S->lmax[g], S->pmax[g]);
    PT.mark("wl lists");
    for (int w = 0; w < N_GROUPS; w++) {
        CK(S->d_work[w].upload(S->work[w]));
    }
    PT.mark("wl uploads");
    CK(S->d_counter.alloc(N_GROUPS));
    CK(S->d_alg.alloc(1));
    CK(cudaMemset(S->d_alg.p, 0, sizeof(unsigned long long)));
    PT.mark("work lists");
    CK(cudaDeviceSynchronize());
    PT.mark("sync");
    int h = ctx->next_handle++;
    T.n_sweeps++;
    ctx->sweeps[h] = std::move(S);
    *sweep_id = h;
    return TRIOSIM_OK;
}

// ------------------------------------------------------------------------------------------
// simulate_batch
// ------------------------------------------------------------------------------------------
// K1b + K2 for every class of the sweep (cheap; part of every step)
static cudaError_t enqueue_k1_k2(triosim_ctx *ctx, Sweep &S, Trace &T, cudaStream_t st) {
    const uint32_t ncls = (uint32_t)S.classes.size();
    cudaError_t e = launch_k1_rescale(S.d_cls.p, ncls, T.dev, S.d_dur.p, st);
    if (e != cudaSuccess) return e;
    if (ncls) ctx->n_k1++;
    e = launch_k2_coll(S.d_cls.p, S.d_coll_list.p, (uint32_t)S.coll_list.size(), T.dev, S.d_dur.p, S.d_hooks.p,
                       S.d_colls.p, S.d_scr_i32.p, st);
    if (e != cudaSuccess) return e;
    if (!S.coll_list.empty()) ctx->n_k2++;
    e = launch_k2_pipe(S.d_cls.p, S.d_pipe_list.p, (uint32_t)S.pipe_list.size(), T.dev, S.d_dur.p, S.d_plans.p,
                       S.d_stages.p, S.d_ents.p, S.d_sends.p, S.d_recvs.p, S.d_scr_u64.p, st);
    if (e != cudaSuccess) return e;
    if (!S.pipe_list.empty()) ctx->n_k2++;
    e = launch_k2_hybrid(S.d_cls.p, S.d_hyb_list.p, (uint32_t)S.hyb_list.size(), T.dev, S.d_plans.p, S.d_stages.p,
                         S.d_hst.p, S.d_hents.p, S.d_hsends.p, S.d_recvs.p, S.d_colls.p, S.d_scr_u64.p, S.d_dur.p, st);
    if (e != cudaSuccess) return e;
    if (!S.hyb_list.empty()) ctx->n_k2++;
    return cudaSuccess;
}

// K3 arguments shared by every launch group w of a sweep
static K3Args k3_args(Sweep &S, int w) {
    K3Args a;
    std::memset(&a, 0, sizeof a);
    a.counter = S.d_counter.p + w;
    a.pts = S.d_pts.p;
    a.cls = S.d_cls.p; a.topo = S.d_topo.p;
    a.link_bw = S.d_bw.p; a.link_lat = S.d_lat.p; a.rt_off = S.d_rt_off.p; a.rt_len = S.d_rt_len.p;
    a.rt_links = S.d_rt_links.p; a.ro = S.d_ro.p;
    a.hooks = S.d_hooks.p; a.colls = S.d_colls.p; a.dur = S.d_dur.p;
    a.stages = S.d_stages.p; a.ents = S.d_ents.p; a.sends = S.d_sends.p; a.recvs = S.d_recvs.p;
    a.hst = S.d_hst.p; a.hents = S.d_hents.p; a.hsends = S.d_hsends.p;
    a.out = S.d_res.p;
    a.alg_ops = S.d_alg.p;
    a.lmax = S.lmax[w];
    a.pmax = S.pmax[w];
    a.rlo = 0;
    a.rhi = 0xffffffffu;
    return a;
}

triosim_status triosim_simulate_batch(triosim_ctx *ctx, int32_t sweep_id, uint64_t first, uint64_t count,
                                      void *cuda_stream) {
    if (!ctx) return TRIOSIM_EINVAL;
    CK(cudaSetDevice(ctx->device));
    CK(cudaGetLastError());  // report sticky errors from earlier asynchronous work
    auto it = ctx->sweeps.find(sweep_id);
    if (it == ctx->sweeps.end()) return fail(ctx, TRIOSIM_ENOTFOUND, "unknown sweep %d", sweep_id);
    Sweep &S = *it->second;
    if (first > S.n_pts || count > S.n_pts - first) return fail(ctx, TRIOSIM_ERANGE, "range [%llu,+%llu) outside sweep of %llu",
                                                              (unsigned long long)first, (unsigned long long)count,
                                                              (unsigned long long)S.n_pts);
    Trace &T = *ctx->traces.at(S.trace_handle);
    cudaStream_t st = (cudaStream_t)cuda_stream;
    S.last_stream = st;
    const uint32_t ncls = (uint32_t)S.classes.size();
    const int slot = ctx->timing ? ctx->n_timed % triosim_ctx::NT : -1;
    if (slot >= 0) CK(cudaEventRecord(ctx->t_begin[slot], st));
    CK(enqueue_k1_k2(ctx, S, T, st));
    const uint32_t L = T.n_layers;
    if (S.bd) {
        CK(launch_k4_layer_compute(S.d_cls.p, ncls, T.dev, S.d_dur.p, S.d_stages.p, S.d_ents.p, S.d_hents.p,
                                   S.d_lcomp.p, st));
        CK(cudaMemsetAsync(S.d_bd_acc.p + first * 3 * L, 0, count * 3 * L * sizeof(double), st));
    }
    // K3 per segment width, forked onto side streams so the widths run concurrently
    const bool full = first == 0 && count == S.n_pts;
    CK(cudaMemsetAsync(S.d_counter.p, 0, N_GROUPS * sizeof(unsigned int), st));
    CK(cudaMemsetAsync(S.d_alg.p, 0, sizeof(unsigned long long), st));
    if (slot >= 0) CK(cudaEventRecord(ctx->t_mid[slot], st));
    CK(cudaEventRecord(ctx->ev_fork, st));
    int launched[N_GROUPS] = {};
    // groups in width order: the narrow groups' few CTAs take their SM slots first and finish early, then the
    // wide groups' persistent grids fill the GPU (launching the most expensive group first was measured 12 %
    // slower on C2: its persistent grid held every slot, serialising the narrow groups behind it)
    for (int w = 0; w < N_GROUPS; w++) {
        const uint32_t *wl = S.d_work[w].p;
        const uint32_t n_all = (uint32_t)S.work[w].size();
        uint32_t n = n_all;   // points of this group in [first, first + count): the kernel skips the rest
        if (!full) {
            n = 0;
            for (uint32_t i : S.work[w]) n += (i >= first && i < first + count) ? 1u : 0u;
        }
        if (n == 0) continue;
        const int W = W_OF[w / N_MODES], mode = w % N_MODES;
        K3Args a = k3_args(S, w);
        a.work = wl; a.n_work = n_all;
        a.rlo = (uint32_t)first;
        a.rhi = (uint32_t)(first + count);
        if (S.bd) {
            a.bd = S.d_bd_acc.p;
            a.layer = T.d_layer.p;
            a.n_layers = L;
        }
        uint64_t blocks;
        if (W <= 32) {
            const int nseg = 32 / W;
            const uint64_t warps = (n + nseg - 1) / nseg;
            blocks = (warps + K3_WARPS - 1) / K3_WARPS;
        } else {
            blocks = n;   // one point per CTA
        }
        const uint64_t cap = (uint64_t)ctx->n_sms * (uint64_t)((S.lmax[w] || S.pmax[w]) ? S.occ[w] : ctx->occ[w]);
        if (blocks > cap) blocks = cap;
        cudaError_t e = cudaStreamWaitEvent(ctx->side[w], ctx->ev_fork, 0);
        if (e == cudaSuccess)
            e = mode == MODE_HYBRID ? launch_k3_hybrid(W, a, (int)blocks, ctx->side[w])
                                    : launch_k3(W, mode, a, (int)blocks, ctx->side[w]);
        if (e == cudaSuccess) {
            ctx->n_k3++;
            e = cudaEventRecord(ctx->ev_join[w], ctx->side[w]);
            if (e == cudaSuccess) launched[w] = 1;
        }
        if (e != cudaSuccess) {
            // join the groups already running back into the caller's stream before reporting
            for (int v = 0; v < N_GROUPS; v++)
                if (launched[v]) cudaStreamWaitEvent(st, ctx->ev_join[v], 0);
            CK(e);
        }
    }
    for (int w = 0; w < N_GROUPS; w++)
        if (launched[w]) CK(cudaStreamWaitEvent(st, ctx->ev_join[w], 0));
    if (!S.ev_done) CK(cudaEventCreateWithFlags(&S.ev_done, cudaEventDisableTiming));
    CK(cudaEventRecord(S.ev_done, st));
    if (slot >= 0) {
        CK(cudaEventRecord(ctx->t_end[slot], st));
        ctx->n_timed++;
    }
    return TRIOSIM_OK;
}

triosim_status triosim_timing(triosim_ctx *ctx, int enable) {
    if (!ctx) return TRIOSIM_EINVAL;
    CK(cudaSetDevice(ctx->device));
    if (enable && !ctx->t_begin[0])
        for (int i = 0; i < triosim_ctx::NT; i++) {
            CK(cudaEventCreate(&ctx->t_begin[i]));
            CK(cudaEventCreate(&ctx->t_mid[i]));
            CK(cudaEventCreate(&ctx->t_end[i]));
        }
    ctx->timing = enable != 0;
    ctx->n_timed = 0;
    return TRIOSIM_OK;
}

int32_t triosim_timings(triosim_ctx *ctx, float *ms_total, float *ms_k3, int32_t max) {
    if (!ctx || !ctx->timing) return TRIOSIM_EINVAL;
    int n = ctx->n_timed < triosim_ctx::NT ? ctx->n_timed : triosim_ctx::NT;
    if (n > max) n = max;
    for (int i = 0; i < n; i++) {
        if (cudaEventSynchronize(ctx->t_end[i]) != cudaSuccess) return TRIOSIM_ECUDA;
        if (ms_total && cudaEventElapsedTime(&ms_total[i], ctx->t_begin[i], ctx->t_end[i]) != cudaSuccess) return TRIOSIM_ECUDA;
        if (ms_k3 && cudaEventElapsedTime(&ms_k3[i], ctx->t_mid[i], ctx->t_end[i]) != cudaSuccess) return TRIOSIM_ECUDA;
    }
    return n;
}

triosim_status triosim_results(triosim_ctx *ctx, int32_t sweep_id, uint64_t first, uint64_t count, triosim_result *out,
                               int out_is_device, void *cuda_stream) {
    if (!ctx || (count && !out)) return fail(ctx, TRIOSIM_EINVAL, "null argument");
    CK(cudaSetDevice(ctx->device));
    auto it = ctx->sweeps.find(sweep_id);
    if (it == ctx->sweeps.end()) return fail(ctx, TRIOSIM_ENOTFOUND, "unknown sweep %d", sweep_id);
    Sweep &S = *it->second;
    if (first > S.n_pts || count > S.n_pts - first) return fail(ctx, TRIOSIM_ERANGE, "range outside sweep");
    if (count == 0) return TRIOSIM_OK;
    cudaStream_t st = (cudaStream_t)cuda_stream;
    if (out_is_device) {
        // stream-ordered after the last simulate_batch even when that ran on another stream
        if (S.ev_done && S.last_stream != st) CK(cudaStreamWaitEvent(st, S.ev_done, 0));
        CK(cudaMemcpyAsync(out, S.d_res.p + first, count * sizeof(triosim_result), cudaMemcpyDeviceToDevice, st));
    } else {
        // the last simulate_batch may have run on another (non-blocking) stream: finish it first
        if (S.last_stream != st) CK(cudaStreamSynchronize(S.last_stream));
        CK(cudaMemcpyAsync(out, S.d_res.p + first, count * sizeof(triosim_result), cudaMemcpyDeviceToHost, st));
        CK(cudaStreamSynchronize(st));
    }
    return TRIOSIM_OK;
}

triosim_status triosim_timeline(triosim_ctx *ctx, int32_t sweep_id, uint64_t point, triosim_task_rec *tasks,
                                uint64_t task_cap, triosim_flow_rec *flows, uint64_t flow_cap, uint64_t *n_tasks,
                                uint64_t *n_flows) {
    if (!ctx || !n_tasks || !n_flows || (task_cap && !tasks) || (flow_cap && !flows))
        return fail(ctx, TRIOSIM_EINVAL, "null argument");
    CK(cudaSetDevice(ctx->device));
    CK(cudaGetLastError());
    auto it = ctx->sweeps.find(sweep_id);
    if (it == ctx->sweeps.end()) return fail(ctx, TRIOSIM_ENOTFOUND, "unknown sweep %d", sweep_id);
    Sweep &S = *it->second;
    if (point >= S.n_pts) return fail(ctx, TRIOSIM_ERANGE, "point %llu outside sweep", (unsigned long long)point);
    Trace &T = *ctx->traces.at(S.trace_handle);
    *n_tasks = *n_flows = 0;
    if (S.status[point] >= 0) return TRIOSIM_OK;   // decided on the host (R3): no timeline
    cudaStream_t st = nullptr;
    // K2's tables, the work counter and the result records are shared with simulate_batch: let its last
    // call (possibly on a non-blocking stream) finish first
    CK(cudaStreamSynchronize(S.last_stream));
    CK(enqueue_k1_k2(ctx, S, T, st));
    if (S.d_tl_tasks.n < task_cap || !S.d_tl_tasks.p) CK(S.d_tl_tasks.alloc(task_cap));
    if (S.d_tl_flows.n < flow_cap || !S.d_tl_flows.p) CK(S.d_tl_flows.alloc(flow_cap));
    if (!S.d_tl_cnt.p) CK(S.d_tl_cnt.alloc(2));
    if (!S.d_one.p) CK(S.d_one.alloc(1));
    const uint32_t pi = (uint32_t)point;
    CK(cudaMemcpyAsync(S.d_one.p, &pi, sizeof pi, cudaMemcpyHostToDevice, st));
    CK(cudaMemsetAsync(S.d_tl_cnt.p, 0, 2 * sizeof(unsigned long long), st));
    const int w = N_MODES * w_index(S.width[point]) + S.mode[point];
    CK(cudaMemsetAsync(S.d_counter.p + w, 0, sizeof(unsigned int), st));
    K3Args a = k3_args(S, w);
    a.work = S.d_one.p;
    a.n_work = 1;
    a.tl_tasks = S.d_tl_tasks.p;
    a.tl_flows = S.d_tl_flows.p;
    a.tl_cnt = S.d_tl_cnt.p;
    a.tl_task_cap = task_cap;
    a.tl_flow_cap = flow_cap;
    const int W = W_OF[w / N_MODES], mode = w % N_MODES;
    if (mode == MODE_HYBRID) CK(launch_k3_hybrid(W, a, 1, st));
    else CK(launch_k3(W, mode, a, 1, st));
    ctx->n_k3++;
    unsigned long long cnt[2] = {0, 0};
    int32_t pst = 0;
    CK(cudaMemcpyAsync(cnt, S.d_tl_cnt.p, sizeof cnt, cudaMemcpyDeviceToHost, st));
    CK(cudaMemcpyAsync(&pst, &S.d_res.p[point].status, sizeof pst, cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));
    if (pst != TRIOSIM_PT_OK) return TRIOSIM_OK;   // rejected in K3 (R3) or deadlocked: no timeline
    if (cnt[0] <= task_cap && cnt[1] <= flow_cap) CK(sort_timeline(S.d_tl_tasks.p, cnt[0], S.d_tl_flows.p, cnt[1], st));
    const uint64_t kt = cnt[0] < task_cap ? cnt[0] : task_cap, kf = cnt[1] < flow_cap ? cnt[1] : flow_cap;
    if (kt) CK(cudaMemcpyAsync(tasks, S.d_tl_tasks.p, kt * sizeof(triosim_task_rec), cudaMemcpyDeviceToHost, st));
    if (kf) CK(cudaMemcpyAsync(flows, S.d_tl_flows.p, kf * sizeof(triosim_flow_rec), cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));
    *n_tasks = cnt[0];
    *n_flows = cnt[1];
    return TRIOSIM_OK;
}

triosim_status triosim_set_breakdown(triosim_ctx *ctx, int32_t sweep_id, int enable) {
    if (!ctx) return TRIOSIM_EINVAL;
    CK(cudaSetDevice(ctx->device));
    auto it = ctx->sweeps.find(sweep_id);
    if (it == ctx->sweeps.end()) return fail(ctx, TRIOSIM_ENOTFOUND, "unknown sweep %d", sweep_id);
    Sweep &S = *it->second;
    const uint64_t L = ctx->traces.at(S.trace_handle)->n_layers;
    CK(cudaDeviceSynchronize());   // no launch of this sweep may still use the buffers
    S.bd = false;
    S.d_lcomp.alloc(0);
    S.d_bd_acc.alloc(0);
    S.d_bd_stage.alloc(0);
    if (!enable) return TRIOSIM_OK;
    if (S.d_lcomp.alloc(S.classes.size() * L) != cudaSuccess || S.d_bd_acc.alloc(S.n_pts * 3 * L) != cudaSuccess) {
        cudaGetLastError();
        S.d_lcomp.alloc(0);
        S.d_bd_acc.alloc(0);
        return fail(ctx, TRIOSIM_ENOMEM, "breakdown buffers: %llu points x %llu layers",
                    (unsigned long long)S.n_pts, (unsigned long long)L);
    }
    CK(cudaMemset(S.d_lcomp.p, 0, S.d_lcomp.n * sizeof(double) + (S.d_lcomp.n ? 0 : sizeof(double))));
    CK(cudaMemset(S.d_bd_acc.p, 0, S.d_bd_acc.n * sizeof(double) + (S.d_bd_acc.n ? 0 : sizeof(double))));
    S.bd = true;
    return TRIOSIM_OK;
}

triosim_status triosim_breakdown(triosim_ctx *ctx, int32_t sweep_id, uint64_t first, uint64_t count,
                                 double *layer_compute_s, double *layer_comm_s, int out_is_device, void *cuda_stream) {
    if (!ctx) return TRIOSIM_EINVAL;
    CK(cudaSetDevice(ctx->device));
    auto it = ctx->sweeps.find(sweep_id);
    if (it == ctx->sweeps.end()) return fail(ctx, TRIOSIM_ENOTFOUND, "unknown sweep %d", sweep_id);
    Sweep &S = *it->second;
    if (!S.bd) return fail(ctx, TRIOSIM_EINVAL, "breakdown not enabled on sweep %d (triosim_set_breakdown)", sweep_id);
    if (first > S.n_pts || count > S.n_pts - first) return fail(ctx, TRIOSIM_ERANGE, "range outside sweep");
    const uint64_t L = ctx->traces.at(S.trace_handle)->n_layers;
    if (count == 0 || L == 0) return TRIOSIM_OK;
    cudaStream_t st = (cudaStream_t)cuda_stream;
    if (out_is_device) {
        CK(launch_k4_breakdown(S.d_pts.p, S.d_res.p, first, count, (uint32_t)L, S.d_lcomp.p, S.d_bd_acc.p,
                               layer_compute_s, layer_comm_s, st));
        return TRIOSIM_OK;
    }
    const uint64_t n = count * L;
    if (S.d_bd_stage.n < 2 * n && S.d_bd_stage.alloc(2 * n) != cudaSuccess) {
        cudaGetLastError();
        return fail(ctx, TRIOSIM_ENOMEM, "breakdown staging buffer");
    }
    CK(launch_k4_breakdown(S.d_pts.p, S.d_res.p, first, count, (uint32_t)L, S.d_lcomp.p, S.d_bd_acc.p,
                           S.d_bd_stage.p, S.d_bd_stage.p + n, st));
    if (layer_compute_s) CK(cudaMemcpyAsync(layer_compute_s, S.d_bd_stage.p, n * sizeof(double), cudaMemcpyDeviceToHost, st));
    if (layer_comm_s) CK(cudaMemcpyAsync(layer_comm_s, S.d_bd_stage.p + n, n * sizeof(double), cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));
    return TRIOSIM_OK;
}

triosim_status triosim_work_counters(triosim_ctx *ctx, int32_t sweep_id, uint64_t *fp64_ops) {
    if (!ctx || !fp64_ops) return fail(ctx, TRIOSIM_EINVAL, "null argument");
    CK(cudaSetDevice(ctx->device));
    auto it = ctx->sweeps.find(sweep_id);
    if (it == ctx->sweeps.end()) return fail(ctx, TRIOSIM_ENOTFOUND, "unknown sweep %d", sweep_id);
    Sweep &S = *it->second;
    unsigned long long v = 0;
    CK(cudaMemcpyAsync(&v, S.d_alg.p, sizeof v, cudaMemcpyDeviceToHost, S.last_stream));
    CK(cudaStreamSynchronize(S.last_stream));
    *fp64_ops = v;
    return TRIOSIM_OK;
}

const void *triosim_results_device_ptr(const triosim_ctx *ctx, int32_t sweep_id) {
    if (!ctx) return nullptr;
    auto it = ctx->sweeps.find(sweep_id);
    return it == ctx->sweeps.end() ? nullptr : (const void *)it->second->d_res.p;
}

triosim_status triosim_release(triosim_ctx *ctx, int32_t handle) {
    if (!ctx) return TRIOSIM_EINVAL;
    cudaSetDevice(ctx->device);
    auto s = ctx->sweeps.find(handle);
    if (s != ctx->sweeps.end()) {
        cudaDeviceSynchronize();
        auto t = ctx->traces.find(s->second->trace_handle);
        if (t != ctx->traces.end()) t->second->n_sweeps--;
        ctx->sweeps.erase(s);
        return TRIOSIM_OK;
    }
    auto t = ctx->traces.find(handle);
    if (t != ctx->traces.end()) {
        if (t->second->n_sweeps > 0) return fail(ctx, TRIOSIM_EINVAL, "trace %d still used by a sweep", handle);
        cudaDeviceSynchronize();
        ctx->traces.erase(t);
        return TRIOSIM_OK;
    }
    return fail(ctx, TRIOSIM_ENOTFOUND, "unknown handle %d", handle);
}

}  // extern "C"
