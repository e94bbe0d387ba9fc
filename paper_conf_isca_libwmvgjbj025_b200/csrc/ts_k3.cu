// ts_k3.cu -- K3, the timeline kernel.
//
// One design point per W-lane segment of a warp (W = 2..32, 32/W points per warp).  Lane i of a
// segment is simulated GPU i: it owns that GPU's in-order compute stream and its single flow slot
// (ring step i -> i+1, tree edge, or the GPU's FIFO P2P send).  Segment-wide decisions are
// ballots / shuffles: collective start (all members ready), ring predecessor progress, the
// bottleneck share of each water-filling round, the next event time.
//
// Instant processing (R17) is ONE ordered pass -- completions, deliveries, activations,
// collective done / finish / start, releases, compute starts -- which is already a fixed point
// because every phase only consumes state produced by earlier phases; the pass repeats only when
// a zero-latency release or a zero-duration operator creates another event at the same instant.
// Then the max-min progressive filling (R14) re-allocates every in-transit flow if the active set
// changed, and the instant repeats if that made a flow drain now.
#include <cuda_runtime.h>
#include <cstdint>
#include <cstdio>
#include "ts_internal.h"

namespace ts {

#define FULL 0xffffffffu

enum { CS_IDLE = 0, CS_RUN = 1 };
enum { FS_NONE = 0, FS_LAT = 1, FS_ACT = 2 };
enum { EV_COLL_START = 1, EV_RELEASE = 2, EV_ACTIVATE = 3, EV_DELIVER = 4, EV_TASK_START = 5, EV_TASK_END = 6 };

__device__ __forceinline__ uint64_t mix64(uint64_t z) {
    z = (z ^ (z >> 30)) * 0xbf58476d1ce4e5b9ull;
    z = (z ^ (z >> 27)) * 0x94d049bb133111ebull;
    return z ^ (z >> 31);
}
__device__ __forceinline__ double dinf() { return __longlong_as_double(0x7ff0000000000000ll); }

#ifndef TS_SEGMIN_REDUX
#define TS_SEGMIN_REDUX 0
#endif
template <int W>
__device__ __forceinline__ double seg_min_shfl(double v) {
#pragma unroll
    for (int o = W / 2; o > 0; o >>= 1) {
        double w = __shfl_xor_sync(FULL, v, o);
        v = w < v ? w : v;
    }
    return v;
}
// minimum of a NON-NEGATIVE double over the lanes of `mask` (this lane's segment): such doubles
// order like their bit patterns, so two 32-bit warp reductions (REDUX) give the exact minimum
__device__ __forceinline__ double seg_min_redux(double v, unsigned mask) {
    const unsigned long long b = (unsigned long long)__double_as_longlong(v);
    const unsigned hi = (unsigned)(b >> 32), lo = (unsigned)b;
    const unsigned mhi = __reduce_min_sync(mask, hi);
    const unsigned mlo = __reduce_min_sync(mask, hi == mhi ? lo : 0xffffffffu);
    return __longlong_as_double((long long)(((unsigned long long)mhi << 32) | mlo));
}
template <int W>
__device__ __forceinline__ double seg_max(double v) {
#pragma unroll
    for (int o = W / 2; o > 0; o >>= 1) {
        double w = __shfl_xor_sync(FULL, v, o);
        v = w > v ? w : v;
    }
    return v;
}
template <int W>
__device__ __forceinline__ unsigned long long seg_sum_u64(unsigned long long v) {
#pragma unroll
    for (int o = W / 2; o > 0; o >>= 1) v += __shfl_xor_sync(FULL, v, o);
    return v;
}
template <int W>
__device__ __forceinline__ uint32_t seg_sum_u32(uint32_t v) {
#pragma unroll
    for (int o = W / 2; o > 0; o >>= 1) v += __shfl_xor_sync(FULL, v, o);
    return v;
}

struct Route {
    uint32_t off;
    int len;
};

// R28: neighbours of worker i in Fig. 16a's communication graphs, as a bit set over the n <= 32 workers
// (so they come out ascending): ring-based -- the ring neighbours and the most distant worker of i's
// group, the group being all n workers; double ring -- the same inside i's half, plus its counterpart
// in the other half.  Returns the degree; nb[] receives the ranks.
__device__ __forceinline__ int hop_nbrs(int n, int graph, int i, int (&nb)[4]) {
    const int h = graph == 1 ? n / 2 : n, base = i - i % h, j = i % h;
    uint32_t set = (1u << (base + (j + 1) % h)) | (1u << (base + (j + h - 1) % h)) | (1u << (base + (j + h / 2) % h));
    if (graph == 1) set |= 1u << ((i + h) % n);
    set &= ~(1u << i);
    int d = 0;
    while (set && d < 4) {
        nb[d++] = __ffs(set) - 1;
        set &= set - 1;
    }
    return d;
}

struct TopoRef {
    uint32_t n_gpus, link_off, rt_off, ro_off;
};

__device__ __forceinline__ Route get_route(const K3Args &a, const TopoRef &T, uint32_t s, uint32_t d) {
    const uint32_t k = T.rt_off + s * T.n_gpus + d;
    Route r;
    r.len = a.rt_len[k];
    r.off = a.rt_off[k];
    return r;
}

// route latency: left fold of link latency x lat_scale (R12); caches the first MAX_HOPS link ids (16
// bit each) in four registers for the water-filling rounds -- hops past them (at most MAX_ROUTE_K3) are
// read from rt_links at the route's offset
__device__ __forceinline__ double load_route(const K3Args &a, const TopoRef &T, Route r, double lat_scale,
                                             uint32_t (&hl)[4]) {
    double L = 0.0;
    hl[0] = hl[1] = hl[2] = hl[3] = 0;
#pragma unroll
    for (int h = 0; h < MAX_HOPS; h++)
        if (h < r.len) {
            const uint32_t e = a.rt_links[r.off + h];
            hl[h >> 1] |= e << (16 * (h & 1));
            L = L + a.link_lat[T.link_off + e] * lat_scale;
        }
    for (int h = MAX_HOPS; h < r.len; h++) L = L + a.link_lat[T.link_off + a.rt_links[r.off + h]] * lat_scale;
    return L;
}
__device__ __forceinline__ int hop(const uint32_t (&hl)[4], int h) { return (hl[h >> 1] >> (16 * (h & 1))) & 0xffff; }

#ifndef TS_K3_MINB
#define TS_K3_MINB 1
#endif
// V & V_BD: also record the per-layer communication breakdown (R22) into a.bd; V & V_LOG: record the
// R23 timeline (every task and flow with its times) -- separate instantiations, so the plain timeline
// carries none of their state
template <int W, int MODE, int V>
__global__ void __launch_bounds__(K3_THREADS, TS_K3_MINB) k3_timeline(const K3Args a) {
    constexpr bool BD = (V & V_BD) != 0;
    constexpr bool LOG = (V & V_LOG) != 0;
    constexpr int NSEG = 32 / W;
    constexpr int LMAX = lmax_warp(W);
    constexpr bool HOPM = MODE == MODE_HOP;    // R28 Hop decentralized training (update / token queues)
    constexpr bool COLL = MODE == MODE_COLL || MODE == MODE_TREE;   // DP / DDP / TP collectives
    constexpr bool TREE = MODE == MODE_TREE;   // ... some of which may be tree AllReduces
    __shared__ double s_res[K3_WARPS][NSEG * LMAX];
    __shared__ int s_n[K3_WARPS][NSEG * LMAX];
    __shared__ int s_k[K3_WARPS][NSEG * LMAX];
    __shared__ uint32_t s_cnt[K3_WARPS][COLL ? 1 : 32];
    // HOP: per worker lane and neighbour slot q, 1 + the last iteration whose update from that neighbour
    // was delivered (FIFO streams make it monotone); s_cnt holds each lane's finished backward passes
    __shared__ uint32_t s_rcv[K3_WARPS][HOPM ? 32 * 4 : 1];

    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    const int seg = lane / W, li = lane % W, sbase = seg * W;
    const unsigned smask = (W == 32 ? FULL : ((1u << (W & 31)) - 1u)) << sbase;
    double *lres = &s_res[wid][seg * LMAX];
    int *ln = &s_n[wid][seg * LMAX];
    int *lk = &s_k[wid][seg * LMAX];
    uint32_t *cnt = &s_cnt[wid][COLL ? 0 : sbase];
    uint32_t *rcv = &s_rcv[wid][HOPM ? sbase * 4 : 0];
    for (int q = lane; q < NSEG * LMAX; q += 32) { s_n[wid][q] = 0; s_k[wid][q] = 0; }
    __syncwarp();

    // ---- per-segment (uniform) state ----
    bool have = false, exhausted = false;
    uint32_t pidx = 0;
    double t = 0.0, bws = 1.0, lats = 1.0;
    int p = 1;
    int pred = 0;   // ring predecessor lane of this lane (li - 1 mod p)
    uint32_t ncoll = 0, m = 1;
    const ClassDesc *C = nullptr;
    TopoRef TR = {0, 0, 0, 0};
    uint32_t ninst = 0, nwf = 0, nrounds = 0, maxact = 0;
    bool bon = false;
    double bstart = 0.0, cbusy = 0.0;
    uint32_t cur = 0;
    bool running = false, tree_cur = false, tree_algo = false, ring_fast = false, ring_uni = false;
    bool rb_algo = false, rb_cur = false;   // R26: AllReduce as ring Reduce + ring Broadcast chains
    bool ring_ff = false;   // uniform ring whose lanes also share one route latency: ring fast-forward
#ifdef TS_WATCHDOG
    unsigned int wd_iter = 0;
#endif
#ifdef TS_PROF
    long long pf_ff = 0, pf_t0 = 0;
    unsigned int pf_gen = 0, pf_entries = 0;
#endif
    int K = 0, Kp = 0;   // this lane's / its ring predecessor's sends in the running collective
    double cS = 0.0, chunk = 0.0;
    // ---- per-lane state ----
    bool used = false;
    uint32_t gpu = 0, pos = 0, run_start = 0, run_end = 0, nprog = 0;
    int cst = CS_IDLE;
    int hwait = -1;           // COLL: cached wait of the head operator
    double t_end = 0.0, busy = 0.0;
    uint32_t ntask = 0, nflow = 0;
    uint32_t trig = 0, donec = 0;
    int D = 0;
    bool ldone = false, uprel = false, upd = false, dnrel = false, dnd = false, fup = false;
    Route rring = {0, 0};
    uint32_t hring[4] = {0, 0, 0, 0};
    double Lring = 0.0, rbw = 0.0;   // ring flow: route latency, min-hop bandwidth
    int fst = FS_NONE;
    double t_act = 0.0, rem = 0.0, rate = 0.0, t_upd = 0.0, t_drain = 0.0, fbytes = 0.0;
    int flen = 0;
    uint32_t hl[4] = {0, 0, 0, 0};
    uint32_t froff = 0;       // route offset of the flow in flight (hops past MAX_HOPS)
    uint64_t fcode = 0;
    StageInfo SI;
    SI.nF = SI.nB = SI.nO = SI.SF = SI.SB = SI.SO = 0;
    SI.ent_off = SI.send_off = SI.recv_off = 0;
    uint32_t sq = 0, nsend_tot = 0, dcnt = 0;
    // PIPE: the head operator's first unmet receive (lane, count it waits for) at program position hc_pos.
    // Counters only grow, so while that receive is still missing the head cannot start: an idle stage
    // re-checks one shared-memory counter per pass instead of re-reading its entry and receive tables
    uint32_t hc_pos = 0xffffffffu, hc_seq = 0;
    int hc_src = 0;
    // HOP (R28): neighbours (ranks, ascending) and this lane's slot in each neighbour's list; iteration
    // structure (ops per iteration, last non-OPT op, first OPT op); finished backward passes; the flow in
    // flight's destination lane, slot and iteration
    int hdeg = 0, hb = 0, hs = 0, hg = 0;
    int hnb[4] = {0, 0, 0, 0}, hsl[4] = {0, 0, 0, 0};
    uint32_t hN = 1, hlast = 0, hfirst = 0, hbwd = 0;
    int hdst = 0, hslot = 0;
    uint32_t hk = 0;
    double hS = 0.0;
    uint64_t acc = 0;            // this lane's part of the order hash (R19)
    uint32_t alg = 0;            // fp64 operations of the method performed by this lane (wraps per point only beyond 4e9)
    uint64_t tmix = 0;           // mix64(bits(t)) of the current instant
    bool nev = false;            // this lane recorded an event at the current instant
    // R22 (BD): the representative rank's current collective (rank 0) / P2P send (every stage):
    // start or release time and the layer it is attributed to; category 0 TP / 1 DP / 2 P2P
    double bd_t0 = 0.0;
    uint32_t bd_l = 0, bd_cat = 0;
    // R23 (LOG): record slot of this lane's flow in flight
    unsigned long long tl_fs = 0;
    auto tl_task = [&](uint32_t g, uint32_t prog, uint32_t op, uint32_t mb, double t0, double t1) {
        const unsigned long long k = atomicAdd(&a.tl_cnt[0], 1ull);
        if (k < a.tl_task_cap) {
            triosim_task_rec r;
            r.gpu = g; r.prog = prog; r.op = op; r.mb = mb; r.start_s = t0; r.end_s = t1;
            a.tl_tasks[k] = r;
        }
    };
    auto tl_release = [&](uint32_t src, uint32_t dst) {
        tl_fs = atomicAdd(&a.tl_cnt[1], 1ull);
        if (tl_fs < a.tl_flow_cap) {
            triosim_flow_rec r;
            r.code = fcode; r.src = src; r.dst = dst; r.bytes = fbytes; r.release_s = t;
            r.start_s = r.delivered_s = 0.0;
            a.tl_flows[tl_fs] = r;
        }
    };
    auto tl_start = [&]() { if (tl_fs < a.tl_flow_cap) a.tl_flows[tl_fs].start_s = t; };
    auto tl_deliver = [&]() { if (tl_fs < a.tl_flow_cap) a.tl_flows[tl_fs].delivered_s = t; };

#define EV(kind, code)                                                  \
    do {                                                                \
        acc += mix64(tmix ^ (((uint64_t)(kind) << 60) | (uint64_t)(code))); \
        nev = true;                                                     \
    } while (0)

    for (;;) {
        // ------------------------------ refill ------------------------------
        const bool need = !have && !exhausted;
        bool fresh = false, rbad = false, rlong = false;
        if (__any_sync(FULL, need)) {
          uint32_t it = 0;
          if (need && li == 0) it = atomicAdd(a.counter, 1u);
          it = __shfl_sync(FULL, it, sbase);
          if (need) {
            if (it >= a.n_work) {
                exhausted = true;
            } else if (a.work[it] < a.rlo || a.work[it] >= a.rhi) {
                // outside [first, first + count) of this simulate_batch call: skipped, refilled next pass
            } else {
                fresh = have = true;
#ifdef TS_PROF
                pf_ff = 0; pf_gen = 0; pf_entries = 0; pf_t0 = clock64();
#endif
#ifdef TS_WATCHDOG
                wd_iter = 0;
#endif
                const PointDesc pd = a.pts[a.work[it]];
                pidx = pd.idx;
                bws = pd.bw_scale;
                lats = pd.lat_scale;
                C = &a.cls[pd.cls];
                p = (int)C->p;
                {
                    const TopoDev td = a.topo[pd.topo];
                    TR.n_gpus = td.n_gpus; TR.link_off = td.link_off; TR.rt_off = td.rt_off; TR.ro_off = td.ro_off;
                    ring_fast = COLL && (p < 32 ? (td.ring_disjoint_lo >> p) & 1u : (td.ring_disjoint_hi >> (p - 32)) & 1u);
                }
                ncoll = C->n_coll;
                m = C->m;
                tree_algo = TREE && C->algo == TRIOSIM_ALGO_TREE;
                rb_algo = COLL && C->algo == TRIOSIM_ALGO_REDBCAST;
                if constexpr (BD) bd_cat = !COLL ? 2u : C->strategy == TRIOSIM_TP ? 0u : 1u;
                t = 0.0;
                tmix = mix64(0ull);
                ninst = nwf = nrounds = maxact = 0;
                bon = false;
                bstart = cbusy = 0.0;
                cur = 0;
                running = false;
                used = li < p;
                pred = sbase + (li == 0 ? p - 1 : li - 1);
                pos = run_start = run_end = 0;
                cst = CS_IDLE;
                t_end = busy = 0.0;
                ntask = nflow = 0;
                trig = donec = 0;
                D = 0;
                ldone = uprel = upd = dnrel = dnd = false;
                fst = FS_NONE;
                sq = dcnt = 0;
                hc_pos = 0xffffffffu;
                acc = alg = 0;
                nev = false;
                if (used) {
                    gpu = a.ro[TR.ro_off + li];
                    if constexpr (COLL) {
                        nprog = C->n_prog_max;
                        hwait = nprog > 0 ? a.hooks[C->hook_off].wait : -1;
                        rring = get_route(a, TR, gpu, a.ro[TR.ro_off + (li + 1) % p]);
                        if (C->need_ring && rring.len == NO_ROUTE) rbad = true;
                        if (rring.len != NO_ROUTE) {
                            Lring = load_route(a, TR, rring, lats, hring);
                            alg += 2 * rring.len;
                            // link-disjoint ring (host-checked): a ring flow is alone on each of its
                            // links, so its max-min share is its smallest bw * bw_scale (R14 with
                            // n_e = 1: res_e / 1.0 == res_e exactly)
                            rbw = dinf();
#pragma unroll
                            for (int h = 0; h < MAX_HOPS; h++)
                                if (h < rring.len) {
                                    const double b = a.link_bw[TR.link_off + hop(hring, h)] * bws;
                                    rbw = b < rbw ? b : rbw;
                                }
                            for (int h = MAX_HOPS; h < rring.len; h++) {
                                const double b = a.link_bw[TR.link_off + a.rt_links[rring.off + h]] * bws;
                                rbw = b < rbw ? b : rbw;
                            }
                            alg += 2 * rring.len;
                        }
                        if (C->need_tree && li >= 1) {
                            const uint32_t par = a.ro[TR.ro_off + (li - 1) / 2];
                            const int l1 = get_route(a, TR, gpu, par).len, l2 = get_route(a, TR, par, gpu).len;
                            if (l1 == NO_ROUTE || l2 == NO_ROUTE) rbad = true;
                        }
                    } else if constexpr (HOPM) {
                        hN = C->n_prog_max;
                        hlast = C->hop_last;
                        hfirst = C->hop_first;
                        hS = C->hop_S;
                        hb = (int)(C->hop & 15u);
                        hs = (int)((C->hop >> 4) & 15u);
                        hg = (int)((C->hop >> 8) & 255u);
                        nprog = m * hN;
                        hbwd = 0;
                        hdeg = hop_nbrs(p, (int)C->tp_mode, li, hnb);
                        nsend_tot = m * (uint32_t)hdeg;
                        for (int q = 0; q < 4; q++) {
                            rcv[li * 4 + q] = 0;
                            if (q < hdeg) {
                                int o4[4];
                                const int od = hop_nbrs(p, (int)C->tp_mode, hnb[q], o4);
                                for (int x = 0; x < od; x++) if (o4[x] == li) hsl[q] = x;
                                const int l = get_route(a, TR, gpu, a.ro[TR.ro_off + hnb[q]]).len;
                                if (l == NO_ROUTE) rbad = true;
                            }
                        }
                    } else {
                        SI = a.stages[C->stage_off + li];
                        nprog = m * (SI.nF + SI.nB) + SI.nO;
                        nsend_tot = m * (SI.SF + SI.SB) + SI.SO;
                        unsigned long long dm = SI.dst_mask;
                        while (dm) {
                            const int d = __ffsll((long long)dm) - 1;
                            dm &= dm - 1;
                            const int l = get_route(a, TR, gpu, a.ro[TR.ro_off + d]).len;
                            if (l == NO_ROUTE) rbad = true;
                        }
                    }
                }
            }
          }
          if constexpr (COLL) {
              // link-disjoint ring whose lanes all see the same min-hop bandwidth: every
              // water-filling call is a single round at that rate (R14)
              const double lo = seg_min_shfl<W>(used ? rbw : dinf());
              const double hi = seg_max<W>(used ? rbw : 0.0);
              const double llo = seg_min_shfl<W>(used ? Lring : dinf());
              const double lhi = seg_max<W>(used ? Lring : 0.0);
              if (fresh) {
                  ring_uni = ring_fast && lo == hi;
                  ring_ff = ring_uni && llo == lhi && llo > 0.0;
              }
          }
          if (__any_sync(FULL, fresh && (rbad || rlong))) {
              // a needed (src, dst) pair without a path (R3) / beyond this kernel's hop limit
              const bool bad = (__ballot_sync(FULL, fresh && rbad) & smask) != 0;
              const bool lng = (__ballot_sync(FULL, fresh && rlong) & smask) != 0;
              if (fresh && (bad || lng)) {
                  if (li == 0) {
                      triosim_result r = {};
                      r.status = bad ? TRIOSIM_PT_NO_ROUTE : TRIOSIM_PT_TOO_LARGE;
                      a.out[pidx] = r;
                  }
                  have = used = false;
              }
          }

        }
        // done when every segment has drained the work list (a segment whose point was just
        // rejected refills on the next iteration)
        if (__all_sync(FULL, !have && exhausted)) break;
#ifdef TS_WATCHDOG
        {
            static __device__ unsigned int wd_printed = 0;
            if (have && ++wd_iter > 2000000u) {
                if (atomicAdd(&wd_printed, 1u) < 16u)
                    printf("WD pidx=%u li=%d used=%d t=%.17g t_end=%.17g cst=%d fst=%d t_act=%.17g t_drain=%.17g D=%d K=%d cur=%u running=%d ring_ff=%d ldone=%d pos=%u nprog=%u\n",
                           pidx, li, (int)used, t, t_end, cst, fst, t_act, t_drain, D, K, cur, (int)running, (int)ring_ff, (int)ldone, pos, nprog);
                if (wd_iter > 2000010u) { have = false; exhausted = true; used = false; }
            }
        }
#endif

        // ------------------------- exact fast-forward of a uniform ring -------------------------
        // While a ring collective runs on a link-disjoint ring with one bandwidth and one route
        // latency, every lane releases, activates and delivers its step at the same instants:
        // activation at t_a (rate = rbw after one progressive-filling round, drain t_a + chunk/rbw)
        // and delivery + release of the next step at t_d (activation t_d + L).  Until the first
        // compute completion t_c (the only other pending event: the lanes' flows are all in this
        // collective and no operator can start before it is done), those instants are processed
        // here lane-locally, with exactly the arithmetic, events, hash terms and counters of the
        // general pass below (R13-R19) -- only without its warp-wide votes.  The collective's last
        // delivery, a zero-length drain / latency and any instant at or after t_c go to the
        // general pass.
#ifdef TS_PROF
        const long long pf_a = clock64();
#endif
        if constexpr (COLL && !LOG) {
            if (__any_sync(FULL, have && running && ring_ff && !tree_cur && !rb_cur)) {
                const double tc = seg_min_shfl<W>(used && cst == CS_RUN ? t_end : dinf());
                const int Dseg = __shfl_sync(FULL, D, sbase);
                // segment-uniform copies (every used lane holds the same values; unused lanes follow them)
                const double rbw0 = __shfl_sync(FULL, rbw, sbase), L0 = __shfl_sync(FULL, Lring, sbase);
                const bool okl = !used || (fst == FS_LAT && t_act == t && D == Dseg && flen > 0);
                const bool allok = (__ballot_sync(FULL, okl) & smask) == smask;   // (every lane votes)
                const bool ok = allok && have && running && ring_ff && !tree_cur && !rb_cur && chunk > 0.0 && Dseg < K && t < tc;
                if (ok) {
#ifdef TS_PROF
                    pf_entries++;
#endif
                    const double x = chunk / rbw0;  // = rem / rate at activation (rem = chunk, rate = rbw)
                    const uint64_t cbase = ((uint64_t)cur << 32) | (uint64_t)li;
                    int Dl = Dseg;                  // steps delivered so far; the flow in flight is step Dl
                    int lastk = -1;                 // kind of the last processed instant: 0 activation, 1 delivery
                    double tl = t;                  // ... and its time
                    bool go = true;
                    // blocks of up to four steps (eight instants): first the instant times (a short
                    // dependent chain of adds), then their hash terms, which are independent of each other
                    while (go) {
                        double ti[8] = {0.0, 0.0, 0.0, 0.0, 0.0, 0.0, 0.0, 0.0};
                        int n = 0;
                        const int D0 = Dl;
#pragma unroll
                        for (int i = 0; i < 8; i++) {
                            if (go) {
                                if ((i & 1) == 0) {   // activation of step Dl: drain at t + x
                                    const double td = t + x;
                                    if (t < tc && td > t) {
                                        ti[i] = tl = t;
                                        lastk = 0;
                                        n = i + 1;
                                        t = tc < td ? tc : td;   // next instant: the drain, or a compute completion first
                                    } else {
                                        go = false;
                                    }
                                } else {              // delivery of step Dl, release of step Dl + 1 (not the last)
                                    const double ta = t + L0;
                                    if (t < tc && Dl + 1 < K && ta > t) {
                                        ti[i] = tl = t;
                                        lastk = 1;
                                        n = i + 1;
                                        Dl++;
                                        t = tc < ta ? tc : ta;
                                    } else {
                                        go = false;
                                    }
                                }
                            }
                        }
                        // order-hash terms (R19).  With spare lanes (W >= 2p) the twin lane li + W/2 hashes
                        // instants 4..7 of member li and the member lane instants 0..3 (the segment's hash is
                        // the sum over all its lanes), halving the warp's mix64 work; else the member lane
                        // takes all eight.  All terms unconditionally (independent chains the compiler
                        // interleaves), the ones past n masked out of the sum
                        const bool split = 2 * p <= W;
                        const bool twin = split && li >= W / 2 && li - W / 2 < p;
                        // mix64 of the eight instant times: the same in every lane of the segment, so with W >= 8
                        // segment lane j computes instant j's and the others read it by shuffle (the block's
                        // control flow is segment-uniform: every lane of the segment is here)
                        uint64_t tmx[8];
                        if constexpr (W >= 8) {
                            const int j = li & 7;
                            double tj = ti[0];
#pragma unroll
                            for (int i = 1; i < 8; i++) tj = j == i ? ti[i] : tj;
                            const uint64_t mj = mix64((uint64_t)__double_as_longlong(tj));
#pragma unroll
                            for (int i = 0; i < 8; i++) tmx[i] = __shfl_sync(smask, mj, sbase + i);
                        }
                        if (used || twin) {
                            const uint64_t cb = ((uint64_t)cur << 32) | (uint64_t)(twin ? li - W / 2 : li);
                            // instant of parity `odd` (0 activation, 1 delivery + release) of step k, m = mix64 of
                            // its time
                            auto term = [&](uint64_t m, bool odd, int kk) -> uint64_t {
                                const uint64_t k = (uint64_t)kk;
                                if (!odd)
                                    return mix64(m ^ (((uint64_t)EV_ACTIVATE << 60) | cb | (k << 16)));
                                return mix64(m ^ (((uint64_t)EV_DELIVER << 60) | cb | (k << 16))) +
                                       mix64(m ^ (((uint64_t)EV_RELEASE << 60) | cb | ((k + 1) << 16)));
                            };
                            uint64_t add = 0;
                            if (split) {
                                const int off = twin ? 4 : 0;
#pragma unroll
                                for (int i = 0; i < 4; i++) {
                                    uint64_t m;
                                    if constexpr (W >= 8) m = twin ? tmx[i + 4] : tmx[i];
                                    else m = mix64((uint64_t)__double_as_longlong(twin ? ti[i + 4] : ti[i]));
                                    const uint64_t tr = term(m, (i & 1) != 0, D0 + ((i + off) >> 1));
                                    add += i + off < n ? tr : 0ull;
                                }
                            } else {
#pragma unroll
                                for (int i = 0; i < 8; i++) {
                                    uint64_t m;
                                    if constexpr (W >= 8) m = tmx[i];
                                    else m = mix64((uint64_t)__double_as_longlong(ti[i]));
                                    const uint64_t tr = term(m, (i & 1) != 0, D0 + (i >> 1));
                                    add += i < n ? tr : 0ull;
                                }
                            }
                            acc += add;
                        }
                        if (used) {
                            alg += 2u * (uint32_t)((n + 1) >> 1) + (uint32_t)(n >> 1);
                            nflow += (uint32_t)(n >> 1);
                        }
                        nrounds += (uint32_t)((n + 1) >> 1);
                        nwf += (uint32_t)n;
                        ninst += (uint32_t)n;
                        go = go && n == 8;
                    }
                    if (lastk >= 0) {
                        maxact = (uint32_t)p > maxact ? (uint32_t)p : maxact;
                        if (used) {
                            if (Dl != Dseg) {
                                D = Dl;
                                fcode = cbase | ((uint64_t)Dl << 16);
                            }
                            if (lastk == 0) {   // the step in flight is active, draining
                                fst = FS_ACT;
                                rem = chunk;
                                t_upd = tl;
                                rate = rbw;
                                t_drain = tl + x;
                            } else {            // the next step was released and is latent
                                fst = FS_LAT;
                                t_act = tl + L0;
                            }
                        }
                        tmix = mix64((uint64_t)__double_as_longlong(t));
                    }
                }
            }
        }

#ifdef TS_PROF
        pf_ff += clock64() - pf_a;
        if (have) pf_gen++;
#endif
        // ------------------------------ one instant at time t ------------------------------
        bool dirty = false;
        for (;;) {
            for (;;) {
                bool more = false;
                // (a) compute completions
                if (used && cst == CS_RUN && t_end == t) {
                    cst = CS_IDLE;
                    pos = run_end;
                    if constexpr (COLL) {
                        const uint32_t ns = a.hooks[C->hook_off + pos - 1].nsig;
                        if (ns) {
                            trig += ns;
                            EV(EV_TASK_END, ((uint64_t)gpu << 40) | (pos - 1));
                        }
                        hwait = pos < nprog ? a.hooks[C->hook_off + pos].wait : -1;
                    } else if constexpr (HOPM) {
                        // the run ends at the iteration's last non-OPT op: its update goes out (R28)
                        if ((pos - 1) % hN == hlast) {
                            hbwd++;
                            EV(EV_TASK_END, ((uint64_t)gpu << 40) | (pos - 1));
                        }
                    } else {
                        const uint32_t q = pos - 1;
                        uint32_t P, idx;
                        if (q < m * SI.nF) { P = 0; idx = q % SI.nF; }
                        else if (q < m * (SI.nF + SI.nB)) { P = 1; idx = (q - m * SI.nF) % SI.nB; }
                        else { P = 2; idx = q - m * (SI.nF + SI.nB); }
                        const uint32_t eo = SI.ent_off + (P == 0 ? 0 : P == 1 ? SI.nF : SI.nF + SI.nB) + idx;
                        if (a.ents[eo].nsend) EV(EV_TASK_END, ((uint64_t)gpu << 40) | q);
                    }
                }
                // (b) deliveries and (c) activations after the route latency (Q19)
                bool delivered = false;
                if (used && fst == FS_ACT && t_drain == t) {
                    fst = FS_NONE;
                    EV(EV_DELIVER, fcode);
                    if constexpr (LOG) tl_deliver();
                    delivered = dirty = true;
                } else if (used && fst == FS_LAT && t_act == t) {
                    EV(EV_ACTIVATE, fcode);
                    if constexpr (LOG) tl_start();
                    if (fbytes == 0.0 || flen == 0) {
                        fst = FS_NONE;
                        EV(EV_DELIVER, fcode);
                        if constexpr (LOG) tl_deliver();
                        delivered = true;
                    } else {
                        fst = FS_ACT;
                        rem = fbytes;
                        t_upd = t;
                        rate = 0.0;
                        t_drain = dinf();
                        dirty = true;
                    }
                }
                if (delivered) {
                    nflow++;
                    if constexpr (COLL) {
                        if (TREE && tree_cur) {
                            if (fup) upd = true; else dnd = true;
                        } else {
                            D++;
                        }
                    } else {
                        dcnt++;
                        if constexpr (HOPM) rcv[hdst * 4 + hslot] = hk + 1;   // update (hk) reached hdst (R28)
                        if constexpr (BD) {   // R22: P2P time of the sending (representative) stage / rank 0
                            if (!HOPM || li == 0) {
                                double *q = a.bd + ((size_t)pidx * 3 + 2) * a.n_layers + bd_l;
                                *q = *q + (t - bd_t0);
                            }
                        }
                    }
                }
                if constexpr (COLL) {
                    // (d) collective progress: done on this GPU, finish, start (R10)
                    const int Dp = __shfl_sync(FULL, D, pred);
                    unsigned upm = 0, dnm = 0;
                    if constexpr (TREE) {
                        if (__any_sync(FULL, tree_cur)) {
                            upm = (__ballot_sync(FULL, upd) & smask) >> sbase;
                            dnm = (__ballot_sync(FULL, dnd) & smask) >> sbase;
                        }
                    }
                    const int c1 = 2 * li + 1, c2 = 2 * li + 2;
                    if (used && running && !ldone) {
                        bool dn;
                        if (!TREE || !tree_cur) {
                            dn = D == K && Dp == Kp;
                        } else {
                            const bool ku = (c1 >= p || ((upm >> c1) & 1u)) && (c2 >= p || ((upm >> c2) & 1u));
                            const bool kd = (c1 >= p || ((dnm >> c1) & 1u)) && (c2 >= p || ((dnm >> c2) & 1u));
                            dn = (li == 0 || (upd && dnd)) && ku && kd;
                        }
                        if (dn) {
                            ldone = true;
                            donec = cur + 1;
                            if constexpr (BD)
                                if (li == 0) {   // R22: collective time on the representative rank
                                    double *q = a.bd + ((size_t)pidx * 3 + bd_cat) * a.n_layers + bd_l;
                                    *q = *q + (t - bd_t0);
                                }
                        }
                    }
                    const bool allfin = (__ballot_sync(FULL, !used || ldone) & smask) == smask;
                    if (have && running && allfin) {
                        running = false;
                        cur++;
                    }
                    const bool allrdy = (__ballot_sync(FULL, !used || trig > cur) & smask) == smask;
                    bool started = false;
                    if (have && !running && cur < ncoll && allrdy) {
                        // every member ready: the collective starts (barrier, Q22)
                        const CollEnt ce = a.colls[C->coll_off + cur];
                        running = started = true;
                        tree_cur = tree_algo && ce.kind == CK_AR;
                        cS = ce.S;
                        // R25: nch chunks of S / p / nch per ring step, sent one at a time (q = k nch + j)
                        chunk = ce.S / (double)p / (double)C->nch;
                        K = ((ce.kind == CK_AR) ? 2 * (p - 1) : (p - 1)) * (int)C->nch;
                        Kp = K;
                        rb_cur = rb_algo && ce.kind == CK_AR;
                        if (rb_cur) {
                            // R26: reduce chunks (members != 0), then broadcast chunks (members != p-1)
                            const int c = (int)C->nch, pl = li == 0 ? p - 1 : li - 1;
                            chunk = ce.S / (double)c;
                            K = (li != 0 ? c : 0) + (li != p - 1 ? c : 0);
                            Kp = (pl != 0 ? c : 0) + (pl != p - 1 ? c : 0);
                        }
                        D = 0;
                        ldone = uprel = upd = dnrel = dnd = false;
                        if (li == 0) { EV(EV_COLL_START, cur); alg += 1; }
                        if constexpr (BD) { bd_t0 = t; bd_l = ce.layer; }
                    }
                    if (used && running && fst == FS_NONE) {
                        bool rel = false;
                        if (!TREE || !tree_cur) {
                            const int c = (int)C->nch;
                            bool go;
                            if (!rb_cur) {
                                go = D < K && (D < c || Dp >= D - c + 1);
                            } else if (li != 0 && D < c) {   // R26 reduce chunk D: after the predecessor's
                                go = li == 1 || (!started && Dp >= D + 1);   // (member 1 starts the chain;
                            } else {                          // Dp is the previous collective's at its start)
                                const int j = D - (li != 0 ? c : 0);   // broadcast chunk j
                                go = D < K && !started && Dp >= (li == 0 || li == 1 ? 0 : c) + j + 1;
                            }
                            if (go) {
                                // ring step (i, k = D): m_i -> m_{i+1}, S/p bytes (Q21); R25: flat
                                // chunk index q = D waits for the predecessor's chunk q - nch
                                rel = true;
                                flen = rring.len;
                                hl[0] = hring[0]; hl[1] = hring[1]; hl[2] = hring[2]; hl[3] = hring[3];
                                froff = rring.off;
                                fbytes = chunk;
                                t_act = t + Lring;
                                alg += 1;
                                fcode = ((uint64_t)cur << 32) | ((uint64_t)D << 16) | (uint64_t)li;
                                if constexpr (LOG) tl_release(gpu, a.ro[TR.ro_off + (li + 1) % p]);
                            }
                        } else if (TREE && li >= 1) {
                            const unsigned um = started ? 0u : upm, dm = started ? 0u : dnm;
                            const bool ku = (c1 >= p || ((um >> c1) & 1u)) && (c2 >= p || ((um >> c2) & 1u));
                            const int par_i = (li - 1) / 2;
                            const uint32_t par = a.ro[TR.ro_off + par_i];
                            if (!uprel && ku) {
                                // tree reduce edge i -> parent(i) (Q25)
                                const Route r = get_route(a, TR, gpu, par);
                                flen = r.len;
                                t_act = t + load_route(a, TR, r, lats, hl);
                                froff = r.off;
                                fcode = ((uint64_t)cur << 32) | (uint64_t)li;
                                fup = uprel = rel = true;
                                if constexpr (LOG) { fbytes = cS; tl_release(gpu, par); }
                            } else if (uprel && upd && !dnrel &&
                                       (par_i == 0 ? ((p <= 1 || ((um >> 1) & 1u)) && (p <= 2 || ((um >> 2) & 1u)))
                                                   : ((dm >> par_i) & 1u))) {
                                // tree broadcast edge parent(i) -> i
                                const Route r = get_route(a, TR, par, gpu);
                                flen = r.len;
                                t_act = t + load_route(a, TR, r, lats, hl);
                                froff = r.off;
                                fcode = ((uint64_t)cur << 32) | (1ull << 16) | (uint64_t)li;
                                fup = false;
                                dnrel = rel = true;
                                if constexpr (LOG) { fbytes = cS; tl_release(par, gpu); }
                            }
                            if (rel) {
                                fbytes = cS;
                                alg += 2 * flen + 1;
                            }
                        }
                        if (rel) {
                            fst = FS_LAT;
                            EV(EV_RELEASE, fcode);
                            if (t_act == t) more = true;
                        }
                    }
                } else if constexpr (HOPM) {
                    // (d) R28 update queues: the lane's FIFO send stream -- iteration k's update to each
                    // neighbour in turn, once the iteration's backward pass is done
                    cnt[li] = hbwd;
                    __syncwarp();
                    if (used && fst == FS_NONE && sq < nsend_tot) {
                        const uint32_t k = sq / (uint32_t)hdeg, q = sq % (uint32_t)hdeg;
                        if (hbwd > k) {
                            const int j = hnb[q];
                            const uint32_t dg = a.ro[TR.ro_off + j];
                            const Route r = get_route(a, TR, gpu, dg);
                            flen = r.len;
                            fst = FS_LAT;
                            fbytes = hS;
                            t_act = t + load_route(a, TR, r, lats, hl);
                                froff = r.off;
                            alg += 2 * flen + 1;
                            fcode = (1ull << 58) | ((uint64_t)k << 32) | ((uint64_t)li << 16) | (uint64_t)j;
                            hdst = j;
                            hslot = hsl[q];
                            hk = k;
                            EV(EV_RELEASE, fcode);
                            if constexpr (LOG) tl_release(gpu, dg);
                            if constexpr (BD) {
                                bd_t0 = t;
                                bd_l = a.layer[hlast];
                            }
                            sq++;
                            if (t_act == t) more = true;
                        }
                    }
                } else {
                    cnt[li] = dcnt;
                    __syncwarp();
                    if (used && fst == FS_NONE && sq < nsend_tot) {
                        // next P2P send of this stage's FIFO stream (R11, Q14)
                        uint32_t P, j, e;
                        if (sq < m * SI.SF) { P = 0; j = sq / SI.SF; e = sq % SI.SF; }
                        else if (sq < m * (SI.SF + SI.SB)) { const uint32_t r = sq - m * SI.SF; P = 1; j = m - 1 - r / SI.SB; e = r % SI.SB; }
                        else { P = 2; j = 0; e = sq - m * (SI.SF + SI.SB); }
                        const SendEnt se = a.sends[SI.send_off + (P == 0 ? 0 : P == 1 ? SI.SF : SI.SF + SI.SB) + e];
                        const uint32_t prodpos = P == 0 ? j * SI.nF + se.pidx
                                               : P == 1 ? m * SI.nF + (m - 1 - j) * SI.nB + se.pidx
                                                        : m * (SI.nF + SI.nB) + se.pidx;
                        const uint32_t donepos = (cst == CS_RUN) ? run_start : pos;
                        if (donepos > prodpos) {
                            const uint32_t dg = a.ro[TR.ro_off + se.dst];
                            const Route r = get_route(a, TR, gpu, dg);
                            flen = r.len;
                            fst = FS_LAT;
                            fbytes = se.bytes;
                            t_act = t + load_route(a, TR, r, lats, hl);
                                froff = r.off;
                            alg += 2 * flen + 1;
                            fcode = (1ull << 59) | ((uint64_t)se.x << 32) | ((uint64_t)j << 16) | (uint64_t)dg;
                            EV(EV_RELEASE, fcode);
                            if constexpr (LOG) tl_release(gpu, dg);
                            if constexpr (BD) {
                                bd_t0 = t;
                                bd_l = a.layer[a.ents[SI.ent_off + (P == 0 ? 0 : P == 1 ? SI.nF : SI.nF + SI.nB) + se.pidx].op];
                            }
                            sq++;
                            if (t_act == t) more = true;
                        }
                    }
                }
                // (e) an idle GPU starts its head operator once its inputs are present
                if (used && cst == CS_IDLE && pos < nprog) {
                    if constexpr (HOPM) {
                        const uint32_t k = pos / hN, o = pos % hN;
                        bool ok = true, ev = false;
                        if (o == 0 && hg > 0 && (int)k >= hg) {
                            // token queues: every neighbour finished computing iteration k - g
                            ev = true;
                            for (int q = 0; q < hdeg; q++)
                                if (cnt[hnb[q]] < k - (uint32_t)hg + 1) ok = false;
                        }
                        if (o == hfirst && (int)k >= hs && hdeg > hb) {
                            // update queues: deg - b neighbours' updates of iteration k - s arrived
                            ev = true;
                            int got = 0;
                            for (int q = 0; q < hdeg; q++) got += rcv[li * 4 + q] >= k - (uint32_t)hs + 1 ? 1 : 0;
                            if (got < hdeg - hb) ok = false;
                        }
                        if (ok) {
                            if (ev) EV(EV_TASK_START, ((uint64_t)gpu << 40) | pos);
                            run_start = pos;
                            // fold (R16) to the next boundary: through the iteration's last non-OPT op (its
                            // completion sends the update), or up to an op that waits (the first OPT op of an
                            // iteration that applies updates, the first op of a gated iteration)
                            double te = t;
                            uint32_t q = pos;
                            for (;;) {
                                const uint32_t oo = q % hN;
                                const double dd = a.dur[C->dur_off + oo];
                                if constexpr (LOG) tl_task(gpu, q, oo, q / hN, te, te + dd);
                                te = te + dd;
                                busy = busy + dd;
                                q++;
                                if (oo == hlast || q >= nprog) break;
                                const uint32_t no = q % hN, nk = q / hN;
                                if (no == hfirst && (int)nk >= hs && hdeg > hb) break;
                                if (no == 0 && hg > 0 && (int)nk >= hg) break;
                            }
                            ntask += q - pos;
                            alg += 2 * (q - pos);
                            run_end = q;
                            t_end = te;
                            cst = CS_RUN;
                            if (te == t) more = true;
                        }
                    } else if constexpr (COLL) {
                        if (hwait < 0 || (int)donec > hwait) {
                            const OpHook *HK = a.hooks + C->hook_off;
                            const OpHook h = HK[pos];
                            if (h.wait >= 0) EV(EV_TASK_START, ((uint64_t)gpu << 40) | pos);
                            run_start = pos;
                            double te = t + h.dur;
                            if constexpr (LOG) tl_task(gpu, pos, pos, 0, t, te);
                            busy = busy + h.dur;
                            uint32_t q = pos + 1, sig = h.nsig;
                            while (sig == 0 && q < nprog) {
                                const OpHook h2 = HK[q];
                                if (h2.wait >= 0) break;
                                if constexpr (LOG) tl_task(gpu, q, q, 0, te, te + h2.dur);
                                te = te + h2.dur;
                                busy = busy + h2.dur;
                                sig = h2.nsig;
                                q++;
                            }
                            ntask += q - pos;
                            alg += 2 * (q - pos);
                            run_end = q;
                            t_end = te;
                            cst = CS_RUN;
                            if (te == t) more = true;
                        }
                    } else if (!(hc_pos == pos && !(cnt[hc_src] > hc_seq))) {
                        uint32_t q = pos, P, j, idx;
                        if (q < m * SI.nF) { P = 0; j = q / SI.nF; idx = q % SI.nF; }
                        else if (q < m * (SI.nF + SI.nB)) { const uint32_t r = q - m * SI.nF; P = 1; j = m - 1 - r / SI.nB; idx = r % SI.nB; }
                        else { P = 2; j = 0; idx = q - m * (SI.nF + SI.nB); }
                        const StageEnt en = a.ents[SI.ent_off + (P == 0 ? 0 : P == 1 ? SI.nF : SI.nF + SI.nB) + idx];
                        bool ok = true;
                        for (uint32_t r = 0; r < en.nrecv && ok; r++) {
                            const RecvEnt re = a.recvs[en.recv_off + r];
                            const StageInfo &ps = a.stages[C->stage_off + re.src];
                            const uint32_t jp = (re.phase == 2 || P == 2) ? 0 : j;
                            const uint32_t seqi = re.phase == 0 ? jp * ps.SF + re.e
                                                : re.phase == 1 ? m * ps.SF + (m - 1 - jp) * ps.SB + re.e
                                                                : m * (ps.SF + ps.SB) + re.e;
                            if (!(cnt[re.src] > seqi)) {
                                ok = false;
                                hc_pos = pos;
                                hc_src = (int)re.src;
                                hc_seq = seqi;
                            }
                        }
                        if (ok) {
                            if (en.nrecv) EV(EV_TASK_START, ((uint64_t)gpu << 40) | q);
                            run_start = pos;
                            // fold (R16): K2's run from the head within its phase list, then on into the
                            // next lists (micro-batch / phase) while the run ends at a list end without a
                            // send and the next list's first operator waits for no receive.  One
                            // sequential fp64 add per operator, over contiguous entries
                            const StageEnt *L = a.ents + SI.ent_off + (P == 0 ? 0 : P == 1 ? SI.nF : SI.nF + SI.nB);
                            uint32_t len = P == 0 ? SI.nF : P == 1 ? SI.nB : SI.nO;
                            uint32_t n = en.run, i0 = idx;
                            double te = t;
                            for (;;) {
#pragma unroll 4
                                for (uint32_t k = 0; k < n; k++) {
                                    const double dd = L[i0 + k].dur;
                                    if constexpr (LOG) tl_task(gpu, q + k, L[i0 + k].op, j, te, te + dd);
                                    te = te + dd;
                                    busy = busy + dd;
                                }
                                q += n;
                                const uint32_t last = i0 + n - 1;
                                if (L[last].nsend != 0 || last + 1 < len || q >= nprog) break;
                                if (q < m * SI.nF) { j = q / SI.nF; L = a.ents + SI.ent_off; len = SI.nF; }
                                else if (q < m * (SI.nF + SI.nB)) { j = m - 1 - (q - m * SI.nF) / SI.nB; L = a.ents + SI.ent_off + SI.nF; len = SI.nB; }
                                else { j = 0; L = a.ents + SI.ent_off + SI.nF + SI.nB; len = SI.nO; }
                                i0 = 0;
                                if (L[0].nrecv) break;
                                n = L[0].run;
                            }
                            ntask += q - pos;
                            alg += 2 * (q - pos);
                            run_end = q;
                            t_end = te;
                            cst = CS_RUN;
                            if (te == t) more = true;
                        }
                    }
                }
                if constexpr (!COLL) __syncwarp();
                if (!__any_sync(FULL, more)) break;
            }

            // (f) bandwidth re-allocation of every in-transit flow: max-min fair
            //     progressive filling (R14, Q18)
            const unsigned dball = __ballot_sync(FULL, dirty);
            if (!dball) break;
            const bool segdirty = (dball & smask) != 0;
            dirty = false;
            const bool act = segdirty && used && fst == FS_ACT;
            // ring_fast is segment-uniform and only set while a ring collective runs (tree_cur off)
            const bool fast = ring_fast && !tree_cur;
            const bool gen = act && !fast;
            if (act && t_upd < t) {
                const double r = rem - rate * (t - t_upd);
                rem = r > 0.0 ? r : 0.0;
                t_upd = t;
                alg += 4;
            }
            const bool anygen = __any_sync(FULL, gen);
            if (anygen) {
                // link counters are 0 here: every complete progressive filling returns them to 0
                if (gen) {
                    alg += flen;
#pragma unroll
                    for (int h = 0; h < MAX_HOPS; h++)
                        if (h < flen) {
                            const int e = hop(hl, h);
                            atomicAdd(&ln[e], 1);
                            lres[e] = a.link_bw[TR.link_off + e] * bws;
                        }
                    for (int h = MAX_HOPS; h < flen; h++) {   // long routes
                        const int e = a.rt_links[froff + h];
                        atomicAdd(&ln[e], 1);
                        lres[e] = a.link_bw[TR.link_off + e] * bws;
                    }
                }
                __syncwarp();
            }
            if (act && fast) rate = rbw;
            // uniform link-disjoint ring: one round at rate rbw, nothing to reduce
            const bool uni = fast && ring_uni;
            const bool segany = (__ballot_sync(FULL, act) & smask) != 0;
            uint32_t rounds = (uni && segany) ? 1u : 0u;
            // link-disjoint ring with different rates: progressive filling freezes, round after round, the
            // flows at the smallest remaining rate, so its rounds are the distinct rates of the active
            // flows -- counted at once (a lane leads its value if it is the lowest segment lane holding it)
            if (COLL && __any_sync(FULL, fast && !uni && segany)) {   // (ring fast path: COLL classes only)
                const unsigned long long key = act ? (unsigned long long)__double_as_longlong(rate)
                                                   : ~(unsigned long long)lane;   // NaN patterns, never a rate
                bool lead;
                if constexpr (W <= 16) {
                    // W - 1 independent shuffles beat one 64-bit match.any here (its issue latency was 14 % of
                    // the C3 K3 stall samples, profiles/r2_c3_k3_lines.txt)
                    bool dup = false;
#pragma unroll
                    for (int d = 1; d < W; d++) {
                        const unsigned long long o = __shfl_up_sync(FULL, key, d, W);
                        dup = dup || (li >= d && o == key);
                    }
                    lead = act && !dup;
                } else {
                    const unsigned mm = __match_any_sync(FULL, key) & smask;
                    lead = act && (__ffs(mm) - 1) == lane;
                }
                const uint32_t nd = __popc(__ballot_sync(FULL, lead) & smask);
                if (fast && !uni) rounds = nd;
            }
            bool unf = act && !fast;
            if (__any_sync(FULL, unf)) {   // guard: keeps the loop's hoisted address math off the fast path
                while (__any_sync(FULL, unf)) {
                    const bool segact = (__ballot_sync(FULL, unf) & smask) != 0;
                    double my = dinf();
                    if (unf) {
                        if (fast) {
                            my = rate;
                        } else {
    #pragma unroll
                            for (int h = 0; h < MAX_HOPS; h++)
                                if (h < flen) {
                                    const int e = hop(hl, h);
                                    const double sh = lres[e] / (double)ln[e];
                                    my = sh < my ? sh : my;
                                }
                            for (int h = MAX_HOPS; h < flen; h++) {
                                const int e = a.rt_links[froff + h];
                                const double sh = lres[e] / (double)ln[e];
                                my = sh < my ? sh : my;
                            }
                            alg += 2 * flen;
                        }
                    }
                    const double s = TS_SEGMIN_REDUX ? seg_min_redux(my, smask) : seg_min_shfl<W>(my);
                    const bool inF = unf && my == s;
                    unsigned own = 0;
                    if (inF && !fast) {
                        rate = s;
    #pragma unroll
                        for (int h = 0; h < MAX_HOPS; h++)
                            if (h < flen && atomicAdd(&lk[hop(hl, h)], 1) == 0) own |= 1u << h;
                        for (int h = MAX_HOPS; h < flen; h++)   // (flen <= MAX_ROUTE_K3 = 32: host-checked)
                            if (atomicAdd(&lk[a.rt_links[froff + h]], 1) == 0) own |= 1u << h;
                    }
                    if (anygen) __syncwarp();
                    if (inF && !fast) {
    #pragma unroll
                        for (int h = 0; h < MAX_HOPS; h++)
                            if ((own >> h) & 1u) {
                                const int e = hop(hl, h);
                                const int kk = lk[e];
                                const double r = lres[e] - s * (double)kk;
                                lres[e] = r > 0.0 ? r : 0.0;
                                ln[e] -= kk;
                                lk[e] = 0;
                                alg += 3;
                            }
                        for (int h = MAX_HOPS; h < flen; h++)
                            if ((own >> h) & 1u) {
                                const int e = a.rt_links[froff + h];
                                const int kk = lk[e];
                                const double r = lres[e] - s * (double)kk;
                                lres[e] = r > 0.0 ? r : 0.0;
                                ln[e] -= kk;
                                lk[e] = 0;
                                alg += 3;
                            }
                    }
                    if (anygen) __syncwarp();
                    if (segact) rounds++;
                    unf = unf && !inF;
                }
            }
            const uint32_t nact = __popc(__ballot_sync(FULL, act) & smask);  // (all lanes vote)
            if (segdirty) {
                nwf++;
                nrounds += rounds;
                if (nact > maxact) maxact = nact;
            }
            bool again = false;
            if (act) {
                t_drain = (rem == 0.0) ? t : t + rem / rate;
                alg += 2;
                again = t_drain == t;
            }
            if (!__any_sync(FULL, again)) break;
        }

        // ------------------------------ end of instant ------------------------------
        const bool any_ev = (__ballot_sync(FULL, nev) & smask) != 0;
        if (have && any_ev) ninst++;
        nev = false;
        const bool infl = (__ballot_sync(FULL, used && fst != FS_NONE) & smask) != 0;
        if (have && infl != bon) {   // an interval with >= 1 flow in flight opens or closes (R18)
            if (bon) cbusy = cbusy + (t - bstart);
            else bstart = t;
            bon = !bon;
        }
        bool lane_done = !used || (cst == CS_IDLE && pos >= nprog && fst == FS_NONE);
        if constexpr (!COLL) lane_done = lane_done && (!used || sq >= nsend_tot);
        const bool alldone = (__ballot_sync(FULL, lane_done) & smask) == smask;
        const bool fin = have && alldone && (!COLL || (cur >= ncoll && !running));
        double cand = dinf();
        if (used) {
            if (cst == CS_RUN) cand = t_end;
            if (fst == FS_LAT && t_act < cand) cand = t_act;
            if (fst == FS_ACT && t_drain < cand) cand = t_drain;
        }
        const double tn = TS_SEGMIN_REDUX ? seg_min_redux(cand, smask) : seg_min_shfl<W>(cand);
        const bool stuck = have && !fin && !(tn < dinf());
        if (__any_sync(FULL, fin || stuck)) {
            const double bmax = seg_max<W>(used ? busy : 0.0);
            const uint32_t ntk = seg_sum_u32<W>(ntask);
            const uint32_t nfl = seg_sum_u32<W>(nflow);
            const unsigned long long alg_s = seg_sum_u64<W>((unsigned long long)alg);
            const unsigned long long H = seg_sum_u64<W>(acc);
            if ((fin || stuck) && li == 0) {
                triosim_result r;
                r.iter_time_s = fin ? t : 0.0;
                r.compute_busy_max_s = fin ? bmax : 0.0;
                r.comm_busy_s = fin ? cbusy : 0.0;
                r.exposed_comm_s = fin ? t - bmax : 0.0;
                r.coll_payload_bytes = fin ? C->coll_payload : 0.0;
                r.n_compute = fin ? (uint64_t)ntk : 0;
                r.n_flows = fin ? (uint64_t)nfl : 0;
                r.n_collectives = fin ? ncoll : 0;
                r.n_p2p = (fin && !COLL) ? (uint64_t)nfl : 0;
                r.n_instants = fin ? ninst : 0;
                r.n_wf_calls = fin ? nwf : 0;
                r.n_wf_rounds = fin ? nrounds : 0;
                r.order_hash = fin ? H : 0;
                r.status = fin ? TRIOSIM_PT_OK : TRIOSIM_PT_DEADLOCK;
                r.max_active_flows = fin ? maxact : 0;
                a.out[pidx] = r;
                if (a.alg_ops) atomicAdd(a.alg_ops, alg_s);
#ifdef TS_PROF
                if (pidx < 4) printf("PROF pidx=%u W=%d inst=%u general=%u ff_entries=%u ff_cycles=%lld total_cycles=%lld\n",
                                     pidx, W, ninst, pf_gen, pf_entries, pf_ff, clock64() - pf_t0);
#endif
            }
            if (fin || stuck) have = used = false;
        }
        if (have) {
            t = tn;
            tmix = mix64((uint64_t)__double_as_longlong(t));
        }
    }
#undef EV
}

template <int W, int MODE>
static cudaError_t launch_wm(const K3Args &a, int grid, cudaStream_t s) {
    if (a.tl_cnt) k3_timeline<W, MODE, V_LOG><<<grid, K3_THREADS, 0, s>>>(a);
    else if (a.bd) k3_timeline<W, MODE, V_BD><<<grid, K3_THREADS, 0, s>>>(a);
    else k3_timeline<W, MODE, 0><<<grid, K3_THREADS, 0, s>>>(a);
    return cudaGetLastError();
}

template <int W>
static cudaError_t launch_w(int mode, const K3Args &a, int grid, cudaStream_t s) {
    switch (mode) {
    case MODE_COLL: return launch_wm<W, MODE_COLL>(a, grid, s);
    case MODE_TREE: return launch_wm<W, MODE_TREE>(a, grid, s);
    case MODE_HOP: return launch_wm<W, MODE_HOP>(a, grid, s);
    default: return launch_wm<W, MODE_PIPE>(a, grid, s);
    }
}

cudaError_t launch_k3(int W, int mode, const K3Args &a, int grid, cudaStream_t s) {
    switch (W) {
    case 2: return launch_w<2>(mode, a, grid, s);
    case 4: return launch_w<4>(mode, a, grid, s);
    case 8: return launch_w<8>(mode, a, grid, s);
    case 16: return launch_w<16>(mode, a, grid, s);
    case 32: return launch_w<32>(mode, a, grid, s);
    default: return cudaErrorInvalidValue;
    }
}

template <int W>
static int occ_w(int mode) {
    int nb = 0;
    if (mode == MODE_COLL) cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, k3_timeline<W, MODE_COLL, 0>, K3_THREADS, 0);
    else if (mode == MODE_TREE) cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, k3_timeline<W, MODE_TREE, 0>, K3_THREADS, 0);
    else if (mode == MODE_HOP) cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, k3_timeline<W, MODE_HOP, 0>, K3_THREADS, 0);
    else cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, k3_timeline<W, MODE_PIPE, 0>, K3_THREADS, 0);
    return nb;
}

int k3_max_blocks_per_sm(int W, int mode) {
    int nb = W == 2 ? occ_w<2>(mode) : W == 4 ? occ_w<4>(mode) : W == 8 ? occ_w<8>(mode)
           : W == 16 ? occ_w<16>(mode) : occ_w<32>(mode);
    return nb > 0 ? nb : 1;
}

}  // namespace ts
