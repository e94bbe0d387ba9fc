// ts_k3h.cu -- K3 for HYBRID DP x TP x PP points (R9; Table 1).
//
// One point per segment: W lanes of a warp (NW = 1), or NW whole warps = one CTA (NW = 2..8, up to
// 1024 ranks).  Lane r = rank (d, s, t) with r = (d*pp + s)*tp + t.  Each lane
// runs its stage's GPipe program (R8) and owns THREE flow slots: its TP-group collective step,
// its DP-group collective step and its FIFO P2P send.  The TP group {(d,s,.)} is a contiguous lane
// range, the DP group {(.,s,t)} a strided one; both run R10's ring / tree collectives through one
// routine parameterised by (first lane, stride, size).  Instants, R14's progressive filling over
// all flow slots and R19's hash follow ts_k3.cu.
#include <cuda_runtime.h>
#include <cstdint>
#include "ts_internal.h"

namespace ts {

#define FULL 0xffffffffu
namespace {

enum { CS_IDLE = 0, CS_RUN = 1 };
enum { FS_NONE = 0, FS_LAT = 1, FS_ACT = 2 };   // FS_ACT: draining (flow network) / transferring (photonic)
enum { PS_REQ = 3, PS_LINKQ = 4, PS_BUFW = 5 };  // photonic (R20): no link yet, queued on a link, awaiting a buffer
enum { EV_COLL_START = 1, EV_RELEASE = 2, EV_ACTIVATE = 3, EV_DELIVER = 4, EV_TASK_START = 5, EV_TASK_END = 6 };

__device__ __forceinline__ uint64_t mix64(uint64_t z) {
    z = (z ^ (z >> 30)) * 0xbf58476d1ce4e5b9ull;
    z = (z ^ (z >> 27)) * 0x94d049bb133111ebull;
    return z ^ (z >> 31);
}
__device__ __forceinline__ double dinf() { return __longlong_as_double(0x7ff0000000000000ll); }

template <int W>
__device__ __forceinline__ double seg_min(double v) {
#pragma unroll
    for (int o = W / 2; o > 0; o >>= 1) {
        const double w = __shfl_xor_sync(FULL, v, o);
        v = w < v ? w : v;
    }
    return v;
}
template <int W>
__device__ __forceinline__ double seg_max(double v) {
#pragma unroll
    for (int o = W / 2; o > 0; o >>= 1) {
        const double w = __shfl_xor_sync(FULL, v, o);
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

struct Topo {
    uint32_t n_gpus, link_off, rt_off, ro_off, n_links;
    bool phot;
};

struct Flow {
    int st;
    double t_act, rem, rate, t_upd, t_drain, bytes;
    int len;
    uint32_t hl[4];               // the first MAX_HOPS link ids (16 bit each) ...
    uint32_t roff;                // ... and where the route sits in rt_links, for the hops beyond them
    uint64_t code;
    uint32_t src, dst;            // endpoints (R23 timeline records only)
    unsigned long long tl;        // R23 (LOG): record slot
};

// one boolean per segment lane: ballot bits (warp segments) or a shared-memory byte array (CTA)
template <bool CTA>
struct LaneFlags {
    uint32_t bits;      // warp segment: ballot bits (0 = all false)
    const uint8_t *p;   // CTA: flag bytes (nullptr = all false)
    uint8_t sel;
    __device__ __forceinline__ bool test(int k) const {
        if constexpr (CTA) return p != nullptr && (p[k] & sel) != 0;
        else return (bits >> k) & 1u;
    }
};
// one collective group (TP or DP) as seen by one member lane
struct Group {
    bool member;
    int p, i;                 // group size, my member index
    int lane0, stride;        // segment lane of member k = lane0 + k * stride
    int pred;                 // segment lane of member (i - 1) mod p
    bool cross;               // segment-uniform: some group of this kind spans several warps (CTA only)
    uint32_t wmask;           // warp-lane bits of the members when the group lies inside this lane's warp
    int slot;                 // counter slot of a cross-warp group (CTA only)
    uint64_t gid;
    uint32_t ncoll, trig, donec, cur;
    bool running, tree_cur, ldone, uprel, upd, dnrel, dnd, fup;
    bool dbt_cur, uprel2, upd2, dnrel2, dnd2, fup2;   // R27 double binary tree: the mirrored tree B's edge state
    bool rb_cur;              // R26: the running AllReduce is a ring Reduce + ring Broadcast
    int K, D, Kp;             // this member's / its predecessor's sends in the running collective
    double cS, chunk;
    uint32_t flow_deliv;      // deliveries of this group's flows (for counts)
    double bd_t0;             // R22 (BD): start time of the running collective
    uint32_t bd_l;            // ... and the layer it is attributed to
};

__device__ __forceinline__ int hop(const uint32_t (&hl)[4], int h) { return (hl[h >> 1] >> (16 * (h & 1))) & 0xffff; }

__device__ __forceinline__ int route_len(const K3Args &a, const Topo &T, uint32_t s, uint32_t d) {
    return a.rt_len[T.rt_off + s * T.n_gpus + d];
}

// release flow f along src -> dst: route latency fold (R12), link ids cached (<= 8 hops).  Photonic
// (R20): a send request keyed by (release time t_upd, code); hl[0] = destination GPU, hl[1] = link slot
__device__ __forceinline__ void release(const K3Args &a, const Topo &T, Flow &f, uint32_t src, uint32_t dst,
                                        double bytes, uint64_t code, double t, double lats, uint64_t &alg) {
    f.src = src;
    f.dst = dst;
    if (T.phot) {
        f.len = 0;
        f.bytes = bytes;
        f.code = code;
        f.hl[0] = dst;
        f.hl[1] = 0;
        f.t_upd = t;
        if (src == dst) {          // nothing to move: activation and delivery now (as an empty route)
            f.st = FS_LAT;
            f.t_act = t;
        } else {
            f.st = PS_REQ;
            f.t_act = __longlong_as_double(0x7ff0000000000000ll);
        }
        return;
    }
    const uint32_t k = T.rt_off + src * T.n_gpus + dst;
    const int len = a.rt_len[k];
    const uint32_t off = a.rt_off[k];
    double L = 0.0;
    f.hl[0] = f.hl[1] = f.hl[2] = f.hl[3] = 0;
#pragma unroll
    for (int h = 0; h < MAX_HOPS; h++)
        if (h < len) {
            const uint32_t e = a.rt_links[off + h];
            f.hl[h >> 1] |= e << (16 * (h & 1));
            L = L + a.link_lat[T.link_off + e] * lats;
        }
    for (int h = MAX_HOPS; h < len; h++) L = L + a.link_lat[T.link_off + a.rt_links[off + h]] * lats;   // long routes
    f.roff = off;
    f.len = len;
    f.st = FS_LAT;
    f.bytes = bytes;
    f.t_act = t + L;
    f.code = code;
    alg += 2 * len + 1;
}

}  // namespace


// V & V_BD: also record the per-layer communication breakdown (R22) into a.bd; V & V_LOG: record the R23
// timeline (separate instantiations)
template <int W, int NW, int V>
__global__ void __launch_bounds__(NW == 1 ? K3_THREADS : 32 * NW, 1) k3_hybrid(const K3Args a) {
    constexpr bool BD = (V & V_BD) != 0;
    constexpr bool LOG = (V & V_LOG) != 0;
    constexpr int SL = NW == 1 ? W : 32 * NW;           // lanes per segment
    constexpr int NSEG = NW == 1 ? 32 / W : 1;          // segments per warp (NW = 1)
    constexpr int LMAXW = lmax_hybrid(W);               // warp segments: static link arrays
    constexpr int NSLOT = NW == 1 ? K3_WARPS : 1;       // segment-array slots of the block
    // warp segments keep their link arrays in static smem; a one-point CTA sizes them to the sweep's
    // largest topology (a.lmax links, dynamic smem: residual f64, share f64, unfrozen and frozen counts)
    __shared__ double s_res[NW == 1 ? NSLOT : 1][NW == 1 ? NSEG * LMAXW : 1];
    __shared__ double s_sh[NW == 1 ? NSLOT : 1][NW == 1 ? NSEG * LMAXW : 1];
    __shared__ int s_n[NW == 1 ? NSLOT : 1][NW == 1 ? NSEG * LMAXW : 1];
    __shared__ int s_k[NW == 1 ? NSLOT : 1][NW == 1 ? NSEG * LMAXW : 1];
    __shared__ int s_own[NW == 1 ? NSLOT : 1][NW == 1 ? NSEG * LMAXW : 1];   // owner of a link reached past MAX_HOPS
    extern __shared__ double s_dyn[];
    const int LMAX = NW == 1 ? LMAXW : (int)a.lmax;
    // photonic tables (R20) after the CTA link arrays: per lane a.pmax logical links {dst GPU, state
    // 0 none / 1 setup / 2 up, t = ready time or last use} and per flow slot its buffer request
    constexpr int NTHR = NW == 1 ? K3_THREADS : 32 * NW;
    const int PM = (int)a.pmax;
    // A one-point CTA keeps them at the start of dynamic smem while it runs a photonic point (which has
    // no link arrays), after the link arrays otherwise; dynamic smem = the larger of the two (k3h_dyn_smem)
    double *p_t;
    int *p_dst, *p_st;
    double *q_t;                    // [3 * NTHR] request key time
    unsigned long long *q_code;
    int *q_dst;                     // destination GPU or -1
    uint8_t *q_st, *q_g;            // 1 waiting for a buffer / 2 transferring; granted
    auto ph_tables = [&](bool phot) {
        p_t = s_dyn + ((NW == 1 || phot) ? 0 : (7 * LMAX + 1) / 2);   // after lres, lsh, ln, lk, lown
        p_dst = (int *)(p_t + NTHR * PM);
        p_st = p_dst + NTHR * PM;
        q_t = (double *)(p_st + NTHR * PM);
        q_code = (unsigned long long *)(q_t + 3 * NTHR);
        q_dst = (int *)(q_code + 3 * NTHR);
        q_st = (uint8_t *)(q_dst + 3 * NTHR);
        q_g = q_st + 3 * NTHR;
    };
    ph_tables(false);
    bool last_phot = false;   // CTA: the previous point ran photonic (its tables overlaid the link arrays)
    __shared__ uint32_t s_cnt[NSLOT][NW == 1 ? 32 : SL];
    __shared__ double s_red[2][NW];
    __shared__ unsigned s_fl3[2][NW];                  // CTA: per-warp end-of-instant votes
    __shared__ unsigned long long s_red64[2][NW];
    // CTA: each lane's group progress D (TP, DP), published with an event-loop pass's first barrier
    __shared__ int s_dx[2][NW == 1 ? 1 : SL];
    // CTA: one round of cross-warp group votes per pass and group -- members done | ready now (16-bit fields),
    // and ready after this collective -- in a rotating triple buffer indexed by group slot (a group that spans
    // warps has >= 2 members, so its slot is < SL / 2).  32-bit adds: a 64-bit shared add is a CAS loop, which
    // an 84-member group turned into a 35 % slower wafer sweep
    __shared__ unsigned s_gca[3][NW == 1 ? 1 : SL / 2], s_gcb[3][NW == 1 ? 1 : SL / 2];
    __shared__ uint8_t s_fl[2][NW == 1 ? 1 : SL];      // tree flags exchange (CTA)
    __shared__ uint32_t s_item;
    __shared__ int s_na;                               // CTA water-filling: active flows of the call

    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    const int seg = NW == 1 ? lane / W : 0;
    const int li = NW == 1 ? lane % W : (int)threadIdx.x;     // lane inside the segment
    const int sbase = NW == 1 ? seg * W : 0;                 // segment's first warp lane (NW = 1)
    const unsigned smask = NW == 1 ? ((W == 32 ? FULL : ((1u << (W & 31)) - 1u)) << sbase) : FULL;
    const int slot = NW == 1 ? wid : 0;
    double *lres = NW == 1 ? &s_res[slot][seg * LMAX] : s_dyn;
    double *lsh = NW == 1 ? &s_sh[slot][seg * LMAX] : s_dyn + LMAX;   // share res / n of links with n > 0
    int *ln = NW == 1 ? &s_n[slot][seg * LMAX] : (int *)(s_dyn + 2 * LMAX);
    int *lk = NW == 1 ? &s_k[slot][seg * LMAX] : (int *)(s_dyn + 2 * LMAX) + LMAX;
    int *lown = NW == 1 ? &s_own[slot][seg * LMAX] : (int *)(s_dyn + 2 * LMAX) + 2 * LMAX;
    uint32_t *cnt = &s_cnt[slot][sbase];                     // indexed by segment lane
    for (int q = (NW == 1 ? lane : (int)threadIdx.x); q < NSEG * LMAX; q += (NW == 1 ? 32 : 32 * NW)) {
        ln[q - seg * LMAX] = 0;   // (NW == 1: each lane clears its warp's slot through segment 0's base)
        lk[q - seg * LMAX] = 0;
    }
    if constexpr (NW > 1) {
        if (threadIdx.x < SL / 2) {
            s_gca[0][threadIdx.x] = s_gca[1][threadIdx.x] = s_gca[2][threadIdx.x] = 0u;
            s_gcb[0][threadIdx.x] = s_gcb[1][threadIdx.x] = s_gcb[2][threadIdx.x] = 0u;
        }
    }
    if (NW == 1 && PM > 0) {   // (a CTA overlays its tables on the link arrays: set up per photonic point)
        for (int k = 0; k < PM; k++) p_st[k * NTHR + threadIdx.x] = 0;
        for (int k = 0; k < 3; k++) q_g[threadIdx.x * 3 + k] = 0;
    }
    int bb = 0;   // double-buffer toggle of the block-level exchanges (NW > 1)
    int fb = 0;   // double-buffer toggle of the tree-flag exchange (NW > 1)
    int gcb3 = 0;  // rotating buffer of the cross-warp group votes (NW > 1)

    // ---- segment primitives: a segment is W lanes of a warp, or the whole CTA ----
    auto ssync = [&]() {
        if constexpr (NW == 1) __syncwarp(); else __syncthreads();
    };
    auto vany = [&](bool p) -> bool {          // any lane of the warp / CTA (loop control)
        if constexpr (NW == 1) return __any_sync(FULL, p); else return __syncthreads_or(p) != 0;
    };
    auto vall = [&](bool p) -> bool {
        if constexpr (NW == 1) return __all_sync(FULL, p); else return __syncthreads_and(p) != 0;
    };
    auto sany = [&](bool p) -> bool {          // any lane of the segment
        if constexpr (NW == 1) return (__ballot_sync(FULL, p) & smask) != 0; else return __syncthreads_or(p) != 0;
    };
    auto scount = [&](bool p) -> uint32_t {    // lanes of the segment with p
        if constexpr (NW == 1) return __popc(__ballot_sync(FULL, p) & smask); else return __syncthreads_count(p);
    };
    // upd / dnd flags of every segment lane (tree collectives)
    using LF = LaneFlags<(NW > 1)>;
    auto flags2 = [&](bool u, bool dn, LF &fu, LF &fd) {
        if constexpr (NW == 1) {
            fu.bits = (__ballot_sync(FULL, u) & smask) >> sbase;
            fd.bits = (__ballot_sync(FULL, dn) & smask) >> sbase;
            fu.p = fd.p = nullptr;
        } else {
            s_fl[fb][threadIdx.x] = (uint8_t)((u ? 1 : 0) | (dn ? 2 : 0));
            __syncthreads();
            fu.p = fd.p = s_fl[fb];
            fu.bits = fd.bits = 0;
            fb ^= 1;
        }
        fu.sel = 1;
        fd.sel = 2;
    };
    // every member of G satisfies pred (called by all lanes; non-members pass anything) -- groups inside a
    // warp; a CTA's cross-warp groups vote in grp_pass
    auto gall = [&](const Group &G, bool pred) -> bool {
        const unsigned b = __ballot_sync(FULL, !G.member || pred);
        return (b & G.wmask) == G.wmask;
    };
    auto smin = [&](double v) -> double {
        if constexpr (NW == 1) {
            return seg_min<W>(v);
        } else {
            v = seg_min<32>(v);
            if (lane == 0) s_red[bb][wid] = v;
            __syncthreads();
            // every warp combines the NW warp minima: serially for a few warps, with a shuffle tree (lane i
            // reads warp i's) for many -- not an NW-long chain
            double r;
            if constexpr (NW <= 4) {
                r = s_red[bb][0];
#pragma unroll
                for (int i = 1; i < NW; i++) r = s_red[bb][i] < r ? s_red[bb][i] : r;
            } else {
                r = seg_min<32>(lane < NW ? s_red[bb][lane] : dinf());
            }
            bb ^= 1;
            return r;
        }
    };
    auto smax = [&](double v) -> double {
        if constexpr (NW == 1) {
            return seg_max<W>(v);
        } else {
            v = seg_max<32>(v);
            if (lane == 0) s_red[bb][wid] = v;
            __syncthreads();
            double r = s_red[bb][0];
#pragma unroll
            for (int i = 1; i < NW; i++) r = s_red[bb][i] > r ? s_red[bb][i] : r;
            bb ^= 1;
            return r;
        }
    };
    auto ssum = [&](unsigned long long v) -> unsigned long long {
        if constexpr (NW == 1) {
            return seg_sum_u64<W>(v);
        } else {
            v = seg_sum_u64<32>(v);
            if (lane == 0) s_red64[bb][wid] = v;
            __syncthreads();
            unsigned long long r = 0;
#pragma unroll
            for (int i = 0; i < NW; i++) r += s_red64[bb][i];
            bb ^= 1;
            return r;
        }
    };
    auto xch = [&](int v, int src) -> int {    // value of segment lane src (warp segments)
        return __shfl_sync(FULL, v, sbase + src);
    };
    ssync();

    // ---- segment-uniform ----
    bool have = false, exhausted = false;
    uint32_t pidx = 0;
    double t = 0.0, bws = 1.0, lats = 1.0;
    double ph_bw = 1.0, ph_set = 0.0, ph_lat = 0.0;   // photonic (R20), scaled by the point
    int ports = 0, bufs = 0;
    int R = 1, S = 1, tp = 1, dp = 1;
    uint32_t m = 1;
    bool tree_algo = false, dbt_algo = false;   // binary-tree AllReduce (R10) / double binary tree (R27)
    const ClassDesc *C = nullptr;
    Topo TR = {0, 0, 0, 0, 0, false};
    uint32_t ninst = 0, nwf = 0, nrounds = 0, maxact = 0;
    bool bon = false;
    double bstart = 0.0, cbusy = 0.0;
    // ---- lane ----
    bool used = false;
    int d = 0, s = 0, tt = 0;
    uint32_t gpu = 0, pos = 0, run_start = 0, run_end = 0, nprog = 0;
    int cst = CS_IDLE;
    double t_end = 0.0, busy = 0.0;
    uint32_t ntask = 0, nflow = 0, np2p = 0;
    StageInfo SI;
    SI.nF = SI.nB = SI.nO = SI.SF = SI.SB = SI.SO = 0;
    SI.ent_off = SI.send_off = SI.recv_off = 0;
    HStage HS;
    HS.TF = HS.TB = HS.TO = HS.tcol_off = HS.ndp = HS.dcol_off = 0;
    HS.first_opt = 0xffffffffu;
    uint32_t sq = 0, nsend_tot = 0, dcnt = 0;
    // the head operator's first unmet condition at program position hc_pos (counters only grow, so while it
    // holds the head cannot start): kind 0 a receive (cnt[hc_a] > hc_b), 1 the TP wait (GT.donec > hc_b),
    // 2 the DP wait of the first OPT op (GD.donec >= GD.ncoll) -- one register / shared-memory test per pass
    uint32_t hc_pos = 0xffffffffu, hc_b = 0;
    int hc_kind = 0, hc_a = 0;
    Group GT, GD;
    GT.member = GD.member = false;
    GT.cross = GD.cross = false;
    GT.tree_cur = GD.tree_cur = GT.dbt_cur = GD.dbt_cur = false;
    Flow FT, FD, FP;
    FT.st = FD.st = FP.st = FS_NONE;
    uint64_t acc = 0, alg = 0, tmix = 0;
    bool nev = false;
    // R22 (BD): this lane is its layers' representative rank (d = 0, t = 0); its P2P send in flight
    bool bd_rep = false;
    double bd_p_t0 = 0.0;
    uint32_t bd_p_l = 0;
    auto bd_add = [&](uint32_t cat, uint32_t l, double dt) {
        double *q = a.bd + ((size_t)pidx * 3 + cat) * a.n_layers + l;
        *q = *q + dt;
    };
    // R23 (LOG): task and flow records
    auto tl_task = [&](uint32_t g, uint32_t prog, uint32_t op, uint32_t mbi, double t0, double t1) {
        const unsigned long long k = atomicAdd(&a.tl_cnt[0], 1ull);
        if (k < a.tl_task_cap) {
            triosim_task_rec r;
            r.gpu = g; r.prog = prog; r.op = op; r.mb = mbi; r.start_s = t0; r.end_s = t1;
            a.tl_tasks[k] = r;
        }
    };
    auto tl_release = [&](Flow &F) {
        F.tl = atomicAdd(&a.tl_cnt[1], 1ull);
        if (F.tl < a.tl_flow_cap) {
            triosim_flow_rec r;
            r.code = F.code; r.src = F.src; r.dst = F.dst; r.bytes = F.bytes; r.release_s = t;
            r.start_s = r.delivered_s = 0.0;
            a.tl_flows[F.tl] = r;
        }
    };
    auto tl_start = [&](const Flow &F) { if (F.tl < a.tl_flow_cap) a.tl_flows[F.tl].start_s = t; };
    auto tl_deliver = [&](const Flow &F) { if (F.tl < a.tl_flow_cap) a.tl_flows[F.tl].delivered_s = t; };

#define EV(kind, code)                                                        \
    do {                                                                      \
        acc += mix64(tmix ^ (((uint64_t)(kind) << 60) | (uint64_t)(code)));   \
        nev = true;                                                           \
    } while (0)
    // TS_PROF_H (profiling builds only): thread 0 accumulates clock64() cycles per phase of an instant and
    // prints them when its point finishes; a point stops after TS_PROF_H instants
#ifdef TS_PROF_H
    long long pf_c[7] = {0, 0, 0, 0, 0, 0, 0}, pf_last = clock64();
    unsigned pf_inner = 0, pf_outer = 0;
#define PFM(k)                                                                 \
    do {                                                                       \
        if (threadIdx.x == 0) { const long long c_ = clock64(); pf_c[k] += c_ - pf_last; pf_last = c_; } \
    } while (0)
#else
#define PFM(k) do {} while (0)
#endif

    auto grp_init = [&](Group &G, bool member, int p, int i, int lane0, int stride, uint64_t gid, uint32_t ncoll,
                        int slot) {
        G.member = member;
        G.p = p;
        G.i = i;
        G.lane0 = lane0;
        G.stride = stride;
        G.pred = lane0 + ((i + p - 1) % p) * stride;
        G.slot = slot;
        G.wmask = 0;
        const int last = lane0 + (p - 1) * stride;
        const bool inwarp = NW == 1 || (lane0 >> 5) == (last >> 5);
        if (member && inwarp)
            for (int k = 0; k < p; k++) G.wmask |= 1u << ((sbase + lane0 + k * stride) & 31);
        if constexpr (NW == 1) G.cross = false;               // (segments of a warp refill independently)
        else G.cross = sany(member && !inwarp);               // (a CTA segment refills as a whole)
        G.gid = gid;
        G.ncoll = ncoll;
        G.trig = G.donec = G.cur = 0;
        G.running = G.tree_cur = G.ldone = G.uprel = G.upd = G.dnrel = G.dnd = G.fup = false;
        G.dbt_cur = G.uprel2 = G.upd2 = G.dnrel2 = G.dnd2 = G.fup2 = false;
        G.K = G.D = G.Kp = 0;
        G.rb_cur = false;
        G.cS = G.chunk = 0.0;
        G.flow_deliv = 0;
        G.bd_t0 = 0.0;
        G.bd_l = 0;
    };
    auto gpu_of_member = [&](const Group &G, int k) -> uint32_t { return a.ro[TR.ro_off + G.lane0 + k * G.stride]; };
    auto tp_seq = [&](uint32_t P, uint32_t j, uint32_t e) -> uint32_t {
        return P == 0 ? j * HS.TF + e : P == 1 ? m * HS.TF + (m - 1 - j) * HS.TB + e : m * (HS.TF + HS.TB) + e;
    };

    // R10 for one group: done on this member, finish, start, releases (all lanes call it)
    auto grp_pass = [&](Group &G, Flow &F, Flow &F2, bool is_tp, bool &more) {
        // the predecessor's progress: a shuffle when every group of this kind lies inside one warp (TP groups;
        // segment-uniform), a shared-memory exchange across warps otherwise
        // (a cross-warp group reads it from s_dx, written before the pass's first barrier: G.D does not change
        // between that barrier and here)
        const int Dp = NW == 1 ? xch(G.D, G.pred)
                     : !G.cross ? __shfl_sync(FULL, G.D, G.pred & 31) : s_dx[is_tp ? 0 : 1][G.pred];
        LF upb, dnb, zero;
        upb.bits = dnb.bits = zero.bits = 0;
        upb.p = dnb.p = zero.p = nullptr;
        upb.sel = dnb.sel = zero.sel = 1;
        // (the vote / ballots must be warp-uniform: the segments of a warp may run different algorithms; a
        // CTA segment skips the vote when its point runs no tree)
        if ((NW == 1 || tree_algo || dbt_algo) && vany(G.tree_cur)) flags2(G.upd, G.dnd, upb, dnb);
        LF upb2 = zero, dnb2 = zero;
        if ((NW == 1 || dbt_algo) && vany(G.dbt_cur)) flags2(G.upd2, G.dnd2, upb2, dnb2);
        auto mb = [&](const LF &b, int k) -> bool { return b.test(G.lane0 + k * G.stride); };
        const int c1 = 2 * G.i + 1, c2 = 2 * G.i + 2;
        // R27's tree B: member i sits at heap position p - 1 - i
        const int hB = G.p - 1 - G.i, b1 = 2 * hB + 1, b2 = 2 * hB + 2;
        auto memB = [&](int h) { return G.p - 1 - h; };
        if (G.member && G.running && !G.ldone) {
            bool dn;
            if (!G.tree_cur) {
                dn = G.D == G.K && Dp == G.Kp;
            } else {
                const bool ku = (c1 >= G.p || mb(upb, c1)) && (c2 >= G.p || mb(upb, c2));
                const bool kd = (c1 >= G.p || mb(dnb, c1)) && (c2 >= G.p || mb(dnb, c2));
                dn = (G.i == 0 || (G.upd && G.dnd)) && ku && kd;
                if (G.dbt_cur) {
                    const bool kuB = (b1 >= G.p || mb(upb2, memB(b1))) && (b2 >= G.p || mb(upb2, memB(b2)));
                    const bool kdB = (b1 >= G.p || mb(dnb2, memB(b1))) && (b2 >= G.p || mb(dnb2, memB(b2)));
                    dn = dn && (hB == 0 || (G.upd2 && G.dnd2)) && kuB && kdB;
                }
            }
            if (dn) {
                G.ldone = true;
                G.donec = G.cur + 1;
                if constexpr (BD)
                    if (bd_rep) bd_add(is_tp ? 0u : 1u, G.bd_l, t - G.bd_t0);
            }
        }
        bool allfin, allrdy;
        if (NW > 1 && G.cross) {
            // one barrier for both votes: a group's members start and finish collectives together (running
            // is group-uniform), so each member also reports readiness for the next collective
            const int cb = gcb3;
            gcb3 = gcb3 == 2 ? 0 : gcb3 + 1;
            if (threadIdx.x < SL / 2) {   // next call's buffer (its last readers passed a barrier since)
                s_gca[gcb3][threadIdx.x] = 0u;
                s_gcb[gcb3][threadIdx.x] = 0u;
            }
            if (G.member) {
                const unsigned va = (G.ldone ? 1u : 0u) | (G.trig > G.cur ? (1u << 16) : 0u);
                if (va) atomicAdd(&s_gca[cb][G.slot], va);
                if (G.trig > G.cur + 1) atomicAdd(&s_gcb[cb][G.slot], 1u);
            }
            __syncthreads();
            const unsigned ca = s_gca[cb][G.slot], cbv = s_gcb[cb][G.slot], P = (unsigned)G.p;
            allfin = !G.member || (ca & 0xffffu) == P;
            const bool adv = G.member && G.running && allfin;
            if (adv) {
                G.running = false;
                G.cur++;
            }
            allrdy = !G.member || (adv ? cbv : (ca >> 16)) == P;
        } else {
            allfin = gall(G, G.ldone);
            if (G.member && G.running && allfin) {
                G.running = false;
                G.cur++;
            }
            allrdy = gall(G, G.trig > G.cur);
        }
        bool started = false;
        if (G.member && !G.running && G.cur < G.ncoll && allrdy) {
            CollEnt ce;
            if (is_tp) {
                const uint32_t c = G.cur;
                uint32_t off;
                if (c < m * HS.TF) off = c % HS.TF;
                else if (c < m * (HS.TF + HS.TB)) off = HS.TF + (c - m * HS.TF) % HS.TB;
                else off = HS.TF + HS.TB + (c - m * (HS.TF + HS.TB));
                ce = a.colls[HS.tcol_off + off];
            } else {
                ce = a.colls[HS.dcol_off + G.cur];
            }
            G.running = started = true;
            G.tree_cur = (tree_algo || dbt_algo) && ce.kind == CK_AR;
            G.dbt_cur = dbt_algo && ce.kind == CK_AR;
            G.cS = G.dbt_cur ? ce.S / 2.0 : ce.S;   // R27: each tree carries half the payload
            G.chunk = ce.S / (double)G.p / (double)C->nch;   // R25
            G.K = (ce.kind == CK_AR ? 2 * (G.p - 1) : (G.p - 1)) * (int)C->nch;
            G.Kp = G.K;
            G.rb_cur = C->algo == TRIOSIM_ALGO_REDBCAST && ce.kind == CK_AR;
            if (G.rb_cur) {
                // R26: reduce chunks (members != 0), then broadcast chunks (members != p-1)
                const int c = (int)C->nch, pl = G.i == 0 ? G.p - 1 : G.i - 1;
                G.chunk = ce.S / (double)c;
                G.K = (G.i != 0 ? c : 0) + (G.i != G.p - 1 ? c : 0);
                G.Kp = (pl != 0 ? c : 0) + (pl != G.p - 1 ? c : 0);
            }
            G.D = 0;
            G.ldone = G.uprel = G.upd = G.dnrel = G.dnd = false;
            G.uprel2 = G.upd2 = G.dnrel2 = G.dnd2 = false;
            if (G.i == 0) {
                EV(EV_COLL_START, (G.gid << 20) | G.cur);
                alg += 1;
            }
            if constexpr (BD) {
                G.bd_t0 = t;
                G.bd_l = ce.layer;
            }
        }
        if (G.member && G.running && F.st == FS_NONE) {
            const uint64_t cc = (G.gid << 20) | G.cur;
            bool rel = false;
            if (!G.tree_cur) {
                const int c = (int)C->nch;
                bool go;
                if (!G.rb_cur) go = G.D < G.K && (G.D < c || Dp >= G.D - c + 1);   // R25 chunk q waits for q - nch
                // R26 (Dp is the previous collective's at this one's start)
                else if (G.i != 0 && G.D < c) go = G.i == 1 || (!started && Dp >= G.D + 1);   // reduce chunk
                else go = G.D < G.K && !started && Dp >= (G.i <= 1 ? 0 : c) + (G.D - (G.i != 0 ? c : 0)) + 1;   // broadcast
                if (go) {
                    release(a, TR, F, gpu, gpu_of_member(G, (G.i + 1) % G.p), G.chunk,
                            (cc << 32) | ((uint64_t)G.D << 16) | (uint64_t)G.i, t, lats, alg);
                    rel = true;
                }
            } else if (G.i >= 1) {
                const LF ub = started ? zero : upb, db = started ? zero : dnb;
                const bool ku = (c1 >= G.p || mb(ub, c1)) && (c2 >= G.p || mb(ub, c2));
                const int par = (G.i - 1) / 2;
                if (!G.uprel && ku) {
                    release(a, TR, F, gpu, gpu_of_member(G, par), G.cS, (cc << 32) | (uint64_t)G.i, t, lats, alg);
                    G.fup = G.uprel = rel = true;
                } else if (G.uprel && G.upd && !G.dnrel &&
                           (par == 0 ? ((G.p <= 1 || mb(ub, 1)) && (G.p <= 2 || mb(ub, 2))) : mb(db, par))) {
                    release(a, TR, F, gpu_of_member(G, par), gpu, G.cS, (cc << 32) | (1ull << 16) | (uint64_t)G.i, t,
                            lats, alg);
                    G.fup = false;
                    G.dnrel = rel = true;
                }
            }
            if (rel) {
                EV(EV_RELEASE, F.code);
                if constexpr (LOG) tl_release(F);
                if (F.t_act == t) more = true;
            }
        }
        // R27 tree B (mirrored heap positions, steps 2 up / 3 down) on the lane's second slot
        if (G.member && G.running && G.dbt_cur && hB >= 1 && F2.st == FS_NONE) {
            const uint64_t cc = (G.gid << 20) | G.cur;
            const LF ub = started ? zero : upb2, db = started ? zero : dnb2;
            const bool ku = (b1 >= G.p || mb(ub, memB(b1))) && (b2 >= G.p || mb(ub, memB(b2)));
            const int parh = (hB - 1) / 2, par = memB(parh);
            bool rel = false;
            if (!G.uprel2 && ku) {
                release(a, TR, F2, gpu, gpu_of_member(G, par), G.cS, (cc << 32) | (2ull << 16) | (uint64_t)G.i, t, lats,
                        alg);
                G.fup2 = G.uprel2 = rel = true;
            } else if (G.uprel2 && G.upd2 && !G.dnrel2 &&
                       (parh == 0 ? ((G.p <= 1 || mb(ub, memB(1))) && (G.p <= 2 || mb(ub, memB(2)))) : mb(db, par))) {
                release(a, TR, F2, gpu_of_member(G, par), gpu, G.cS, (cc << 32) | (3ull << 16) | (uint64_t)G.i, t, lats,
                        alg);
                G.fup2 = false;
                G.dnrel2 = rel = true;
            }
            if (rel) {
                EV(EV_RELEASE, F2.code);
                if constexpr (LOG) tl_release(F2);
                if (F2.t_act == t) more = true;
            }
        }
    };
    // (b)/(c) for one flow slot; returns true if delivered
    auto flow_step = [&](Flow &F, bool &dirty) -> bool {
        if (F.st == FS_ACT && F.t_drain == t) {
            F.st = FS_NONE;
            EV(EV_DELIVER, F.code);
            if constexpr (LOG) tl_deliver(F);
            if (TR.phot) p_t[F.hl[1] * NTHR + threadIdx.x] = t;   // R20: the logical link was last used now
            else dirty = true;
            return true;
        }
        if (F.st == FS_LAT && F.t_act == t) {
            EV(EV_ACTIVATE, F.code);
            if constexpr (LOG) tl_start(F);
            if (F.bytes == 0.0 || F.len == 0) {
                F.st = FS_NONE;
                EV(EV_DELIVER, F.code);
                if constexpr (LOG) tl_deliver(F);
                return true;
            }
            F.st = FS_ACT;
            F.rem = F.bytes;
            F.t_upd = t;
            F.rate = 0.0;
            F.t_drain = dinf();
            dirty = true;
        }
        return false;
    };
    auto grp_delivered = [&](Group &G) {
        G.flow_deliv++;
        if (G.tree_cur) {
            if (G.fup) G.upd = true; else G.dnd = true;
        } else {
            G.D++;
        }
    };
    auto grp_delivered2 = [&](Group &G) {   // R27: a tree-B edge of G (on the lane's second slot)
        G.flow_deliv++;
        if (G.fup2) G.upd2 = true; else G.dnd2 = true;
    };
    // decode program position q of this stage -> (phase, micro-batch, index in phase list)
    auto decode = [&](uint32_t q, uint32_t &P, uint32_t &j, uint32_t &idx) {
        if (q < m * SI.nF) { P = 0; j = q / SI.nF; idx = q % SI.nF; }
        else if (q < m * (SI.nF + SI.nB)) { const uint32_t r = q - m * SI.nF; P = 1; j = m - 1 - r / SI.nB; idx = r % SI.nB; }
        else { P = 2; j = 0; idx = q - m * (SI.nF + SI.nB); }
    };
    auto ent_at = [&](uint32_t P, uint32_t idx) -> HEnt {
        return a.hents[SI.ent_off + (P == 0 ? 0 : P == 1 ? SI.nF : SI.nF + SI.nB) + idx];
    };
    auto has_wait = [&](const HEnt &en, uint32_t P, uint32_t idx) -> bool {
        return en.nrecv > 0 || en.tpw >= 0 || (P == 2 && idx == HS.first_opt && GD.ncoll > 0);
    };
    auto has_sig = [&](const HEnt &en, uint32_t j) -> bool {
        return en.nsend > 0 || en.tp_nsig > 0 || (en.dp_nsig > 0 && j == 0);
    };

    for (;;) {
        // ------------------------------ refill ------------------------------
        const bool need = !have && !exhausted;
        bool fresh = false, rbad = false, rlong = false;
        // (a CTA is one segment: have / exhausted are block-uniform, so it needs no vote here)
        if (NW > 1 ? need : vany(need)) {
            uint32_t it = 0;
            if constexpr (NW == 1) {
                if (need && li == 0) it = atomicAdd(a.counter, 1u);
                it = __shfl_sync(FULL, it, sbase);
            } else {
                if (need && threadIdx.x == 0) s_item = atomicAdd(a.counter, 1u);
                __syncthreads();
                it = s_item;
                __syncthreads();
            }
            if (need) {
                if (it >= a.n_work) {
                    exhausted = true;
                } else if (a.work[it] < a.rlo || a.work[it] >= a.rhi) {
                    // outside [first, first + count) of this simulate_batch call: skipped, refilled next pass
                } else {
                    fresh = have = true;
                    const PointDesc pd = a.pts[a.work[it]];
                    pidx = pd.idx;
                    bws = pd.bw_scale;
                    lats = pd.lat_scale;
                    C = &a.cls[pd.cls];
                    {
                        const TopoDev td = a.topo[pd.topo];
                        TR.n_gpus = td.n_gpus; TR.link_off = td.link_off; TR.rt_off = td.rt_off; TR.ro_off = td.ro_off;
                        TR.n_links = td.n_links;
                        TR.phot = td.net == TRIOSIM_NET_PHOTONIC;
                        ports = (int)td.ports;
                        bufs = (int)td.buf_slots;
                        ph_bw = td.ph_bw * bws;
                        ph_set = td.ph_setup * lats;
                        ph_lat = td.ph_lat * lats;
                    }
                    S = (int)C->p;
                    tp = (int)C->tpdeg;
                    dp = (int)C->dp;
                    R = dp * S * tp;
                    m = C->m;
                    tree_algo = C->algo == TRIOSIM_ALGO_TREE;
                    dbt_algo = C->algo == TRIOSIM_ALGO_DBTREE;
                    t = 0.0;
                    tmix = mix64(0ull);
                    ninst = nwf = nrounds = maxact = 0;
                    bon = false;
                    bstart = cbusy = 0.0;
                    used = li < R;
                    pos = run_start = run_end = 0;
                    cst = CS_IDLE;
                    t_end = busy = 0.0;
                    ntask = nflow = np2p = 0;
                    sq = dcnt = 0;
                    hc_pos = 0xffffffffu;
                    FT.st = FD.st = FP.st = FS_NONE;
                    acc = alg = 0;
                    nev = false;
                    const int r = used ? li : 0;
                    d = r / (S * tp);
                    s = (r / tp) % S;
                    tt = r % tp;
                    bd_rep = used && d == 0 && tt == 0;
                    SI = a.stages[C->stage_off + s];
                    HS = a.hst[C->hst_off + s];
                    nprog = used ? m * (SI.nF + SI.nB) + SI.nO : 0;
                    nsend_tot = used ? m * (SI.SF + SI.SB) + SI.SO : 0;
                    gpu = a.ro[TR.ro_off + r];
                    const uint32_t ntp = tp > 1 ? m * (HS.TF + HS.TB) + HS.TO : 0;
                    const uint32_t ndp = dp > 1 ? HS.ndp : 0;
                    grp_init(GT, used && tp > 1, tp, tt, (d * S + s) * tp, 1, (uint64_t)(d * S + s), ntp, d * S + s);
                    grp_init(GD, used && dp > 1, dp, d, s * tp + tt, S * tp,
                             (uint64_t)((tp > 1 ? dp * S : 0) + s * tp + tt), ndp, s * tp + tt);
                    if constexpr (NW > 1) {
                        ph_tables(TR.phot);
                        if (!TR.phot && last_phot)   // the link counters must start at 0 again
                            for (int q = (int)threadIdx.x; q < LMAX; q += NTHR) { ln[q] = 0; lk[q] = 0; }
                        last_phot = TR.phot;
                    }
                    if (TR.phot) {
                        for (int k = 0; k < ports; k++) p_st[k * NTHR + threadIdx.x] = 0;
                        for (int k = 0; k < 3; k++) q_g[threadIdx.x * 3 + k] = 0;
                    }
                    if (used && !TR.phot) {
                        // route checks of every pair this rank's flows will use (R3)
                        auto chk = [&](uint32_t x, uint32_t y) {
                            const int l = route_len(a, TR, x, y);
                            if (l == NO_ROUTE) rbad = true;   // (any length: hops past MAX_HOPS are read from rt_links)
                        };
                        for (int gk = 0; gk < 2; gk++) {
                            const Group &G = gk == 0 ? GT : GD;
                            if (!G.member || G.ncoll == 0) continue;
                            if (C->need_ring) chk(gpu, gpu_of_member(G, (G.i + 1) % G.p));
                            if (C->need_tree && G.i >= 1) {
                                const uint32_t par = gpu_of_member(G, (G.i - 1) / 2);
                                chk(gpu, par);
                                chk(par, gpu);
                            }
                            if (C->need_tree && dbt_algo && G.p - 1 - G.i >= 1) {   // R27 tree B's edge to its parent
                                const uint32_t par = gpu_of_member(G, G.p - 1 - (G.p - 2 - G.i) / 2);
                                chk(gpu, par);
                                chk(par, gpu);
                            }
                        }
                        unsigned long long dm = SI.dst_mask;
                        while (dm) {
                            const int ds = __ffsll((long long)dm) - 1;
                            dm &= dm - 1;
                            chk(gpu, a.ro[TR.ro_off + (d * S + ds) * tp + tt]);
                        }
                    }
                }
            }
            if (vany(fresh && (rbad || rlong))) {
                const bool bad = sany(fresh && rbad);
                const bool lng = sany(fresh && rlong);
                if (fresh && (bad || lng)) {
                    if (li == 0) {
                        triosim_result rr = {};
                        rr.status = bad ? TRIOSIM_PT_NO_ROUTE : TRIOSIM_PT_TOO_LARGE;
                        a.out[pidx] = rr;
                    }
                    have = used = false;
                    GT.member = GD.member = false;
                }
            }
        }
        if (NW > 1 ? (!have && exhausted) : vall(!have && exhausted)) break;

        // ------------------------------ one instant ------------------------------
        PFM(0);
        bool dirty = false;
        if (TR.phot && used)   // R20: logical links whose setup completes now are up (last use = now)
            for (int k = 0; k < ports; k++)
                if (p_st[k * NTHR + threadIdx.x] == 1 && p_t[k * NTHR + threadIdx.x] == t) p_st[k * NTHR + threadIdx.x] = 2;
        for (;;) {
            for (;;) {
                bool more = false;
                // (a) completions
                if (used && cst == CS_RUN && t_end == t) {
                    cst = CS_IDLE;
                    pos = run_end;
                    uint32_t P, j, idx;
                    decode(pos - 1, P, j, idx);
                    const HEnt en = ent_at(P, idx);
                    GT.trig += en.tp_nsig;
                    if (j == 0) GD.trig += en.dp_nsig;
                    if (has_sig(en, j)) EV(EV_TASK_END, ((uint64_t)gpu << 40) | (pos - 1));
                }
                // (b) / (c) for the three flow slots
                if (used) {
                    // R27: with a double binary tree, the group's tree B runs on the other group's (absent) slot
                    if (flow_step(FT, dirty)) { nflow++; if (dbt_algo && dp > 1) grp_delivered2(GD); else grp_delivered(GT); }
                    if (flow_step(FD, dirty)) { nflow++; if (dbt_algo && tp > 1) grp_delivered2(GT); else grp_delivered(GD); }
                    if (flow_step(FP, dirty)) {
                        nflow++; np2p++; dcnt++;
                        if constexpr (BD)
                            if (bd_rep) bd_add(2u, bd_p_l, t - bd_p_t0);
                    }
                }
                cnt[li] = dcnt;
                if constexpr (NW > 1) {
                    s_dx[0][threadIdx.x] = GT.D;
                    s_dx[1][threadIdx.x] = GD.D;
                }
                ssync();
                // (d) both groups, then this rank's next P2P send
                grp_pass(GT, FT, FD, true, more);
                grp_pass(GD, FD, FT, false, more);
                if (used && FP.st == FS_NONE && sq < nsend_tot) {
                    uint32_t P, j, e;
                    if (sq < m * SI.SF) { P = 0; j = sq / SI.SF; e = sq % SI.SF; }
                    else if (sq < m * (SI.SF + SI.SB)) { const uint32_t r = sq - m * SI.SF; P = 1; j = m - 1 - r / SI.SB; e = r % SI.SB; }
                    else { P = 2; j = 0; e = sq - m * (SI.SF + SI.SB); }
                    const HSend se = a.hsends[SI.send_off + (P == 0 ? 0 : P == 1 ? SI.SF : SI.SF + SI.SB) + e];
                    const uint32_t prodpos = P == 0 ? j * SI.nF + se.pidx
                                           : P == 1 ? m * SI.nF + (m - 1 - j) * SI.nB + se.pidx
                                                    : m * (SI.nF + SI.nB) + se.pidx;
                    const uint32_t donepos = (cst == CS_RUN) ? run_start : pos;
                    const bool gate = se.tpg < 0 ||
                                      GT.donec > tp_seq((uint32_t)se.tpg >> 24, j, (uint32_t)se.tpg & 0xffffffu);
                    if (donepos > prodpos && gate) {
                        const uint32_t dg = a.ro[TR.ro_off + (d * S + se.dst) * tp + tt];
                        release(a, TR, FP, gpu, dg, se.bytes,
                                (1ull << 59) | ((uint64_t)se.x << 32) | ((uint64_t)j << 16) | (uint64_t)dg, t, lats, alg);
                        EV(EV_RELEASE, FP.code);
                        if constexpr (LOG) tl_release(FP);
                        if constexpr (BD) {
                            bd_p_t0 = t;
                            bd_p_l = a.layer[ent_at(P, se.pidx).op];
                        }
                        sq++;
                        if (FP.t_act == t) more = true;
                    }
                }
                // (e) compute start
                const bool hc_blocked = hc_pos == pos && (hc_kind == 0 ? !(cnt[hc_a] > hc_b)
                                                          : hc_kind == 1 ? !(GT.donec > hc_b) : GD.donec < GD.ncoll);
                if (used && cst == CS_IDLE && pos < nprog && !hc_blocked) {
                    uint32_t P, j, idx;
                    decode(pos, P, j, idx);
                    HEnt en = ent_at(P, idx);
                    bool ok = true;
                    for (uint32_t r = 0; r < en.nrecv && ok; r++) {
                        const RecvEnt re = a.recvs[en.recv_off + r];
                        const StageInfo &ps = a.stages[C->stage_off + re.src];
                        const uint32_t jp = (re.phase == 2 || P == 2) ? 0 : j;
                        const uint32_t seqi = re.phase == 0 ? jp * ps.SF + re.e
                                            : re.phase == 1 ? m * ps.SF + (m - 1 - jp) * ps.SB + re.e
                                                            : m * (ps.SF + ps.SB) + re.e;
                        if (!(cnt[(d * S + re.src) * tp + tt] > seqi)) {
                            ok = false;
                            hc_pos = pos; hc_kind = 0; hc_a = (d * S + re.src) * tp + tt; hc_b = seqi;
                        }
                    }
                    if (ok && en.tpw >= 0) {
                        const uint32_t pp_ = (uint32_t)en.tpw >> 24, ee = (uint32_t)en.tpw & 0xffffffu;
                        const uint32_t jp = (pp_ == 2 || P == 2) ? 0 : j;
                        if (!(GT.donec > tp_seq(pp_, jp, ee))) {
                            ok = false;
                            hc_pos = pos; hc_kind = 1; hc_b = tp_seq(pp_, jp, ee);
                        }
                    }
                    if (ok && P == 2 && idx == HS.first_opt && GD.ncoll > 0 && GD.donec < GD.ncoll) {
                        ok = false;
                        hc_pos = pos; hc_kind = 2;
                    }
                    if (ok) {
                        if (has_wait(en, P, idx)) EV(EV_TASK_START, ((uint64_t)gpu << 40) | pos);
                        run_start = pos;
                        // fold (R16): K2's run from the head within its phase list (run0 for micro-batch
                        // instance 0), then on into the next lists while a run ends at a list end
                        // without a signal and the next list's first operator waits for nothing
                        const HEnt *L = a.hents + SI.ent_off + (P == 0 ? 0 : P == 1 ? SI.nF : SI.nF + SI.nB);
                        uint32_t len = P == 0 ? SI.nF : P == 1 ? SI.nB : SI.nO;
                        uint32_t n = j == 0 ? en.run0 : en.run, i0 = idx, q = pos;
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
                            if (has_sig(L[last], j) || last + 1 < len || q >= nprog) break;
                            decode(q, P, j, i0);
                            L = a.hents + SI.ent_off + (P == 0 ? 0 : P == 1 ? SI.nF : SI.nF + SI.nB);
                            len = P == 0 ? SI.nF : P == 1 ? SI.nB : SI.nO;
                            if (has_wait(L[0], P, 0)) break;
                            n = j == 0 ? L[0].run0 : L[0].run;
                        }
                        ntask += q - pos;
                        alg += 2 * (q - pos);
                        run_end = q;
                        t_end = te;
                        cst = CS_RUN;
                        if (te == t) more = true;
                    }
                }
                if constexpr (NW == 1) ssync();   // (a CTA's vote below is a barrier itself)
#ifdef TS_PROF_H
                pf_inner++;
#endif
                if (!vany(more)) break;
            }
            PFM(1);
#ifdef TS_PROF_H
            pf_outer++;
#endif

            bool again = false;
            // (f') R20 photonic network: (i) a logical link per request, (ii) link heads ask for a
            // receive buffer, (iii) destinations grant buffers in (release time, code) order
            const bool phw = TR.phot && used && (FT.st >= PS_REQ || FD.st >= PS_REQ || FP.st >= PS_REQ);
            if ((NW == 1 || TR.phot) && vany(phw)) {   // (a CTA segment runs one point: TR.phot is uniform)
                const int me = (int)threadIdx.x;
                auto onlink = [&](int k) -> bool {   // a transfer of this lane is queued on / using link k
                    auto u = [&](const Flow &F) { return (F.st >= PS_LINKQ || F.st == FS_ACT) && (int)F.hl[1] == k; };
                    return u(FT) || u(FD) || u(FP);
                };
                auto klt = [](double ta, uint64_t ca, double tb, uint64_t cb) { return ta < tb || (ta == tb && ca < cb); };
                if (phw) {
                    // (i) requests in key order: existing link, free port, else tear down the link idle longest
                    // (the slots are chosen by index, never by address: a Flow whose address is taken would
                    // live in local memory for the whole kernel)
                    auto with_slot = [&](int k, auto &&fn) { if (k == 0) fn(FT); else if (k == 1) fn(FD); else fn(FP); };
                    for (int r = 0; r < 3; r++) {
                        int bi = -1;
                        double bt = 0.0;
                        uint64_t bc = 0;
                        auto pick = [&](const Flow &F, int k) {
                            if (F.st == PS_REQ && F.len == 0 && (bi < 0 || klt(F.t_upd, F.code, bt, bc))) { bi = k; bt = F.t_upd; bc = F.code; }
                        };
                        pick(FT, 0); pick(FD, 1); pick(FP, 2);
                        if (bi < 0) break;
                        with_slot(bi, [&](Flow &F) {
                        F.len = 1;   // visited in this pass
                        const int dg = (int)F.hl[0];
                        int k = -1;
                        for (int q = 0; q < ports; q++)
                            if (p_st[q * NTHR + me] != 0 && p_dst[q * NTHR + me] == dg) k = q;
                        if (k < 0) {
                            int nk = -1;
                            for (int q = 0; q < ports && nk < 0; q++) if (p_st[q * NTHR + me] == 0) nk = q;
                            if (nk < 0)
                                for (int q = 0; q < ports; q++) {
                                    if (p_st[q * NTHR + me] != 2 || onlink(q)) continue;
                                    if (nk < 0 || p_t[q * NTHR + me] < p_t[nk * NTHR + me] ||
                                        (p_t[q * NTHR + me] == p_t[nk * NTHR + me] && p_dst[q * NTHR + me] < p_dst[nk * NTHR + me]))
                                        nk = q;
                                }
                            if (nk >= 0) {
                                const double tr = t + ph_set;
                                p_dst[nk * NTHR + me] = dg;
                                p_st[nk * NTHR + me] = tr == t ? 2 : 1;
                                p_t[nk * NTHR + me] = tr;
                                k = nk;
                                alg += 1;
                            }
                        }
                        if (k >= 0) { F.st = PS_LINKQ; F.hl[1] = (uint32_t)k; }
                        });
                    }
                    FT.len = FT.st == PS_REQ ? 0 : FT.len;
                    FD.len = FD.st == PS_REQ ? 0 : FD.len;
                    FP.len = FP.st == PS_REQ ? 0 : FP.len;
                    // (ii) an up link with nothing waiting for a buffer or moving passes its queue head on
                    for (int r = 0; r < 3; r++) {
                        int hi = -1;
                        double ht = 0.0;
                        uint64_t hc = 0;
                        auto hd = [&](const Flow &F, int q) {
                            if (F.st != PS_LINKQ) return;
                            const int k = (int)F.hl[1];
                            if (p_st[k * NTHR + me] != 2) return;
                            auto busy = [&](const Flow &G) { return (G.st == PS_BUFW || G.st == FS_ACT) && (int)G.hl[1] == k; };
                            if (busy(FT) || busy(FD) || busy(FP)) return;
                            if (hi < 0 || klt(F.t_upd, F.code, ht, hc)) { hi = q; ht = F.t_upd; hc = F.code; }
                        };
                        hd(FT, 0); hd(FD, 1); hd(FP, 2);
                        if (hi < 0) break;
                        with_slot(hi, [&](Flow &F) { F.st = PS_BUFW; });
                    }
                }
                // (iii) publish buffer requests and transfers, each destination grants in key order
                auto pub = [&](const Flow &F, int k) {
                    const int e = me * 3 + k;
                    const bool w = TR.phot && used && (F.st == PS_BUFW || (F.st == FS_ACT && F.len == 0));
                    q_dst[e] = w ? (int)F.hl[0] : -1;
                    q_st[e] = F.st == PS_BUFW ? 1 : 2;
                    q_t[e] = F.t_upd;
                    q_code[e] = F.code;
                };
                pub(FT, 0);
                pub(FD, 1);
                pub(FP, 2);
                ssync();
                if (TR.phot && used) {
                    const int e0 = NW == 1 ? (wid * 32 + sbase) * 3 : 0, e1 = e0 + 3 * SL;
                    const int g = (int)gpu;
                    int occ = 0, nc = 0;
                    for (int e = e0; e < e1; e++)
                        if (q_dst[e] == g) { if (q_st[e] == 2) occ++; else nc++; }
                    if (nc > 0) {
                        const int fr = bufs > 0 ? bufs - occ : nc;
                        if (fr >= nc) {
                            for (int e = e0; e < e1; e++) if (q_dst[e] == g && q_st[e] == 1) q_g[e] = 1;
                        } else {
                            for (int r = 0; r < fr; r++) {
                                int be = -1;
                                for (int e = e0; e < e1; e++)
                                    if (q_dst[e] == g && q_st[e] == 1 && !q_g[e] &&
                                        (be < 0 || klt(q_t[e], q_code[e], q_t[be], q_code[be])))
                                        be = e;
                                q_g[be] = 1;
                            }
                        }
                    }
                }
                ssync();
                auto take = [&](Flow &F, int k) {
                    const int e = me * 3 + k;
                    if (q_g[e]) {
                        q_g[e] = 0;
                        F.st = FS_ACT;
                        F.len = 0;
                        F.t_drain = (t + ph_lat) + F.bytes / ph_bw;
                        alg += 3;
                        EV(EV_ACTIVATE, F.code);
                        if constexpr (LOG) tl_start(F);
                        if (F.t_drain == t) again = true;
                    }
                };
                take(FT, 0);
                take(FD, 1);
                take(FP, 2);
                const uint32_t nx = scount(TR.phot && used && FT.st == FS_ACT) + scount(TR.phot && used && FD.st == FS_ACT) +
                                    scount(TR.phot && used && FP.st == FS_ACT);
                if (TR.phot && have && nx > maxact) maxact = nx;
            }

            PFM(2);
            // (f) R14 over every in-transit flow of the segment (up to three per lane)
            if (!vany(dirty)) {
                if (!vany(again)) break;
                continue;
            }
            if constexpr (NW > 1)
            {
                if (threadIdx.x == 0) s_na = 0;   // (its last readers passed barriers since)
                // the call's link masks (s_dx's words: the event loop's progress exchange is over): bit j of
                // thread i's word = link j * NTHR + i is counted / has flows frozen in this round
                s_dx[0][threadIdx.x] = 0;
                s_dx[1][threadIdx.x] = 0;
            }
            const bool segdirty = sany(dirty);
            dirty = false;
            const bool aT = segdirty && used && FT.st == FS_ACT;
            const bool aD = segdirty && used && FD.st == FS_ACT;
            const bool aP = segdirty && used && FP.st == FS_ACT;
            auto progress = [&](Flow &F, bool on) {
                if (on && F.t_upd < t) {
                    const double r = F.rem - F.rate * (t - F.t_upd);
                    F.rem = r > 0.0 ? r : 0.0;
                    F.t_upd = t;
                    alg += 4;
                }
            };
            progress(FT, aT);
            progress(FD, aD);
            progress(FP, aP);
            // link counters are 0 here: every complete progressive filling returns them to 0
            // progressive filling: each round freezes every unfrozen flow crossing a link whose share is
            // the minimum s; the owners then update those links' residual, count and share
            auto fmin = [&](const Flow &F, bool on) -> double {
                double my = dinf();
                if (on) {
#pragma unroll
                    for (int h = 0; h < MAX_HOPS; h++)
                        if (h < F.len) {
                            const double sh = lsh[hop(F.hl, h)];
                            my = sh < my ? sh : my;
                        }
                    for (int h = MAX_HOPS; h < F.len; h++) {
                        const double sh = lsh[a.rt_links[F.roff + h]];
                        my = sh < my ? sh : my;
                    }
                }
                return my;
            };
            uint32_t rounds = 0;
            uint32_t nact;
            if constexpr (NW > 1) {
                // CTA: flows count their links with fire-and-forget shared-memory adds (no returned value on
                // the critical path); then the topology's links are spread over all threads, which set
                // residual and share of every counted link, and after each round's freezes update every link
                // with frozen flows.  Same per-link expressions (R14), so the same bits as the warp path.
                const int nl = (int)TR.n_links;
                const bool lmask = nl <= 32 * NTHR;   // block-uniform: the links fit the per-thread masks
                unsigned *um = reinterpret_cast<unsigned *>(s_dx[0]), *dm = reinterpret_cast<unsigned *>(s_dx[1]);
                auto mark = [&](unsigned *mk, int e) {
                    if (lmask) atomicOr(&mk[e & (NTHR - 1)], 1u << (e / NTHR));
                };
                auto count_c = [&](const Flow &F, bool on) {
                    if (on) {
                        alg += F.len;
                        auto c1 = [&](int e) { atomicAdd(&ln[e], 1); mark(um, e); };
#pragma unroll
                        for (int h = 0; h < MAX_HOPS; h++)
                            if (h < F.len) c1(hop(F.hl, h));
                        for (int h = MAX_HOPS; h < F.len; h++) c1(a.rt_links[F.roff + h]);
                    }
                };
                count_c(FT, aT);
                count_c(FD, aD);
                count_c(FP, aP);
                const int na = (aT ? 1 : 0) + (aD ? 1 : 0) + (aP ? 1 : 0);
                if (na) atomicAdd(&s_na, na);
                __syncthreads();
                nact = (uint32_t)s_na;
                auto init1 = [&](int e) {
                    const int c = ln[e];
                    if (c > 0) {
                        const double r0 = a.link_bw[TR.link_off + e] * bws;
                        lres[e] = r0;
                        lsh[e] = r0 / (double)c;
                        alg += 2;
                    }
                };
                if (lmask) {
                    for (unsigned mm = um[threadIdx.x]; mm; mm &= mm - 1) init1((__ffs(mm) - 1) * NTHR + (int)threadIdx.x);
                } else {
                    for (int e = (int)threadIdx.x; e < nl; e += NTHR) init1(e);
                }
                __syncthreads();
                PFM(3);
                bool uT = aT, uD = aD, uP = aP;
                for (;;) {
                    const double mT = fmin(FT, uT), mD = fmin(FD, uD), mP = fmin(FP, uP);
                    double my = mT < mD ? mT : mD;
                    my = mP < my ? mP : my;
                    const double sm = smin(my);   // block-uniform; +inf: nothing left to freeze
                    if (!(sm < dinf())) break;
                    const bool iT = uT && mT == sm, iD = uD && mD == sm, iP = uP && mP == sm;
                    auto freeze_c = [&](Flow &F, bool in) {
                        if (in) {
                            F.rate = sm;
                            auto f1 = [&](int e) { atomicAdd(&lk[e], 1); mark(dm, e); };
#pragma unroll
                            for (int h = 0; h < MAX_HOPS; h++)
                                if (h < F.len) f1(hop(F.hl, h));
                            for (int h = MAX_HOPS; h < F.len; h++) f1(a.rt_links[F.roff + h]);
                        }
                    };
                    freeze_c(FT, iT);
                    freeze_c(FD, iD);
                    freeze_c(FP, iP);
                    __syncthreads();
                    auto upd1 = [&](int e) {
                        const int kk = lk[e];
                        if (kk) {
                            const double r = lres[e] - sm * (double)kk;
                            const double rr = r > 0.0 ? r : 0.0;
                            const int nn = ln[e] - kk;
                            lres[e] = rr;
                            ln[e] = nn;
                            lk[e] = 0;
                            if (nn > 0) lsh[e] = rr / (double)nn;
                            alg += 5;
                        }
                    };
                    if (lmask) {
                        const unsigned mm0 = dm[threadIdx.x];
                        dm[threadIdx.x] = 0;   // (the next round's marks follow this round's closing barrier)
                        for (unsigned mm = mm0; mm; mm &= mm - 1) upd1((__ffs(mm) - 1) * NTHR + (int)threadIdx.x);
                    } else {
                        for (int e = (int)threadIdx.x; e < nl; e += NTHR) upd1(e);
                    }
                    __syncthreads();
                    rounds++;
                    uT = uT && !iT;
                    uD = uD && !iD;
                    uP = uP && !iP;
                }
            } else {
                // warp segments: the first flow to count a link owns it for this call: it sets the residual,
                // computes the share and updates both whenever flows on the link freeze (R14's single
                // per-link expression)
                unsigned lo = 0;   // owned links: bit slot * 8 + hop (the first MAX_HOPS hops)
                unsigned lt = 0;   // bit slot: this slot owns links past MAX_HOPS (marked in lown)
                auto count = [&](const Flow &F, bool on, int slot) {
                    if (on) {
                        alg += F.len;
    #pragma unroll
                        for (int h = 0; h < MAX_HOPS; h++)
                            if (h < F.len) {
                                const int e = hop(F.hl, h);
                                if (atomicAdd(&ln[e], 1) == 0) {
                                    lo |= 1u << (slot * 8 + h);
                                    lown[e] = li * 4 + slot;   // (so no stale owner mark of an earlier call matches)
                                    lres[e] = a.link_bw[TR.link_off + e] * bws;
                                }
                            }
                        for (int h = MAX_HOPS; h < F.len; h++) {   // long routes
                            const int e = a.rt_links[F.roff + h];
                            if (atomicAdd(&ln[e], 1) == 0) {
                                lown[e] = li * 4 + slot;
                                lt |= 1u << slot;
                                lres[e] = a.link_bw[TR.link_off + e] * bws;
                            }
                        }
                    }
                };
                count(FT, aT, 0);
                count(FD, aD, 1);
                count(FP, aP, 2);
                ssync();
                auto owned = [&](auto &&fn) {   // fn(link) for every link this lane owns
                    // the cached hops: one bit scan (one copy of fn); the slot's words are selected, not
                    // addressed, so the flow slots stay in registers
                    for (unsigned m = lo; m; m &= m - 1) {
                        const int b = __ffs(m) - 1, sl = b >> 3, h = b & 7, q = h >> 1;
                        const uint32_t x0 = sl == 0 ? FT.hl[0] : sl == 1 ? FD.hl[0] : FP.hl[0];
                        const uint32_t x1 = sl == 0 ? FT.hl[1] : sl == 1 ? FD.hl[1] : FP.hl[1];
                        const uint32_t x2 = sl == 0 ? FT.hl[2] : sl == 1 ? FD.hl[2] : FP.hl[2];
                        const uint32_t x3 = sl == 0 ? FT.hl[3] : sl == 1 ? FD.hl[3] : FP.hl[3];
                        const uint32_t w = q == 0 ? x0 : q == 1 ? x1 : q == 2 ? x2 : x3;
                        fn((int)((w >> (16 * (h & 1))) & 0xffffu));
                    }
                    if (lt) {   // hops past the cache (long routes): the owner marks
                        auto tail = [&](const Flow &F, int slot) {
                            if ((lt >> slot) & 1u)
                                for (int h = MAX_HOPS; h < F.len; h++) {
                                    const int e = a.rt_links[F.roff + h];
                                    if (lown[e] == li * 4 + slot) fn(e);
                                }
                        };
                        tail(FT, 0);
                        tail(FD, 1);
                        tail(FP, 2);
                    }
                };
                owned([&](int e) { lsh[e] = lres[e] / (double)ln[e]; alg += 2; });
                ssync();
                PFM(3);
                // warp segments: every lane its own (up to three) flows, segment minimum per round
                bool uT = aT, uD = aD, uP = aP;
                for (;;) {
                    const double mT = fmin(FT, uT), mD = fmin(FD, uD), mP = fmin(FP, uP);
                    double my = mT < mD ? mT : mD;
                    my = mP < my ? mP : my;
                    const double sm = smin(my);   // segment-uniform; +inf: nothing left to freeze
                    const bool segact = sm < dinf();
                    if constexpr (NW == 1) {
                        if (!__any_sync(FULL, segact)) break;
                    } else {
                        if (!segact) break;
                    }
                    const bool iT = uT && mT == sm, iD = uD && mD == sm, iP = uP && mP == sm;
                    auto freeze = [&](Flow &F, bool in) {
                        if (in) {
                            F.rate = sm;
    #pragma unroll
                            for (int h = 0; h < MAX_HOPS; h++)
                                if (h < F.len) atomicAdd(&lk[hop(F.hl, h)], 1);
                            for (int h = MAX_HOPS; h < F.len; h++) atomicAdd(&lk[a.rt_links[F.roff + h]], 1);
                        }
                    };
                    freeze(FT, iT);
                    freeze(FD, iD);
                    freeze(FP, iP);
                    ssync();
                    owned([&](int e) {
                        const int kk = lk[e];
                        if (kk) {
                            const double r = lres[e] - sm * (double)kk;
                            const double rr = r > 0.0 ? r : 0.0;
                            const int nn = ln[e] - kk;
                            lres[e] = rr;
                            ln[e] = nn;
                            lk[e] = 0;
                            if (nn > 0) lsh[e] = rr / (double)nn;
                            alg += 5;
                        }
                    });
                    ssync();
                    if (segact) rounds++;
                    uT = uT && !iT;
                    uD = uD && !iD;
                    uP = uP && !iP;
                }
                nact = scount(aT) + scount(aD) + scount(aP);
            }
            PFM(4);
            // every link's count is back to 0 (all its flows froze)
            if (segdirty) {
                nwf++;
                nrounds += rounds;
                if (nact > maxact) maxact = nact;
            }
            auto drain = [&](Flow &F, bool on) {
                if (on) {
                    F.t_drain = (F.rem == 0.0) ? t : t + F.rem / F.rate;
                    alg += 2;
                    if (F.t_drain == t) again = true;
                }
            };
            drain(FT, aT);
            drain(FD, aD);
            drain(FP, aP);
            PFM(5);
            if (!vany(again)) break;
        }

        // ------------------------------ end of instant ------------------------------
        // the instant's end: did anything happen (R19 n_instants), is a flow in flight (R18 comm_busy),
        // is every lane done, and the next event time -- one exchange in a CTA, segment votes in a warp
        const bool myinfl = used && (FT.st != FS_NONE || FD.st != FS_NONE || FP.st != FS_NONE);
        const bool lane_done = !used || (cst == CS_IDLE && pos >= nprog && FT.st == FS_NONE && FD.st == FS_NONE &&
                                         FP.st == FS_NONE && sq >= nsend_tot && GT.cur >= GT.ncoll * (GT.member ? 1u : 0u) &&
                                         GD.cur >= GD.ncoll * (GD.member ? 1u : 0u) && !GT.running && !GD.running);
        double cand = dinf();
        if (used) {
            if (cst == CS_RUN) cand = t_end;
            auto cf = [&](const Flow &F) {
                if (F.st == FS_LAT && F.t_act < cand) cand = F.t_act;
                if (F.st == FS_ACT && F.t_drain < cand) cand = F.t_drain;
            };
            cf(FT);
            cf(FD);
            cf(FP);
            if (TR.phot)
                for (int k = 0; k < ports; k++)
                    if (p_st[k * NTHR + threadIdx.x] == 1 && p_t[k * NTHR + threadIdx.x] < cand) cand = p_t[k * NTHR + threadIdx.x];
        }
        bool any_ev, infl, alldone;
        double tn;
        if constexpr (NW == 1) {
            any_ev = sany(nev);
            infl = sany(myinfl);
            alldone = !sany(!lane_done);
            tn = smin(cand);
        } else {
            const double wmin = seg_min<32>(cand);
            const unsigned f = (__any_sync(FULL, nev) ? 1u : 0u) | (__any_sync(FULL, myinfl) ? 2u : 0u) |
                               (__any_sync(FULL, !lane_done) ? 4u : 0u);
            if (lane == 0) {
                s_red[bb][wid] = wmin;
                s_fl3[bb][wid] = f;
            }
            __syncthreads();
            const double r = seg_min<32>(lane < NW ? s_red[bb][lane] : dinf());
            unsigned fa = lane < NW ? s_fl3[bb][lane] : 0u;
#pragma unroll
            for (int o = 16; o > 0; o >>= 1) fa |= __shfl_xor_sync(FULL, fa, o);
            bb ^= 1;
            any_ev = (fa & 1u) != 0;
            infl = (fa & 2u) != 0;
            alldone = (fa & 4u) == 0;
            tn = r;
        }
        if (have && any_ev) ninst++;
        nev = false;
        if (have) {
            if (infl && !bon) { bon = true; bstart = t; }
            else if (!infl && bon) { bon = false; cbusy = cbusy + (t - bstart); }
        }
        PFM(6);
#ifdef TS_PROF_H
        const bool fin = have && (alldone || ninst >= (uint32_t)TS_PROF_H);
        if (fin && threadIdx.x == 0)
            printf("PFH pidx=%u W=%d NW=%d inst=%u wf=%u rounds=%u inner=%u outer=%u cyc refill+end=%lld inner=%lld phot=%lld wfsetup=%lld rounds=%lld drain=%lld endinst=%lld\n",
                   pidx, W, NW, ninst, nwf, nrounds, pf_inner, pf_outer, pf_c[0], pf_c[1], pf_c[2], pf_c[3], pf_c[4], pf_c[5], pf_c[6]);
        if (fin) { for (int k = 0; k < 7; k++) pf_c[k] = 0; pf_inner = pf_outer = 0; }
#else
        const bool fin = have && alldone;
#endif
        const bool stuck = have && !fin && !(tn < dinf());
        if ((NW > 1) ? (fin || stuck) : vany(fin || stuck)) {   // (a CTA segment: uniform, no vote needed)
            const double bmax = smax(used ? busy : 0.0);
            const unsigned long long ntk = ssum(ntask);
            const unsigned long long nfl = ssum(nflow);
            const unsigned long long npp = ssum(np2p);
            const unsigned long long alg_s = ssum(alg);
            const unsigned long long H = ssum(acc);
            if ((fin || stuck) && li == 0) {
                triosim_result rr;
                rr.iter_time_s = fin ? t : 0.0;
                rr.compute_busy_max_s = fin ? bmax : 0.0;
                rr.comm_busy_s = fin ? cbusy : 0.0;
                rr.exposed_comm_s = fin ? t - bmax : 0.0;
                rr.coll_payload_bytes = fin ? C->coll_payload : 0.0;
                rr.n_compute = fin ? ntk : 0;
                rr.n_flows = fin ? nfl : 0;
                rr.n_collectives = fin ? C->n_coll : 0;
                rr.n_p2p = fin ? npp : 0;
                rr.n_instants = fin ? ninst : 0;
                rr.n_wf_calls = fin ? nwf : 0;
                rr.n_wf_rounds = fin ? nrounds : 0;
                rr.order_hash = fin ? H : 0;
                rr.status = fin ? TRIOSIM_PT_OK : TRIOSIM_PT_DEADLOCK;
                rr.max_active_flows = fin ? maxact : 0;
                a.out[pidx] = rr;
                if (a.alg_ops) atomicAdd(a.alg_ops, alg_s);
            }
            if (fin || stuck) {
                have = used = false;
                GT.member = GD.member = false;
            }
        }
        if (have) {
            t = tn;
            tmix = mix64((uint64_t)__double_as_longlong(t));
        }
    }
#undef EV
#undef PFM
}

size_t k3h_dyn_smem(int W, uint32_t lmax, uint32_t pmax) {
    const size_t nthr = W <= 32 ? K3_THREADS : (size_t)W;
    const size_t ph = pmax ? nthr * pmax * 16 + nthr * 3 * (8 + 8 + 4 + 1 + 1) : 0;
    if (W <= 32) return ph;
    const size_t links = (size_t)lmax * 28 + 8;   // lres, lsh (f64); ln, lk, lown (i32)
    return links > ph ? links : ph;   // a one-point CTA runs either a flow-network or a photonic point
}

template <int W, int NW, int V>
static cudaError_t launch_hb(const K3Args &a, int grid, cudaStream_t s) {
    const size_t dyn = k3h_dyn_smem(NW == 1 ? W : 32 * NW, a.lmax, a.pmax);
    if (dyn > 0) {
        const cudaError_t e = cudaFuncSetAttribute(k3_hybrid<W, NW, V>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)dyn);
        if (e != cudaSuccess) return e;
    }
    k3_hybrid<W, NW, V><<<grid, NW == 1 ? K3_THREADS : 32 * NW, dyn, s>>>(a);
    return cudaGetLastError();
}
template <int W, int NW>
static cudaError_t launch_h(const K3Args &a, int grid, cudaStream_t s) {
    return a.tl_cnt ? launch_hb<W, NW, V_LOG>(a, grid, s)
         : a.bd ? launch_hb<W, NW, V_BD>(a, grid, s) : launch_hb<W, NW, 0>(a, grid, s);
}

// W <= 32: W-lane segments in 256-thread CTAs; W = 64..1024: one point per CTA of W threads
cudaError_t launch_k3_hybrid(int W, const K3Args &a, int grid, cudaStream_t s) {
    switch (W) {
    case 2: return launch_h<2, 1>(a, grid, s);
    case 4: return launch_h<4, 1>(a, grid, s);
    case 8: return launch_h<8, 1>(a, grid, s);
    case 16: return launch_h<16, 1>(a, grid, s);
    case 32: return launch_h<32, 1>(a, grid, s);
    case 64: return launch_h<32, 2>(a, grid, s);
    case 128: return launch_h<32, 4>(a, grid, s);
    case 256: return launch_h<32, 8>(a, grid, s);
    case 512: return launch_h<32, 16>(a, grid, s);
    case 1024: return launch_h<32, 32>(a, grid, s);
    default: return cudaErrorInvalidValue;
    }
}

template <int W, int NW>
static int occ_h(uint32_t lmax, uint32_t pmax) {
    const size_t dyn = k3h_dyn_smem(NW == 1 ? W : 32 * NW, lmax, pmax);
    if (dyn > 0 && cudaFuncSetAttribute(k3_hybrid<W, NW, 0>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)dyn) != cudaSuccess)
        return 0;
    int nb = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, k3_hybrid<W, NW, 0>, NW == 1 ? K3_THREADS : 32 * NW, dyn);
    return nb;
}

int k3h_max_blocks_per_sm(int W, uint32_t lmax, uint32_t pmax) {
    int nb;
    switch (W) {
    case 2: nb = occ_h<2, 1>(lmax, pmax); break;
    case 4: nb = occ_h<4, 1>(lmax, pmax); break;
    case 8: nb = occ_h<8, 1>(lmax, pmax); break;
    case 16: nb = occ_h<16, 1>(lmax, pmax); break;
    case 32: nb = occ_h<32, 1>(lmax, pmax); break;
    case 64: nb = occ_h<32, 2>(lmax, pmax); break;
    case 128: nb = occ_h<32, 4>(lmax, pmax); break;
    case 256: nb = occ_h<32, 8>(lmax, pmax); break;
    case 512: nb = occ_h<32, 16>(lmax, pmax); break;
    default: nb = occ_h<32, 32>(lmax, pmax); break;
    }
    return nb > 0 ? nb : 1;
}

}  // namespace ts
