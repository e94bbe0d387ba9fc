// ts_kernels.cu -- sm_100a kernels of libtriosim.
//
//  K1a  k1_ingest      trace ingest: SoA staging, producer table, WGRAD production order,
//                      first-OPT / last-non-OPT indices
//  K1b  k1_rescale     operator-time model t' = t * rho per (class, op)
//  K2   k2_coll        DP / DDP buckets and TP collectives -> per-op hooks
//       k2_pipe        GPipe stage programs, P2P send / receive lists
//  K3   k3_timeline    event-driven timeline + max-min progressive filling, one design point
//                      per W-lane warp segment (W = 2..32 simulated GPUs)
//
// Numerics: compiled with --fmad=false (no FMA contraction), IEEE division; every sum is a
// left fold in the order DESIGN.md states, so results match the oracle bit for bit.
#include <cuda_runtime.h>
#include <climits>
#include <cstdint>
#include "ts_internal.h"

namespace ts {

#define FULL 0xffffffffu

__device__ __forceinline__ uint64_t mix64(uint64_t z) {
    z = (z ^ (z >> 30)) * 0xbf58476d1ce4e5b9ull;
    z = (z ^ (z >> 27)) * 0x94d049bb133111ebull;
    return z ^ (z >> 31);
}
__device__ __forceinline__ uint64_t fnv_u64(uint64_t h, uint64_t v) {
#pragma unroll
    for (int b = 0; b < 8; b++) {
        h ^= (v >> (8 * b)) & 0xffull;
        h *= 0x100000001b3ull;
    }
    return h;
}

// ------------------------------------------------------------------------------------
// K1a: trace ingest (one CTA; once per trace)
// ------------------------------------------------------------------------------------
__global__ void __launch_bounds__(1024) k1_ingest(TraceDev T) {
    __shared__ int s_scan[1024];
    __shared__ int s_base;
    const int tid = threadIdx.x, nt = blockDim.x;
    for (uint32_t o = tid; o < T.n_ops; o += nt) {
        const triosim_op op = T.ops[o];
        T.time[o] = op.time_s;
        T.info[o] = (uint32_t)op.phase | ((uint32_t)(op.tp_role & 7) << INFO_ROLE_SHIFT) |
                    ((op.flags & TRIOSIM_OPF_BATCH_SCALED) ? INFO_SCALED : 0u);
        T.layer[o] = op.layer;
        for (uint32_t k = 0; k < op.n_out; k++) T.prod[T.io[op.io_off + op.n_in + k]] = (int32_t)o;
        if (op.phase == PH_OPT) atomicMin(&T.scal[1], (int)o);
        else atomicMax(&T.scal[2], (int)o);
    }
    if (tid == 0) s_base = 0;
    __syncthreads();
    // weight gradients in production order: producer op ascending, then tensor id
    for (uint32_t start = 0; start < T.n_ops; start += nt) {
        uint32_t o = start + tid;
        int c = 0;
        triosim_op op;
        if (o < T.n_ops) {
            op = T.ops[o];
            if (op.phase != PH_OPT)
                for (uint32_t k = 0; k < op.n_out; k++)
                    c += T.ts[T.io[op.io_off + op.n_in + k]].category == TRIOSIM_CAT_WGRAD;
        }
        s_scan[tid] = c;
        __syncthreads();
        for (int off = 1; off < nt; off <<= 1) {  // Hillis-Steele inclusive scan
            int v = tid >= off ? s_scan[tid - off] : 0;
            __syncthreads();
            s_scan[tid] += v;
            __syncthreads();
        }
        int excl = s_scan[tid] - c + s_base;
        if (c > 0) {
            int w = excl;
            uint32_t last = 0;
            bool first = true;
            for (int r = 0; r < c; r++) {  // emit this op's WGRAD outputs in ascending tensor id
                uint32_t best = UINT_MAX;
                for (uint32_t k = 0; k < op.n_out; k++) {
                    uint32_t x = T.io[op.io_off + op.n_in + k];
                    if (T.ts[x].category == TRIOSIM_CAT_WGRAD && (first || x > last) && x < best) best = x;
                }
                T.wgrad[w++] = best;
                last = best;
                first = false;
            }
        }
        __syncthreads();
        if (tid == nt - 1) s_base += s_scan[nt - 1];
        __syncthreads();
    }
    if (tid == 0) T.scal[0] = s_base;
}

cudaError_t launch_k1_ingest(const TraceDev &T, cudaStream_t s) {
    k1_ingest<<<1, 1024, 0, s>>>(T);
    return cudaGetLastError();
}

// ------------------------------------------------------------------------------------
// K1b: operator-time model (R4): rho = 1; *r_b if batch-scaled; /tp if TP-split;
//      t' = t if rho == 1 else t * rho
// ------------------------------------------------------------------------------------
__device__ __forceinline__ bool split_of(uint32_t info, uint32_t tp_mode) {
    uint32_t role = (info >> INFO_ROLE_SHIFT) & 7u;
    return tp_mode == TRIOSIM_TP_PAPER ? (role & TRIOSIM_ROLE_GATHER) != 0 : (role & 3u) != 0;
}

__global__ void k1_rescale(const ClassDesc *cls, TraceDev T, double *dur) {
    const ClassDesc &C = cls[blockIdx.y];
    for (uint32_t o = blockIdx.x * blockDim.x + threadIdx.x; o < T.n_ops; o += gridDim.x * blockDim.x) {
        uint32_t info = T.info[o];
        double rho = 1.0;
        if (info & INFO_SCALED) rho = C.r_b;
        if (C.tpdeg > 1 && split_of(info, C.tp_mode)) rho = rho / (double)C.tpdeg;
        double t = T.time[o];
        dur[C.dur_off + o] = (rho == 1.0) ? t : t * rho;
    }
}

cudaError_t launch_k1_rescale(const ClassDesc *cls, uint32_t n_cls, const TraceDev &T, double *dur, cudaStream_t s) {
    if (n_cls == 0) return cudaSuccess;
    dim3 grid((T.n_ops + 255) / 256, n_cls);
    if (grid.x > 64) grid.x = 64;
    k1_rescale<<<grid, 256, 0, s>>>(cls, T, dur);
    return cudaGetLastError();
}

// bytes of a tensor instance (R5)
__device__ __forceinline__ double tensor_bytes(const TraceDev &T, uint32_t x, double r_b, uint32_t tp,
                                               uint32_t tp_mode) {
    const triosim_tensor tt = T.ts[x];
    double b = (double)tt.bytes_b0;
    if (tt.batch_scaled) b = b * r_b;
    if (tp > 1 && tt.category == TRIOSIM_CAT_WGRAD && T.prod[x] >= 0 && split_of(T.info[T.prod[x]], tp_mode))
        b = b / (double)tp;
    return b;
}

// ------------------------------------------------------------------------------------
// K2 (COLL): one CTA per DP/DDP/TP class
// ------------------------------------------------------------------------------------
__global__ void __launch_bounds__(256) k2_coll(ClassDesc *cls, const uint32_t *list, TraceDev T, const double *dur,
                                               OpHook *hooks, CollEnt *colls, int32_t *scratch) {
    ClassDesc &C = cls[list[blockIdx.x]];
    const int tid = threadIdx.x, nt = blockDim.x;
    OpHook *H = hooks + C.hook_off;
    CollEnt *CE = colls + C.coll_off;
    for (uint32_t o = tid; o < T.n_ops; o += nt) {
        H[o].dur = dur[C.dur_off + o];
        H[o].wait = -1;
        H[o].nsig = 0;
    }
    const bool is_dp = C.strategy == TRIOSIM_DP || C.strategy == TRIOSIM_DDP;
    int32_t *coll_of = scratch + C.scratch_off;
    if (!is_dp)
        for (uint32_t x = tid; x < T.n_ts; x += nt) coll_of[x] = -1;
    __syncthreads();
    if (is_dp) {
        if (tid == 0) {
            uint32_t nc = 0;
            double payload = 0.0;
            const int nw = T.scal[0], first_opt = T.scal[1], last_nonopt = T.scal[2];
            if (C.p > 1) {
                int i = 0;
                while (i < nw) {
                    // gradient bucket (reading Q5): greedy on the u64 byte sum
                    uint64_t sum = 0;
                    double S = 0.0;
                    int j = i;
                    for (;;) {
                        uint32_t x = T.wgrad[j];
                        sum += T.ts[x].bytes_b0;
                        S = S + tensor_bytes(T, x, C.r_b, 1, C.tp_mode);
                        j++;
                        if (C.bucket_bytes == 0 || sum >= C.bucket_bytes || j == nw) break;
                    }
                    int trig = (C.strategy == TRIOSIM_DDP) ? T.prod[T.wgrad[j - 1]] : last_nonopt;
                    CE[nc].S = S;
                    CE[nc].kind = CK_AR;
                    H[trig].nsig += 1;
                    payload = payload + S;
                    nc++;
                    i = j;
                }
                if (nc > 0 && first_opt != INT_MAX) H[first_opt].wait = (int32_t)nc - 1;
            }
            C.n_coll = nc;
            C.coll_payload = payload;
            C.need_ring = nc > 0 && C.algo == TRIOSIM_ALGO_RING;
            C.need_tree = nc > 0 && C.algo == TRIOSIM_ALGO_TREE;
            C.n_compute = (uint64_t)C.p * T.n_ops;
            uint64_t fl = C.algo == TRIOSIM_ALGO_RING ? 2ull * (C.p - 1) * C.p : 2ull * (C.p - 1);
            C.n_flows = fl * nc;
            C.n_prog_max = T.n_ops;
        }
    } else {
        if (tid == 0) {
            uint32_t nc = 0, any_ag = 0, any_ar = 0;
            double payload = 0.0;
            uint64_t nfl = 0;
            if (C.p > 1) {
                for (uint32_t o = 0; o < T.n_ops; o++) {
                    const triosim_op op = T.ops[o];
                    const uint32_t role = op.tp_role;
                    for (uint32_t k = 0; k < op.n_out; k++) {
                        uint32_t x = T.io[op.io_off + op.n_in + k];
                        int kind = -1;
                        const uint8_t cat = T.ts[x].category;
                        if (C.tp_mode == TRIOSIM_TP_PAPER) {
                            if ((role & TRIOSIM_ROLE_GATHER) && op.phase == PH_FWD) kind = CK_AG;
                            if ((role & TRIOSIM_ROLE_GATHER) && op.phase == PH_BWD && cat == TRIOSIM_CAT_AGRAD) kind = CK_AR;
                        } else {
                            if ((role & 3u) == TRIOSIM_ROLE_ROW && op.phase == PH_FWD) kind = CK_AR;
                            if ((role & 3u) == TRIOSIM_ROLE_COL && op.phase == PH_BWD && cat == TRIOSIM_CAT_AGRAD) kind = CK_AR;
                        }
                        if (kind < 0) continue;
                        double S = (double)T.ts[x].bytes_b0;
                        if (T.ts[x].batch_scaled) S = S * C.r_b;
                        CE[nc].S = S;
                        CE[nc].kind = (uint32_t)kind;
                        H[o].nsig += 1;
                        coll_of[x] = (int32_t)nc;
                        payload = payload + S;
                        if (kind == CK_AG) any_ag = 1; else any_ar = 1;
                        if (kind == CK_AR && C.algo == TRIOSIM_ALGO_TREE) nfl += 2ull * (C.p - 1);
                        else nfl += (kind == CK_AR ? 2ull : 1ull) * (C.p - 1) * C.p;
                        nc++;
                    }
                }
            }
            C.n_coll = nc;
            C.coll_payload = payload;
            C.need_ring = any_ag || (any_ar && C.algo == TRIOSIM_ALGO_RING);
            C.need_tree = any_ar && C.algo == TRIOSIM_ALGO_TREE;
            C.n_compute = (uint64_t)C.p * T.n_ops;
            C.n_flows = nfl;
            C.n_prog_max = T.n_ops;
        }
        __syncthreads();
        // an operator reading a communicated tensor waits for that collective on its GPU; FIFO
        // completion order lets the largest index stand for all
        for (uint32_t o = tid; o < T.n_ops; o += nt) {
            const triosim_op op = T.ops[o];
            int32_t w = -1;
            for (uint32_t k = 0; k < op.n_in; k++) {
                int32_t c = coll_of[T.io[op.io_off + k]];
                if (c > w) w = c;
            }
            H[o].wait = w;
        }
    }
}

cudaError_t launch_k2_coll(ClassDesc *cls, const uint32_t *list, uint32_t n, const TraceDev &T, const double *dur,
                           OpHook *hooks, CollEnt *colls, int32_t *scratch, cudaStream_t s) {
    if (n == 0) return cudaSuccess;
    k2_coll<<<n, 256, 0, s>>>(cls, list, T, dur, hooks, colls, scratch);
    return cudaGetLastError();
}

// ------------------------------------------------------------------------------------
// K2 (PIPE): one CTA per GPipe class; thread s builds stage s
// ------------------------------------------------------------------------------------
constexpr int K2P_THREADS = 64;
constexpr int K2P_MAX_LAYERS = 2048;

__global__ void __launch_bounds__(K2P_THREADS) k2_pipe(ClassDesc *cls, const uint32_t *list, TraceDev T,
                                                       const double *dur, const uint32_t *plan_pool,
                                                       StageInfo *stages, StageEnt *ents, SendEnt *sends,
                                                       RecvEnt *recvs, unsigned long long *scratch) {
    ClassDesc &C = cls[list[blockIdx.x]];
    __shared__ uint16_t s_stage[K2P_MAX_LAYERS];
    __shared__ uint32_t s_cnt[64][4];
    const int tid = threadIdx.x, nt = blockDim.x;
    const int S = (int)C.p;
    const uint32_t *fl = plan_pool + C.plan_off;
    for (uint32_t l = tid; l < T.n_layers; l += nt) {
        int s = 0;
        while (s + 1 < S && fl[s + 1] <= l) s++;
        s_stage[l] = (uint16_t)s;
    }
    unsigned long long *readers = scratch + C.scratch_off;
    for (uint32_t x = tid; x < T.n_ts; x += nt) readers[x] = 0ull;
    __syncthreads();
    for (uint32_t o = tid; o < T.n_ops; o += nt) {
        const triosim_op op = T.ops[o];
        unsigned long long bit = 1ull << s_stage[op.layer];
        for (uint32_t k = 0; k < op.n_in; k++) atomicOr(&readers[T.io[op.io_off + k]], bit);
    }
    __syncthreads();
    // pass 1: sizes per stage
    StageInfo *SI = stages + C.stage_off;
    if (tid < S) {
        const int s = tid;
        uint32_t n[3] = {0, 0, 0}, sn[3] = {0, 0, 0}, nrecv = 0;
        unsigned long long dmask = 0;
        for (uint32_t o = 0; o < T.n_ops; o++) {
            const triosim_op op = T.ops[o];
            if (s_stage[op.layer] != s) continue;
            n[op.phase]++;
            for (uint32_t k = 0; k < op.n_out; k++) {
                unsigned long long r = readers[T.io[op.io_off + op.n_in + k]] & ~(1ull << s);
                sn[op.phase] += __popcll(r);
                dmask |= r;
            }
            for (uint32_t k = 0; k < op.n_in; k++) {
                int32_t po = T.prod[T.io[op.io_off + k]];
                if (po >= 0 && s_stage[T.layer[po]] != s) nrecv++;
            }
        }
        SI[s].nF = n[0]; SI[s].nB = n[1]; SI[s].nO = n[2];
        SI[s].SF = sn[0]; SI[s].SB = sn[1]; SI[s].SO = sn[2];
        SI[s].dst_mask = dmask;
        s_cnt[s][0] = n[0] + n[1] + n[2];
        s_cnt[s][1] = sn[0] + sn[1] + sn[2];
        s_cnt[s][2] = nrecv;
    }
    __syncthreads();
    if (tid == 0) {
        uint32_t e = 0, sd = 0, rv = 0;
        uint64_t ncomp = 0, nflow = 0;
        uint32_t pmax = 0;
        for (int s = 0; s < S; s++) {
            SI[s].ent_off = C.ent_off + e;
            SI[s].send_off = C.send_off + sd;
            SI[s].recv_off = C.recv_off + rv;
            e += s_cnt[s][0]; sd += s_cnt[s][1]; rv += s_cnt[s][2];
            uint32_t prog = C.m * (SI[s].nF + SI[s].nB) + SI[s].nO;
            ncomp += prog;
            if (prog > pmax) pmax = prog;
            nflow += (uint64_t)C.m * (SI[s].SF + SI[s].SB) + SI[s].SO;
        }
        C.n_compute = ncomp;
        C.n_flows = nflow;
        C.n_prog_max = pmax;
        C.n_coll = 0;
        C.coll_payload = 0.0;
        C.need_ring = C.need_tree = 0;
    }
    __syncthreads();
    // pass 2: stage op lists and send lists, in program order (producer op, io order, dst ascending)
    if (tid < S) {
        const int s = tid;
        StageInfo si = SI[s];
        uint32_t eoff[3] = {si.ent_off, si.ent_off + si.nF, si.ent_off + si.nF + si.nB};
        uint32_t soff[3] = {si.send_off, si.send_off + si.SF, si.send_off + si.SF + si.SB};
        uint32_t ei[3] = {0, 0, 0}, sj[3] = {0, 0, 0};
        for (uint32_t o = 0; o < T.n_ops; o++) {
            const triosim_op op = T.ops[o];
            if (s_stage[op.layer] != s) continue;
            const int P = op.phase;
            uint32_t nsend = 0;
            for (uint32_t k = 0; k < op.n_out; k++) {
                uint32_t x = T.io[op.io_off + op.n_in + k];
                unsigned long long r = readers[x] & ~(1ull << s);
                while (r) {
                    int d = __ffsll((long long)r) - 1;
                    r &= r - 1;
                    SendEnt se;
                    se.bytes = tensor_bytes(T, x, C.r_b, 1, C.tp_mode);
                    se.x = x;
                    se.dst = (uint16_t)d;
                    se.pidx = (uint16_t)ei[P];
                    sends[soff[P] + sj[P]++] = se;
                    nsend++;
                }
            }
            StageEnt en;
            en.op = o;
            en.nsend = (uint16_t)nsend;
            en.nrecv = 0;
            en.recv_off = 0;
            en.pad = 0;
            ents[eoff[P] + ei[P]++] = en;
        }
    }
    __syncthreads();
    // pass 3: receive lists (which send of which stage delivers each remote input)
    if (tid < S) {
        const int s = tid;
        StageInfo si = SI[s];
        uint32_t rv = si.recv_off;
        uint32_t total = si.nF + si.nB + si.nO;
        for (uint32_t q = 0; q < total; q++) {
            StageEnt &en = ents[si.ent_off + q];
            const triosim_op op = T.ops[en.op];
            en.recv_off = rv;
            uint32_t nr = 0;
            for (uint32_t k = 0; k < op.n_in; k++) {
                uint32_t x = T.io[op.io_off + k];
                int32_t po = T.prod[x];
                if (po < 0) continue;
                int ps = s_stage[T.layer[po]];
                if (ps == s) continue;
                int pph = (int)(T.info[po] & INFO_PHASE_MASK);
                StageInfo pi = SI[ps];
                uint32_t base = pi.send_off + (pph == 0 ? 0 : pph == 1 ? pi.SF : pi.SF + pi.SB);
                uint32_t cnt = pph == 0 ? pi.SF : pph == 1 ? pi.SB : pi.SO;
                uint32_t e = 0;
                while (e < cnt && !(sends[base + e].x == x && sends[base + e].dst == s)) e++;
                RecvEnt re;
                re.src = (uint16_t)ps;
                re.phase = (uint8_t)pph;
                re.pad = 0;
                re.e = e;
                recvs[rv++] = re;
                nr++;
            }
            en.nrecv = (uint16_t)nr;
        }
    }
}

cudaError_t launch_k2_pipe(ClassDesc *cls, const uint32_t *list, uint32_t n, const TraceDev &T, const double *dur,
                           const uint32_t *plan_pool, StageInfo *stages, StageEnt *ents, SendEnt *sends,
                           RecvEnt *recvs, unsigned long long *scratch, cudaStream_t s) {
    if (n == 0) return cudaSuccess;
    k2_pipe<<<n, K2P_THREADS, 0, s>>>(cls, list, T, dur, plan_pool, stages, ents, sends, recvs, scratch);
    return cudaGetLastError();
}

// ------------------------------------------------------------------------------------
// K3: the timeline.  One design point per W-lane segment of a warp; lane i of a segment
// is simulated GPU (rank / stage) i and owns that GPU's in-order compute stream and its one
// in-flight flow (ring step i->i+1, tree edge, or P2P send).  Segment-wide decisions
// (collective start, bottleneck share, next event time) are ballots / shuffles.
// ------------------------------------------------------------------------------------
enum { CS_IDLE = 0, CS_RUN = 1 };
enum { FS_NONE = 0, FS_LAT = 1, FS_ACT = 2 };
enum { EV_COLL_START = 1, EV_RELEASE = 2, EV_ACTIVATE = 3, EV_DELIVER = 4, EV_TASK_START = 5, EV_TASK_END = 6 };


template <int W>
__device__ __forceinline__ double seg_min(double v) {
#pragma unroll
    for (int o = W / 2; o > 0; o >>= 1) {
        double w = __shfl_xor_sync(FULL, v, o);
        v = w < v ? w : v;
    }
    return v;
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
__device__ __forceinline__ int seg_sum_i(int v) {
#pragma unroll
    for (int o = W / 2; o > 0; o >>= 1) v += __shfl_xor_sync(FULL, v, o);
    return v;
}

struct Route {
    uint32_t off;
    int len;
};

__device__ __forceinline__ Route get_route(const K3Args &a, const TopoDev &T, uint32_t s, uint32_t d) {
    uint32_t k = T.rt_off + s * T.n_gpus + d;
    Route r;
    r.len = a.rt_len[k];
    r.off = a.rt_off[k];
    return r;
}
__device__ __forceinline__ double route_lat(const K3Args &a, const TopoDev &T, Route r, double lat_scale) {
    double L = 0.0;
    for (int h = 0; h < r.len; h++) L = L + a.link_lat[T.link_off + a.rt_links[r.off + h]] * lat_scale;
    return L;
}

template <int W>
__global__ void __launch_bounds__(K3_THREADS) k3_timeline(const K3Args a) {
    constexpr int NSEG = 32 / W;
    constexpr int LMAX = (4 * W < 8) ? 8 : 4 * W;
    __shared__ double s_res[K3_WARPS][NSEG * LMAX];
    __shared__ int s_n[K3_WARPS][NSEG * LMAX];
    __shared__ int s_k[K3_WARPS][NSEG * LMAX];
    __shared__ uint32_t s_cnt[K3_WARPS][32];

    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    const int seg = lane / W, li = lane % W, sbase = seg * W;
    const unsigned smask = (W == 32 ? 0xffffffffu : ((1u << (W & 31)) - 1u)) << sbase;
    double *lres = &s_res[wid][seg * LMAX];
    int *ln = &s_n[wid][seg * LMAX];
    int *lk = &s_k[wid][seg * LMAX];
    uint32_t *cnt = &s_cnt[wid][sbase];
    for (int q = lane; q < NSEG * LMAX; q += 32) { s_n[wid][q] = 0; s_k[wid][q] = 0; }
    __syncwarp();

    // ---- per-segment (uniform) state ----
    bool have = false, exhausted = false;
    uint32_t pidx = 0;
    double t = 0.0, bws = 1.0, lats = 1.0;
    int p = 0, mode = 0, algo = 0;
    uint32_t ncoll = 0, m = 1;
    const ClassDesc *C = nullptr;
    TopoDev TD;
    uint64_t H = 0, ninst = 0, nwf = 0, nrounds = 0;
    uint32_t maxact = 0;
    bool bon = false;
    double bstart = 0.0, cbusy = 0.0;
    // collective (COLL)
    uint32_t cur = 0;
    bool running = false;
    int K = 0;
    uint32_t ckind = 0;
    double cS = 0.0, chunk = 0.0;
    // ---- per-lane state ----
    bool used = false;
    uint32_t gpu = 0;
    uint32_t pos = 0, run_start = 0, run_end = 0, nprog = 0;
    int cst = CS_IDLE;
    double t_end = 0.0, busy = 0.0;
    uint32_t ntask = 0, nflow = 0;
    uint32_t trig = 0, donec = 0;
    int D = 0;
    bool ldone = false, uprel = false, upd = false, dnrel = false, dnd = false, flow_is_up = false;
    Route rring = {0, 0};
    double Lring = 0.0;
    // flow slot
    int fst = FS_NONE;
    double t_act = 0.0, rem = 0.0, rate = 0.0, t_upd = 0.0, t_drain = 0.0, fbytes = 0.0;
    Route fr = {0, 0};
    uint64_t fcode = 0;
    // PIPE
    StageInfo SI;
    SI.nF = SI.nB = SI.nO = SI.SF = SI.SB = SI.SO = 0;
    SI.ent_off = SI.send_off = SI.recv_off = 0;
    uint32_t sq = 0, nsend_tot = 0, dcnt = 0;
    // event accumulation
    uint64_t acc = 0;
    int nev = 0;
    uint64_t alg = 0;   // fp64 operations of the method (R4-R17) performed by this lane

#define EV(kind, code)                                                  \
    do {                                                                \
        acc += mix64(((uint64_t)(kind) << 60) | (uint64_t)(code));      \
        nev++;                                                          \
    } while (0)

    for (;;) {
        // ------------------------------ refill ------------------------------
        bool need = !have && !exhausted;
        uint32_t it = 0;
        if (need && li == 0) it = atomicAdd(a.counter, 1u);
        it = __shfl_sync(FULL, it, sbase);
        bool fresh = false, rbad = false, rlong = false;
        if (need) {
            if (it >= a.n_work) {
                exhausted = true;
            } else {
                fresh = true;
                have = true;
                const PointDesc pd = a.pts[a.work[it]];
                pidx = pd.idx;
                bws = pd.bw_scale;
                lats = pd.lat_scale;
                C = &a.cls[pd.cls];
                TD = a.topo[pd.topo];
                p = (int)C->p;
                mode = (int)C->mode;
                algo = (int)C->algo;
                ncoll = C->n_coll;
                m = C->m;
                t = 0.0;
                H = 0xcbf29ce484222325ull;
                ninst = nwf = nrounds = 0;
                maxact = 0;
                bon = false;
                bstart = cbusy = 0.0;
                cur = 0;
                running = false;
                used = li < p;
                pos = run_start = run_end = 0;
                cst = CS_IDLE;
                t_end = busy = 0.0;
                ntask = nflow = 0;
                trig = donec = 0;
                D = 0;
                ldone = uprel = upd = dnrel = dnd = false;
                fst = FS_NONE;
                sq = dcnt = 0;
                acc = 0;
                nev = 0;
                alg = 0;
                if (used) {
                    gpu = a.ro[TD.ro_off + li];
                    if (mode == MODE_COLL) {
                        nprog = C->n_prog_max;
                        uint32_t succ = a.ro[TD.ro_off + (li + 1) % p];
                        rring = get_route(a, TD, gpu, succ);
                        if (C->need_ring && rring.len == NO_ROUTE) rbad = true;
                        if (C->need_ring && rring.len != NO_ROUTE && rring.len > MAX_HOPS) rlong = true;
                        if (rring.len != NO_ROUTE) { Lring = route_lat(a, TD, rring, lats); alg += 2 * rring.len; }
                        if (C->need_tree && li >= 1) {
                            uint32_t par = a.ro[TD.ro_off + (li - 1) / 2];
                            const int l1 = get_route(a, TD, gpu, par).len, l2 = get_route(a, TD, par, gpu).len;
                            if (l1 == NO_ROUTE || l2 == NO_ROUTE) rbad = true;
                            else if (l1 > MAX_HOPS || l2 > MAX_HOPS) rlong = true;
                        }
                    } else {
                        SI = a.stages[C->stage_off + li];
                        nprog = m * (SI.nF + SI.nB) + SI.nO;
                        nsend_tot = m * (SI.SF + SI.SB) + SI.SO;
                        unsigned long long dm = SI.dst_mask;
                        while (dm) {
                            int d = __ffsll((long long)dm) - 1;
                            dm &= dm - 1;
                            const int l = get_route(a, TD, gpu, a.ro[TD.ro_off + d]).len;
                            if (l == NO_ROUTE) rbad = true;
                            else if (l > MAX_HOPS) rlong = true;
                        }
                    }
                }
            }
        }
        if (__all_sync(FULL, !have)) break;
        {
            // a needed (src, dst) pair without a path (R3) / beyond this kernel's hop limit
            const bool bad = (__ballot_sync(FULL, fresh && rbad) & smask) != 0;
            const bool lng = (__ballot_sync(FULL, fresh && rlong) & smask) != 0;
            if (fresh && (bad || lng)) {
                if (li == 0) {
                    triosim_result r = {};
                    r.status = bad ? TRIOSIM_PT_NO_ROUTE : TRIOSIM_PT_TOO_LARGE;
                    a.out[pidx] = r;
                }
                have = false;
                used = false;
            }
        }

        // ------------------------------ one instant at time t ------------------------------
        bool dirty = false;
        for (;;) {
            for (;;) {
                bool ch = false;
                // (a) compute completions
                if (used && cst == CS_RUN && t_end == t) {
                    cst = CS_IDLE;
                    pos = run_end;
                    if (mode == MODE_COLL) {
                        uint32_t ns = a.hooks[C->hook_off + pos - 1].nsig;
                        if (ns) {
                            trig += ns;
                            EV(EV_TASK_END, ((uint64_t)gpu << 40) | (pos - 1));
                        }
                    } else {
                        // the last task of a run is the only one that may send
                        uint32_t q = pos - 1, P, idx;
                        if (q < m * SI.nF) { P = 0; idx = q % SI.nF; }
                        else if (q < m * (SI.nF + SI.nB)) { P = 1; idx = (q - m * SI.nF) % SI.nB; }
                        else { P = 2; idx = q - m * (SI.nF + SI.nB); }
                        uint32_t eo = SI.ent_off + (P == 0 ? 0 : P == 1 ? SI.nF : SI.nF + SI.nB) + idx;
                        if (a.ents[eo].nsend) EV(EV_TASK_END, ((uint64_t)gpu << 40) | q);
                    }
                    ch = true;
                }
                // (b) deliveries
                bool delivered = false;
                if (used && fst == FS_ACT && t_drain == t) {
                    fst = FS_NONE;
                    EV(EV_DELIVER, fcode);
                    delivered = true;
                    dirty = true;
                    ch = true;
                }
                // (c) activations after the route latency (reading Q19)
                if (used && fst == FS_LAT && t_act == t) {
                    EV(EV_ACTIVATE, fcode);
                    if (fbytes == 0.0 || fr.len == 0) {
                        fst = FS_NONE;
                        EV(EV_DELIVER, fcode);
                        delivered = true;
                    } else {
                        fst = FS_ACT;
                        rem = fbytes;
                        t_upd = t;
                        rate = 0.0;
                        t_drain = __longlong_as_double(0x7ff0000000000000ll);
                        dirty = true;
                    }
                    ch = true;
                }
                if (delivered) {
                    nflow++;
                    if (mode == MODE_COLL) {
                        if (algo == TRIOSIM_ALGO_TREE && ckind == CK_AR) {
                            if (flow_is_up) upd = true; else dnd = true;
                        } else {
                            D++;
                        }
                    } else {
                        dcnt++;
                    }
                }
                if (used && mode == MODE_PIPE) cnt[li] = dcnt;
                __syncwarp();

                // (d) dependency resolution
                const int pred = (li + p - 1) % (p > 0 ? p : 1);
                const int Dp = __shfl_sync(FULL, D, sbase + (pred < W ? pred : 0));
                const unsigned upm = (__ballot_sync(FULL, upd) & smask) >> sbase;
                const unsigned dnm = (__ballot_sync(FULL, dnd) & smask) >> sbase;
                if (used && mode == MODE_COLL && running) {
                    const bool tree = algo == TRIOSIM_ALGO_TREE && ckind == CK_AR;
                    if (!tree) {
                        if (fst == FS_NONE && D < K && (D == 0 || Dp >= D)) {
                            // ring step (i, k = D): m_i -> m_{i+1}, S/p bytes (reading Q21)
                            fst = FS_LAT;
                            fr = rring;
                            fbytes = chunk;
                            t_act = t + Lring;
                            alg += 1;
                            fcode = ((uint64_t)cur << 32) | ((uint64_t)D << 16) | (uint64_t)li;
                            EV(EV_RELEASE, fcode);
                            ch = true;
                        }
                        if (!ldone && D == K && Dp == K) {
                            ldone = true;
                            donec = cur + 1;
                            ch = true;
                        }
                    } else {
                        const int c1 = 2 * li + 1, c2 = 2 * li + 2;
                        const bool kids_up = (c1 >= p || ((upm >> c1) & 1u)) && (c2 >= p || ((upm >> c2) & 1u));
                        const bool kids_dn = (c1 >= p || ((dnm >> c1) & 1u)) && (c2 >= p || ((dnm >> c2) & 1u));
                        if (li >= 1 && fst == FS_NONE && !uprel && kids_up) {
                            uint32_t par = a.ro[TD.ro_off + (li - 1) / 2];
                            fr = get_route(a, TD, gpu, par);
                            fst = FS_LAT;
                            fbytes = cS;
                            t_act = t + route_lat(a, TD, fr, lats);
                            alg += 2 * fr.len + 1;
                            fcode = ((uint64_t)cur << 32) | (0ull << 16) | (uint64_t)li;
                            flow_is_up = true;
                            uprel = true;
                            EV(EV_RELEASE, fcode);
                            ch = true;
                        }
                        if (li >= 1 && fst == FS_NONE && uprel && upd && !dnrel) {
                            const int par_i = (li - 1) / 2;
                            bool pready;
                            if (par_i == 0) pready = (p <= 1 || ((upm >> 1) & 1u)) && (p <= 2 || ((upm >> 2) & 1u));
                            else pready = (dnm >> par_i) & 1u;
                            if (pready) {
                                uint32_t par = a.ro[TD.ro_off + par_i];
                                fr = get_route(a, TD, par, gpu);
                                fst = FS_LAT;
                                fbytes = cS;
                                t_act = t + route_lat(a, TD, fr, lats);
                                alg += 2 * fr.len + 1;
                                fcode = ((uint64_t)cur << 32) | (1ull << 16) | (uint64_t)li;
                                flow_is_up = false;
                                dnrel = true;
                                EV(EV_RELEASE, fcode);
                                ch = true;
                            }
                        }
                        if (!ldone && (li == 0 || (upd && dnd)) && kids_up && kids_dn) {
                            ldone = true;
                            donec = cur + 1;
                            ch = true;
                        }
                    }
                }
                {
                    const bool allfin = (__ballot_sync(FULL, !used || ldone) & smask) == smask;
                    if (have && mode == MODE_COLL && running && allfin) {
                        running = false;
                        cur++;
                        ch = true;
                    }
                    const bool allrdy = (__ballot_sync(FULL, !used || trig > cur) & smask) == smask;
                    if (have && mode == MODE_COLL && !running && cur < ncoll && allrdy) {
                        // collective start: every member ready (barrier, reading Q22)
                        const CollEnt ce = a.colls[C->coll_off + cur];
                        running = true;
                        ckind = ce.kind;
                        cS = ce.S;
                        chunk = ce.S / (double)p;
                        K = (ce.kind == CK_AR) ? 2 * (p - 1) : (p - 1);
                        D = 0;
                        ldone = uprel = upd = dnrel = dnd = false;
                        if (li == 0) { EV(EV_COLL_START, cur); alg += 1; }
                        ch = true;
                    }
                }
                if (used && mode == MODE_PIPE && fst == FS_NONE && sq < nsend_tot) {
                    // next P2P send of this stage's FIFO stream (reading Q14)
                    uint32_t P, j, e;
                    if (sq < m * SI.SF) { P = 0; j = sq / SI.SF; e = sq % SI.SF; }
                    else if (sq < m * (SI.SF + SI.SB)) { uint32_t r = sq - m * SI.SF; P = 1; j = m - 1 - r / SI.SB; e = r % SI.SB; }
                    else { P = 2; j = 0; e = sq - m * (SI.SF + SI.SB); }
                    const SendEnt se = a.sends[SI.send_off + (P == 0 ? 0 : P == 1 ? SI.SF : SI.SF + SI.SB) + e];
                    uint32_t prodpos = P == 0 ? j * SI.nF + se.pidx
                                     : P == 1 ? m * SI.nF + (m - 1 - j) * SI.nB + se.pidx
                                              : m * (SI.nF + SI.nB) + se.pidx;
                    uint32_t donepos = (cst == CS_RUN) ? run_start : pos;
                    if (donepos > prodpos) {
                        uint32_t dg = a.ro[TD.ro_off + se.dst];
                        fr = get_route(a, TD, gpu, dg);
                        fst = FS_LAT;
                        fbytes = se.bytes;
                        t_act = t + route_lat(a, TD, fr, lats);
                        alg += 2 * fr.len + 1;
                        fcode = (1ull << 59) | ((uint64_t)se.x << 32) | ((uint64_t)j << 16) | (uint64_t)dg;
                        EV(EV_RELEASE, fcode);
                        sq++;
                        ch = true;
                    }
                }
                // (e) an idle GPU starts its head operator once its inputs are present
                if (used && cst == CS_IDLE && pos < nprog) {
                    if (mode == MODE_COLL) {
                        const OpHook *HK = a.hooks + C->hook_off;
                        OpHook h = HK[pos];
                        if (h.wait < 0 || (int)donec > h.wait) {
                            if (h.wait >= 0) EV(EV_TASK_START, ((uint64_t)gpu << 40) | pos);
                            run_start = pos;
                            double te = t + h.dur;
                            busy = busy + h.dur;
                            uint32_t q = pos + 1, sig = h.nsig;
                            while (sig == 0 && q < nprog) {
                                OpHook h2 = HK[q];
                                if (h2.wait >= 0) break;
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
                            ch = true;
                        }
                    } else {
                        uint32_t q = pos, P, j, idx;
                        if (q < m * SI.nF) { P = 0; j = q / SI.nF; idx = q % SI.nF; }
                        else if (q < m * (SI.nF + SI.nB)) { uint32_t r = q - m * SI.nF; P = 1; j = m - 1 - r / SI.nB; idx = r % SI.nB; }
                        else { P = 2; j = 0; idx = q - m * (SI.nF + SI.nB); }
                        StageEnt en = a.ents[SI.ent_off + (P == 0 ? 0 : P == 1 ? SI.nF : SI.nF + SI.nB) + idx];
                        bool ok = true;
                        for (uint32_t r = 0; r < en.nrecv && ok; r++) {
                            const RecvEnt re = a.recvs[en.recv_off + r];
                            const StageInfo &ps = a.stages[C->stage_off + re.src];
                            uint32_t jp = (re.phase == 2 || P == 2) ? 0 : j;
                            uint32_t seqi = re.phase == 0 ? jp * ps.SF + re.e
                                          : re.phase == 1 ? m * ps.SF + (m - 1 - jp) * ps.SB + re.e
                                                          : m * (ps.SF + ps.SB) + re.e;
                            if (!(cnt[re.src] > seqi)) ok = false;
                        }
                        if (ok) {
                            if (en.nrecv) EV(EV_TASK_START, ((uint64_t)gpu << 40) | q);
                            run_start = pos;
                            const double *du = a.dur + C->dur_off;
                            double d0 = du[en.op];
                            double te = t + d0;
                            busy = busy + d0;
                            uint32_t ns = en.nsend;
                            q++;
                            while (ns == 0 && q < nprog) {
                                if (q < m * SI.nF) { P = 0; idx = q % SI.nF; }
                                else if (q < m * (SI.nF + SI.nB)) { P = 1; idx = (q - m * SI.nF) % SI.nB; }
                                else { P = 2; idx = q - m * (SI.nF + SI.nB); }
                                StageEnt e2 = a.ents[SI.ent_off + (P == 0 ? 0 : P == 1 ? SI.nF : SI.nF + SI.nB) + idx];
                                if (e2.nrecv) break;
                                double dd = du[e2.op];
                                te = te + dd;
                                busy = busy + dd;
                                ns = e2.nsend;
                                q++;
                            }
                            ntask += q - pos;
                            alg += 2 * (q - pos);
                            run_end = q;
                            t_end = te;
                            cst = CS_RUN;
                            ch = true;
                        }
                    }
                }
                __syncwarp();
                if (!__any_sync(FULL, ch)) break;
            }

            // (f) bandwidth re-allocation of every in-transit flow:
            //     max-min fair progressive filling (reading Q18)
            const bool segdirty = (__ballot_sync(FULL, dirty) & smask) != 0;
            dirty = false;
            const bool act = segdirty && used && fst == FS_ACT;
            uint16_t hl[MAX_HOPS];
#pragma unroll
            for (int h = 0; h < MAX_HOPS; h++) hl[h] = (act && h < fr.len) ? a.rt_links[fr.off + h] : 0;
            if (act && t_upd < t) {
                double r = rem - rate * (t - t_upd);
                rem = r > 0.0 ? r : 0.0;
                t_upd = t;
                alg += 4;
            }
            if (act) alg += fr.len;  // link residual initialisation bw * scale
            if (act) {
#pragma unroll
                for (int h = 0; h < MAX_HOPS; h++) if (h < fr.len) ln[hl[h]] = 0;
            }
            __syncwarp();
            if (act) {
#pragma unroll
                for (int h = 0; h < MAX_HOPS; h++)
                    if (h < fr.len) {
                        atomicAdd(&ln[hl[h]], 1);
                        lres[hl[h]] = a.link_bw[TD.link_off + hl[h]] * bws;
                    }
            }
            __syncwarp();
            bool unf = act;
            uint32_t rounds = 0;
            while (__any_sync(FULL, unf)) {
                const bool segact = (__ballot_sync(FULL, unf) & smask) != 0;
                double my = __longlong_as_double(0x7ff0000000000000ll);
                if (unf) {
#pragma unroll
                    for (int h = 0; h < MAX_HOPS; h++)
                        if (h < fr.len) {
                            double sh = lres[hl[h]] / (double)ln[hl[h]];
                            my = sh < my ? sh : my;
                            alg += 2;
                        }
                }
                const double s = seg_min<W>(my);
                const bool inF = unf && my == s;
                unsigned own = 0;
                if (inF) {
                    rate = s;
#pragma unroll
                    for (int h = 0; h < MAX_HOPS; h++)
                        if (h < fr.len && atomicAdd(&lk[hl[h]], 1) == 0) own |= 1u << h;
                }
                __syncwarp();
                if (inF) {
#pragma unroll
                    for (int h = 0; h < MAX_HOPS; h++)
                        if ((own >> h) & 1u) {
                            const int e = hl[h];
                            const int kk = lk[e];
                            double r = lres[e] - s * (double)kk;
                            lres[e] = r > 0.0 ? r : 0.0;
                            alg += 3;
                            ln[e] -= kk;
                            lk[e] = 0;
                        }
                }
                __syncwarp();
                if (segact) rounds++;
                unf = unf && !inF;
            }
            const int nact = __popc(__ballot_sync(FULL, act) & smask);
            if (segdirty) {
                nwf++;
                nrounds += rounds;
                if ((uint32_t)nact > maxact) maxact = (uint32_t)nact;
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
        const unsigned long long acc_s = seg_sum_u64<W>(acc);
        const int nev_s = seg_sum_i<W>(nev);
        acc = 0;
        nev = 0;
        if (have && nev_s > 0) {
            H = fnv_u64(H, (uint64_t)__double_as_longlong(t));
            H = fnv_u64(H, acc_s);
            ninst++;
        }
        const int infl = seg_sum_i<W>(used && fst != FS_NONE ? 1 : 0);
        if (have) {
            if (infl > 0 && !bon) { bon = true; bstart = t; }
            else if (infl == 0 && bon) { bon = false; cbusy = cbusy + (t - bstart); }
        }
        const bool lane_done = !used || (cst == CS_IDLE && pos >= nprog && fst == FS_NONE &&
                                         (mode == MODE_COLL || sq >= nsend_tot));
        const bool alldone = (__ballot_sync(FULL, lane_done) & smask) == smask;
        const bool fin = have && alldone && (mode == MODE_PIPE || (cur >= ncoll && !running));
        double cand = __longlong_as_double(0x7ff0000000000000ll);
        if (used) {
            if (cst == CS_RUN) cand = t_end;
            if (fst == FS_LAT && t_act < cand) cand = t_act;
            if (fst == FS_ACT && t_drain < cand) cand = t_drain;
        }
        const double tn = seg_min<W>(cand);
        const bool stuck = have && !fin && !(tn < __longlong_as_double(0x7ff0000000000000ll));
        if (__any_sync(FULL, fin || stuck)) {
            const double bmax = seg_max<W>(used ? busy : 0.0);
            const int ntk = seg_sum_i<W>((int)ntask);
            const int nfl = seg_sum_i<W>((int)nflow);
            const unsigned long long alg_s = seg_sum_u64<W>(alg);
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
                r.n_p2p = (fin && mode == MODE_PIPE) ? (uint64_t)nfl : 0;
                r.n_instants = fin ? ninst : 0;
                r.n_wf_calls = fin ? nwf : 0;
                r.n_wf_rounds = fin ? nrounds : 0;
                r.order_hash = fin ? H : 0;
                r.status = fin ? TRIOSIM_PT_OK : TRIOSIM_PT_DEADLOCK;
                r.max_active_flows = fin ? maxact : 0;
                a.out[pidx] = r;
                if (a.alg_ops) atomicAdd(a.alg_ops, alg_s);
            }
            if (fin || stuck) {
                have = false;
                used = false;
            }
        }
        if (have) t = tn;
    }
#undef EV
}

template <int W>
static cudaError_t launch_w(const K3Args &a, int grid, cudaStream_t s) {
    k3_timeline<W><<<grid, K3_THREADS, 0, s>>>(a);
    return cudaGetLastError();
}

cudaError_t launch_k3(int W, const K3Args &a, int grid, cudaStream_t s) {
    switch (W) {
    case 2: return launch_w<2>(a, grid, s);
    case 4: return launch_w<4>(a, grid, s);
    case 8: return launch_w<8>(a, grid, s);
    case 16: return launch_w<16>(a, grid, s);
    case 32: return launch_w<32>(a, grid, s);
    default: return cudaErrorInvalidValue;
    }
}

int k3_max_blocks_per_sm(int W) {
    int nb = 0;
    switch (W) {
    case 2: cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, k3_timeline<2>, K3_THREADS, 0); break;
    case 4: cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, k3_timeline<4>, K3_THREADS, 0); break;
    case 8: cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, k3_timeline<8>, K3_THREADS, 0); break;
    case 16: cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, k3_timeline<16>, K3_THREADS, 0); break;
    case 32: cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, k3_timeline<32>, K3_THREADS, 0); break;
    }
    return nb > 0 ? nb : 1;
}

}  // namespace ts
