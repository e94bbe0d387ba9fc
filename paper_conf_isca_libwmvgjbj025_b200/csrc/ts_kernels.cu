// ts_kernels.cu -- sm_100a kernels of libtriosim.
//
//  K1a  k1_ingest      trace ingest: SoA staging, producer table, WGRAD production order,
//                      first-OPT / last-non-OPT indices
//  K1b  k1_rescale     operator-time model t' = t * rho per (class, op)
//  K2   k2_coll        DP / DDP buckets and TP collectives -> per-op hooks
//       k2_pipe        GPipe stage programs, P2P send / receive lists
//  K3   k3_timeline    (ts_k3.cu) event-driven timeline + max-min progressive filling, one point
//                      per W-lane warp segment (W = 2..32 simulated GPUs)
//  K4   k4_layer_compute, k4_breakdown   per-layer compute / comm breakdown (R22; Fig. 13)
//
// Numerics: compiled with --fmad=false (no FMA contraction), IEEE division; every sum is a
// left fold in the order DESIGN.md states, so results match the oracle bit for bit.
#include <cuda_runtime.h>
#include <climits>
#include <cstdint>
#include "ts_internal.h"

namespace ts {

#define FULL 0xffffffffu

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

// R24: cap of gradient bucket number k of a group (PyTorch DDP's first-bucket rule); 0 = one tensor per
// AllReduce (Q5)
__device__ __forceinline__ uint64_t bucket_cap(const ClassDesc &C, uint32_t k) {
    if (C.bucket_bytes == 0) return 0;
    return (k == 0 && C.first_bucket != 0) ? (uint64_t)C.first_bucket : C.bucket_bytes;
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
    if (C.strategy == TRIOSIM_HOP) {
        // R28: the update every worker sends each neighbour per iteration -- the left fold of its weight
        // gradients' bytes' in production order -- and the iteration's boundaries
        if (tid == 0) {
            double S = 0.0;
            for (int i = 0; i < T.scal[0]; i++) S = S + tensor_bytes(T, T.wgrad[i], C.r_b, 1, C.tp_mode);
            const uint32_t n = C.p, h = C.tp_mode == TRIOSIM_HOP_DOUBLE_RING ? n / 2 : n;
            const uint32_t deg = (h > 2 ? 3u : h == 2 ? 1u : 0u) + (C.tp_mode == TRIOSIM_HOP_DOUBLE_RING ? 1u : 0u);
            C.hop_S = S;
            C.hop_last = (uint32_t)T.scal[2];
            C.hop_first = (uint32_t)T.scal[1];
            C.n_coll = 0;
            C.coll_payload = 0.0;
            C.need_ring = C.need_tree = 0;
            C.n_prog_max = T.n_ops;
            C.n_compute = (uint64_t)n * C.m * T.n_ops;
            C.n_flows = (uint64_t)n * C.m * deg;
        }
        return;
    }
    const bool is_dp = C.strategy == TRIOSIM_DP || C.strategy == TRIOSIM_DDP;
    int32_t *coll_of = scratch + C.scratch_off;
    if (!is_dp)
        for (uint32_t x = tid; x < T.n_ts; x += nt) coll_of[x] = -1;
    __syncthreads();
    if (is_dp) {
        if (tid == 0) {
            uint32_t nc = 0, nb = 0;   // collectives, gradient buckets
            double payload = 0.0;
            const int nw = T.scal[0], first_opt = T.scal[1], last_nonopt = T.scal[2];
            if (C.p > 1) {
                int i = 0;
                while (i < nw) {
                    // gradient bucket (reading Q5): greedy on the u64 byte sum, first cap per R24
                    const uint64_t cap = bucket_cap(C, nb);
                    uint64_t sum = 0;
                    double S = 0.0;
                    int j = i;
                    for (;;) {
                        uint32_t x = T.wgrad[j];
                        sum += T.ts[x].bytes_b0;
                        S = S + tensor_bytes(T, x, C.r_b, 1, C.tp_mode);
                        j++;
                        if (cap == 0 || sum >= cap || j == nw) break;
                    }
                    int trig = (C.strategy == TRIOSIM_DDP) ? T.prod[T.wgrad[j - 1]] : last_nonopt;
                    // R29: an AllReduce, or its ReduceScatter + AllGather pair (two collectives)
                    const int parts = C.algo == TRIOSIM_ALGO_RSAG ? 2 : 1;
                    for (int h = 0; h < parts; h++) {
                        CE[nc].S = S;
                        CE[nc].kind = parts == 1 ? CK_AR : h == 0 ? CK_RS : CK_AG;
                        CE[nc].layer = T.layer[trig];
                        H[trig].nsig += 1;
                        payload = payload + S;
                        nc++;
                    }
                    nb++;
                    i = j;
                }
                if (nc > 0 && first_opt != INT_MAX) H[first_opt].wait = (int32_t)nc - 1;
            }
            C.n_coll = nc;
            C.coll_payload = payload;
            C.need_ring = nc > 0 && C.algo != TRIOSIM_ALGO_TREE;
            C.need_tree = nc > 0 && C.algo == TRIOSIM_ALGO_TREE;
            C.n_compute = (uint64_t)C.p * T.n_ops;
            uint64_t fl = (C.algo == TRIOSIM_ALGO_RING || C.algo == TRIOSIM_ALGO_RSAG) ? 2ull * (C.p - 1) * C.p * C.nch
                        : C.algo == TRIOSIM_ALGO_REDBCAST ? 2ull * (C.p - 1) * C.nch : 2ull * (C.p - 1);
            C.n_flows = fl * nb;
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
                        const bool split = kind == CK_AR && C.algo == TRIOSIM_ALGO_RSAG;
                        if (split) {   // R29: ReduceScatter, then AllGather
                            CE[nc].S = S;
                            CE[nc].kind = CK_RS;
                            CE[nc].layer = T.layer[o];
                            H[o].nsig += 1;
                            payload = payload + S;
                            nc++;
                            kind = CK_AG;
                        }
                        CE[nc].S = S;
                        CE[nc].kind = (uint32_t)kind;
                        CE[nc].layer = T.layer[o];
                        H[o].nsig += 1;
                        coll_of[x] = (int32_t)nc;
                        payload = payload + S;
                        if (kind == CK_AG) any_ag = 1; else any_ar = 1;
                        if (kind == CK_AR && C.algo == TRIOSIM_ALGO_TREE) nfl += 2ull * (C.p - 1);
                        else if (kind == CK_AR && C.algo == TRIOSIM_ALGO_REDBCAST) nfl += 2ull * (C.p - 1) * C.nch;
                        else nfl += (kind == CK_AR || split ? 2ull : 1ull) * (C.p - 1) * C.p * C.nch;
                        nc++;
                    }
                }
            }
            C.n_coll = nc;
            C.coll_payload = payload;
            C.need_ring = any_ag || (any_ar && C.algo != TRIOSIM_ALGO_TREE);
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
            en.dur = dur[C.dur_off + o];
            en.op = o;
            en.nsend = (uint16_t)nsend;
            en.nrecv = 0;
            en.recv_off = 0;
            en.run = 1;
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
        // pass 4: fold run lengths per phase list, back to front
        const uint32_t base[3] = {si.ent_off, si.ent_off + si.nF, si.ent_off + si.nF + si.nB};
        const uint32_t len[3] = {si.nF, si.nB, si.nO};
        for (int P = 0; P < 3; P++)
            for (int e = (int)len[P] - 2; e >= 0; e--) {
                StageEnt &x = ents[base[P] + e];
                const StageEnt &y = ents[base[P] + e + 1];
                x.run = (x.nsend == 0 && y.nrecv == 0) ? y.run + 1 : 1;
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
// K2 (HYBRID): one CTA per DP x TP x PP class; thread s builds stage s (R9)
// ------------------------------------------------------------------------------------
__device__ __forceinline__ int tp_kind_dev(uint32_t role, uint32_t phase, uint8_t cat, uint32_t tp_mode) {
    if (tp_mode == TRIOSIM_TP_PAPER) {
        if ((role & TRIOSIM_ROLE_GATHER) && phase == PH_FWD) return CK_AG;
        if ((role & TRIOSIM_ROLE_GATHER) && phase == PH_BWD && cat == TRIOSIM_CAT_AGRAD) return CK_AR;
    } else {
        if ((role & 3u) == TRIOSIM_ROLE_ROW && phase == PH_FWD) return CK_AR;
        if ((role & 3u) == TRIOSIM_ROLE_COL && phase == PH_BWD && cat == TRIOSIM_CAT_AGRAD) return CK_AR;
    }
    return -1;
}

__global__ void __launch_bounds__(K2P_THREADS) k2_hybrid(ClassDesc *cls, const uint32_t *list, TraceDev T,
                                                         const uint32_t *plan_pool, StageInfo *stages, HStage *hst,
                                                         HEnt *ents, HSend *sends, RecvEnt *recvs, CollEnt *colls,
                                                         unsigned long long *scratch, const double *dur) {
    ClassDesc &C = cls[list[blockIdx.x]];
    __shared__ uint16_t s_stage[K2P_MAX_LAYERS];
    __shared__ uint32_t s_cnt[64][6];
    const int tid = threadIdx.x, nt = blockDim.x;
    const int S = (int)C.p, tp = (int)C.tpdeg, dp = (int)C.dp;
    const uint32_t m = C.m;
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
        const unsigned long long bit = 1ull << s_stage[op.layer];
        for (uint32_t k = 0; k < op.n_in; k++) atomicOr(&readers[T.io[op.io_off + k]], bit);
    }
    __syncthreads();
    StageInfo *SI = stages + C.stage_off;
    HStage *HS = hst + C.hst_off;
    // pass 1: sizes of every per-stage list
    if (tid < S) {
        const int s = tid;
        uint32_t n[3] = {0, 0, 0}, sn[3] = {0, 0, 0}, tn[3] = {0, 0, 0}, nrecv = 0;
        unsigned long long dmask = 0;
        for (uint32_t o = 0; o < T.n_ops; o++) {
            const triosim_op op = T.ops[o];
            if (s_stage[op.layer] != s) continue;
            n[op.phase]++;
            for (uint32_t k = 0; k < op.n_out; k++) {
                const uint32_t x = T.io[op.io_off + op.n_in + k];
                const unsigned long long r = readers[x] & ~(1ull << s);
                sn[op.phase] += __popcll(r);
                dmask |= r;
                if (tp > 1) {
                    const int kd = tp_kind_dev(op.tp_role, op.phase, T.ts[x].category, C.tp_mode);
                    if (kd >= 0) tn[op.phase] += (kd == CK_AR && C.algo == TRIOSIM_ALGO_RSAG) ? 2 : 1;   // R29 pairs
                }
            }
            for (uint32_t k = 0; k < op.n_in; k++) {
                const int32_t po = T.prod[T.io[op.io_off + k]];
                if (po >= 0 && s_stage[T.layer[po]] != s) nrecv++;
            }
        }
        uint32_t nb = 0;
        if (dp > 1) {
            const int nw = T.scal[0];
            uint64_t sum = 0;
            bool open = false;
            for (int i = 0; i < nw; i++) {
                const uint32_t x = T.wgrad[i];
                if (s_stage[T.layer[T.prod[x]]] != s) continue;
                sum += T.ts[x].bytes_b0;
                open = true;
                const uint64_t cap = bucket_cap(C, nb);
                if (cap == 0 || sum >= cap) { nb++; sum = 0; open = false; }
            }
            if (open) nb++;
        }
        SI[s].nF = n[0]; SI[s].nB = n[1]; SI[s].nO = n[2];
        SI[s].SF = sn[0]; SI[s].SB = sn[1]; SI[s].SO = sn[2];
        SI[s].dst_mask = dmask;
        if (C.algo == TRIOSIM_ALGO_RSAG) nb *= 2;   // R29: each bucket's ReduceScatter + AllGather
        HS[s].TF = tn[0]; HS[s].TB = tn[1]; HS[s].TO = tn[2];
        HS[s].ndp = nb;
        HS[s].first_opt = n[2] > 0 ? 0u : 0xffffffffu;
        s_cnt[s][0] = n[0] + n[1] + n[2];
        s_cnt[s][1] = sn[0] + sn[1] + sn[2];
        s_cnt[s][2] = nrecv;
        s_cnt[s][3] = tn[0] + tn[1] + tn[2];
        s_cnt[s][4] = nb;
    }
    __syncthreads();
    if (tid == 0) {
        uint32_t e = 0, sd = 0, rv = 0, tc = 0, dc = 0;
        for (int s = 0; s < S; s++) {
            SI[s].ent_off = C.ent_off + e;
            SI[s].send_off = C.send_off + sd;
            SI[s].recv_off = C.recv_off + rv;
            HS[s].tcol_off = C.tcol_off + tc;
            HS[s].dcol_off = C.dcol_off + dc;
            e += s_cnt[s][0]; sd += s_cnt[s][1]; rv += s_cnt[s][2]; tc += s_cnt[s][3]; dc += s_cnt[s][4];
        }
    }
    __syncthreads();
    // pass 2: op entries, sends, TP lists (program order), DP buckets (production order)
    if (tid < S) {
        const int s = tid;
        const StageInfo si = SI[s];
        const HStage hs = HS[s];
        const uint32_t eoff[3] = {si.ent_off, si.ent_off + si.nF, si.ent_off + si.nF + si.nB};
        const uint32_t soff[3] = {si.send_off, si.send_off + si.SF, si.send_off + si.SF + si.SB};
        const uint32_t toff[3] = {hs.tcol_off, hs.tcol_off + hs.TF, hs.tcol_off + hs.TF + hs.TB};
        uint32_t ei[3] = {0, 0, 0}, sj[3] = {0, 0, 0}, tj[3] = {0, 0, 0};
        for (uint32_t o = 0; o < T.n_ops; o++) {
            const triosim_op op = T.ops[o];
            if (s_stage[op.layer] != s) continue;
            const int P = op.phase;
            uint32_t nsend = 0, ntp = 0;
            for (uint32_t k = 0; k < op.n_out; k++) {
                const uint32_t x = T.io[op.io_off + op.n_in + k];
                unsigned long long r = readers[x] & ~(1ull << s);
                while (r) {
                    const int d = __ffsll((long long)r) - 1;
                    r &= r - 1;
                    HSend se;
                    se.bytes = tensor_bytes(T, x, C.r_b, C.tpdeg, C.tp_mode);
                    se.x = x;
                    se.dst = (uint16_t)d;
                    se.pidx = (uint16_t)ei[P];
                    se.tpg = -1;
                    se.pad = 0;
                    sends[soff[P] + sj[P]++] = se;
                    nsend++;
                }
                if (tp > 1) {
                    int kind = tp_kind_dev(op.tp_role, op.phase, T.ts[x].category, C.tp_mode);
                    if (kind >= 0) {
                        CollEnt ce;
                        ce.S = (double)T.ts[x].bytes_b0;
                        if (T.ts[x].batch_scaled) ce.S = ce.S * C.r_b;
                        ce.layer = op.layer;
                        ce.pad2 = 0;
                        if (kind == CK_AR && C.algo == TRIOSIM_ALGO_RSAG) {
                            // R29: the ReduceScatter half (no reader waits on it: pad = no tensor), then the AllGather
                            ce.kind = CK_RS;
                            ce.pad = 0xffffffffu;
                            colls[toff[P] + tj[P]++] = ce;
                            ntp++;
                            kind = CK_AG;
                        }
                        ce.kind = (uint32_t)kind;
                        ce.pad = x;
                        colls[toff[P] + tj[P]++] = ce;
                        ntp++;
                    }
                }
            }
            HEnt en;
            en.dur = dur[C.dur_off + o];
            en.run = en.run0 = 1;
            en.op = o;
            en.nsend = (uint16_t)nsend;
            en.nrecv = 0;
            en.recv_off = 0;
            en.tp_nsig = (uint16_t)ntp;
            en.dp_nsig = 0;
            en.tpw = -1;
            en.pad = 0;
            ents[eoff[P] + ei[P]++] = en;
        }
        if (dp > 1) {
            const int nw = T.scal[0];
            uint64_t sum = 0;
            double Sb = 0.0;
            uint32_t b = 0;
            int32_t last_prod = -1;
            bool open = false;
            for (int i = 0; i <= nw; i++) {
                const bool end = i == nw;
                if (!end) {
                    const uint32_t x = T.wgrad[i];
                    if (s_stage[T.layer[T.prod[x]]] != s) continue;
                    sum += T.ts[x].bytes_b0;
                    Sb = Sb + tensor_bytes(T, x, C.r_b, C.tpdeg, C.tp_mode);
                    last_prod = T.prod[x];
                    open = true;
                }
                const uint64_t cap = bucket_cap(C, C.algo == TRIOSIM_ALGO_RSAG ? b / 2 : b);   // b counts collectives (R29: 2 per bucket)
                if (open && (end || cap == 0 || sum >= cap)) {
                    CollEnt ce;
                    ce.S = Sb;
                    ce.kind = CK_AR;
                    ce.pad = 0;
                    ce.layer = T.layer[last_prod];
                    ce.pad2 = 0;
                    // trigger: (producer of the bucket's last gradient, micro-batch 0); the HYBRID form
                    // of DataParallel (R6) triggers every bucket after the stage's last non-OPT op
                    const uint16_t parts = C.algo == TRIOSIM_ALGO_RSAG ? 2 : 1;   // R29: RS + AG pair
                    if (C.dp_after_bwd && (si.nB > 0 || si.nF > 0)) {
                        HEnt &te = ents[si.nB > 0 ? eoff[1] + si.nB - 1 : eoff[0] + si.nF - 1];
                        te.dp_nsig += parts;
                        ce.layer = T.layer[te.op];
                    } else {
                        const int P = (int)(T.info[last_prod] & INFO_PHASE_MASK);
                        const uint32_t cntP = P == 0 ? si.nF : P == 1 ? si.nB : si.nO;
                        for (uint32_t q = 0; q < cntP; q++)
                            if (ents[eoff[P] + q].op == (uint32_t)last_prod) { ents[eoff[P] + q].dp_nsig += parts; break; }
                    }
                    if (parts == 2) {
                        ce.kind = CK_RS;
                        colls[hs.dcol_off + b++] = ce;
                        ce.kind = CK_AG;
                    }
                    colls[hs.dcol_off + b++] = ce;
                    sum = 0;
                    Sb = 0.0;
                    open = false;
                }
            }
        }
    }
    __syncthreads();
    // pass 3: receive lists, TP waits of same-stage readers, TP gates of sends
    if (tid < S) {
        const int s = tid;
        const StageInfo si = SI[s];
        const HStage hs = HS[s];
        const uint32_t tcnt[3] = {hs.TF, hs.TB, hs.TO};
        const uint32_t toff[3] = {hs.tcol_off, hs.tcol_off + hs.TF, hs.tcol_off + hs.TF + hs.TB};
        uint32_t rv = si.recv_off;
        const uint32_t total = si.nF + si.nB + si.nO;
        for (uint32_t q = 0; q < total; q++) {
            HEnt &en = ents[si.ent_off + q];
            const triosim_op op = T.ops[en.op];
            en.recv_off = rv;
            uint32_t nr = 0;
            int32_t tpw = -1;
            for (uint32_t k = 0; k < op.n_in; k++) {
                const uint32_t x = T.io[op.io_off + k];
                const int32_t po = T.prod[x];
                if (po < 0) continue;
                const int ps = s_stage[T.layer[po]];
                const int pph = (int)(T.info[po] & INFO_PHASE_MASK);
                if (ps == s) {
                    if (tp > 1)
                        for (uint32_t e = 0; e < tcnt[pph]; e++)
                            if (colls[toff[pph] + e].pad == x) {
                                const int32_t key = (pph << 24) | (int32_t)e;
                                if (key > tpw) tpw = key;
                                break;
                            }
                    continue;
                }
                const StageInfo pi = SI[ps];
                const uint32_t base = pi.send_off + (pph == 0 ? 0 : pph == 1 ? pi.SF : pi.SF + pi.SB);
                const uint32_t cnt = pph == 0 ? pi.SF : pph == 1 ? pi.SB : pi.SO;
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
            en.tpw = tpw;
        }
        {
            // fold run lengths per phase list, back to front (K3h's has_wait / has_sig, R16): entry e
            // folds e + 1 when e signals nothing and e + 1 waits for nothing; run0 counts DP triggers
            // as signals (micro-batch instance 0)
            const uint32_t base[3] = {si.ent_off, si.ent_off + si.nF, si.ent_off + si.nF + si.nB};
            const uint32_t len[3] = {si.nF, si.nB, si.nO};
            const bool dpw = dp > 1 && hs.ndp > 0;
            for (int P = 0; P < 3; P++)
                for (int e = (int)len[P] - 2; e >= 0; e--) {
                    HEnt &x = ents[base[P] + e];
                    const HEnt &y = ents[base[P] + e + 1];
                    const bool yw = y.nrecv > 0 || y.tpw >= 0 || (P == 2 && (uint32_t)(e + 1) == hs.first_opt && dpw);
                    const bool xs = x.nsend > 0 || x.tp_nsig > 0;
                    x.run = (!xs && !yw) ? y.run + 1 : 1;
                    x.run0 = (!xs && x.dp_nsig == 0 && !yw) ? y.run0 + 1 : 1;
                }
        }
        if (tp > 1) {
            const uint32_t scnt = si.SF + si.SB + si.SO;
            for (uint32_t q = 0; q < scnt; q++) {
                HSend &se = sends[si.send_off + q];
                const int P = q < si.SF ? 0 : q < si.SF + si.SB ? 1 : 2;
                for (uint32_t e = 0; e < tcnt[P]; e++)
                    if (colls[toff[P] + e].pad == se.x) { se.tpg = (P << 24) | (int32_t)e; break; }
            }
        }
    }
    __syncthreads();
    if (tid == 0) {
        // class totals; collective payloads folded in canonical creation order (R9): TP groups
        // (d, s) then DP groups (s, t)
        uint64_t ncomp = 0, nflow = 0, ncoll = 0;
        uint32_t pmax = 0, any_ag = 0, any_ar = 0;
        double payload = 0.0;
        for (int s = 0; s < S; s++) {
            const uint32_t prog = m * (SI[s].nF + SI[s].nB) + SI[s].nO;
            ncomp += (uint64_t)prog * dp * tp;
            if (prog > pmax) pmax = prog;
            nflow += ((uint64_t)m * (SI[s].SF + SI[s].SB) + SI[s].SO) * dp * tp;
        }
        for (int d = 0; d < dp && tp > 1; d++)
            for (int s = 0; s < S; s++) {
                const HStage hs = HS[s];
                const uint32_t part[3][2] = {{hs.tcol_off, hs.TF}, {hs.tcol_off + hs.TF, hs.TB},
                                             {hs.tcol_off + hs.TF + hs.TB, hs.TO}};
                for (uint32_t j = 0; j < m; j++)
                    for (uint32_t e = 0; e < part[0][1]; e++) payload = payload + colls[part[0][0] + e].S;
                for (uint32_t j = 0; j < m; j++)
                    for (uint32_t e = 0; e < part[1][1]; e++) payload = payload + colls[part[1][0] + e].S;
                for (uint32_t e = 0; e < part[2][1]; e++) payload = payload + colls[part[2][0] + e].S;
                for (uint32_t e = 0; e < hs.TF + hs.TB + hs.TO; e++) {
                    const uint32_t kind = colls[hs.tcol_off + e].kind;
                    const uint64_t reps = e < hs.TF + hs.TB ? m : 1;
                    const uint64_t per = (kind == CK_AG || kind == CK_RS) ? (uint64_t)(tp - 1) * tp * C.nch
                                       : C.algo == TRIOSIM_ALGO_TREE ? 2ull * (tp - 1)
                                       : C.algo == TRIOSIM_ALGO_DBTREE ? 4ull * (tp - 1)
                                       : C.algo == TRIOSIM_ALGO_REDBCAST ? 2ull * (tp - 1) * C.nch : 2ull * (tp - 1) * tp * C.nch;
                    nflow += reps * per;
                    ncoll += reps;
                    if (kind == CK_AG) any_ag = 1; else any_ar = 1;
                }
            }
        for (int s = 0; s < S && dp > 1; s++)
            for (int t = 0; t < tp; t++)
                for (uint32_t b = 0; b < HS[s].ndp; b++) {
                    payload = payload + colls[HS[s].dcol_off + b].S;
                    nflow += C.algo == TRIOSIM_ALGO_TREE ? 2ull * (dp - 1)
                           : C.algo == TRIOSIM_ALGO_DBTREE ? 4ull * (dp - 1)
                           : C.algo == TRIOSIM_ALGO_REDBCAST ? 2ull * (dp - 1) * C.nch
                           : C.algo == TRIOSIM_ALGO_RSAG ? 1ull * (dp - 1) * dp * C.nch : 2ull * (dp - 1) * dp * C.nch;
                    ncoll++;
                    any_ar = 1;
                }
        C.n_compute = ncomp;
        C.n_flows = nflow;
        C.n_coll = (uint32_t)ncoll;
        C.coll_payload = payload;
        C.n_prog_max = pmax;
        C.need_ring = any_ag || (any_ar && C.algo != TRIOSIM_ALGO_TREE && C.algo != TRIOSIM_ALGO_DBTREE);
        C.need_tree = any_ar && (C.algo == TRIOSIM_ALGO_TREE || C.algo == TRIOSIM_ALGO_DBTREE);
    }
}

cudaError_t launch_k2_hybrid(ClassDesc *cls, const uint32_t *list, uint32_t n, const TraceDev &T,
                             const uint32_t *plan_pool, StageInfo *stages, HStage *hst, HEnt *ents, HSend *sends,
                             RecvEnt *recvs, CollEnt *colls, unsigned long long *scratch, const double *dur,
                             cudaStream_t s) {
    if (n == 0) return cudaSuccess;
    k2_hybrid<<<n, K2P_THREADS, 0, s>>>(cls, list, T, plan_pool, stages, hst, ents, sends, recvs, colls, scratch, dur);
    return cudaGetLastError();
}

// ------------------------------------------------------------------------------------
// K4 (R22): per-layer breakdown.  k4_layer_compute: per class, one thread per layer, the left fold
// of t' over the representative rank's program instances of that layer in program order (rank 0
// runs every operator in DP / DDP / TP; in GPipe / HYBRID the layer's stage runs FWD of
// micro-batches 0..m-1, BWD of m-1..0, OPT once).  k4_breakdown: per (point, layer), the class's
// compute and comm = (TP-group + DP-group collective time) + P2P time from K3's accumulators.
// ------------------------------------------------------------------------------------
__global__ void __launch_bounds__(128) k4_layer_compute(const ClassDesc *cls, TraceDev T, const double *dur,
                                                        const StageInfo *stages, const StageEnt *ents,
                                                        const HEnt *hents, double *lcomp) {
    const ClassDesc &C = cls[blockIdx.x];
    const uint32_t L = T.n_layers;
    const double *du = dur + C.dur_off;
    for (uint32_t l = threadIdx.x; l < L; l += blockDim.x) {
        double acc = 0.0;
        if (C.mode == MODE_COLL || C.mode == MODE_TREE) {
            for (uint32_t o = 0; o < T.n_ops; o++)
                if (T.layer[o] == l) acc = acc + du[o];
        } else if (C.mode == MODE_HOP) {   // R28: rank 0 runs every operator once per iteration
            for (uint32_t k = 0; k < C.m; k++)
                for (uint32_t o = 0; o < T.n_ops; o++)
                    if (T.layer[o] == l) acc = acc + du[o];
        } else {
            const bool hyb = C.mode == MODE_HYBRID;
            auto op_at = [&](uint32_t e) -> uint32_t { return hyb ? hents[e].op : ents[e].op; };
            // the stage that runs layer l (stages hold contiguous layers, every op of l in one stage)
            int st = -1;
            for (uint32_t s = 0; s < C.p && st < 0; s++) {
                const StageInfo SI = stages[C.stage_off + s];
                const uint32_t n = SI.nF + SI.nB + SI.nO;
                for (uint32_t e = 0; e < n; e++)
                    if (T.layer[op_at(SI.ent_off + e)] == l) { st = (int)s; break; }
            }
            if (st >= 0) {
                const StageInfo SI = stages[C.stage_off + st];
                for (uint32_t j = 0; j < C.m; j++)
                    for (uint32_t e = 0; e < SI.nF; e++) {
                        const uint32_t o = op_at(SI.ent_off + e);
                        if (T.layer[o] == l) acc = acc + du[o];
                    }
                for (uint32_t j = 0; j < C.m; j++)
                    for (uint32_t e = 0; e < SI.nB; e++) {
                        const uint32_t o = op_at(SI.ent_off + SI.nF + e);
                        if (T.layer[o] == l) acc = acc + du[o];
                    }
                for (uint32_t e = 0; e < SI.nO; e++) {
                    const uint32_t o = op_at(SI.ent_off + SI.nF + SI.nB + e);
                    if (T.layer[o] == l) acc = acc + du[o];
                }
            }
        }
        lcomp[(size_t)blockIdx.x * L + l] = acc;
    }
}

cudaError_t launch_k4_layer_compute(const ClassDesc *cls, uint32_t n_cls, const TraceDev &T, const double *dur,
                                    const StageInfo *stages, const StageEnt *ents, const HEnt *hents,
                                    double *lcomp, cudaStream_t s) {
    if (n_cls == 0 || T.n_layers == 0) return cudaSuccess;
    k4_layer_compute<<<n_cls, 128, 0, s>>>(cls, T, dur, stages, ents, hents, lcomp);
    return cudaGetLastError();
}

__global__ void k4_breakdown(const PointDesc *pts, const triosim_result *res, uint64_t first, uint64_t count,
                             uint32_t L, const double *lcomp, const double *acc, double *out_comp, double *out_comm) {
    const uint64_t n = count * L;
    for (uint64_t q = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; q < n; q += (uint64_t)gridDim.x * blockDim.x) {
        const uint64_t i = first + q / L;
        const uint32_t l = (uint32_t)(q % L);
        double c = 0.0, m = 0.0;
        if (res[i].status == TRIOSIM_PT_OK) {
            const double *A = acc + i * 3ull * L;
            c = lcomp[(size_t)pts[i].cls * L + l];
            m = (A[l] + A[L + l]) + A[2 * L + l];
        }
        if (out_comp) out_comp[q] = c;
        if (out_comm) out_comm[q] = m;
    }
}

cudaError_t launch_k4_breakdown(const PointDesc *pts, const triosim_result *res, uint64_t first, uint64_t count,
                                uint32_t n_layers, const double *lcomp, const double *acc, double *out_comp,
                                double *out_comm, cudaStream_t s) {
    const uint64_t n = count * n_layers;
    if (n == 0) return cudaSuccess;
    uint64_t blocks = (n + 255) / 256;
    if (blocks > 148 * 16) blocks = 148 * 16;
    k4_breakdown<<<(unsigned)blocks, 256, 0, s>>>(pts, res, first, count, n_layers, lcomp, acc, out_comp, out_comm);
    return cudaGetLastError();
}

}  // namespace ts
