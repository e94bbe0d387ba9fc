// ts_internal.h -- device-side data layout of libtriosim.
// Shared only by ts_host.cu and ts_kernels.cu (product path).  Nothing here is shared
// with oracle/.
#pragma once
#include <cstdint>
#include "triosim.h"

namespace ts {

enum { MODE_COLL = 0, MODE_PIPE = 1, MODE_TREE = 2, MODE_HYBRID = 3, MODE_HOP = 4 };  // K3 variants: ring-only collectives, GPipe, tree-capable collectives, DP x TP x PP, Hop (R28)
enum { CK_AR = 0, CK_AG = 1, CK_RS = 2 };
enum { PH_FWD = 0, PH_BWD = 1, PH_OPT = 2 };
constexpr int MAX_HOPS = 8;   // route hops cached in registers per flow; longer routes read the rest from rt_links
constexpr uint32_t MAX_ROUTE_K3 = 32;   // longest route of a warp-kernel (K3) topology (its owner bits); beyond: K3h
constexpr uint8_t NO_ROUTE = 0xFF;
#ifndef TS_K3_THREADS
#define TS_K3_THREADS 128
#endif
constexpr int K3_THREADS = TS_K3_THREADS;   // threads per CTA of the warp-segment K3 kernels
constexpr int K3_WARPS = K3_THREADS / 32;

// per-op packed info written by the ingest kernel
constexpr uint32_t INFO_PHASE_MASK = 3u;
constexpr uint32_t INFO_ROLE_SHIFT = 2;   // 3 bits of tp_role
constexpr uint32_t INFO_SCALED = 1u << 5;

struct TraceDev {
    // raw staged records
    const triosim_op *ops;
    const triosim_tensor *ts;
    const uint32_t *io;
    // SoA produced by K1a (ingest)
    double *time;       // n_ops
    uint32_t *info;     // n_ops: phase | role << 2 | scaled << 5
    uint32_t *layer;    // n_ops
    int32_t *prod;      // n_ts: producing op or -1
    uint32_t *wgrad;    // weight gradients in production order (non-OPT producers)
    int32_t *scal;      // [0] n_wgrad, [1] first OPT op (INT_MAX = none), [2] last non-OPT op (-1 = none)
    uint32_t n_ops, n_ts, n_io, b0, n_layers, pad;
};

// COLL mode (DP / DDP / TP): one entry per operator of a class
struct OpHook {
    double dur;       // t' (K1b)
    int32_t wait;     // collective index that must be done on this GPU before the op starts, or -1
    uint32_t nsig;    // number of collectives triggered by this op's completion
};
struct CollEnt {
    double S;         // payload bytes
    uint32_t kind;    // CK_*
    uint32_t pad;     // HYBRID K2: the communicated tensor
    uint32_t layer;   // layer of the triggering operator (R22 per-layer breakdown)
    uint32_t pad2;
};

// PIPE mode (GPipe): per stage of a class
struct StageInfo {
    uint32_t nF, nB, nO;      // ops of the stage per phase
    uint32_t SF, SB, SO;      // P2P sends per micro-batch (F, B) and once (O)
    uint32_t ent_off;         // StageEnt list: [F nF][B nB][O nO]
    uint32_t send_off;        // SendEnt list: [F SF][B SB][O SO]
    uint32_t recv_off;        // RecvEnt pool base of this stage
    uint32_t pad;
    uint64_t dst_mask;        // stages this stage sends to (route check)
};
struct StageEnt {
    double dur;       // t' of the operator (K2 copy of K1b's dur[op]): the compute fold reads one array
    uint32_t op;
    uint16_t nsend, nrecv;
    uint32_t recv_off;
    uint32_t run;     // entries from here on (within this phase list) that one start folds (R16): the
                      // next one has no receive and none before the last has a send
};
struct SendEnt {
    double bytes;
    uint32_t x;
    uint16_t dst;    // destination stage
    uint16_t pidx;   // producer index inside its phase list
};
struct RecvEnt {
    uint16_t src;    // producing stage
    uint8_t phase;   // producer phase
    uint8_t pad;
    uint32_t e;      // index in the producer stage's send list of that phase
};

// HYBRID (DP x TP x PP): per stage, on top of StageInfo
struct HStage {
    uint32_t TF, TB, TO;      // TP collectives per micro-batch (F, B) and once (O) of one TP group
    uint32_t tcol_off;        // CollEnt list [F TF][B TB][O TO]
    uint32_t ndp, dcol_off;   // DP buckets of this stage (one DP group per t)
    uint32_t first_opt;       // index of the first OPT op inside the stage's OPT list, or 0xffffffff
    uint32_t pad;
};
struct HEnt {                 // per stage op entry (hybrid): the PIPE entry plus TP / DP hooks
    double dur;                  // t' of the operator (K2 copy of K1b's dur[op]) for the compute fold
    uint32_t op;
    uint16_t nsend, nrecv;
    uint32_t recv_off;
    uint16_t tp_nsig, dp_nsig;   // TP collectives triggered (every instance); DP buckets (instance 0)
    int32_t tpw;                 // TP collective to wait for: (phase << 24) | index, or -1
    uint32_t run, run0;          // fold run lengths from here within the phase list (R16) for micro-batch
                                 // instances j > 0 / j == 0 (DP triggers only signal on instance 0)
    uint32_t pad;
};
struct HSend {
    double bytes;
    uint32_t x;
    uint16_t dst, pidx;
    int32_t tpg;                 // TP collective of the tensor on the sender: (phase << 24) | index, or -1
    uint32_t pad;
};

struct ClassDesc {
    // set by the host
    uint32_t mode, strategy, tp_mode, algo;
    uint32_t p, m, tpdeg, b_loc;
    uint64_t bucket_bytes;
    double r_b;
    uint32_t dur_off, hook_off, coll_off, coll_cap;
    uint32_t plan_off, stage_off, ent_off, ent_cap;
    uint32_t send_off, send_cap, recv_off, recv_cap;
    uint32_t scratch_off, dp;            // dp: HYBRID data-parallel degree
    uint32_t hst_off, tcol_off, tcol_cap, dcol_off, dcol_cap;   // HYBRID pools
    uint32_t dp_after_bwd;               // HYBRID form of DataParallel: DP buckets trigger after the backward pass
    uint32_t first_bucket;               // R24: cap of each gradient group's first bucket (0 = bucket_bytes)
    uint32_t nch, pad_nch;               // R25: chunks per ring step (>= 1)
    // written by K2
    uint32_t n_coll, need_ring, need_tree, n_prog_max;
    double coll_payload;
    uint64_t n_compute, n_flows;
    // R28 Hop: backup | staleness << 4 | gap << 8 (host); K2: update bytes, last non-OPT op, first OPT op
    uint32_t hop, hop_last, hop_first, hop_pad;
    double hop_S;
};

struct TopoDev {
    uint32_t n_nodes, n_gpus, n_links, link_off;
    uint32_t rt_off, ro_off;
    // bit p (p = 2..32 over the two words): the routes ring_order[i] -> ring_order[(i+1) % p] of
    // the first p GPUs are pairwise link-disjoint, so ring flows never share a link (K3 fast path)
    uint32_t ring_disjoint_lo, ring_disjoint_hi;
    // photonic circuit-switched network (R20); net == TRIOSIM_NET_FLOW: unused
    uint32_t net, ports, buf_slots, pad;
    double ph_bw, ph_setup, ph_lat;
};

struct PointDesc {
    double bw_scale, lat_scale;
    uint32_t cls, topo, idx, pad;
};

struct K3Args {
    const PointDesc *pts;
    const uint32_t *work;
    uint32_t n_work, lmax;         // lmax: links per segment in dynamic smem (one-point-per-CTA hybrid)
    uint32_t rlo, rhi;             // simulate only work items (point indices) in [rlo, rhi)
    uint32_t pmax, pad2;           // pmax: photonic ports per lane in dynamic smem (hybrid, R20)
    unsigned int *counter;
    const ClassDesc *cls;
    const TopoDev *topo;
    const double *link_bw, *link_lat;
    const uint32_t *rt_off;
    const uint8_t *rt_len;
    const uint16_t *rt_links;
    const uint32_t *ro;
    const OpHook *hooks;
    const CollEnt *colls;
    const double *dur;
    const StageInfo *stages;
    const StageEnt *ents;
    const SendEnt *sends;
    const RecvEnt *recvs;
    const HStage *hst;
    const HEnt *hents;
    const HSend *hsends;
    triosim_result *out;
    unsigned long long *alg_ops;   // method fp64 operations performed
    // R22 per-layer breakdown (kernel variant BD only): per point [3][n_layers] communication
    // accumulators (TP-group collectives, DP-group collectives, P2P sends of the layer's
    // representative rank), zeroed by the host before the launch
    double *bd;
    const uint32_t *layer;         // trace: layer of each operator
    uint32_t n_layers, pad3;
    // R23 timeline (kernel variant LOG only): record slots counted in tl_cnt[0] (tasks), [1] (flows)
    triosim_task_rec *tl_tasks;
    triosim_flow_rec *tl_flows;
    unsigned long long *tl_cnt;
    uint64_t tl_task_cap, tl_flow_cap;
};

// K3 instantiations: V bit 0 = BD (R22 breakdown), bit 1 = LOG (R23 timeline; no ring fast-forward)
constexpr int V_BD = 1, V_LOG = 2;
__host__ __device__ constexpr int k3_variant(bool bd, bool log) { return (bd ? V_BD : 0) | (log ? V_LOG : 0); }

// launchers (ts_kernels.cu)
cudaError_t launch_k1_ingest(const TraceDev &T, cudaStream_t s);
cudaError_t launch_k1_rescale(const ClassDesc *cls, uint32_t n_cls, const TraceDev &T, double *dur, cudaStream_t s);
cudaError_t launch_k2_coll(ClassDesc *cls, const uint32_t *list, uint32_t n, const TraceDev &T, const double *dur,
                           OpHook *hooks, CollEnt *colls, int32_t *scratch_i32, cudaStream_t s);
cudaError_t launch_k2_pipe(ClassDesc *cls, const uint32_t *list, uint32_t n, const TraceDev &T, const double *dur,
                           const uint32_t *plan_pool, StageInfo *stages, StageEnt *ents, SendEnt *sends,
                           RecvEnt *recvs, unsigned long long *scratch_u64, cudaStream_t s);
cudaError_t launch_k2_hybrid(ClassDesc *cls, const uint32_t *list, uint32_t n, const TraceDev &T,
                             const uint32_t *plan_pool, StageInfo *stages, HStage *hst, HEnt *ents, HSend *sends,
                             RecvEnt *recvs, CollEnt *colls, unsigned long long *scratch_u64, const double *dur,
                             cudaStream_t s);
// K3 variants: a.bd != nullptr selects the breakdown-recording (BD) instantiation, a.tl_cnt != nullptr the
// timeline-recording (LOG) one
cudaError_t launch_k3(int W, int mode, const K3Args &a, int grid, cudaStream_t s);   // ts_k3.cu
cudaError_t launch_k3_hybrid(int W, const K3Args &a, int grid, cudaStream_t s);      // ts_k3h.cu
// R22: per-class layer compute (left fold of t' over the representative rank's program) and the
// per-point finalisation into caller buffers (ts_kernels.cu)
cudaError_t launch_k4_layer_compute(const ClassDesc *cls, uint32_t n_cls, const TraceDev &T, const double *dur,
                                    const StageInfo *stages, const StageEnt *ents, const HEnt *hents,
                                    double *lcomp, cudaStream_t s);
cudaError_t launch_k4_breakdown(const PointDesc *pts, const triosim_result *res, uint64_t first, uint64_t count,
                                uint32_t n_layers, const double *lcomp, const double *acc, double *out_comp,
                                double *out_comm, cudaStream_t s);
// R23: canonical order of the recorded timeline (ts_timeline.cu)
cudaError_t sort_timeline(triosim_task_rec *tasks, uint64_t nt, triosim_flow_rec *flows, uint64_t nf, cudaStream_t s);
int k3h_max_blocks_per_sm(int W, uint32_t lmax, uint32_t pmax);   // dynamic smem: links (W > 32), ports
size_t k3h_dyn_smem(int W, uint32_t lmax, uint32_t pmax);
int k3_max_blocks_per_sm(int W, int mode);
// links per segment the K3 kernels keep in shared memory
__host__ __device__ constexpr int lmax_warp(int W) { return 4 * W < 8 ? 8 : 4 * W; }
__host__ __device__ constexpr int lmax_hybrid(int W) { return 8 * W < 16 ? 16 : 8 * W; }
constexpr int LMAX_CTA = 6144;          // links of a one-point-per-CTA hybrid segment (dynamic smem, 28 B/link)
constexpr int N_WIDTHS = 10;            // W = 2, 4, 8, 16, 32 (warp segments), 64 ... 1024 (hybrid CTAs)
constexpr int N_MODES = 5;
constexpr int N_GROUPS = N_MODES * N_WIDTHS;  // (width, mode) launch groups
constexpr int MAX_PORTS = 8;            // photonic ports per GPU the hybrid kernel holds (R20)
constexpr uint32_t K2P_MAX_LAYERS = 2048;   // trace layers the PP / HYBRID expansion (K2) stages in shared memory

}  // namespace ts
