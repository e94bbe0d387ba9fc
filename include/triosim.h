/*
 * triosim.h -- C ABI of libtriosim.so, the B200-native batched design-point
 * simulator of TrioSim (Li et al., ISCA'25; PAPER.md = "P:N" line refs).
 *
 * A design point = (parallelism strategy, degrees, topology + bandwidth /
 * latency scale, batch size, ...).  For every point the library runs the three
 * steps of the paper's method on the GPU (DESIGN.md "Semantics" R1-R19):
 *   1. operator-time model on the single-GPU trace,
 *   2. trace extrapolation of DP / DDP / TP / PP into compute tasks and
 *      collective / point-to-point flows,
 *   3. an event-driven timeline whose in-transit flows share link bandwidth by
 *      max-min fair progressive filling, re-allocated whenever a flow starts or
 *      completes (Fig. 5),
 * and returns the predicted iteration time plus breakdowns.
 *
 * Conventions: all structs are little-endian with natural alignment (sizes are
 * asserted below).  Times are seconds, bandwidths bytes/s, sizes bytes, IEEE
 * binary64.  Entry points return a triosim_status (0 = OK, < 0 = error); the
 * message of the last error is available from triosim_last_error().  A context
 * is bound to one CUDA device and is not thread-safe (use one per thread).
 * Every input array is deep-copied during the call: the caller may free it as
 * soon as the call returns.  There is no CPU fallback: if the CUDA device is
 * missing or not sm_100, triosim_create fails with TRIOSIM_EUNSUPPORTED.
 */
#ifndef TRIOSIM_H
#define TRIOSIM_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef int32_t triosim_status;
#define TRIOSIM_OK 0
#define TRIOSIM_EINVAL (-1)       /* malformed input table / argument */
#define TRIOSIM_ENOMEM (-2)       /* host or device allocation failed */
#define TRIOSIM_ECUDA (-3)        /* CUDA runtime error (sticky errors reported on the next call) */
#define TRIOSIM_ENOTFOUND (-4)    /* unknown trace / sweep handle */
#define TRIOSIM_ERANGE (-5)       /* point range outside the sweep */
#define TRIOSIM_EUNSUPPORTED (-6) /* no sm_100 device */

/* per-point status in triosim_result.status (R3) */
#define TRIOSIM_PT_OK 0
#define TRIOSIM_PT_BAD_BATCH 1   /* global_batch not divisible by dp * microbatches (Q3, Q12) */
#define TRIOSIM_PT_BAD_DEGREES 2 /* zero / inconsistent degrees, dp*tp*pp > GPUs, pp > layers or > 64 */
#define TRIOSIM_PT_NO_ROUTE 3    /* a needed (src, dst) GPU pair has no path */
#define TRIOSIM_PT_TOO_LARGE 4   /* exceeds this GPU kernel's limits: > 1024 ranks, > 6144 links on a > 32-rank point,
                                    tree collectives over photonic links, a double binary tree on a HYBRID
                                    point with both TP and DP groups, Hop beyond 32 workers (R3) */
#define TRIOSIM_PT_DEADLOCK 5    /* the task graph cannot make progress */
#define TRIOSIM_PT_BAD_PLAN 6    /* explicit stage plan invalid for this point */
#define TRIOSIM_PT_BAD_CONFIG 7  /* unknown enum, topology index out of range, bw_scale <= 0, lat_scale < 0 */

/* operator phases, tensor categories, TP roles */
#define TRIOSIM_PHASE_FWD 0
#define TRIOSIM_PHASE_BWD 1
#define TRIOSIM_PHASE_OPT 2
#define TRIOSIM_CAT_INPUT 0
#define TRIOSIM_CAT_WEIGHT 1
#define TRIOSIM_CAT_WGRAD 2
#define TRIOSIM_CAT_ACT 3
#define TRIOSIM_CAT_AGRAD 4
#define TRIOSIM_CAT_OTHER 5
#define TRIOSIM_ROLE_NONE 0   /* bits 0-1: Megatron role */
#define TRIOSIM_ROLE_COL 1
#define TRIOSIM_ROLE_ROW 2
#define TRIOSIM_ROLE_LOCAL 3
#define TRIOSIM_ROLE_GATHER 4 /* bit 2: paper-mode split layer (conv / linear / embedding) */
#define TRIOSIM_OPF_BATCH_SCALED 1u

/* One operator of the single-GPU trace, in program order ("operator name, measured
 * execution time, and input/output as a list of tensor IDs").  Phases must be FWD* BWD* OPT*;
 * layer ids are numbered by first FWD appearance (0, 1, 2, ...).  io[io_off .. io_off+n_in)
 * are the inputs, the next n_out entries the outputs. */
typedef struct {
    uint32_t kind;    /* operator name id (informational) */
    uint32_t layer;
    uint8_t phase;
    uint8_t tp_role;
    uint16_t flags;   /* TRIOSIM_OPF_* */
    uint32_t io_off;
    uint16_t n_in, n_out;
    uint32_t pad;
    double time_s;    /* measured time on the trace GPU at trace_batch */
    double flops;     /* informational */
} triosim_op;         /* 40 B */

/* One tensor: bytes at the trace batch, category, batch dependence. */
typedef struct {
    uint64_t bytes_b0;
    uint8_t category;
    uint8_t batch_scaled;
    uint16_t pad;
    uint32_t param_id;
} triosim_tensor;     /* 16 B */

typedef struct {
    uint32_t n_ops, n_tensors, n_io, trace_batch;
    const triosim_op *ops;          /* host pointers */
    const triosim_tensor *tensors;
    const uint32_t *io;
} triosim_trace_desc;

/* Directed link (P:142 topology input, P:226 bandwidth is a user input). */
typedef struct {
    uint32_t src, dst;  /* node ids; GPUs are nodes [0, n_gpus), switches after */
    double bw_Bps;      /* > 0 */
    double lat_s;       /* >= 0 */
} triosim_link;         /* 24 B */

/* Photonic circuit-switched interconnect (Lightmatter Passage case study; R20).
 * A send (1) establishes a directed logical link src -> dst if none exists, taking setup_s, on one of
 * the sender's `ports` photonic ports; with no free port it tears down the sender's link that has been
 * idle the longest; (2) waits for a receive buffer at the destination (buf_slots per GPU,
 * 0 = unlimited); (3) moves the data at the link's dedicated bandwidth: delivered lat_s + bytes /
 * link_bw_Bps after the buffer is granted.  Requests are served in (release time, flow id) order.
 * The point's bw_scale multiplies link_bw_Bps, lat_scale multiplies setup_s and lat_s. */
typedef struct {
    uint32_t ports;       /* 1..8 */
    uint32_t buf_slots;   /* receive buffers per GPU, 0 = unlimited */
    double link_bw_Bps;   /* > 0: bandwidth of one logical link (484 GB/s across 8 links) */
    double setup_s;       /* >= 0: latency of establishing a logical link (20 ms) */
    double lat_s;         /* >= 0: latency of one transfer */
} triosim_photonic;       /* 32 B */

#define TRIOSIM_NET_FLOW 0      /* links + routes, max-min fair flow model (R12-R15) */
#define TRIOSIM_NET_PHOTONIC 1  /* logical links of a circuit-switched photonic interposer (R20) */

typedef struct {
    uint32_t n_nodes, n_gpus, n_links;
    uint32_t net_model;             /* TRIOSIM_NET_*; PHOTONIC ignores links (n_links may be 0) */
    const triosim_link *links;      /* at most one link per ordered pair */
    const uint32_t *ring_order;     /* permutation of [0, n_gpus) or NULL (= identity) */
    const triosim_photonic *photonic;  /* required iff net_model == PHOTONIC, else ignored */
} triosim_topology;

/* Explicit PP stage plans: plan k has first_layer[off[k] .. off[k+1]) (first must be 0,
 * strictly increasing); a point selects one with stage_plan = k, or -1 = automatic. */
typedef struct {
    uint32_t n_plans;
    const uint32_t *off;            /* n_plans + 1 entries */
    const uint32_t *first_layer;
} triosim_stage_plans;

#define TRIOSIM_DP 0      /* DataParallel: gradient AllReduce after the backward pass */
#define TRIOSIM_DDP 1     /* DistributedDataParallel: AllReduce overlapped with backward */
#define TRIOSIM_TP 2      /* tensor parallel */
#define TRIOSIM_PP 3      /* GPipe pipeline parallel */
#define TRIOSIM_HYBRID 4  /* DP x TP x PP (extension, R9) */
#define TRIOSIM_HOP 5     /* Hop heterogeneity-aware decentralized training (R28): dp = workers
                             (even; <= 32 on this library's kernel), microbatches = iterations, tp_mode = the
                             communication graph (TRIOSIM_HOP_*), hop = backup | staleness << 4 | max gap << 8 */
#define TRIOSIM_HOP_RING_BASED 0   /* Fig. 16a top: ring plus each worker's most distant worker */
#define TRIOSIM_HOP_DOUBLE_RING 1  /* Fig. 16a bottom: two ring-based graphs joined node to node (dp % 4 == 0) */
#define TRIOSIM_TP_PAPER 0
#define TRIOSIM_TP_MEGATRON 1
#define TRIOSIM_ALGO_RING 0
#define TRIOSIM_ALGO_TREE 1
#define TRIOSIM_ALGO_REDBCAST 2   /* AllReduce as ring Reduce to member 0 + ring Broadcast from it, pipelined in
                                     ring_chunks chunks (R26); AllGather / ReduceScatter stay rings */
#define TRIOSIM_ALGO_RSAG 4       /* AllReduce as a ring ReduceScatter followed by a ring AllGather: two collectives
                                     of the group, the AllGather starting once every member finished the
                                     ReduceScatter ("reduce, scatter, and gather"; R29) */
#define TRIOSIM_ALGO_DBTREE 3     /* NCCL-style double binary tree AllReduce: two heap trees over mirrored member
                                     positions, S/2 each, both at once (R27); runs in the hybrid kernel,
                                     whose lanes hold the second tree on a spare flow slot -- TRIOSIM_PT_TOO_LARGE
                                     for HYBRID points with both dp > 1 and tp > 1, and over photonic links */

typedef struct {
    uint32_t topo;
    uint8_t strategy, tp_mode, coll_algo;
    uint8_t ring_chunks;     /* chunks per ring step, pipelined (NCCL-style; R25): each ring step's
                                slice S/p is sent as ring_chunks flows of S/(p*ring_chunks), one at a time per
                                member; 0 or 1 = unchunked (R10); > 16 -> TRIOSIM_PT_BAD_CONFIG; ignored by
                                tree AllReduces */
    uint16_t dp, tp, pp;
    uint16_t hop;            /* TRIOSIM_HOP only (R28): backup workers (bits 0-3) | staleness (4-7) | max iteration
                                gap, 0 = unbounded (8-15); ignored otherwise */
    uint32_t microbatches, global_batch;
    int32_t stage_plan;      /* -1 = automatic balanced partition */
    uint32_t first_bucket_bytes;  /* cap of each gradient group's first bucket (PyTorch DDP's first-bucket
                                     rule, R24); 0 = bucket_bytes; ignored when bucket_bytes == 0 */
    uint64_t bucket_bytes;   /* DP/DDP/HYBRID gradient bucket; 0 = one AllReduce per tensor */
    double bw_scale;         /* multiplies every link bandwidth (> 0) */
    double lat_scale;        /* multiplies every link latency (>= 0) */
} triosim_point;             /* 56 B */

typedef struct {
    double iter_time_s;          /* predicted iteration time T */
    double compute_busy_max_s;   /* max over GPUs of summed operator time */
    double comm_busy_s;          /* time with >= 1 flow in flight */
    double exposed_comm_s;       /* T - compute_busy_max_s */
    double coll_payload_bytes;   /* summed collective payloads ("amount of data ... AllReduce") */
    uint64_t n_compute, n_flows, n_collectives, n_p2p;
    uint64_t n_instants, n_wf_calls, n_wf_rounds, order_hash; /* DESIGN.md R19 */
    int32_t status;              /* TRIOSIM_PT_* */
    uint32_t max_active_flows;
} triosim_result;                /* 112 B */

/* Timeline records (R23; "the timeline of the communication process among GPUs or the
 * computation process on each GPU").  A task is one operator instance on one simulated GPU; a
 * flow is one ring / tree step, P2P send or photonic transfer. */
typedef struct {
    uint32_t gpu;        /* simulated GPU (topology node id) */
    uint32_t prog;       /* position in that GPU's program (micro-batch instances included) */
    uint32_t op;         /* trace operator */
    uint32_t mb;         /* micro-batch (0 outside GPipe / HYBRID) */
    double start_s, end_s;
} triosim_task_rec;      /* 32 B */
typedef struct {
    uint64_t code;       /* the flow's order-hash code (R19): collective (c<<32 | step<<16 | member, tree
                            broadcast edges step = 1), P2P (1<<59 | tensor<<32 | micro-batch<<16 | dst) */
    uint32_t src, dst;   /* GPU node ids */
    double bytes;
    double release_s;    /* dependencies met (R10, R11) */
    double start_s;      /* activation after the route latency (R13) / photonic buffer grant (R20) */
    double delivered_s;
} triosim_flow_rec;      /* 48 B */

#ifdef __cplusplus
static_assert(sizeof(triosim_op) == 40, "op");
static_assert(sizeof(triosim_tensor) == 16, "tensor");
static_assert(sizeof(triosim_link) == 24, "link");
static_assert(sizeof(triosim_point) == 56, "point");
static_assert(sizeof(triosim_photonic) == 32, "photonic");
static_assert(sizeof(triosim_result) == 112, "result");
static_assert(sizeof(triosim_task_rec) == 32, "task rec");
static_assert(sizeof(triosim_flow_rec) == 48, "flow rec");
#endif

typedef struct triosim_ctx triosim_ctx;

/* Create a context on CUDA device `cuda_device` (must be sm_100).  *out owns every device and
 * host copy made later; free with triosim_destroy.  Errors: EUNSUPPORTED, ECUDA, ENOMEM. */
triosim_status triosim_create(int cuda_device, triosim_ctx **out);
void triosim_destroy(triosim_ctx *ctx);

/* Message for the last error on ctx (owned by ctx, valid until the next call). */
const char *triosim_last_error(const triosim_ctx *ctx);

/* Trace ingest (S1).  Validates the tables (EINVAL: ids out of range, a tensor
 * produced twice or read before it is produced, phases not FWD* BWD* OPT*, layers not numbered
 * by first FWD appearance, negative / non-finite time, trace_batch == 0), copies them to the
 * device and runs the ingest kernel.  Synchronous.  *trace_id receives the handle. */
triosim_status triosim_load_trace(triosim_ctx *ctx, const triosim_trace_desc *t, int32_t *trace_id);

/* Build a sweep of n_pts design points over trace_id (P:142 inputs).  Validates topologies
 * (EINVAL: bad endpoints, bw <= 0, lat < 0, duplicate ordered pair, bad ring_order, unknown net_model,
 * photonic parameters missing or out of range), computes
 * routes (S5) and stage partitions on the host, groups points into structural classes and
 * stages everything in device memory.  Invalid design points do NOT fail the call: they get a
 * per-point status.  plans may be NULL.  Synchronous.  *sweep_id receives the handle. */
triosim_status triosim_build_sweep(triosim_ctx *ctx, int32_t trace_id, const triosim_topology *topos,
                                   uint32_t n_topos, const triosim_stage_plans *plans, const triosim_point *pts,
                                   uint64_t n_pts, int32_t *sweep_id);

/* Simulate points [first, first+count) of sweep_id: operator rescale (K1), task-graph
 * expansion (K2) and the timeline kernel (K3) on `cuda_stream` (cudaStream_t; NULL = the
 * legacy default stream).  Asynchronous and stream-ordered; returns after enqueue, for partial
 * ranges too (the kernels skip the points outside the range).
 * Errors: ERANGE, ENOTFOUND, ECUDA. */
triosim_status triosim_simulate_batch(triosim_ctx *ctx, int32_t sweep_id, uint64_t first, uint64_t count,
                                      void *cuda_stream);

/* Copy result records [first, first+count) to out.  out_is_device == 0: host memory; the call first
 * synchronises the stream of the sweep's last simulate_batch (if it is not cuda_stream), then copies on
 * cuda_stream and synchronises it.  out_is_device != 0: a device pointer on the context's GPU; the copy
 * is enqueued on `cuda_stream`, after an event the sweep's last simulate_batch recorded on its own stream
 * (so the copy is ordered after that batch on any stream; asynchronous, no host synchronisation). */
triosim_status triosim_results(triosim_ctx *ctx, int32_t sweep_id, uint64_t first, uint64_t count,
                               triosim_result *out, int out_is_device, void *cuda_stream);

/* Free a trace or sweep handle (a trace must outlive its sweeps).  Its device blocks go to a per-process
 * cache that later load_trace / build_sweep calls reuse (at most TS_BLOCK_CACHE_MB, default 512 MiB, of idle
 * blocks; TS_NO_BLOCK_CACHE=1 disables it; triosim_destroy returns them to the driver). */
triosim_status triosim_release(triosim_ctx *ctx, int32_t handle);

/* Per-layer breakdown ("the communication time and computation time of each layer or stage";
 * Fig. 13; R22).  enable != 0 allocates, for the sweep, per-class layer tables and
 * 3 x n_layers f64 accumulators per point (24 B x n_layers x n_pts of device memory; ENOMEM if that
 * fails) and makes every later triosim_simulate_batch on the sweep also record the breakdown (a
 * separate instantiation of the timeline kernels; the plain path is unchanged).  enable == 0 frees
 * them.  Synchronises the device.  Errors: ENOTFOUND, ENOMEM, ECUDA. */
triosim_status triosim_set_breakdown(triosim_ctx *ctx, int32_t sweep_id, int enable);

/* Per-layer times of points [first, first+count) as two row-major [count][n_layers] f64 arrays
 * (layer ids as in the trace, R1), of the layer's representative rank -- the lowest rank that runs
 * it: rank 0 for DP / DDP / TP, the stage's GPU for PP, rank (d = 0, its stage, t = 0) for HYBRID:
 *   layer_compute_s[l] = left fold, in that rank's program order, of t' over its operator instances
 *                        of layer l (R4);
 *   layer_comm_s[l]    = (TP-group + DP-group collective time) + P2P time, where a collective counts
 *                        (done on the rank - start) and is attributed to the layer of the operator
 *                        that triggers it (R6, R7, R9), and a P2P send of the rank counts
 *                        (delivery - release) attributed to the producing operator's layer (R11);
 *                        each term a left fold in creation order.
 * Points whose status is not OK get zeros.  Values are those of the most recent simulate_batch that
 * covered the point after the breakdown was enabled.  Either output may be NULL.  out_is_device == 0:
 * host memory, the call runs the finalising kernel on `cuda_stream` and synchronises it;
 * out_is_device != 0: device pointers on the context's GPU, stream-ordered and asynchronous.
 * Errors: EINVAL (breakdown not enabled), ENOTFOUND, ERANGE, ENOMEM, ECUDA. */
triosim_status triosim_breakdown(triosim_ctx *ctx, int32_t sweep_id, uint64_t first, uint64_t count,
                                 double *layer_compute_s, double *layer_comm_s, int out_is_device,
                                 void *cuda_stream);

/* Timeline of one design point (R23): runs the path for point `point` of sweep_id alone with a
 * recording instantiation of the timeline kernel (same results, bit for bit; the point's result record
 * is rewritten with them), then sorts the records on the device: tasks by (gpu, prog), flows by
 * (release_s, code).  *n_tasks / *n_flows receive the totals (= the result's n_compute / n_flows); at
 * most task_cap / flow_cap records are written to the caller-owned host arrays, and only when the
 * totals fit are they the complete sorted timeline (call again with larger arrays otherwise).  A point
 * whose status is not OK has no records.  Synchronous.  Errors: EINVAL, ENOTFOUND, ERANGE, ENOMEM, ECUDA. */
triosim_status triosim_timeline(triosim_ctx *ctx, int32_t sweep_id, uint64_t point, triosim_task_rec *tasks,
                                uint64_t task_cap, triosim_flow_rec *flows, uint64_t flow_cap, uint64_t *n_tasks,
                                uint64_t *n_flows);

/* Automatic GPipe stage plan (R8; P:188 user-specified stages, "automatically assigns layers to
 * GPUs to balance workloads"), the one build_sweep uses for stage_plan = -1: the contiguous split of the
 * trace's layers (n_layers = 1 + the largest FWD layer id) into n_stages stages minimising the largest
 * stage cost -- the left fold in layer order of the per-layer sums of time_s -- ties broken towards the
 * lexicographically smallest first_layer vector.  Host-only (no context, no device); writes n_stages
 * first layers (first_layer[0] = 0).  Errors: EINVAL (NULL pointers, no ops, n_stages == 0 or
 * > n_layers, an op layer >= n_layers, a negative / non-finite time). */
triosim_status triosim_stage_partition(const triosim_trace_desc *t, uint32_t n_stages, uint32_t *first_layer);

/* Kernel launch counters since the context was created (K1, K2, K3 launches), for the bench. */
triosim_status triosim_launch_counts(const triosim_ctx *ctx, uint64_t *k1, uint64_t *k2, uint64_t *k3);

/* fp64 operations of the method (folds, latencies, progress, shares,
 * residual updates, drain times) performed by the last simulate_batch of sweep_id.  Synchronises
 * that call's stream. */
triosim_status triosim_work_counters(triosim_ctx *ctx, int32_t sweep_id, uint64_t *fp64_ops);

/* CUDA-event timing of simulate_batch calls (events recorded on the call's stream): enable
 * resets the log; triosim_timings returns how many calls were logged (<= 512, <= max) and their
 * durations in ms: whole call (K1b+K2+K3) and the K3 timeline phase (fork to join). */
triosim_status triosim_timing(triosim_ctx *ctx, int enable);
int32_t triosim_timings(triosim_ctx *ctx, float *ms_total, float *ms_k3, int32_t max);

/* Device pointer of the sweep's result records (for stream-ordered gathers), or NULL. */
const void *triosim_results_device_ptr(const triosim_ctx *ctx, int32_t sweep_id);

#ifdef __cplusplus
}
#endif
#endif /* TRIOSIM_H */
