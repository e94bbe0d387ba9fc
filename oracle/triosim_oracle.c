/*
 * triosim_oracle.c -- TEST INFRASTRUCTURE ONLY.
 *
 * A plain, slow, single-threaded CPU discrete-event simulator of TrioSim's
 * per-design-point method (Li et al., "TrioSim", ISCA'25; PAPER.md = P:N line
 * refs).  Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
 * --impl reference leg may load this library.  It shares NO code, header,
 * table or helper with the CUDA product path (paper_conf_isca_libwmvgjbj025_b200/):
 * it restates the binary record layouts itself and re-derives everything
 * (routes, partitions, buckets, task graph) from the paper and the readings in
 * DESIGN.md ("Semantics" R1-R19; readings Q1-Q31).
 *
 * Structure, in the paper's order (Sec. 4.3-4.5):
 *   1. trace checks + producer table
 *   2. operator-time model t' = t * rho                   (R4)
 *   3. trace extrapolation into an explicit task graph    (R6-R11)
 *        nodes: compute TASKs (per-GPU in-order queues),
 *               FLOWs (data movement / collective steps),
 *               BARRIERs (zero-time joins: collective start, "done on GPU g")
 *   4. routing: BFS shortest path, lexicographic tie break (R12)
 *   5. event-driven timeline (R13-R17) with the
 *      flow-based network model: route -> bandwidth allocation (max-min
 *      progressive filling) -> progress update -> delivery, re-allocating every
 *      in-transit flow whenever one starts or completes (Fig. 5).
 *   6. outputs (R18-R19).
 *
 * Arithmetic: IEEE binary64, compiled with -O2 -ffp-contract=off (no FMA
 * contraction), no fast-math; every sum is a left fold in the stated order.
 *
 * Parity pins (tests/test_oracle_*.py): closed forms CF1-CF14 (DESIGN.md
 * "Pins"), brute-force routing and partitioning, max-min invariants of the
 * progressive filling, and an exact-rational Python re-simulation of exported
 * task graphs.  Extensions R20-R26 (photonic network, per-layer breakdown,
 * timeline, DDP first bucket, pipelined ring, reduce + broadcast AllReduce, double
 * binary tree) and R28 (Hop decentralized training) carry their own pins
 * (tests/test_oracle_{photonic,breakdown,timeline,closed_forms,chunked_ring,
 * reduce_broadcast,double_tree,hop,hash}.py).
 * Unpinned: absolute accuracy vs real hardware (P:244-300,
 * needs the paper's traces and machines) -- "parity unpinned" for that only.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <math.h>
#include <stdio.h>

/* ------------------------------------------------------------------ */
/* Record layouts (the binary formats of DESIGN.md "Inputs"),          */
/* restated here independently of include/triosim.h.                   */
/* ------------------------------------------------------------------ */
typedef struct {
    uint32_t kind, layer;
    uint8_t phase, tp_role;
    uint16_t flags;
    uint32_t io_off;
    uint16_t n_in, n_out;
    uint32_t pad;
    double time_s, flops;
} OOp; /* 40 B */

typedef struct {
    uint64_t bytes_b0;
    uint8_t category, batch_scaled;
    uint16_t pad;
    uint32_t param_id;
} OTensor; /* 16 B */

typedef struct {
    uint32_t src, dst;
    double bw, lat;
} OLink; /* 24 B */

typedef struct {
    uint32_t topo;
    uint8_t strategy, tp_mode, coll_algo;
    uint8_t ring_chunks;           /* R25: chunks per ring step (0 or 1 = unchunked, R10) */
    uint16_t dp, tp, pp, pad1;
    uint32_t microbatches, global_batch;
    int32_t stage_plan;
    uint32_t first_bucket_bytes;   /* R24: cap of a group's first gradient bucket, 0 = bucket_bytes */
    uint64_t bucket_bytes;
    double bw_scale, lat_scale;
} OPoint; /* 56 B */

/* R24 (PyTorch DDP's first-bucket rule): the cap of bucket number k of a gradient group -- the first
 * bucket closes at first_bucket_bytes when that is set, every later one at bucket_bytes; bucket_bytes
 * == 0 keeps one tensor per AllReduce (the paper-literal reading of Q5) */
static uint64_t bucket_cap(const OPoint *pt, int k) {
    if (pt->bucket_bytes == 0) return 0;
    return (k == 0 && pt->first_bucket_bytes != 0) ? (uint64_t)pt->first_bucket_bytes : pt->bucket_bytes;
}

typedef struct {
    double iter_time_s, compute_busy_max_s, comm_busy_s, exposed_comm_s, coll_payload_bytes;
    uint64_t n_compute, n_flows, n_collectives, n_p2p, n_instants, n_wf_calls, n_wf_rounds, order_hash;
    int32_t status;
    uint32_t max_active_flows;
} OResult; /* 112 B */

/* Photonic circuit-switched interconnect parameters (R20) */
typedef struct {
    uint32_t ports;      /* photonic ports per GPU (logical links it can hold) */
    uint32_t buf_slots;  /* receive buffers per destination GPU (0 = unlimited) */
    double link_bw;      /* bandwidth of one logical link, B/s */
    double setup_s;      /* latency of establishing a logical link */
    double lat_s;        /* per-transfer latency */
} OPhot; /* 32 B */

_Static_assert(sizeof(OPhot) == 32, "photonic record");
_Static_assert(sizeof(OOp) == 40, "op record");
_Static_assert(sizeof(OTensor) == 16, "tensor record");
_Static_assert(sizeof(OLink) == 24, "link record");
_Static_assert(sizeof(OPoint) == 56, "point record");
_Static_assert(sizeof(OResult) == 112, "result record");

enum { PH_FWD = 0, PH_BWD = 1, PH_OPT = 2 };
enum { CAT_INPUT = 0, CAT_WEIGHT = 1, CAT_WGRAD = 2, CAT_ACT = 3, CAT_AGRAD = 4, CAT_OTHER = 5 };
enum { ST_DP = 0, ST_DDP = 1, ST_TP = 2, ST_PP = 3, ST_HYBRID = 4, ST_HOP = 5 };
enum { HOP_RING_BASED = 0, HOP_DOUBLE_RING = 1 };   /* R28 communication graphs (Fig. 16a) */
enum { TPM_PAPER = 0, TPM_MEGATRON = 1 };
enum { ALG_RING = 0, ALG_TREE = 1, ALG_REDBCAST = 2, ALG_DBTREE = 3, ALG_RSAG = 4 };
enum { ROLE_NONE = 0, ROLE_COL = 1, ROLE_ROW = 2, ROLE_LOCAL = 3, ROLE_GATHER = 4 };
enum { CK_AR = 0, CK_AG = 1, CK_RS = 2 };
#define OPF_BATCH_SCALED 1u

#define O_OK 0
#define O_EINVAL (-1)
#define O_ENOMEM (-2)

enum { PT_OK = 0, PT_BAD_BATCH = 1, PT_BAD_DEGREES = 2, PT_NO_ROUTE = 3, PT_TOO_LARGE = 4,
       PT_DEADLOCK = 5, PT_BAD_PLAN = 6, PT_BAD_CONFIG = 7 };

/* event kinds of the order hash (R19) */
enum { EV_COLL_START = 1, EV_RELEASE = 2, EV_ACTIVATE = 3, EV_DELIVER = 4, EV_TASK_START = 5, EV_TASK_END = 6 };

/* ------------------------------------------------------------------ */
/* small growable arrays                                               */
/* ------------------------------------------------------------------ */
typedef struct { int *v; long n, cap; } IVec;
static int iv_push(IVec *a, int x) {
    if (a->n == a->cap) {
        long nc = a->cap ? a->cap * 2 : 64;
        int *p = (int *)realloc(a->v, (size_t)nc * sizeof(int));
        if (!p) return -1;
        a->v = p; a->cap = nc;
    }
    a->v[a->n++] = x;
    return 0;
}
static void iv_free(IVec *a) { free(a->v); a->v = NULL; a->n = a->cap = 0; }

/* ------------------------------------------------------------------ */
/* Trace checks: SSA tensors, producers precede readers,*/
/* phases FWD* BWD* OPT*, layers numbered by first FWD appearance.     */
/* ------------------------------------------------------------------ */
typedef struct {
    const OOp *ops; uint32_t n_ops;
    const OTensor *ts; uint32_t n_ts;
    const uint32_t *io; uint32_t n_io;
    uint32_t b0;
    int *prod;        /* producing op of each tensor, -1 = none (resident input/weight) */
    uint32_t n_layers;
} Trace;

static int trace_check(Trace *T) {
    if (T->n_ops == 0 || T->b0 == 0) return O_EINVAL;
    T->prod = (int *)malloc(sizeof(int) * (T->n_ts ? T->n_ts : 1));
    if (!T->prod) return O_ENOMEM;
    for (uint32_t x = 0; x < T->n_ts; x++) {
        T->prod[x] = -1;
        if (T->ts[x].category > CAT_OTHER) return O_EINVAL;
    }
    int last_phase = 0;
    uint32_t next_layer = 0;
    for (uint32_t o = 0; o < T->n_ops; o++) {
        const OOp *op = &T->ops[o];
        if (op->phase > PH_OPT || op->phase < last_phase) return O_EINVAL;
        last_phase = op->phase;
        if (!(op->time_s >= 0.0) || isinf(op->time_s)) return O_EINVAL;
        if ((uint64_t)op->io_off + op->n_in + op->n_out > T->n_io) return O_EINVAL;
        if (op->tp_role > 7) return O_EINVAL;
        if (op->phase == PH_FWD) {
            if (op->layer == next_layer) next_layer++;
            else if (op->layer > next_layer) return O_EINVAL;
        } else if (op->layer >= next_layer) {
            return O_EINVAL;
        }
        for (uint32_t k = 0; k < op->n_in; k++) {
            uint32_t x = T->io[op->io_off + k];
            if (x >= T->n_ts) return O_EINVAL;
            if (T->prod[x] == (int)o) return O_EINVAL; /* read-own-output */
        }
        for (uint32_t k = 0; k < op->n_out; k++) {
            uint32_t x = T->io[op->io_off + op->n_in + k];
            if (x >= T->n_ts) return O_EINVAL;
            if (T->prod[x] != -1) return O_EINVAL; /* each tensor produced once */
            T->prod[x] = (int)o;
        }
    }
    /* a reader must come after the producer (checked after all producers are known) */
    for (uint32_t o = 0; o < T->n_ops; o++) {
        const OOp *op = &T->ops[o];
        for (uint32_t k = 0; k < op->n_in; k++) {
            uint32_t x = T->io[op->io_off + k];
            if (T->prod[x] >= (int)o) return O_EINVAL;
        }
    }
    T->n_layers = next_layer;
    if (T->n_layers == 0) return O_EINVAL;
    return O_OK;
}

/* ------------------------------------------------------------------ */
/* Operator-time model (R4; P:178 batch change, P:200 trace time when   */
/* nothing changes, P:202 FLOPs-ratio rescale).                        */
/* ------------------------------------------------------------------ */
static int op_split(const OOp *op, int tp_mode) {
    if (tp_mode == TPM_PAPER) return (op->tp_role & ROLE_GATHER) != 0;   /* conv/linear/embedding */
    return (op->tp_role & 3) != 0;                                      /* Megatron COL/ROW/LOCAL */
}

static double op_time(const Trace *T, uint32_t o, double r_b, int tp, int tp_mode) {
    const OOp *op = &T->ops[o];
    double rho = 1.0;
    if (op->flags & OPF_BATCH_SCALED) rho = r_b;
    if (tp > 1 && op_split(op, tp_mode)) rho = rho / (double)tp;
    if (rho == 1.0) return op->time_s;      /* the trace time itself */
    return op->time_s * rho;                /* FLOPs-ratio rescale */
}

/* R5: bytes of a tensor instance under the point's batch and TP split */
static double tensor_bytes(const Trace *T, uint32_t x, double r_b, int tp, int tp_mode) {
    const OTensor *t = &T->ts[x];
    double b = (double)t->bytes_b0;
    if (t->batch_scaled) b = b * r_b;
    if (tp > 1 && t->category == CAT_WGRAD && T->prod[x] >= 0 && op_split(&T->ops[T->prod[x]], tp_mode))
        b = b / (double)tp;
    return b;
}

/* ------------------------------------------------------------------ */
/* Task graph                                                          */
/* ------------------------------------------------------------------ */
enum { N_TASK = 0, N_FLOW = 1, N_BARRIER = 2 };
#define NF_COLL_START 1 /* barrier that is a collective start (hashed) */
#define NF_P2P 2        /* flow is a point-to-point data movement */
#define NF_NEED_SHIFT 8 /* barrier: (flags >> 8) - 1 = dependencies it needs (0 = all of them; R28 threshold) */

typedef struct {
    int type;
    int gpu;          /* task: simulated GPU node */
    double dur;       /* task: t' */
    int src, dst;     /* flow endpoints (GPU nodes) */
    double bytes;     /* flow size */
    uint64_t code;    /* canonical id for the order hash */
    int flags;
    int layer;        /* task: its operator's layer (R22 breakdown); -1 otherwise */
    int op, mb;       /* task: trace operator and micro-batch (R23 timeline) */
} GNode;

typedef struct {
    GNode *n; long count, cap;
    IVec dep_from, dep_to;   /* edge list: node dep_from[i] waits for node dep_to[i] */
    int n_coll;
    int nch;                 /* R25: chunks per ring step of this point's ring collectives (>= 1) */
    double coll_payload;     /* left fold of collective payloads in creation order */
    /* R22 per-layer breakdown: the representative rank of each layer, and the communications it
     * takes part in, attributed to the layer of the operator that triggers / produces them */
    int want_bd, n_layers;
    int *rep;                /* per layer: GPU of the representative rank */
    int cur_layer, cur_cat;  /* attribution of the next collective: layer, 0 = TP / 1 = DP group */
    IVec rc_s, rc_e, rc_l, rc_c;   /* records: start node, end node, layer, category (2 = P2P) */
} Graph;

static int g_add(Graph *G, GNode nd) {
    if (G->count == G->cap) {
        long nc = G->cap ? G->cap * 2 : 256;
        GNode *p = (GNode *)realloc(G->n, (size_t)nc * sizeof(GNode));
        if (!p) return -1;
        G->n = p; G->cap = nc;
    }
    G->n[G->count] = nd;
    return (int)G->count++;
}
static int g_dep(Graph *G, int node, int on) {
    if (iv_push(&G->dep_from, node) || iv_push(&G->dep_to, on)) return -1;
    return 0;
}
static void g_free(Graph *G) {
    free(G->n); G->n = NULL; G->count = G->cap = 0;
    iv_free(&G->dep_from); iv_free(&G->dep_to);
    free(G->rep); G->rep = NULL;
    iv_free(&G->rc_s); iv_free(&G->rc_e); iv_free(&G->rc_l); iv_free(&G->rc_c);
}
static void g_record(Graph *G, int start, int end, int layer, int cat) {
    iv_push(&G->rc_s, start); iv_push(&G->rc_e, end); iv_push(&G->rc_l, layer); iv_push(&G->rc_c, cat);
}
static int add_task(Graph *G, int gpu, long prog, double dur, int layer, int op, int mb) {
    GNode n; memset(&n, 0, sizeof n);
    n.type = N_TASK; n.gpu = gpu; n.dur = dur; n.layer = layer; n.op = op; n.mb = mb;
    n.code = ((uint64_t)(uint32_t)gpu << 40) | (uint64_t)prog;
    return g_add(G, n);
}
static int add_barrier(Graph *G, int flags, uint64_t code) {
    GNode n; memset(&n, 0, sizeof n);
    n.type = N_BARRIER; n.flags = flags; n.code = code; n.layer = -1;
    return g_add(G, n);
}
static int add_flow(Graph *G, int src, int dst, double bytes, uint64_t code, int flags) {
    GNode n; memset(&n, 0, sizeof n);
    n.type = N_FLOW; n.src = src; n.dst = dst; n.bytes = bytes; n.code = code; n.flags = flags; n.layer = -1;
    return g_add(G, n);
}
static uint64_t coll_flow_code(uint64_t c, int step, int member) {
    return (c << 32) | ((uint64_t)(uint32_t)step << 16) | (uint64_t)(uint32_t)member;
}
static uint64_t p2p_flow_code(uint32_t x, int j, int dst) {
    return (1ull << 59) | ((uint64_t)x << 32) | ((uint64_t)(uint32_t)j << 16) | (uint64_t)(uint32_t)dst;
}

/*
 * One binary-heap tree AllReduce over the members (R10 tree, reading Q25): heap position h holds
 * member h (mirror = 0) or member p-1-h (mirror = 1, R27's second tree).  The child at position h
 * reduces to its parent carrying Sx once all of its own children's reduces arrived (leaves at the
 * collective start sb); the parent broadcasts back once it holds the result (the root once both of
 * its children's reduces arrived).  Flow code step = 2*mirror + {0 up, 1 down}, member = the
 * child's member index.  Appends the flows to fl.
 */
static int heap_tree(Graph *G, uint64_t c, const int *members, int p, int mirror, double Sx, int sb, IVec *fl) {
    int *up = (int *)malloc(sizeof(int) * (size_t)(p > 0 ? p : 1)), *dn = (int *)malloc(sizeof(int) * (size_t)(p > 0 ? p : 1));
    if (!up || !dn) { free(up); free(dn); return -1; }
    for (int h = 0; h < p; h++) up[h] = dn[h] = -1;
#define MEM_AT(h) (mirror ? p - 1 - (h) : (h))
    for (int h = p - 1; h >= 1; h--) {
        up[h] = add_flow(G, members[MEM_AT(h)], members[MEM_AT((h - 1) / 2)], Sx, coll_flow_code(c, 2 * mirror, MEM_AT(h)), 0);
        if (up[h] < 0) { free(up); free(dn); return -1; }
        iv_push(fl, up[h]);
    }
    for (int h = 1; h < p; h++) {
        dn[h] = add_flow(G, members[MEM_AT((h - 1) / 2)], members[MEM_AT(h)], Sx, coll_flow_code(c, 2 * mirror + 1, MEM_AT(h)), 0);
        if (dn[h] < 0) { free(up); free(dn); return -1; }
        iv_push(fl, dn[h]);
    }
#undef MEM_AT
    for (int h = 1; h < p; h++) {
        int nchild = 0;
        for (int ch = 2 * h + 1; ch <= 2 * h + 2 && ch < p; ch++) { g_dep(G, up[h], up[ch]); nchild++; }
        if (nchild == 0) g_dep(G, up[h], sb);
        int par = (h - 1) / 2;
        if (par == 0) {
            for (int ch = 1; ch <= 2 && ch < p; ch++) g_dep(G, dn[h], up[ch]);
        } else {
            g_dep(G, dn[h], dn[par]);
        }
    }
    free(up); free(dn);
    return 0;
}

/*
 * One collective (R10; P:87-89 ring AllReduce, P:174 reduce/scatter/gather,
 * P:192 ring tasks handed to the network model).  members[] are GPU nodes in
 * ring order.  trig[i] = task whose completion makes member i's input ready;
 * prev_done[i] = "previous collective of this group done on member i" (FIFO
 * per (GPU, group), reading Q24) or NULL.  Writes done[i] = barrier "this
 * collective is done on member i" (last flow touching it delivered).
 */
static int build_collective_code(Graph *G, uint64_t c, const int *members, int p, int kind, int algo, int nch,
                                 double S, const int *trig, const int *prev_done, int *done) {
    G->n_coll++;
    G->coll_payload = G->coll_payload + S;
    int sb = add_barrier(G, NF_COLL_START, (uint64_t)c);
    if (sb < 0) return -1;
    for (int i = 0; i < p; i++) {
        if (g_dep(G, sb, trig[i])) return -1;
        if (prev_done && g_dep(G, sb, prev_done[i])) return -1;
    }
    IVec fl = {0}; /* all flows of this collective */
    if (algo == ALG_REDBCAST && kind == CK_AR) {
        /* R26 AllReduce as NCCL-style ring Reduce to member 0 followed by ring Broadcast from member 0
         * ("reduce, scatter, and gather"), each a chain along the ring pipelined in nch chunks of
         * S/nch.  Member i sends its flows one at a time (R25's single send engine) to m_(i+1): first
         * its reduce chunks (i != 0), then its broadcast chunks (i != p-1); q = own send index.
         *   reduce chunk j of i: after its own previous send; for i >= 2 after reduce chunk j of i-1
         *     arrived (i = 1 starts the chain at the collective start);
         *   broadcast chunk j of 0: after reduce chunk j of p-1 arrived (the reduced chunk is at 0);
         *   broadcast chunk j of i >= 1: after its own previous send and broadcast chunk j of i-1. */
        int **id = (int **)malloc(sizeof(int *) * (size_t)(p > 0 ? p : 1));
        if (!id) return -1;
        for (int i = 0; i < p; i++) {
            id[i] = (int *)malloc(sizeof(int) * (size_t)(2 * nch));
            if (!id[i]) return -1;
        }
        /* creation order: reduce chain (members 1..p-1, chunk-major), then broadcast chain (0..p-2) */
        for (int j = 0; j < nch && p > 1; j++)
            for (int i = 1; i < p; i++) {
                int f = add_flow(G, members[i], members[(i + 1) % p], S / (double)nch, coll_flow_code(c, j, i), 0);
                if (f < 0) return -1;
                id[i][j] = f;
                iv_push(&fl, f);
                if (j == 0 && i == 1) g_dep(G, f, sb);
                if (j > 0) g_dep(G, f, id[i][j - 1]);
                if (i >= 2) g_dep(G, f, id[i - 1][j]);
            }
        for (int j = 0; j < nch && p > 1; j++)
            for (int i = 0; i < p - 1; i++) {
                int q = (i != 0 ? nch : 0) + j;
                int f = add_flow(G, members[i], members[i + 1], S / (double)nch, coll_flow_code(c, q, i), 0);
                if (f < 0) return -1;
                id[i][q] = f;
                iv_push(&fl, f);
                if (q > 0) g_dep(G, f, id[i][q - 1]);
                if (i == 0) g_dep(G, f, id[p - 1][j]);
                else g_dep(G, f, id[i - 1][(i - 1 != 0 ? nch : 0) + j]);
            }
        for (int i = 0; i < p; i++) free(id[i]);
        free(id);
    } else if ((algo != ALG_TREE && algo != ALG_DBTREE) || kind != CK_AR) {
        /* ring: K steps; flow (i,k) goes m_i -> m_(i+1); released at start if k == 0,
         * else when (i-1,k-1) [predecessor's chunk arrived] and (i,k-1) [own previous
         * send] are both delivered (reading Q21).
         * R25 pipelined ring (NCCL chunking): each step's slice S/p is cut into
         * nch chunks of S/(p*nch); member i sends its flows one at a time in the order
         * q = k*nch + j; flow (i,q) is released when (i,q-1) [own previous chunk] and,
         * for k >= 1, (i-1,q-nch) [chunk j of the predecessor's step k-1] are delivered.
         * nch == 1 is the rule above. */
        int K = ((kind == CK_AR) ? 2 * (p - 1) : (p - 1)) * nch;
        double chunk = S / (double)p / (double)nch;
        int *id = (int *)malloc(sizeof(int) * (size_t)(p * (K > 0 ? K : 1)));
        if (!id) return -1;
        for (int k = 0; k < K; k++)
            for (int i = 0; i < p; i++) {
                int f = add_flow(G, members[i], members[(i + 1) % p], chunk, coll_flow_code(c, k, i), 0);
                if (f < 0) { free(id); return -1; }
                id[k * p + i] = f;
                iv_push(&fl, f);
                if (k == 0) {
                    g_dep(G, f, sb);
                } else {
                    if (k >= nch) g_dep(G, f, id[(k - nch) * p + (i - 1 + p) % p]);
                    g_dep(G, f, id[(k - 1) * p + i]);
                }
            }
        free(id);
    } else if (algo == ALG_DBTREE) {
        /* R27 double binary tree AllReduce (NCCL's trees, P:174 / P:398; reading in DESIGN.md R27): the
         * payload is split in two halves S/2; half A runs the R10 tree over heap position = member
         * index, half B the same tree over the mirrored positions (member i at position p-1-i), so
         * for even p every interior node of one tree is a leaf of the other.  Both trees run at
         * once; flow steps 0/1 (A up/down) and 2/3 (B up/down), member field = the child. */
        if (heap_tree(G, c, members, p, 0, S / 2.0, sb, &fl) || heap_tree(G, c, members, p, 1, S / 2.0, sb, &fl)) {
            iv_free(&fl);
            return -1;
        }
    } else {
        /* tree AllReduce (extension, reading Q25): binary heap over member index,
         * reduce i -> parent(i) carrying S once all children's reduces arrived;
         * broadcast parent(i) -> i once parent(i) holds the result. */
        if (heap_tree(G, c, members, p, 0, S, sb, &fl)) { iv_free(&fl); return -1; }
    }
    for (int i = 0; i < p; i++) {
        done[i] = add_barrier(G, 0, 0);
        if (done[i] < 0) { iv_free(&fl); return -1; }
        /* done on member i: every flow with src or dst = m_i delivered (R10) */
        int any = 0;
        for (long q = 0; q < fl.n; q++) {
            const GNode *f = &G->n[fl.v[q]];
            if (f->src == members[i] || f->dst == members[i]) { g_dep(G, done[i], fl.v[q]); any = 1; }
        }
        if (!any) g_dep(G, done[i], sb);
    }
    iv_free(&fl);
    /* R22: the layer's representative rank times this collective from its start to "done" on it */
    if (G->want_bd && G->cur_layer >= 0)
        for (int i = 0; i < p; i++)
            if (members[i] == G->rep[G->cur_layer]) { g_record(G, sb, done[i], G->cur_layer, G->cur_cat); break; }
    return 0;
}

/* R29 (NEXT 3; "NCCL-style collective communication, including reduce, scatter, and gather"):
 * coll_algo = RSAG runs every AllReduce as two collectives of its group -- a ring ReduceScatter, then a
 * ring AllGather of the same payload S, codes c and c + 1 -- so the AllGather starts (R10 barrier) once
 * every member has finished the ReduceScatter.  *used = collectives created (1 or 2). */
static int build_allreduce(Graph *G, uint64_t c, const int *members, int p, int kind, int algo, double S,
                           const int *trig, const int *prev_done, int *done, uint64_t *used) {
    if (algo == ALG_RSAG && kind == CK_AR) {
        int *mid = (int *)malloc(sizeof(int) * (size_t)(p > 0 ? p : 1));
        if (!mid) return -1;
        int rc = build_collective_code(G, c, members, p, CK_RS, ALG_RING, G->nch, S, trig, prev_done, mid);
        if (!rc) rc = build_collective_code(G, c + 1, members, p, CK_AG, ALG_RING, G->nch, S, trig, mid, done);
        free(mid);
        *used = 2;
        return rc;
    }
    *used = 1;
    return build_collective_code(G, c, members, p, kind, algo == ALG_RSAG ? ALG_RING : algo, G->nch, S, trig,
                                 prev_done, done);
}

/* collectives of DP / DDP / TP: one group, numbered in creation order */
static int build_collective(Graph *G, const int *members, int p, int kind, int algo, double S,
                            const int *trig, const int *prev_done, int *done) {
    uint64_t used;
    return build_allreduce(G, (uint64_t)G->n_coll, members, p, kind, algo, S, trig, prev_done, done, &used);
}

/* ------------------------------------------------------------------ */
/* Routing (R12; "we use the shortest path algorithm"):           */
/* BFS by hop count, neighbours expanded in ascending node id, first    */
/* discovery fixes the parent -> lexicographically smallest node path.  */
/* ------------------------------------------------------------------ */
typedef struct {
    uint32_t n_nodes, n_gpus, n_links;
    const OLink *links;
    int *adj_off, *adj_link;   /* per node, out-links sorted by dst */
    const OPhot *ph;           /* non-NULL: photonic circuit-switched network (R20) instead of R12-R15 */
} Topo;

static const OLink *g_sort_links;
static int cmp_by_dst(const void *a, const void *b) {
    int la = *(const int *)a, lb = *(const int *)b;
    uint32_t da = g_sort_links[la].dst, db = g_sort_links[lb].dst;
    return (da > db) - (da < db);
}

static int topo_init(Topo *tp, uint32_t n_nodes, uint32_t n_gpus, const OLink *links, uint32_t n_links,
                     const OPhot *ph) {
    tp->n_nodes = n_nodes; tp->n_gpus = n_gpus; tp->n_links = n_links; tp->links = links; tp->ph = ph;
    if (n_gpus == 0 || n_gpus > n_nodes) return O_EINVAL;
    if (ph && (ph->ports == 0 || !(ph->link_bw > 0.0) || isinf(ph->link_bw) || !(ph->setup_s >= 0.0) ||
               isinf(ph->setup_s) || !(ph->lat_s >= 0.0) || isinf(ph->lat_s)))
        return O_EINVAL;
    tp->adj_off = (int *)calloc(n_nodes + 1, sizeof(int));
    tp->adj_link = (int *)malloc(sizeof(int) * (n_links ? n_links : 1));
    if (!tp->adj_off || !tp->adj_link) return O_ENOMEM;
    for (uint32_t e = 0; e < n_links; e++) {
        const OLink *l = &links[e];
        if (l->src >= n_nodes || l->dst >= n_nodes || l->src == l->dst) return O_EINVAL;
        if (!(l->bw > 0.0) || isinf(l->bw) || !(l->lat >= 0.0) || isinf(l->lat)) return O_EINVAL;
        for (uint32_t f = 0; f < e; f++)
            if (links[f].src == l->src && links[f].dst == l->dst) return O_EINVAL; /* one link per ordered pair */
        tp->adj_off[l->src + 1]++;
    }
    for (uint32_t v = 0; v < n_nodes; v++) tp->adj_off[v + 1] += tp->adj_off[v];
    int *fill = (int *)calloc(n_nodes, sizeof(int));
    if (!fill) return O_ENOMEM;
    for (uint32_t e = 0; e < n_links; e++) {
        uint32_t s = links[e].src;
        tp->adj_link[tp->adj_off[s] + fill[s]++] = (int)e;
    }
    free(fill);
    g_sort_links = links;
    for (uint32_t v = 0; v < n_nodes; v++)
        qsort(tp->adj_link + tp->adj_off[v], (size_t)(tp->adj_off[v + 1] - tp->adj_off[v]), sizeof(int), cmp_by_dst);
    return O_OK;
}
static void topo_free(Topo *tp) { free(tp->adj_off); free(tp->adj_link); tp->adj_off = tp->adj_link = NULL; }

/* returns hop count (>=0) and writes link ids src->dst into out[]; -1 = no route */
static int bfs_route(const Topo *tp, int src, int dst, int *out, int out_cap) {
    if (src == dst) return 0;
    int n = (int)tp->n_nodes;
    int *par_link = (int *)malloc(sizeof(int) * (size_t)n), *queue = (int *)malloc(sizeof(int) * (size_t)n);
    char *seen = (char *)calloc((size_t)n, 1);
    if (!par_link || !queue || !seen) { free(par_link); free(queue); free(seen); return -2; }
    int qh = 0, qt = 0;
    queue[qt++] = src; seen[src] = 1; par_link[src] = -1;
    while (qh < qt && !seen[dst]) {
        int u = queue[qh++];
        for (int a = tp->adj_off[u]; a < tp->adj_off[u + 1]; a++) {
            int e = tp->adj_link[a];
            int v = (int)tp->links[e].dst;
            if (!seen[v]) { seen[v] = 1; par_link[v] = e; queue[qt++] = v; }
        }
    }
    int hops = -1;
    if (seen[dst]) {
        int len = 0;
        for (int v = dst; v != src; v = (int)tp->links[par_link[v]].src) len++;
        if (len <= out_cap) {
            int v = dst;
            for (int k = len - 1; k >= 0; k--) { out[k] = par_link[v]; v = (int)tp->links[par_link[v]].src; }
            hops = len;
        } else {
            hops = -3;
        }
    }
    free(par_link); free(queue); free(seen);
    return hops;
}

/* ------------------------------------------------------------------ */
/* PP stage partition (R8; P:188 user-specified, "automatically   */
/* assigns layers to GPUs to balance workloads"): contiguous layers,    */
/* minimise the max stage cost (left fold of trace times t), ties to    */
/* the lexicographically smallest boundary vector.                      */
/* ------------------------------------------------------------------ */
static int auto_partition(const Trace *T, int S, uint32_t *first_layer) {
    int L = (int)T->n_layers;
    if (S < 1 || S > L) return -1;
    double *lc = (double *)calloc((size_t)L, sizeof(double));
    double *cost = (double *)malloc(sizeof(double) * (size_t)L * (size_t)L); /* cost[a*L+b] = layers a..b */
    double *best = (double *)malloc(sizeof(double) * (size_t)(S + 1) * (size_t)(L + 1));
    if (!lc || !cost || !best) { free(lc); free(cost); free(best); return -2; }
    for (uint32_t o = 0; o < T->n_ops; o++) lc[T->ops[o].layer] = lc[T->ops[o].layer] + T->ops[o].time_s;
    for (int a = 0; a < L; a++) {
        double s = 0.0;
        for (int b = a; b < L; b++) { s = s + lc[b]; cost[a * L + b] = s; }
    }
    /* best[s][i]: min over partitions of layers i..L-1 into s stages of the max stage cost */
#define BEST(s, i) best[(size_t)(s) * (size_t)(L + 1) + (size_t)(i)]
    for (int i = 0; i < L; i++) BEST(1, i) = cost[i * L + L - 1];
    for (int s = 2; s <= S; s++)
        for (int i = 0; i + s <= L; i++) {
            double b = INFINITY;
            for (int j = i + 1; L - j >= s - 1; j++) {
                double a = cost[i * L + j - 1];
                double r = BEST(s - 1, j);
                double m = a > r ? a : r;
                if (m < b) b = m;
            }
            BEST(s, i) = b;
        }
    double V = BEST(S, 0);
    int i = 0;
    first_layer[0] = 0;
    for (int s = S; s >= 2; s--) {
        int jj = -1;
        for (int j = i + 1; L - j >= s - 1; j++)
            if (cost[i * L + j - 1] <= V && BEST(s - 1, j) <= V) { jj = j; break; }
        if (jj < 0) { free(lc); free(cost); free(best); return -3; }
        first_layer[S - s + 1] = (uint32_t)jj;
        i = jj;
    }
#undef BEST
    free(lc); free(cost); free(best);
    return 0;
}

/* ------------------------------------------------------------------ */
/* Point validation (R3) -- same order of checks as DESIGN.md R3.       */
/* ------------------------------------------------------------------ */
static int point_check(const Trace *T, const Topo *tp, const OPoint *pt, const uint32_t *plan, uint32_t plan_len,
                       int have_plan) {
    if (pt->strategy > ST_HOP || (pt->strategy != ST_HOP && pt->tp_mode > TPM_MEGATRON) || pt->coll_algo > ALG_RSAG ||
        pt->ring_chunks > 16) return PT_BAD_CONFIG;   /* R25: at most 16 chunks per ring step */
    if (!(pt->bw_scale > 0.0) || isinf(pt->bw_scale) || !(pt->lat_scale >= 0.0) || isinf(pt->lat_scale))
        return PT_BAD_CONFIG;
    uint32_t dp = pt->dp, tpd = pt->tp, pp = pt->pp, m = pt->microbatches;
    if (dp == 0 || tpd == 0 || pp == 0) return PT_BAD_DEGREES;
    if (pt->strategy == ST_HOP) {   /* R28 */
        if (pt->tp_mode > HOP_DOUBLE_RING) return PT_BAD_CONFIG;
        int first_opt = 0;
        for (uint32_t o = 0; o < T->n_ops; o++) if (T->ops[o].phase == PH_OPT) first_opt = 1;
        if (!first_opt) return PT_BAD_CONFIG;
        if (tpd != 1 || pp != 1 || m == 0 || dp < 2 || dp % 2 || (pt->tp_mode == HOP_DOUBLE_RING && dp % 4))
            return PT_BAD_DEGREES;
        if (dp > tp->n_gpus) return PT_BAD_DEGREES;
        if (pt->global_batch == 0 || pt->global_batch % dp != 0) return PT_BAD_BATCH;
        return PT_OK;
    }
    switch (pt->strategy) {
    case ST_DP: case ST_DDP: if (tpd != 1 || pp != 1) return PT_BAD_DEGREES; break;
    case ST_TP: if (dp != 1 || pp != 1) return PT_BAD_DEGREES; break;
    case ST_PP: if (dp != 1 || tpd != 1) return PT_BAD_DEGREES; break;
    default: break;
    }
    int piped = (pt->strategy == ST_PP || pt->strategy == ST_HYBRID);
    if (piped && m == 0) return PT_BAD_DEGREES;
    if ((uint64_t)dp * tpd * pp > tp->n_gpus) return PT_BAD_DEGREES;
    if (pp > T->n_layers || pp > 64) return PT_BAD_DEGREES;
    uint64_t mm = piped ? m : 1;
    if (pt->global_batch == 0 || pt->global_batch % ((uint64_t)dp * mm) != 0) return PT_BAD_BATCH;
    if (piped && have_plan) {
        if (plan_len != pp || plan[0] != 0) return PT_BAD_PLAN;
        for (uint32_t s = 1; s < pp; s++)
            if (plan[s] <= plan[s - 1] || plan[s] >= T->n_layers) return PT_BAD_PLAN;
    }
    return PT_OK;
}

static const int *ring_order_of(const uint32_t *ro, uint32_t n_gpus, int *buf) {
    for (uint32_t i = 0; i < n_gpus; i++) buf[i] = ro ? (int)ro[i] : (int)i;
    return buf;
}

/* ------------------------------------------------------------------ */
/* Extrapolation: DP / DDP (R6)                           */
/* ------------------------------------------------------------------ */
typedef struct { uint32_t x; int prod; } WEnt;
static int cmp_went(const void *a, const void *b) {
    const WEnt *p = (const WEnt *)a, *q = (const WEnt *)b;
    if (p->prod != q->prod) return (p->prod > q->prod) - (p->prod < q->prod);
    return (p->x > q->x) - (p->x < q->x);
}

static int expand_dp(const Trace *T, const OPoint *pt, const int *ro, Graph *G) {
    int dp = pt->dp;
    uint32_t N = T->n_ops;
    double r_b = (double)(pt->global_batch / dp) / (double)T->b0;
    int *task = (int *)malloc(sizeof(int) * (size_t)dp * N);
    if (!task) return -1;
    /* every rank duplicates every operator */
    for (int r = 0; r < dp; r++)
        for (uint32_t o = 0; o < N; o++)
            task[(size_t)r * N + o] = add_task(G, ro[r], o, op_time(T, o, r_b, 1, pt->tp_mode), (int)T->ops[o].layer, (int)o, 0);
    if (dp > 1) {
        /* weight gradients in production order (reading Q4: produced by the backward pass) */
        WEnt *w = (WEnt *)malloc(sizeof(WEnt) * (T->n_ts ? T->n_ts : 1));
        int nw = 0;
        for (uint32_t x = 0; x < T->n_ts; x++)
            if (T->ts[x].category == CAT_WGRAD && T->prod[x] >= 0 && T->ops[T->prod[x]].phase != PH_OPT) {
                w[nw].x = x; w[nw].prod = T->prod[x]; nw++;
            }
        qsort(w, (size_t)nw, sizeof(WEnt), cmp_went);
        int last_nonopt = -1;
        for (uint32_t o = 0; o < N; o++) if (T->ops[o].phase != PH_OPT) last_nonopt = (int)o;
        int first_opt = -1;
        for (uint32_t o = 0; o < N; o++) if (T->ops[o].phase == PH_OPT) { first_opt = (int)o; break; }
        int *trig = (int *)malloc(sizeof(int) * (size_t)dp), *prev = (int *)malloc(sizeof(int) * (size_t)dp),
            *done = (int *)malloc(sizeof(int) * (size_t)dp);
        int have_prev = 0;
        int i = 0, nb = 0;
        while (i < nw) {
            /* bucket (reading Q5): bucket_bytes == 0 -> one tensor per AllReduce (paper-literal);
             * else greedy: close the bucket once its u64 byte sum reaches its cap (R24) */
            const uint64_t cap = bucket_cap(pt, nb++);
            int j = i;
            uint64_t sum = 0;
            double S = 0.0;
            for (;;) {
                sum += T->ts[w[j].x].bytes_b0;
                S = S + tensor_bytes(T, w[j].x, r_b, 1, pt->tp_mode);
                j++;
                if (cap == 0 || sum >= cap || j == nw) break;
            }
            /* DDP: AllReduce parallel with backward, triggered by the op producing the bucket's
             * last gradient; DP (DataParallel): after the backward pass (reading Q6) */
            int trig_op = (pt->strategy == ST_DDP) ? w[j - 1].prod : last_nonopt;
            for (int r = 0; r < dp; r++) trig[r] = task[(size_t)r * N + trig_op];
            G->cur_layer = (int)T->ops[trig_op].layer;
            G->cur_cat = 1;
            if (build_collective(G, ro, dp, CK_AR, pt->coll_algo, S, trig, have_prev ? prev : NULL, done)) return -1;
            memcpy(prev, done, sizeof(int) * (size_t)dp);
            have_prev = 1;
            i = j;
        }
        /* optimizer waits for this GPU's gradient collectives (reading Q7) */
        if (have_prev && first_opt >= 0)
            for (int r = 0; r < dp; r++) g_dep(G, task[(size_t)r * N + first_opt], prev[r]);
        free(w); free(trig); free(prev); free(done);
    }
    free(task);
    return 0;
}

/* ------------------------------------------------------------------ */
/* Extrapolation: TP (R7)                              */
/* ------------------------------------------------------------------ */
static int expand_tp(const Trace *T, const OPoint *pt, const int *ro, Graph *G) {
    int tp = pt->tp;
    uint32_t N = T->n_ops;
    double r_b = (double)pt->global_batch / (double)T->b0;
    int *task = (int *)malloc(sizeof(int) * (size_t)tp * N);
    if (!task) return -1;
    for (int r = 0; r < tp; r++)
        for (uint32_t o = 0; o < N; o++)
            task[(size_t)r * N + o] = add_task(G, ro[r], o, op_time(T, o, r_b, tp, pt->tp_mode), (int)T->ops[o].layer, (int)o, 0);
    if (tp > 1) {
        int *done_of = (int *)malloc(sizeof(int) * (size_t)(T->n_ts ? T->n_ts : 1) * (size_t)tp);
        char *has = (char *)calloc(T->n_ts ? T->n_ts : 1, 1);
        int *trig = (int *)malloc(sizeof(int) * (size_t)tp), *prev = (int *)malloc(sizeof(int) * (size_t)tp);
        int have_prev = 0;
        for (uint32_t o = 0; o < N; o++) {
            const OOp *op = &T->ops[o];
            for (uint32_t k = 0; k < op->n_out; k++) {
                uint32_t x = T->io[op->io_off + op->n_in + k];
                int kind = -1;
                if (pt->tp_mode == TPM_PAPER) {
                    /* "collects the partial outputs from all devices" */
                    if ((op->tp_role & ROLE_GATHER) && op->phase == PH_FWD) kind = CK_AG;
                    if ((op->tp_role & ROLE_GATHER) && op->phase == PH_BWD && T->ts[x].category == CAT_AGRAD) kind = CK_AR;
                } else {
                    if ((op->tp_role & 3) == ROLE_ROW && op->phase == PH_FWD) kind = CK_AR;
                    if ((op->tp_role & 3) == ROLE_COL && op->phase == PH_BWD && T->ts[x].category == CAT_AGRAD) kind = CK_AR;
                }
                if (kind < 0) continue;
                /* payload = the full tensor (not divided by tp), reading Q8 */
                double S = (double)T->ts[x].bytes_b0;
                if (T->ts[x].batch_scaled) S = S * r_b;
                for (int r = 0; r < tp; r++) trig[r] = task[(size_t)r * N + o];
                G->cur_layer = (int)op->layer;
                G->cur_cat = 0;
                if (build_collective(G, ro, tp, kind, pt->coll_algo, S, trig, have_prev ? prev : NULL,
                                     done_of + (size_t)x * tp)) return -1;
                memcpy(prev, done_of + (size_t)x * tp, sizeof(int) * (size_t)tp);
                have_prev = 1;
                has[x] = 1;
            }
        }
        /* a later operator that reads a communicated tensor waits for it on its GPU */
        for (uint32_t o = 0; o < N; o++) {
            const OOp *op = &T->ops[o];
            for (uint32_t k = 0; k < op->n_in; k++) {
                uint32_t x = T->io[op->io_off + k];
                if (has[x])
                    for (int r = 0; r < tp; r++) g_dep(G, task[(size_t)r * N + o], done_of[(size_t)x * tp + r]);
            }
        }
        free(done_of); free(has); free(trig); free(prev);
    }
    free(task);
    return 0;
}

/* ------------------------------------------------------------------ */
/* Extrapolation: Hop decentralized training (R28, Hop [42]) */
/* ------------------------------------------------------------------ */
/* Neighbours of worker i in the communication graph (Fig. 16a), ascending, without i itself:
 * ring-based on n workers (n even): i-1, i+1 and the most distant worker i+n/2 (mod n);
 * double ring (n % 4 == 0): two ring-based graphs on the halves {0..n/2-1}, {n/2..n-1}, plus the
 * node-to-node edge i <-> i+n/2 between them. */
static int hop_ring_based(int n, int i, int *nb) {
    int c = 0, cand[3] = {(i + n - 1) % n, (i + 1) % n, (i + n / 2) % n};
    for (int a = 0; a < 3; a++) {
        if (cand[a] == i) continue;
        int dup = 0;
        for (int b = 0; b < c; b++) if (nb[b] == cand[a]) dup = 1;
        if (!dup) nb[c++] = cand[a];
    }
    for (int x = 1; x < c; x++)   /* insertion sort */
        for (int y = x; y > 0 && nb[y] < nb[y - 1]; y--) { int t = nb[y]; nb[y] = nb[y - 1]; nb[y - 1] = t; }
    return c;
}
static int hop_neighbors(int n, int graph, int i, int *nb) {
    if (graph == HOP_RING_BASED) return hop_ring_based(n, i, nb);
    const int h = n / 2, half = i / h;
    int c = hop_ring_based(h, i % h, nb);
    for (int a = 0; a < c; a++) nb[a] += half * h;
    nb[c++] = (i + h) % n;
    for (int x = 1; x < c; x++)
        for (int y = x; y > 0 && nb[y] < nb[y - 1]; y--) { int t = nb[y]; nb[y] = nb[y - 1]; nb[y - 1] = t; }
    return c;
}
static uint64_t hop_flow_code(int k, int src, int dst) {
    return (1ull << 58) | ((uint64_t)(uint32_t)k << 32) | ((uint64_t)(uint32_t)src << 16) | (uint64_t)(uint32_t)dst;
}

/*
 * Worker r (GPU ro[r]) runs K = microbatches iterations of the whole trace (FWD, BWD, OPT ops in program
 * order, t' at b_loc = B / n).  Reading of the paper's protocol (R28):
 *   - update queues: after its last non-OPT op of iteration k the worker sends its update u(r, k) --
 *     S bytes, the left fold of its weight-gradient sizes -- to every neighbour, ascending, on its FIFO
 *     send stream (R11: one send at a time, across iterations too);
 *   - bounded staleness s and backup workers b: the first OPT op of iteration k (applying the update)
 *     waits until u(j, k - s) has been delivered from at least deg - b neighbours j (nothing to wait
 *     for when k < s or deg <= b) -- a threshold barrier;
 *   - token queues, bounded iteration gap g >= 1 (0 = unbounded): the first op of iteration k waits
 *     until every neighbour has finished computing iteration k - g (its last non-OPT op).
 * hop = backup | staleness << 4 | gap << 8 (point field pad1); tp_mode selects the graph.
 */
static int expand_hop(const Trace *T, const OPoint *pt, const int *ro, Graph *G) {
    const int n = pt->dp, K = (int)pt->microbatches, graph = pt->tp_mode;
    const int b = pt->pad1 & 15, s = (pt->pad1 >> 4) & 15, g = (pt->pad1 >> 8) & 255;
    const uint32_t N = T->n_ops;
    const double r_b = (double)(pt->global_batch / (uint32_t)n) / (double)T->b0;
    int last_nonopt = -1, first_opt = -1;
    for (uint32_t o = 0; o < N; o++) {
        if (T->ops[o].phase != PH_OPT) last_nonopt = (int)o;
        else if (first_opt < 0) first_opt = (int)o;
    }
    /* update size: left fold of the weight-gradient bytes' in production order (as R6's buckets) */
    WEnt *w = (WEnt *)malloc(sizeof(WEnt) * (T->n_ts ? T->n_ts : 1));
    int nw = 0;
    for (uint32_t x = 0; x < T->n_ts; x++)
        if (T->ts[x].category == CAT_WGRAD && T->prod[x] >= 0 && T->ops[T->prod[x]].phase != PH_OPT) {
            w[nw].x = x; w[nw].prod = T->prod[x]; nw++;
        }
    qsort(w, (size_t)nw, sizeof(WEnt), cmp_went);
    double S = 0.0;
    for (int a = 0; a < nw; a++) S = S + tensor_bytes(T, w[a].x, r_b, 1, pt->tp_mode);
    free(w);
    int *nbr = (int *)malloc(sizeof(int) * (size_t)n * 4), *ndeg = (int *)malloc(sizeof(int) * (size_t)n);
    int *task = (int *)malloc(sizeof(int) * (size_t)n * K * (N ? N : 1));
    int *flow = (int *)malloc(sizeof(int) * (size_t)n * K * 4);
    if (!nbr || !ndeg || !task || !flow) return -1;
    for (int r = 0; r < n; r++) ndeg[r] = hop_neighbors(n, graph, r, nbr + r * 4);
#define TSK(r, k, o) task[((size_t)(r) * K + (k)) * N + (o)]
#define FLW(r, k, q) flow[((size_t)(r) * K + (k)) * 4 + (q)]
    for (int r = 0; r < n; r++)
        for (int k = 0; k < K; k++)
            for (uint32_t o = 0; o < N; o++)
                TSK(r, k, o) = add_task(G, ro[r], (long)k * N + o, op_time(T, o, r_b, 1, pt->tp_mode),
                                        (int)T->ops[o].layer, (int)o, k);
    for (int r = 0; r < n; r++) {
        int prev = -1;   /* this worker's previous send (FIFO stream) */
        for (int k = 0; k < K; k++)
            for (int q = 0; q < ndeg[r]; q++) {
                const int j = nbr[r * 4 + q];
                const int f = add_flow(G, ro[r], ro[j], S, hop_flow_code(k, r, j), NF_P2P);
                FLW(r, k, q) = f;
                if (q == 0) g_dep(G, f, TSK(r, k, last_nonopt));
                if (prev >= 0) g_dep(G, f, prev);
                prev = f;
                if (G->want_bd && ro[r] == G->rep[0]) g_record(G, f, f, (int)T->ops[last_nonopt].layer, 2);
            }
    }
    for (int r = 0; r < n; r++)
        for (int k = 0; k < K; k++) {
            /* token queues: iteration k starts after every neighbour finished computing k - g */
            if (g > 0 && k >= g)
                for (int q = 0; q < ndeg[r]; q++) g_dep(G, TSK(r, k, 0), TSK(nbr[r * 4 + q], k - g, last_nonopt));
            /* update queues with backup workers and bounded staleness */
            const int need = ndeg[r] - b;
            if (k >= s && need > 0) {
                const int a = add_barrier(G, (need + 1) << NF_NEED_SHIFT, 0);
                if (a < 0) return -1;
                for (int q = 0; q < ndeg[r]; q++) {
                    const int j = nbr[r * 4 + q];
                    int qq = 0;
                    while (nbr[j * 4 + qq] != r) qq++;   /* r's place in j's neighbour list */
                    g_dep(G, a, FLW(j, k - s, qq));
                }
                g_dep(G, TSK(r, k, first_opt), a);
            }
        }
#undef TSK
#undef FLW
    free(nbr); free(ndeg); free(task); free(flow);
    return 0;
}

/* ------------------------------------------------------------------ */
/* Extrapolation: PP / GPipe (R8; Fig. 4)                    */
/* ------------------------------------------------------------------ */
static int expand_pp(const Trace *T, const OPoint *pt, const int *ro, const uint32_t *first_layer, Graph *G) {
    int S = pt->pp, m = (int)pt->microbatches;
    uint32_t N = T->n_ops, L = T->n_layers;
    double r_b = (double)(pt->global_batch / (uint32_t)m) / (double)T->b0;
    int *stage_of_layer = (int *)malloc(sizeof(int) * L);
    for (uint32_t l = 0, s = 0; l < L; l++) {
        while ((int)s + 1 < S && first_layer[s + 1] <= l) s++;
        stage_of_layer[l] = (int)s;
    }
    /* task id of instance (o, j); OPT ops use j = 0 */
    int *inst = (int *)malloc(sizeof(int) * (size_t)N * (size_t)m);
    int *prog_op = (int *)malloc(sizeof(int) * ((size_t)N * (size_t)m + 1));
    int *prog_mb = (int *)malloc(sizeof(int) * ((size_t)N * (size_t)m + 1));
    /* readers: for each tensor, which stages read it (bitmask over <=64 stages) */
    uint64_t *readers = (uint64_t *)calloc(T->n_ts ? T->n_ts : 1, sizeof(uint64_t));
    if (!stage_of_layer || !inst || !prog_op || !prog_mb || !readers) return -1;
    for (uint32_t o = 0; o < N; o++) {
        const OOp *op = &T->ops[o];
        for (uint32_t k = 0; k < op->n_in; k++) readers[T->io[op->io_off + k]] |= 1ull << stage_of_layer[op->layer];
    }
    /* cross-stage transfers: (tensor, producer instance, destination) -> flow id */
    int *xidx = (int *)malloc(sizeof(int) * (T->n_ts ? T->n_ts : 1));
    int ncross = 0;
    for (uint32_t x = 0; x < T->n_ts; x++) {
        xidx[x] = -1;
        if (T->prod[x] >= 0) {
            int ps = stage_of_layer[T->ops[T->prod[x]].layer];
            if (readers[x] & ~(1ull << ps)) xidx[x] = ncross++;
        }
    }
    int *p2p = (int *)malloc(sizeof(int) * ((size_t)ncross * (size_t)m * (size_t)S + 1));
    for (size_t q = 0; q < (size_t)ncross * (size_t)m * (size_t)S; q++) p2p[q] = -1;

    for (int s = 0; s < S; s++) {
        /* GPipe program on stage s: FWD of micro-batches 0..m-1, BWD of m-1..0, then OPT once */
        long np = 0;
        for (int j = 0; j < m; j++)
            for (uint32_t o = 0; o < N; o++)
                if (T->ops[o].phase == PH_FWD && stage_of_layer[T->ops[o].layer] == s) { prog_op[np] = (int)o; prog_mb[np++] = j; }
        for (int j = m - 1; j >= 0; j--)
            for (uint32_t o = 0; o < N; o++)
                if (T->ops[o].phase == PH_BWD && stage_of_layer[T->ops[o].layer] == s) { prog_op[np] = (int)o; prog_mb[np++] = j; }
        for (uint32_t o = 0; o < N; o++)
            if (T->ops[o].phase == PH_OPT && stage_of_layer[T->ops[o].layer] == s) { prog_op[np] = (int)o; prog_mb[np++] = 0; }
        int prev_send = -1;
        for (long q = 0; q < np; q++) {
            int o = prog_op[q], j = prog_mb[q];
            int t = add_task(G, ro[s], q, op_time(T, (uint32_t)o, r_b, 1, pt->tp_mode), (int)T->ops[o].layer, o, j);
            inst[(size_t)o * m + j] = t;
            /* "send its output data to the next GPU. Simultaneously ... the next micro-batch"
             * (P:190): push every produced tensor to each other stage that reads it, FIFO per
             * sending GPU (reading Q14/Q15) */
            const OOp *op = &T->ops[o];
            for (uint32_t k = 0; k < op->n_out; k++) {
                uint32_t x = T->io[op->io_off + op->n_in + k];
                if (xidx[x] < 0) continue;
                for (int d = 0; d < S; d++) {
                    if (d == s || !(readers[x] & (1ull << d))) continue;
                    double b = tensor_bytes(T, x, r_b, 1, pt->tp_mode);
                    int f = add_flow(G, ro[s], ro[d], b, p2p_flow_code(x, j, ro[d]), NF_P2P);
                    g_dep(G, f, t);
                    if (G->want_bd && ro[s] == G->rep[op->layer]) g_record(G, f, f, (int)op->layer, 2);
                    if (prev_send >= 0) g_dep(G, f, prev_send);
                    prev_send = f;
                    p2p[((size_t)xidx[x] * m + j) * S + d] = f;
                }
            }
        }
    }
    /* consumers wait for the delivery of every remote input ("execution cannot start
     * until the data is available") */
    for (uint32_t o = 0; o < N; o++) {
        const OOp *op = &T->ops[o];
        int s = stage_of_layer[op->layer];
        int nj = (op->phase == PH_OPT) ? 1 : m;
        for (int j = 0; j < nj; j++) {
            int t = inst[(size_t)o * m + j];
            for (uint32_t k = 0; k < op->n_in; k++) {
                uint32_t x = T->io[op->io_off + k];
                int po = T->prod[x];
                if (po < 0 || stage_of_layer[T->ops[po].layer] == s) continue;
                int jp = (T->ops[po].phase == PH_OPT || op->phase == PH_OPT) ? 0 : j;
                int f = p2p[((size_t)xidx[x] * m + jp) * S + s];
                if (f < 0) return -1;
                g_dep(G, t, f);
            }
        }
    }
    free(stage_of_layer); free(inst); free(prog_op); free(prog_mb); free(readers); free(xidx); free(p2p);
    return 0;
}

/* ------------------------------------------------------------------ */
/* Extrapolation: HYBRID DP x TP x PP (R9; "often combined as      */
/* hybrid parallelism"; Table 1 P:102 -- an extension, reading Q26)     */
/* ------------------------------------------------------------------ */
/* tiny open-addressing map uint64 -> int (plain, test infrastructure) */
typedef struct { uint64_t *k; int *v; long cap, n; } HMap;
static int hm_init(HMap *h, long cap) {
    h->cap = 64; while (h->cap < 2 * cap + 64) h->cap *= 2; h->n = 0;
    h->k = (uint64_t *)malloc(sizeof(uint64_t) * (size_t)h->cap); h->v = (int *)malloc(sizeof(int) * (size_t)h->cap);
    if (!h->k || !h->v) return -1;
    for (long i = 0; i < h->cap; i++) h->k[i] = ~0ull;
    return 0;
}
static void hm_free(HMap *h) { free(h->k); free(h->v); h->k = NULL; h->v = NULL; }
static int hm_put(HMap *h, uint64_t key, int val) {
    if (2 * (h->n + 1) > h->cap) {
        HMap g; if (hm_init(&g, h->cap)) return -1;
        for (long i = 0; i < h->cap; i++) if (h->k[i] != ~0ull) hm_put(&g, h->k[i], h->v[i]);
        hm_free(h); *h = g;
    }
    long i = (long)((key * 0x9e3779b97f4a7c15ull) >> 20) & (h->cap - 1);
    while (h->k[i] != ~0ull && h->k[i] != key) i = (i + 1) & (h->cap - 1);
    if (h->k[i] == ~0ull) h->n++;
    h->k[i] = key; h->v[i] = val;
    return 0;
}
static int hm_get(const HMap *h, uint64_t key) {
    long i = (long)((key * 0x9e3779b97f4a7c15ull) >> 20) & (h->cap - 1);
    while (h->k[i] != ~0ull) { if (h->k[i] == key) return h->v[i]; i = (i + 1) & (h->cap - 1); }
    return -1;
}

/* R7's TP collective rule for one output of one op (-1 = none) */
static int tp_kind(const Trace *T, const OOp *op, uint32_t x, int tp_mode) {
    if (tp_mode == TPM_PAPER) {
        if ((op->tp_role & ROLE_GATHER) && op->phase == PH_FWD) return CK_AG;
        if ((op->tp_role & ROLE_GATHER) && op->phase == PH_BWD && T->ts[x].category == CAT_AGRAD) return CK_AR;
    } else {
        if ((op->tp_role & 3) == ROLE_ROW && op->phase == PH_FWD) return CK_AR;
        if ((op->tp_role & 3) == ROLE_COL && op->phase == PH_BWD && T->ts[x].category == CAT_AGRAD) return CK_AR;
    }
    return -1;
}

static int expand_hybrid(const Trace *T, const OPoint *pt, const int *ro, const uint32_t *first_layer, Graph *G) {
    const int dp = pt->dp, tp = pt->tp, S = pt->pp, m = (int)pt->microbatches;
    const uint32_t N = T->n_ops, L = T->n_layers;
    const double r_b = (double)(pt->global_batch / ((uint32_t)dp * (uint32_t)m)) / (double)T->b0;
    const int R = dp * S * tp;
    int rc = -1;
    int *stage_of_layer = (int *)malloc(sizeof(int) * L);
    uint64_t *readers = (uint64_t *)calloc(T->n_ts ? T->n_ts : 1, sizeof(uint64_t));
    int **pop = (int **)calloc((size_t)S, sizeof(int *)), **pmb = (int **)calloc((size_t)S, sizeof(int *));
    long *plen = (long *)calloc((size_t)S, sizeof(long));
    int **task = (int **)calloc((size_t)R, sizeof(int *));
    int *members = (int *)malloc(sizeof(int) * (size_t)(dp > tp ? dp : tp) + sizeof(int));
    int *trig = (int *)malloc(sizeof(int) * (size_t)(dp > tp ? dp : tp) + sizeof(int));
    int *prev = (int *)malloc(sizeof(int) * (size_t)(dp > tp ? dp : tp) + sizeof(int));
    int *done = (int *)malloc(sizeof(int) * (size_t)(dp > tp ? dp : tp) + sizeof(int));
    IVec dtab = {0};          /* done barriers of TP collectives, tp per collective */
    HMap tpc = {0}, p2p = {0};
    if (!stage_of_layer || !readers || !pop || !pmb || !plen || !task || !members || !trig || !prev || !done) goto out;
    if (hm_init(&tpc, 1024) || hm_init(&p2p, 1024)) goto out;
    for (uint32_t l = 0, s = 0; l < L; l++) {
        while ((int)s + 1 < S && first_layer[s + 1] <= l) s++;
        stage_of_layer[l] = (int)s;
    }
    for (uint32_t o = 0; o < N; o++) {
        const OOp *op = &T->ops[o];
        for (uint32_t k = 0; k < op->n_in; k++) readers[T->io[op->io_off + k]] |= 1ull << stage_of_layer[op->layer];
    }
    /* the GPipe program of each stage (R8): FWD of 0..m-1, BWD of m-1..0, OPT once */
    for (int s = 0; s < S; s++) {
        pop[s] = (int *)malloc(sizeof(int) * ((size_t)N * (size_t)m + 1));
        pmb[s] = (int *)malloc(sizeof(int) * ((size_t)N * (size_t)m + 1));
        if (!pop[s] || !pmb[s]) goto out;
        long np = 0;
        for (int j = 0; j < m; j++)
            for (uint32_t o = 0; o < N; o++)
                if (T->ops[o].phase == PH_FWD && stage_of_layer[T->ops[o].layer] == s) { pop[s][np] = (int)o; pmb[s][np++] = j; }
        for (int j = m - 1; j >= 0; j--)
            for (uint32_t o = 0; o < N; o++)
                if (T->ops[o].phase == PH_BWD && stage_of_layer[T->ops[o].layer] == s) { pop[s][np] = (int)o; pmb[s][np++] = j; }
        for (uint32_t o = 0; o < N; o++)
            if (T->ops[o].phase == PH_OPT && stage_of_layer[T->ops[o].layer] == s) { pop[s][np] = (int)o; pmb[s][np++] = 0; }
        plen[s] = np;
    }
    /* rank r = (d*pp + s)*tp + t on GPU ring_order[r] (TP innermost) */
    for (int r = 0; r < R; r++) {
        const int s = (r / tp) % S;
        task[r] = (int *)malloc(sizeof(int) * ((size_t)plen[s] + 1));
        if (!task[r]) goto out;
        for (long q = 0; q < plen[s]; q++)
            task[r][q] = add_task(G, ro[r], q, op_time(T, (uint32_t)pop[s][q], r_b, tp, pt->tp_mode),
                                  (int)T->ops[pop[s][q]].layer, pop[s][q], pmb[s][q]);
    }
    /* TP collectives: per group (d, s), one per (op, output, micro-batch) instance in program order */
    if (tp > 1) {
        for (int d = 0; d < dp; d++)
            for (int s = 0; s < S; s++) {
                const uint64_t gid = (uint64_t)(d * S + s);
                const int base = (d * S + s) * tp;
                for (int t = 0; t < tp; t++) members[t] = ro[base + t];
                int have_prev = 0;
                uint64_t seq = 0;
                for (long q = 0; q < plen[s]; q++) {
                    const OOp *op = &T->ops[pop[s][q]];
                    for (uint32_t k = 0; k < op->n_out; k++) {
                        const uint32_t x = T->io[op->io_off + op->n_in + k];
                        const int kind = tp_kind(T, op, x, pt->tp_mode);
                        if (kind < 0) continue;
                        double Sb = (double)T->ts[x].bytes_b0;      /* full tensor (Q8) */
                        if (T->ts[x].batch_scaled) Sb = Sb * r_b;
                        for (int t = 0; t < tp; t++) trig[t] = task[base + t][q];
                        G->cur_layer = (int)op->layer;
                        G->cur_cat = 0;
                        uint64_t used = 1;
                        if (build_allreduce(G, (gid << 20) | seq, members, tp, kind, pt->coll_algo, Sb, trig,
                                            have_prev ? prev : NULL, done, &used)) goto out;
                        seq += used;
                        memcpy(prev, done, sizeof(int) * (size_t)tp);
                        have_prev = 1;
                        if (hm_put(&tpc, (gid << 40) | ((uint64_t)x << 16) | (uint64_t)pmb[s][q], (int)dtab.n)) goto out;
                        for (int t = 0; t < tp; t++) iv_push(&dtab, done[t]);
                    }
                }
            }
        /* same-stage readers of a communicated tensor wait for it on their GPU */
        for (int r = 0; r < R; r++) {
            const int d = r / (S * tp), s = (r / tp) % S, t = r % tp;
            const uint64_t gid = (uint64_t)(d * S + s);
            for (long q = 0; q < plen[s]; q++) {
                const OOp *op = &T->ops[pop[s][q]];
                for (uint32_t k = 0; k < op->n_in; k++) {
                    const uint32_t x = T->io[op->io_off + k];
                    const int po = T->prod[x];
                    if (po < 0 || stage_of_layer[T->ops[po].layer] != s) continue;
                    const int jp = (T->ops[po].phase == PH_OPT || op->phase == PH_OPT) ? 0 : pmb[s][q];
                    const int di = hm_get(&tpc, (gid << 40) | ((uint64_t)x << 16) | (uint64_t)jp);
                    if (di >= 0) g_dep(G, task[r][q], dtab.v[di + t]);
                }
            }
        }
    }
    /* P2P along each pipeline (d, t): push every produced tensor to each other reading stage,
     * FIFO per sending GPU; a TP-communicated tensor leaves after its collective is done there */
    for (int r = 0; r < R; r++) {
        const int d = r / (S * tp), s = (r / tp) % S, t = r % tp;
        const uint64_t gid = (uint64_t)(d * S + s), pipe = (uint64_t)(d * tp + t);
        int prev_send = -1;
        for (long q = 0; q < plen[s]; q++) {
            const int o = pop[s][q], j = pmb[s][q];
            const OOp *op = &T->ops[o];
            for (uint32_t k = 0; k < op->n_out; k++) {
                const uint32_t x = T->io[op->io_off + op->n_in + k];
                for (int ds = 0; ds < S; ds++) {
                    if (ds == s || !(readers[x] & (1ull << ds))) continue;
                    const int dg = ro[(d * S + ds) * tp + t];
                    const int f = add_flow(G, ro[r], dg, tensor_bytes(T, x, r_b, tp, pt->tp_mode),
                                           p2p_flow_code(x, j, dg), NF_P2P);
                    g_dep(G, f, task[r][q]);
                    if (G->want_bd && ro[r] == G->rep[op->layer]) g_record(G, f, f, (int)op->layer, 2);
                    if (prev_send >= 0) g_dep(G, f, prev_send);
                    if (tp > 1) {
                        const int di = hm_get(&tpc, (gid << 40) | ((uint64_t)x << 16) | (uint64_t)j);
                        if (di >= 0) g_dep(G, f, dtab.v[di + t]);
                    }
                    prev_send = f;
                    if (hm_put(&p2p, (((pipe << 24) | x) << 22) | ((uint64_t)j << 6) | (uint64_t)ds, f)) goto out;
                }
            }
        }
    }
    for (int r = 0; r < R; r++) {
        const int d = r / (S * tp), s = (r / tp) % S, t = r % tp;
        const uint64_t pipe = (uint64_t)(d * tp + t);
        for (long q = 0; q < plen[s]; q++) {
            const OOp *op = &T->ops[pop[s][q]];
            for (uint32_t k = 0; k < op->n_in; k++) {
                const uint32_t x = T->io[op->io_off + k];
                const int po = T->prod[x];
                if (po < 0 || stage_of_layer[T->ops[po].layer] == s) continue;
                const int jp = (T->ops[po].phase == PH_OPT || op->phase == PH_OPT) ? 0 : pmb[s][q];
                const int f = hm_get(&p2p, (((pipe << 24) | x) << 22) | ((uint64_t)jp << 6) | (uint64_t)s);
                if (f < 0) goto out;
                g_dep(G, task[r][q], f);
            }
        }
    }
    /* DP: per group (s, t), one AllReduce per bucket of the stage's weight gradients, triggered by
     * micro-batch 0's producer (the last one GPipe's backward runs); OPT waits for the last one */
    if (dp > 1) {
        WEnt *w = (WEnt *)malloc(sizeof(WEnt) * (T->n_ts ? T->n_ts : 1));
        if (!w) goto out;
        for (int s = 0; s < S; s++) {
            int nw = 0;
            for (uint32_t x = 0; x < T->n_ts; x++)
                if (T->ts[x].category == CAT_WGRAD && T->prod[x] >= 0 && T->ops[T->prod[x]].phase != PH_OPT &&
                    stage_of_layer[T->ops[T->prod[x]].layer] == s) {
                    w[nw].x = x; w[nw].prod = T->prod[x]; nw++;
                }
            qsort(w, (size_t)nw, sizeof(WEnt), cmp_went);
            long first_opt = -1;
            for (long q = 0; q < plen[s]; q++) if (T->ops[pop[s][q]].phase == PH_OPT) { first_opt = q; break; }
            for (int t = 0; t < tp; t++) {
                const uint64_t gid = (uint64_t)((tp > 1 ? dp * S : 0) + s * tp + t);
                for (int d = 0; d < dp; d++) members[d] = ro[(d * S + s) * tp + t];
                int have_prev = 0;
                uint64_t seq = 0;
                int i = 0, nb = 0;
                while (i < nw) {
                    const uint64_t cap = bucket_cap(pt, nb++);   /* R24, per stage's DP group */
                    int j = i;
                    uint64_t sum = 0;
                    double Sb = 0.0;
                    for (;;) {
                        sum += T->ts[w[j].x].bytes_b0;
                        Sb = Sb + tensor_bytes(T, w[j].x, r_b, tp, pt->tp_mode);
                        j++;
                        if (cap == 0 || sum >= cap || j == nw) break;
                    }
                    /* program position of (producer of the bucket's last gradient, micro-batch 0) */
                    long qt = -1;
                    for (long q = 0; q < plen[s]; q++)
                        if (pop[s][q] == w[j - 1].prod && pmb[s][q] == 0) { qt = q; break; }
                    if (qt < 0) { free(w); goto out; }
                    for (int d = 0; d < dp; d++) trig[d] = task[(d * S + s) * tp + t][qt];
                    G->cur_layer = (int)T->ops[pop[s][qt]].layer;
                    G->cur_cat = 1;
                    uint64_t used = 1;
                    if (build_allreduce(G, (gid << 20) | seq, members, dp, CK_AR, pt->coll_algo, Sb, trig,
                                        have_prev ? prev : NULL, done, &used)) { free(w); goto out; }
                    seq += used;
                    memcpy(prev, done, sizeof(int) * (size_t)dp);
                    have_prev = 1;
                    i = j;
                }
                if (have_prev && first_opt >= 0)
                    for (int d = 0; d < dp; d++) g_dep(G, task[(d * S + s) * tp + t][first_opt], prev[d]);
            }
        }
        free(w);
    }
    rc = 0;
out:
    free(stage_of_layer); free(readers);
    if (pop) for (int s = 0; s < S; s++) { free(pop[s]); free(pmb[s]); }
    free(pop); free(pmb); free(plen);
    if (task) for (int r = 0; r < R; r++) free(task[r]);
    free(task); free(members); free(trig); free(prev); free(done);
    iv_free(&dtab); hm_free(&tpc); hm_free(&p2p);
    return rc;
}

/* ------------------------------------------------------------------ */
/* Water-filling (R14; "bandwidth sharing between streams",        */
/* P:210 "allocate bandwidth for the links on the route", reading Q18:  */
/* max-min fair progressive filling).                                   */
/* ------------------------------------------------------------------ */
typedef struct {
    int n_links;
    double *bw;      /* per-point link bandwidth */
    int *n_e, *k_e;
    double *res, *share;
} WF;

/* flows[0..nf): route given by (roff, rlen) into rlinks; writes rate[]; returns rounds */
static long waterfill(WF *w, int nf, const int *flows, const long *roff, const int *rlen, const int *rlinks,
                      double *rate, char *unfrozen) {
    for (int e = 0; e < w->n_links; e++) { w->n_e[e] = 0; w->k_e[e] = 0; w->res[e] = w->bw[e]; }
    for (int a = 0; a < nf; a++) {
        int f = flows[a];
        for (int h = 0; h < rlen[f]; h++) w->n_e[rlinks[roff[f] + h]]++;
        unfrozen[a] = 1;
    }
    int left = nf;
    long rounds = 0;
    while (left > 0) {
        double s = INFINITY;
        for (int e = 0; e < w->n_links; e++)
            if (w->n_e[e] > 0) {
                w->share[e] = w->res[e] / (double)w->n_e[e];
                if (w->share[e] < s) s = w->share[e];
            }
        /* F_r: unfrozen flows crossing a link whose share equals the minimum */
        for (int a = 0; a < nf; a++) {
            if (!unfrozen[a]) continue;
            int f = flows[a], inb = 0;
            for (int h = 0; h < rlen[f]; h++) {
                int e = rlinks[roff[f] + h];
                if (w->n_e[e] > 0 && w->share[e] == s) inb = 1;
            }
            if (inb) {
                rate[a] = s;
                unfrozen[a] = 2; /* mark: frozen this round */
                for (int h = 0; h < rlen[f]; h++) w->k_e[rlinks[roff[f] + h]]++;
            }
        }
        for (int e = 0; e < w->n_links; e++)
            if (w->k_e[e] > 0) {
                double r = w->res[e] - s * (double)w->k_e[e];
                w->res[e] = r > 0.0 ? r : 0.0;
                w->n_e[e] -= w->k_e[e];
                w->k_e[e] = 0;
            }
        for (int a = 0; a < nf; a++)
            if (unfrozen[a] == 2) { unfrozen[a] = 0; left--; }
        rounds++;
    }
    return rounds;
}

/* ------------------------------------------------------------------ */
/* Order hash helpers (R19)                                             */
/* ------------------------------------------------------------------ */
static uint64_t mix64(uint64_t z) {
    z = (z ^ (z >> 30)) * 0xbf58476d1ce4e5b9ull;
    z = (z ^ (z >> 27)) * 0x94d049bb133111ebull;
    return z ^ (z >> 31);
}
static uint64_t dbits(double d) { uint64_t u; memcpy(&u, &d, 8); return u; }

/* ------------------------------------------------------------------ */
/* The event-driven timeline (R13-R17)                                  */
/* ------------------------------------------------------------------ */
enum { S_WAIT = 0, S_QUEUED = 1, S_RUN = 2, S_LATENT = 3, S_ACTIVE = 4, S_DONE = 5 };

static int simulate(Graph *G, const Topo *tp, double bw_scale, double lat_scale, OResult *res, double *t_done,
                    double *l_comp, double *l_comm, double *tl_s, double *tl_a) {
    long NN = G->count;
    const int bd = l_comp != NULL && G->want_bd;
    double *td_own = NULL, *t_rel = NULL;
    if (bd) {
        t_rel = (double *)calloc((size_t)(NN ? NN : 1), sizeof(double));
        if (!t_done) t_done = td_own = (double *)calloc((size_t)(NN ? NN : 1), sizeof(double));
        if (!t_rel || !t_done) { free(t_rel); free(td_own); return -1; }
    }
    int n_nodes_topo = (int)tp->n_nodes;
    /* dependency CSR (forward) and dependents CSR (reverse) */
    long NE = G->dep_from.n;
    long *doff = (long *)calloc((size_t)NN + 1, sizeof(long)), *roff = (long *)calloc((size_t)NN + 1, sizeof(long));
    int *dlist = (int *)malloc(sizeof(int) * (size_t)(NE ? NE : 1)), *rlist = (int *)malloc(sizeof(int) * (size_t)(NE ? NE : 1));
    int *pending = (int *)calloc((size_t)(NN ? NN : 1), sizeof(int));
    if (!doff || !roff || !dlist || !rlist || !pending) return -1;
    for (long e = 0; e < NE; e++) { doff[G->dep_from.v[e] + 1]++; roff[G->dep_to.v[e] + 1]++; }
    for (long i = 0; i < NN; i++) { doff[i + 1] += doff[i]; roff[i + 1] += roff[i]; }
    {
        long *fd = (long *)calloc((size_t)NN + 1, sizeof(long)), *fr = (long *)calloc((size_t)NN + 1, sizeof(long));
        for (long e = 0; e < NE; e++) {
            int a = G->dep_from.v[e], b = G->dep_to.v[e];
            dlist[doff[a] + fd[a]++] = b;
            rlist[roff[b] + fr[b]++] = a;
        }
        free(fd); free(fr);
    }
    for (long i = 0; i < NN; i++) {
        pending[i] = (int)(doff[i + 1] - doff[i]);
        /* R28: a threshold barrier completes once `need` of its dependencies are done */
        if (G->n[i].type == N_BARRIER && (G->n[i].flags >> NF_NEED_SHIFT) > 0) pending[i] = (G->n[i].flags >> NF_NEED_SHIFT) - 1;
    }

    /* per-GPU in-order queues */
    int *qoff = (int *)calloc((size_t)n_nodes_topo + 1, sizeof(int));
    for (long i = 0; i < NN; i++) if (G->n[i].type == N_TASK) qoff[G->n[i].gpu + 1]++;
    for (int g = 0; g < n_nodes_topo; g++) qoff[g + 1] += qoff[g];
    int *qlist = (int *)malloc(sizeof(int) * (size_t)(qoff[n_nodes_topo] ? qoff[n_nodes_topo] : 1));
    {
        int *fq = (int *)calloc((size_t)n_nodes_topo, sizeof(int));
        for (long i = 0; i < NN; i++) if (G->n[i].type == N_TASK) { int g = G->n[i].gpu; qlist[qoff[g] + fq[g]++] = (int)i; }
        free(fq);
    }
    int *head = (int *)calloc((size_t)n_nodes_topo, sizeof(int)), *running = (int *)malloc(sizeof(int) * (size_t)n_nodes_topo);
    for (int g = 0; g < n_nodes_topo; g++) running[g] = -1;

    /* compute_busy_max: per GPU left fold of t' in program order (R18) */
    double cbmax = 0.0;
    long n_tasks = 0, n_flows = 0, n_p2p = 0;
    for (int g = 0; g < n_nodes_topo; g++) {
        double b = 0.0;
        for (int q = qoff[g]; q < qoff[g + 1]; q++) b = b + G->n[qlist[q]].dur;
        if (b > cbmax) cbmax = b;
    }

    /* routes: per flow, BFS route (cached per ordered GPU pair) */
    long *froff = (long *)calloc((size_t)(NN ? NN : 1), sizeof(long));
    int *frlen = (int *)calloc((size_t)(NN ? NN : 1), sizeof(int));
    IVec rpool = {0};
    long *pair_off = (long *)malloc(sizeof(long) * (size_t)n_nodes_topo * (size_t)n_nodes_topo);
    int *pair_len = (int *)malloc(sizeof(int) * (size_t)n_nodes_topo * (size_t)n_nodes_topo);
    for (long q = 0; q < (long)n_nodes_topo * n_nodes_topo; q++) pair_len[q] = -9;
    int *tmp = (int *)malloc(sizeof(int) * (size_t)(n_nodes_topo + 1));
    double *lat = (double *)calloc((size_t)(NN ? NN : 1), sizeof(double));
    int status = PT_OK;
    for (long i = 0; i < NN; i++) {
        if (G->n[i].type != N_FLOW) continue;
        n_flows++;
        if (G->n[i].flags & NF_P2P) n_p2p++;
        if (tp->ph) continue;   /* photonic: logical links instead of physical routes (R20) */
        int s = G->n[i].src, d = G->n[i].dst;
        long key = (long)s * n_nodes_topo + d;
        if (pair_len[key] == -9) {
            int h = bfs_route(tp, s, d, tmp, n_nodes_topo);
            pair_off[key] = rpool.n;
            pair_len[key] = h;
            for (int k = 0; k < h; k++) iv_push(&rpool, tmp[k]);
        }
        if (pair_len[key] < 0) { status = PT_NO_ROUTE; break; }
        froff[i] = pair_off[key];
        frlen[i] = pair_len[key];
        /* route latency: left fold of per-link latencies (R12/R13) */
        double L = 0.0;
        for (int k = 0; k < frlen[i]; k++) L = L + tp->links[rpool.v[froff[i] + k]].lat * lat_scale;
        lat[i] = L;
    }
    for (long i = 0; i < NN; i++) if (G->n[i].type == N_TASK) n_tasks++;

    memset(res, 0, sizeof *res);
    if (status != PT_OK) {
        res->status = status;
        goto out;
    }
    {
        WF w;
        w.n_links = (int)tp->n_links;
        w.bw = (double *)malloc(sizeof(double) * (size_t)(w.n_links ? w.n_links : 1));
        w.n_e = (int *)malloc(sizeof(int) * (size_t)(w.n_links ? w.n_links : 1));
        w.k_e = (int *)malloc(sizeof(int) * (size_t)(w.n_links ? w.n_links : 1));
        w.res = (double *)malloc(sizeof(double) * (size_t)(w.n_links ? w.n_links : 1));
        w.share = (double *)malloc(sizeof(double) * (size_t)(w.n_links ? w.n_links : 1));
        for (int e = 0; e < w.n_links; e++) w.bw[e] = tp->links[e].bw * bw_scale;

        int *state = (int *)calloc((size_t)(NN ? NN : 1), sizeof(int));
        double *t_end = (double *)calloc((size_t)(NN ? NN : 1), sizeof(double));
        double *t_act = (double *)calloc((size_t)(NN ? NN : 1), sizeof(double));
        double *rem = (double *)calloc((size_t)(NN ? NN : 1), sizeof(double));
        double *rate = (double *)calloc((size_t)(NN ? NN : 1), sizeof(double));
        double *t_upd = (double *)calloc((size_t)(NN ? NN : 1), sizeof(double));
        double *t_drain = (double *)calloc((size_t)(NN ? NN : 1), sizeof(double));
        char *has_dependents = (char *)calloc((size_t)(NN ? NN : 1), 1);
        for (long i = 0; i < NN; i++) has_dependents[i] = roff[i + 1] > roff[i];
        IVec ready = {0}, latent = {0}, active = {0};
        int *wf_flows = (int *)malloc(sizeof(int) * (size_t)(NN ? NN : 1));
        double *wf_rate = (double *)malloc(sizeof(double) * (size_t)(NN ? NN : 1));
        char *wf_unf = (char *)malloc((size_t)(NN ? NN : 1));
        for (long i = 0; i < NN; i++)
            if (pending[i] == 0 && G->n[i].type != N_TASK) { iv_push(&ready, (int)i); state[i] = S_QUEUED; }

        /* R20 photonic circuit-switched network: per source GPU `ports` directed logical
         * links {dst, state NONE/SETUP/UP, t = ready time (SETUP) or last use (UP)}; per flow a stage
         * REQ (released, no link) -> LINKQ (queued on a link) -> BUFW (link head, waiting for a receive
         * buffer at dst) -> XFER (delivered at t_drain).  Requests are ordered by (release time, code). */
        const OPhot *ph = tp->ph;
        const int PP_ = ph ? (int)ph->ports : 1;
        int *lk_dst = NULL, *lk_st = NULL, *ph_st = NULL, *ph_lk = NULL, *tmpf = NULL;
        double *lk_t = NULL;
        IVec phl = {0};
        double ph_setup = 0.0, ph_lat = 0.0, ph_bw = 1.0;
        if (ph) {
            lk_dst = (int *)malloc(sizeof(int) * (size_t)n_nodes_topo * PP_);
            lk_st = (int *)calloc((size_t)n_nodes_topo * PP_, sizeof(int));
            lk_t = (double *)calloc((size_t)n_nodes_topo * PP_, sizeof(double));
            ph_st = (int *)calloc((size_t)(NN ? NN : 1), sizeof(int));
            ph_lk = (int *)calloc((size_t)(NN ? NN : 1), sizeof(int));
            tmpf = (int *)malloc(sizeof(int) * (size_t)(NN ? NN : 1));
            for (long q = 0; q < (long)n_nodes_topo * PP_; q++) lk_dst[q] = -1;
            ph_setup = ph->setup_s * lat_scale;
            ph_lat = ph->lat_s * lat_scale;
            ph_bw = ph->link_bw * bw_scale;
        }
        enum { PS_NONE = 0, PS_REQ = 1, PS_LINKQ = 2, PS_BUFW = 3, PS_XFER = 4 };
#define PKEY_LT(a, b) (t_act[a] < t_act[b] || (t_act[a] == t_act[b] && G->n[a].code < G->n[b].code))

        long n_done = 0;
        double t = 0.0;
        uint64_t H = 0;
        uint64_t n_inst = 0, n_wf = 0, n_rounds = 0;
        uint32_t max_act = 0;
        int busy_on = 0;
        double busy_start = 0.0, comm_busy = 0.0;
        long inflight = 0;

#define COMPLETE(i)                                                          \
    do {                                                                     \
        state[i] = S_DONE; n_done++;                                         \
        if (t_done) t_done[i] = t;                                           \
        for (long _r = roff[i]; _r < roff[(i) + 1]; _r++) {                  \
            int _d = rlist[_r];                                              \
            if (--pending[_d] == 0 && G->n[_d].type != N_TASK) {             \
                iv_push(&ready, _d); state[_d] = S_QUEUED;                   \
            }                                                                \
        }                                                                    \
    } while (0)
/* R19: order hash = sum mod 2^64 over events of mix64(mix64(bits(t)) ^ (kind << 60 | code)) */
#define EVENT(kind, code) do { acc += mix64(tmix ^ (((uint64_t)(kind) << 60) | (code))); nev++; } while (0)

        for (;;) {
            uint64_t acc = 0;
            const uint64_t tmix = mix64(dbits(t));
            long nev = 0;
            int again;
            int dirty = 0;
            /* R20: logical links whose setup completes now are up (last use = now) */
            if (ph)
                for (long q = 0; q < (long)n_nodes_topo * PP_; q++)
                    if (lk_st[q] == 1 && lk_t[q] == t) lk_st[q] = 2;
            do {
                int changed;
                do {
                    changed = 0;
                    /* (a) compute completions */
                    for (int g = 0; g < n_nodes_topo; g++) {
                        int k = running[g];
                        if (k >= 0 && t_end[k] == t) {
                            COMPLETE(k);
                            if (has_dependents[k]) EVENT(EV_TASK_END, G->n[k].code);
                            running[g] = -1;
                            changed = 1;
                        }
                    }
                    /* (b) deliveries: push to the destination, notify the receiver */
                    for (long a = 0; a < active.n;) {
                        int f = active.v[a];
                        if (t_drain[f] == t) {
                            active.v[a] = active.v[--active.n];
                            COMPLETE(f);
                            EVENT(EV_DELIVER, G->n[f].code);
                            inflight--;
                            dirty = 1; changed = 1;
                        } else {
                            a++;
                        }
                    }
                    /* (b') photonic deliveries: the logical link was last used now (R20) */
                    for (long a = 0; a < phl.n;) {
                        int f = phl.v[a];
                        if (ph_st[f] == PS_XFER && t_drain[f] == t) {
                            phl.v[a] = phl.v[--phl.n];
                            ph_st[f] = PS_NONE;
                            lk_t[G->n[f].src * PP_ + ph_lk[f]] = t;
                            COMPLETE(f);
                            EVENT(EV_DELIVER, G->n[f].code);
                            inflight--;
                            changed = 1;
                        } else {
                            a++;
                        }
                    }
                    /* (c) activations after the route latency (reading Q19: latency first) */
                    for (long a = 0; a < latent.n;) {
                        int f = latent.v[a];
                        if (t_act[f] == t) {
                            latent.v[a] = latent.v[--latent.n];
                            EVENT(EV_ACTIVATE, G->n[f].code);
                            if (tl_a) tl_a[f] = t;
                            if (G->n[f].bytes == 0.0 || frlen[f] == 0) {
                                COMPLETE(f);
                                EVENT(EV_DELIVER, G->n[f].code);
                                inflight--;
                            } else {
                                state[f] = S_ACTIVE;
                                rem[f] = G->n[f].bytes; t_upd[f] = t; rate[f] = 0.0; t_drain[f] = INFINITY;
                                iv_push(&active, f);
                                dirty = 1;
                            }
                            changed = 1;
                        } else {
                            a++;
                        }
                    }
                    /* (d) dependency resolution: barriers fire, flows are released */
                    while (ready.n > 0) {
                        int k = ready.v[--ready.n];
                        if (G->n[k].type == N_BARRIER) {
                            COMPLETE(k);
                            if (G->n[k].flags & NF_COLL_START) EVENT(EV_COLL_START, G->n[k].code);
                        } else if (ph) {
                            /* R20: a send request; t_act holds its release time (the FIFO key) */
                            if (t_rel) t_rel[k] = t;
                            if (tl_s) tl_s[k] = t;
                            EVENT(EV_RELEASE, G->n[k].code);
                            inflight++;
                            if (G->n[k].src == G->n[k].dst) {
                                EVENT(EV_ACTIVATE, G->n[k].code);
                                if (tl_a) tl_a[k] = t;
                                COMPLETE(k);
                                EVENT(EV_DELIVER, G->n[k].code);
                                inflight--;
                            } else {
                                state[k] = S_LATENT;
                                t_act[k] = t;
                                ph_st[k] = PS_REQ;
                                iv_push(&phl, k);
                            }
                        } else {
                            state[k] = S_LATENT;
                            t_act[k] = t + lat[k];
                            if (t_rel) t_rel[k] = t;
                            if (tl_s) tl_s[k] = t;
                            EVENT(EV_RELEASE, G->n[k].code);
                            iv_push(&latent, k);
                            inflight++;
                        }
                        changed = 1;
                    }
                    /* (e) an idle GPU starts its head operator once its data is present */
                    for (int g = 0; g < n_nodes_topo; g++) {
                        if (running[g] >= 0 || head[g] >= qoff[g + 1] - qoff[g]) continue;
                        int k = qlist[qoff[g] + head[g]];
                        if (pending[k] > 0) continue;
                        running[g] = k; head[g]++;
                        state[k] = S_RUN;
                        t_end[k] = t + G->n[k].dur;
                        if (tl_s) tl_s[k] = t;
                        if (doff[k + 1] > doff[k]) EVENT(EV_TASK_START, G->n[k].code);
                        changed = 1;
                    }
                } while (changed);
                again = 0;
                if (ph) {
                    /* R20: (i) link per request: an existing link to dst, else a free port,
                     * else tear down the source's link idle the longest (ties: smaller dst), else wait */
                    for (int g = 0; g < n_nodes_topo; g++) {
                        int nr = 0;
                        for (long a = 0; a < phl.n; a++)
                            if (ph_st[phl.v[a]] == PS_REQ && G->n[phl.v[a]].src == g) tmpf[nr++] = phl.v[a];
                        for (int x = 1; x < nr; x++)   /* insertion sort by (release time, code) */
                            for (int y = x; y > 0 && PKEY_LT(tmpf[y], tmpf[y - 1]); y--) {
                                int sw = tmpf[y]; tmpf[y] = tmpf[y - 1]; tmpf[y - 1] = sw;
                            }
                        for (int x = 0; x < nr; x++) {
                            int f = tmpf[x], d = G->n[f].dst, k = -1;
                            for (int q = 0; q < PP_; q++) if (lk_st[g * PP_ + q] != 0 && lk_dst[g * PP_ + q] == d) k = q;
                            if (k < 0) {
                                int nk = -1;
                                for (int q = 0; q < PP_ && nk < 0; q++) if (lk_st[g * PP_ + q] == 0) nk = q;
                                if (nk < 0) {
                                    for (int q = 0; q < PP_; q++) {
                                        if (lk_st[g * PP_ + q] != 2) continue;
                                        int used = 0;
                                        for (long a = 0; a < phl.n && !used; a++) {
                                            int h = phl.v[a];
                                            if (G->n[h].src == g && ph_st[h] >= PS_LINKQ && ph_lk[h] == q) used = 1;
                                        }
                                        if (used) continue;
                                        if (nk < 0 || lk_t[g * PP_ + q] < lk_t[g * PP_ + nk] ||
                                            (lk_t[g * PP_ + q] == lk_t[g * PP_ + nk] && lk_dst[g * PP_ + q] < lk_dst[g * PP_ + nk]))
                                            nk = q;
                                    }
                                }
                                if (nk >= 0) {
                                    const double tr = t + ph_setup;
                                    lk_dst[g * PP_ + nk] = d;
                                    if (tr == t) { lk_st[g * PP_ + nk] = 2; lk_t[g * PP_ + nk] = t; }
                                    else { lk_st[g * PP_ + nk] = 1; lk_t[g * PP_ + nk] = tr; }
                                    k = nk;
                                }
                            }
                            if (k >= 0) { ph_st[f] = PS_LINKQ; ph_lk[f] = k; }
                        }
                    }
                    /* (ii) an up link with no transfer waiting or running passes its queue head on */
                    for (int g = 0; g < n_nodes_topo; g++)
                        for (int q = 0; q < PP_; q++) {
                            if (lk_st[g * PP_ + q] != 2) continue;
                            int busy = 0, head = -1;
                            for (long a = 0; a < phl.n; a++) {
                                int h = phl.v[a];
                                if (G->n[h].src != g || ph_lk[h] != q || ph_st[h] < PS_LINKQ) continue;
                                if (ph_st[h] >= PS_BUFW) busy = 1;
                                else if (head < 0 || PKEY_LT(h, head)) head = h;
                            }
                            if (!busy && head >= 0) ph_st[head] = PS_BUFW;
                        }
                    /* (iii) receive buffers at each destination, granted in (release time, code) order;
                     * a granted transfer owns the link's dedicated bandwidth: t + lat + bytes / bw */
                    int nx = 0;
                    for (int d = 0; d < n_nodes_topo; d++) {
                        int occ = 0, nc = 0;
                        for (long a = 0; a < phl.n; a++) {
                            int h = phl.v[a];
                            if (G->n[h].dst != d) continue;
                            if (ph_st[h] == PS_XFER) occ++;
                            else if (ph_st[h] == PS_BUFW) tmpf[nc++] = h;
                        }
                        for (int x = 1; x < nc; x++)
                            for (int y = x; y > 0 && PKEY_LT(tmpf[y], tmpf[y - 1]); y--) {
                                int sw = tmpf[y]; tmpf[y] = tmpf[y - 1]; tmpf[y - 1] = sw;
                            }
                        int fr = ph->buf_slots ? (int)ph->buf_slots - occ : nc;
                        for (int x = 0; x < nc && x < fr; x++) {
                            int f = tmpf[x];
                            ph_st[f] = PS_XFER;
                            t_drain[f] = (t + ph_lat) + G->n[f].bytes / ph_bw;
                            EVENT(EV_ACTIVATE, G->n[f].code);
                            if (tl_a) tl_a[f] = t;
                            if (t_drain[f] == t) again = 1;
                        }
                    }
                    for (long a = 0; a < phl.n; a++) if (ph_st[phl.v[a]] == PS_XFER) nx++;
                    if ((uint32_t)nx > max_act) max_act = (uint32_t)nx;
                }
                /* (f) re-allocate bandwidth of every in-transit flow */
                if (!ph && dirty) {
                    dirty = 0;
                    int nf = (int)active.n;
                    for (int a = 0; a < nf; a++) {
                        int f = active.v[a];
                        wf_flows[a] = f;
                        if (t_upd[f] < t) {
                            double r = rem[f] - rate[f] * (t - t_upd[f]);
                            rem[f] = r > 0.0 ? r : 0.0;
                            t_upd[f] = t;
                        }
                    }
                    n_rounds += (uint64_t)waterfill(&w, nf, wf_flows, froff, frlen, rpool.v, wf_rate, wf_unf);
                    n_wf++;
                    if ((uint32_t)nf > max_act) max_act = (uint32_t)nf;
                    for (int a = 0; a < nf; a++) {
                        int f = wf_flows[a];
                        rate[f] = wf_rate[a];
                        t_drain[f] = (rem[f] == 0.0) ? t : t + rem[f] / rate[f];
                        if (t_drain[f] == t) again = 1;
                    }
                }
            } while (again);

            if (nev > 0) { n_inst++; H = H + acc; }
            if (inflight > 0 && !busy_on) { busy_on = 1; busy_start = t; }
            else if (inflight == 0 && busy_on) { busy_on = 0; comm_busy = comm_busy + (t - busy_start); }
            if (n_done == NN) break;
            double tn = INFINITY;
            for (int g = 0; g < n_nodes_topo; g++) if (running[g] >= 0 && t_end[running[g]] < tn) tn = t_end[running[g]];
            for (long a = 0; a < latent.n; a++) if (t_act[latent.v[a]] < tn) tn = t_act[latent.v[a]];
            for (long a = 0; a < active.n; a++) if (t_drain[active.v[a]] < tn) tn = t_drain[active.v[a]];
            if (ph) {
                for (long a = 0; a < phl.n; a++) if (ph_st[phl.v[a]] == PS_XFER && t_drain[phl.v[a]] < tn) tn = t_drain[phl.v[a]];
                for (long q = 0; q < (long)n_nodes_topo * PP_; q++) if (lk_st[q] == 1 && lk_t[q] < tn) tn = lk_t[q];
            }
            if (!(tn < INFINITY)) { status = PT_DEADLOCK; break; }
            t = tn;
        }
#undef COMPLETE
#undef EVENT
#undef PKEY_LT
        if (status == PT_OK) {
            res->iter_time_s = t;
            res->compute_busy_max_s = cbmax;
            res->comm_busy_s = comm_busy;
            res->exposed_comm_s = t - cbmax;
            res->coll_payload_bytes = G->coll_payload;
            res->n_compute = (uint64_t)n_tasks;
            res->n_flows = (uint64_t)n_flows;
            res->n_collectives = (uint64_t)G->n_coll;
            res->n_p2p = (uint64_t)n_p2p;
            res->n_instants = n_inst;
            res->n_wf_calls = n_wf;
            res->n_wf_rounds = n_rounds;
            res->order_hash = H;
            res->max_active_flows = max_act;
            if (bd) {
                /* R22: compute = left fold of t' over the representative rank's op instances of the layer
                 * in program order; comm = (TP-group + DP-group collective time) + P2P time, each a left
                 * fold in creation order of (done on the rank - start) / (delivery - release) */
                int L = G->n_layers;
                double *acc3 = (double *)calloc((size_t)(3 * (L ? L : 1)), sizeof(double));
                for (int l = 0; l < L; l++) l_comp[l] = 0.0;
                for (long i = 0; i < NN; i++)
                    if (G->n[i].type == N_TASK && G->n[i].gpu == G->rep[G->n[i].layer])
                        l_comp[G->n[i].layer] = l_comp[G->n[i].layer] + G->n[i].dur;
                for (long r = 0; r < G->rc_s.n; r++) {
                    const int c = G->rc_c.v[r], l = G->rc_l.v[r], a0 = G->rc_s.v[r], a1 = G->rc_e.v[r];
                    const double d = t_done[a1] - (c == 2 ? t_rel[a0] : t_done[a0]);
                    acc3[c * L + l] = acc3[c * L + l] + d;
                }
                for (int l = 0; l < L; l++) l_comm[l] = (acc3[l] + acc3[L + l]) + acc3[2 * L + l];
                free(acc3);
            }
        }
        res->status = status;
        free(w.bw); free(w.n_e); free(w.k_e); free(w.res); free(w.share);
        free(state); free(t_end); free(t_act); free(rem); free(rate); free(t_upd); free(t_drain); free(has_dependents);
        iv_free(&ready); iv_free(&latent); iv_free(&active);
        free(wf_flows); free(wf_rate); free(wf_unf);
        free(lk_dst); free(lk_st); free(lk_t); free(ph_st); free(ph_lk); free(tmpf); iv_free(&phl);
    }
out:
    free(doff); free(roff); free(dlist); free(rlist); free(pending);
    free(qoff); free(qlist); free(head); free(running);
    free(froff); free(frlen); iv_free(&rpool); free(pair_off); free(pair_len); free(tmp); free(lat);
    free(t_rel); free(td_own);
    return 0;
}

/* ------------------------------------------------------------------ */
/* Public entry points (called through ctypes by tests / bench only)   */
/* ------------------------------------------------------------------ */
static int build_graph(const Trace *T, const Topo *tp, const uint32_t *ring_order, const uint32_t *plan,
                       uint32_t plan_len, int have_plan, const OPoint *pt, Graph *G, int *status) {
    *status = point_check(T, tp, pt, plan, plan_len, have_plan);
    if (*status != PT_OK) return 0;
    int *ro = (int *)malloc(sizeof(int) * tp->n_gpus);
    if (!ro) return -1;
    ring_order_of(ring_order, tp->n_gpus, ro);
    int rc = 0;
    /* R22: the representative rank of layer l = the lowest rank running it: rank 0 (DP/DDP/TP), the
     * stage's GPU (PP), rank (d=0, s(l), t=0) (HYBRID) */
    G->n_layers = (int)T->n_layers;
    G->rep = (int *)malloc(sizeof(int) * (T->n_layers ? T->n_layers : 1));
    if (!G->rep) { free(ro); return -1; }
    for (uint32_t l = 0; l < T->n_layers; l++) G->rep[l] = ro[0];
    G->cur_layer = -1;
    G->nch = pt->ring_chunks > 1 ? (int)pt->ring_chunks : 1;   /* R25 */
    switch (pt->strategy) {
    case ST_DP: case ST_DDP: rc = expand_dp(T, pt, ro, G); break;
    case ST_TP: rc = expand_tp(T, pt, ro, G); break;
    case ST_HOP: rc = expand_hop(T, pt, ro, G); break;
    case ST_PP: case ST_HYBRID: {
        uint32_t *fl = (uint32_t *)malloc(sizeof(uint32_t) * pt->pp);
        if (have_plan) memcpy(fl, plan, sizeof(uint32_t) * pt->pp);
        else if (auto_partition(T, pt->pp, fl)) { free(fl); free(ro); return -1; }
        for (uint32_t l = 0; l < T->n_layers; l++) {
            uint32_t st = 0;
            while (st + 1 < pt->pp && fl[st + 1] <= l) st++;
            G->rep[l] = ro[pt->strategy == ST_PP ? st : st * pt->tp];
        }
        rc = pt->strategy == ST_PP ? expand_pp(T, pt, ro, fl, G) : expand_hybrid(T, pt, ro, fl, G);
        free(fl);
        break;
    }
    default:
        *status = PT_BAD_CONFIG;
        break;
    }
    free(ro);
    return rc;
}

/* R23 timeline records: every compute task (its simulated GPU, program position, trace operator,
 * micro-batch, start and end) and every flow (code, endpoints, bytes, release, activation -- the
 * photonic grant --, delivery), tasks ordered by (gpu, prog), flows by (release, code) */
typedef struct { uint32_t gpu, prog, op, mb; double start, end; } OTaskRec;
typedef struct { uint64_t code; uint32_t src, dst; double bytes, release, start, delivered; } OFlowRec;

static int task_cmp(const void *a, const void *b) {
    const OTaskRec *x = (const OTaskRec *)a, *y = (const OTaskRec *)b;
    if (x->gpu != y->gpu) return x->gpu < y->gpu ? -1 : 1;
    return x->prog < y->prog ? -1 : x->prog > y->prog;
}
static int flow_cmp(const void *a, const void *b) {
    const OFlowRec *x = (const OFlowRec *)a, *y = (const OFlowRec *)b;
    if (x->release != y->release) return x->release < y->release ? -1 : 1;
    return x->code < y->code ? -1 : x->code > y->code;
}

int oracle_run_point(const OOp *ops, uint32_t n_ops, const OTensor *ts, uint32_t n_ts, const uint32_t *io,
                     uint32_t n_io, uint32_t trace_batch, uint32_t n_nodes, uint32_t n_gpus, const OLink *links,
                     uint32_t n_links, const uint32_t *ring_order, const uint32_t *plan, uint32_t plan_len,
                     int have_plan, const OPoint *pt, OResult *out, const OPhot *ph, double *l_comp,
                     double *l_comm, OTaskRec *tasks, int64_t task_cap, OFlowRec *flows, int64_t flow_cap,
                     int64_t *n_tasks, int64_t *n_flows) {
    Trace T = {ops, n_ops, ts, n_ts, io, n_io, trace_batch, NULL, 0};
    Topo tp; memset(&tp, 0, sizeof tp);
    int rc = trace_check(&T);
    if (rc == O_OK) rc = topo_init(&tp, n_nodes, n_gpus, links, n_links, ph);
    if (rc == O_OK && ring_order) {
        for (uint32_t i = 0; i < n_gpus; i++) {
            if (ring_order[i] >= n_gpus) rc = O_EINVAL;
            for (uint32_t j = 0; j < i; j++) if (ring_order[j] == ring_order[i]) rc = O_EINVAL;
        }
    }
    if (rc != O_OK) { free(T.prod); topo_free(&tp); return rc; }
    Graph G; memset(&G, 0, sizeof G);
    G.want_bd = l_comp != NULL && l_comm != NULL;
    int status = PT_OK;
    memset(out, 0, sizeof *out);
    if (l_comp) for (uint32_t l = 0; l < T.n_layers; l++) l_comp[l] = l_comm[l] = 0.0;
    if (n_tasks && n_flows) *n_tasks = *n_flows = 0;
    if (build_graph(&T, &tp, ring_order, plan, plan_len, have_plan, pt, &G, &status)) rc = O_ENOMEM;
    else if (status != PT_OK) out->status = status;
    else {
        double *t_done = NULL, *tl_s = NULL, *tl_a = NULL;
        const int tl = n_tasks != NULL && n_flows != NULL;
        if (tl) {
            const size_t nn = (size_t)(G.count ? G.count : 1);
            t_done = (double *)calloc(nn, sizeof(double));
            tl_s = (double *)calloc(nn, sizeof(double));
            tl_a = (double *)calloc(nn, sizeof(double));
            if (!t_done || !tl_s || !tl_a) rc = O_ENOMEM;
        }
        if (rc == O_OK && simulate(&G, &tp, pt->bw_scale, pt->lat_scale, out, t_done, l_comp, l_comm, tl_s, tl_a))
            rc = O_ENOMEM;
        if (rc == O_OK && tl && out->status == PT_OK) {
            int64_t nt = 0, nf = 0;
            for (long i = 0; i < G.count; i++) {
                const GNode *nd = &G.n[i];
                if (nd->type == N_TASK) {
                    if (tasks && nt < task_cap) {
                        OTaskRec r = {(uint32_t)nd->gpu, (uint32_t)(nd->code & ((1ull << 40) - 1)), (uint32_t)nd->op,
                                      (uint32_t)nd->mb, tl_s[i], t_done[i]};
                        tasks[nt] = r;
                    }
                    nt++;
                } else if (nd->type == N_FLOW) {
                    if (flows && nf < flow_cap) {
                        OFlowRec r = {nd->code, (uint32_t)nd->src, (uint32_t)nd->dst, nd->bytes, tl_s[i], tl_a[i], t_done[i]};
                        flows[nf] = r;
                    }
                    nf++;
                }
            }
            if (tasks && nt <= task_cap) qsort(tasks, (size_t)nt, sizeof(OTaskRec), task_cmp);
            if (flows && nf <= flow_cap) qsort(flows, (size_t)nf, sizeof(OFlowRec), flow_cmp);
            *n_tasks = nt;
            *n_flows = nf;
        } else if (tl) {
            *n_tasks = *n_flows = 0;
        }
        free(t_done); free(tl_s); free(tl_a);
    }
    g_free(&G); free(T.prod); topo_free(&tp);
    return rc;
}

/* Export the explicit task graph of one point (for the exact-rational re-simulation in
 * tests/).  Two calls: with arrays NULL to get the sizes, then with arrays to fill. */
int oracle_export_graph(const OOp *ops, uint32_t n_ops, const OTensor *ts, uint32_t n_ts, const uint32_t *io,
                        uint32_t n_io, uint32_t trace_batch, uint32_t n_nodes, uint32_t n_gpus, const OLink *links,
                        uint32_t n_links, const uint32_t *ring_order, const uint32_t *plan, uint32_t plan_len,
                        int have_plan, const OPoint *pt, int64_t *n_graph_nodes, int64_t *n_graph_deps,
                        int32_t *type, int32_t *gpu, double *dur, int32_t *src, int32_t *dst, double *bytes,
                        uint64_t *code, int32_t *flags, int64_t *dep_off, int32_t *dep_ids, int32_t *status) {
    Trace T = {ops, n_ops, ts, n_ts, io, n_io, trace_batch, NULL, 0};
    Topo tp; memset(&tp, 0, sizeof tp);
    int rc = trace_check(&T);
    if (rc == O_OK) rc = topo_init(&tp, n_nodes, n_gpus, links, n_links, NULL);
    if (rc != O_OK) { free(T.prod); topo_free(&tp); return rc; }
    Graph G; memset(&G, 0, sizeof G);
    int st = PT_OK;
    if (build_graph(&T, &tp, ring_order, plan, plan_len, have_plan, pt, &G, &st)) rc = O_ENOMEM;
    *status = st;
    *n_graph_nodes = G.count;
    *n_graph_deps = G.dep_from.n;
    if (rc == O_OK && type) {
        for (long i = 0; i < G.count; i++) {
            type[i] = G.n[i].type; gpu[i] = G.n[i].gpu; dur[i] = G.n[i].dur;
            src[i] = G.n[i].src; dst[i] = G.n[i].dst; bytes[i] = G.n[i].bytes;
            code[i] = G.n[i].code; flags[i] = G.n[i].flags;
        }
        for (long i = 0; i <= G.count; i++) dep_off[i] = 0;
        for (long e = 0; e < G.dep_from.n; e++) dep_off[G.dep_from.v[e] + 1]++;
        for (long i = 0; i < G.count; i++) dep_off[i + 1] += dep_off[i];
        int64_t *fill = (int64_t *)calloc((size_t)(G.count > 0 ? G.count : 0) + 1, sizeof(int64_t));
        for (long e = 0; e < G.dep_from.n; e++) {
            int a = G.dep_from.v[e];
            dep_ids[dep_off[a] + fill[a]++] = G.dep_to.v[e];
        }
        free(fill);
    }
    g_free(&G); free(T.prod); topo_free(&tp);
    return rc;
}

/* Simulate an explicit task graph given as arrays (same layout as the export). */
int oracle_sim_graph(int64_t n, const int32_t *type, const int32_t *gpu, const double *dur, const int32_t *src,
                     const int32_t *dst, const double *bytes, const uint64_t *code, const int32_t *flags,
                     const int64_t *dep_off, const int32_t *dep_ids, int32_t n_coll, double coll_payload,
                     uint32_t n_nodes, uint32_t n_gpus, const OLink *links, uint32_t n_links, double bw_scale,
                     double lat_scale, OResult *out, double *t_done, const OPhot *ph) {
    Topo tp; memset(&tp, 0, sizeof tp);
    int rc = topo_init(&tp, n_nodes, n_gpus, links, n_links, ph);
    if (rc != O_OK) { topo_free(&tp); return rc; }
    Graph G; memset(&G, 0, sizeof G);
    for (int64_t i = 0; i < n; i++) {
        GNode nd; memset(&nd, 0, sizeof nd);
        nd.type = type[i]; nd.gpu = gpu[i]; nd.dur = dur[i]; nd.src = src[i]; nd.dst = dst[i];
        nd.bytes = bytes[i]; nd.code = code[i]; nd.flags = flags[i];
        if (nd.type == N_TASK && (nd.gpu < 0 || (uint32_t)nd.gpu >= n_nodes)) { rc = O_EINVAL; break; }
        if (nd.type == N_FLOW && (nd.src < 0 || nd.dst < 0 || (uint32_t)nd.src >= n_nodes || (uint32_t)nd.dst >= n_nodes)) { rc = O_EINVAL; break; }
        if (g_add(&G, nd) < 0) { rc = O_ENOMEM; break; }
        for (int64_t q = dep_off[i]; q < dep_off[i + 1]; q++) {
            if (dep_ids[q] < 0 || dep_ids[q] >= n) { rc = O_EINVAL; break; }
            g_dep(&G, (int)i, dep_ids[q]);
        }
        if (rc) break;
    }
    G.n_coll = n_coll;
    G.coll_payload = coll_payload;
    if (rc == O_OK && simulate(&G, &tp, bw_scale, lat_scale, out, t_done, NULL, NULL, NULL, NULL)) rc = O_ENOMEM;
    g_free(&G); topo_free(&tp);
    return rc;
}

/* Standalone pieces for the pin tests */
int oracle_route(uint32_t n_nodes, uint32_t n_gpus, const OLink *links, uint32_t n_links, uint32_t src, uint32_t dst,
                 int32_t *out_links, int32_t cap) {
    Topo tp; memset(&tp, 0, sizeof tp);
    int rc = topo_init(&tp, n_nodes, n_gpus, links, n_links, NULL);
    if (rc != O_OK) { topo_free(&tp); return -100 + rc; }
    int *tmp = (int *)malloc(sizeof(int) * (size_t)(n_nodes + 1));
    int h = bfs_route(&tp, (int)src, (int)dst, tmp, (int)n_nodes);
    for (int k = 0; k < h && k < cap; k++) out_links[k] = tmp[k];
    free(tmp); topo_free(&tp);
    return h;
}

int64_t oracle_waterfill(int32_t n_links, const double *bw, int32_t n_flows, const int64_t *route_off,
                         const int32_t *route_len, const int32_t *route_links, double *rate_out) {
    WF w;
    w.n_links = n_links;
    w.bw = (double *)malloc(sizeof(double) * (size_t)(n_links ? n_links : 1));
    w.n_e = (int *)malloc(sizeof(int) * (size_t)(n_links ? n_links : 1));
    w.k_e = (int *)malloc(sizeof(int) * (size_t)(n_links ? n_links : 1));
    w.res = (double *)malloc(sizeof(double) * (size_t)(n_links ? n_links : 1));
    w.share = (double *)malloc(sizeof(double) * (size_t)(n_links ? n_links : 1));
    memcpy(w.bw, bw, sizeof(double) * (size_t)n_links);
    int *flows = (int *)malloc(sizeof(int) * (size_t)(n_flows ? n_flows : 1));
    long *roff = (long *)malloc(sizeof(long) * (size_t)(n_flows ? n_flows : 1));
    int *rlen = (int *)malloc(sizeof(int) * (size_t)(n_flows ? n_flows : 1));
    char *unf = (char *)malloc((size_t)(n_flows ? n_flows : 1));
    long tot = 0;
    for (int f = 0; f < n_flows; f++) { flows[f] = f; roff[f] = (long)route_off[f]; rlen[f] = route_len[f]; tot = roff[f] + rlen[f] > tot ? roff[f] + rlen[f] : tot; }
    int *rl = (int *)malloc(sizeof(int) * (size_t)(tot ? tot : 1));
    for (long q = 0; q < tot; q++) rl[q] = route_links[q];
    long rounds = waterfill(&w, n_flows, flows, roff, rlen, rl, rate_out, unf);
    free(w.bw); free(w.n_e); free(w.k_e); free(w.res); free(w.share);
    free(flows); free(roff); free(rlen); free(unf); free(rl);
    return rounds;
}

int oracle_partition(const OOp *ops, uint32_t n_ops, const OTensor *ts, uint32_t n_ts, const uint32_t *io,
                     uint32_t n_io, uint32_t trace_batch, uint32_t n_stages, uint32_t *first_layer) {
    Trace T = {ops, n_ops, ts, n_ts, io, n_io, trace_batch, NULL, 0};
    int rc = trace_check(&T);
    if (rc == O_OK) rc = auto_partition(&T, (int)n_stages, first_layer) ? O_EINVAL : O_OK;
    free(T.prod);
    return rc;
}

int oracle_check_trace(const OOp *ops, uint32_t n_ops, const OTensor *ts, uint32_t n_ts, const uint32_t *io,
                       uint32_t n_io, uint32_t trace_batch, uint32_t *n_layers) {
    Trace T = {ops, n_ops, ts, n_ts, io, n_io, trace_batch, NULL, 0};
    int rc = trace_check(&T);
    if (n_layers) *n_layers = T.n_layers;
    free(T.prod);
    return rc;
}
