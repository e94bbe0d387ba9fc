"""Seeded random sweeps shared by the GPU parity tests (results and the R22 breakdown)."""
import numpy as np

from paper_conf_isca_libwmvgjbj025_b200 import workloads as W


def random_small(seed):
    rng = np.random.Generator(np.random.PCG64(500 + seed))
    tr = W.random_trace(rng, n_layers=int(rng.integers(3, 7)), max_ops_per_layer=4, b0=4)
    topos = [W.random_topology(rng, n_gpus=g, n_switch=int(rng.integers(0, 3)), p_edge=0.25)
             for g in (2, 3, 4, 5, 8, 12)]
    topos += [W.ring(16, 40e9, 1e-6), W.star(8, 80e9, 2e-6), W.mesh(2, 4, 60e9, 1e-6), W.cube_mesh8(50e9, 1e-6),
              W.double_ring(8, 30e9, 3e-6), W.perturb(W.ring_graph(8, 90e9, 1e-6), seed)]
    pts = []
    for _ in range(400):
        ti = int(rng.integers(len(topos)))
        G = topos[ti].n_gpus
        st = int(rng.integers(0, 4))
        bw, lat = float(rng.uniform(0.2, 3.0)), float(rng.uniform(0.0, 2.0))
        algo = int(rng.integers(0, 2))
        if st in (W.ST_DP, W.ST_DDP):
            dp = int(rng.integers(1, G + 1))
            pts.append(W.make_point(ti, st, dp=dp, B=dp * int(rng.integers(1, 9)), algo=algo, bw=bw, lat=lat,
                                    bucket=int(rng.choice([0, 1 << 10, 1 << 14, 1 << 30]))))
        elif st == W.ST_TP:
            tpd = int(rng.integers(1, G + 1))
            pts.append(W.make_point(ti, st, tp=tpd, B=int(rng.integers(1, 9)), algo=algo, bw=bw, lat=lat,
                                    tp_mode=int(rng.integers(0, 2))))
        else:
            pp = int(rng.integers(1, min(G, tr.n_layers) + 1))
            m = int(rng.integers(1, 6))
            pts.append(W.make_point(ti, st, pp=pp, m=m, B=m * int(rng.integers(1, 4)), bw=bw, lat=lat))
    sw = W.Sweep("rand", tr, topos, W.points_array(pts))
    return sw


def random_hybrid(seed):
    rng = np.random.Generator(np.random.PCG64(900 + seed))
    tr = W.random_trace(rng, n_layers=int(rng.integers(3, 7)), max_ops_per_layer=4, b0=2)
    topos = [W.random_topology(rng, n_gpus=g, n_switch=int(rng.integers(0, 3)), p_edge=0.2) for g in (4, 8, 12)]
    topos += [W.star(16, 50e9, 1e-6), W.mesh(4, 4, 40e9, 2e-6), W.perturb(W.cube_mesh8(60e9, 1e-6), seed)]
    pts = []
    for _ in range(250):
        ti = int(rng.integers(len(topos)))
        G = topos[ti].n_gpus
        while True:
            dp, tp, pp = (int(rng.integers(1, 5)), int(rng.choice([1, 2, 4])), int(rng.integers(1, 4)))
            if dp * tp * pp <= G and pp <= tr.n_layers:
                break
        m = int(rng.integers(1, 4))
        pts.append(W.make_point(ti, W.ST_HYBRID, dp=dp, tp=tp, pp=pp, m=m, B=dp * m * int(rng.integers(1, 3)),
                                bucket=int(rng.choice([0, 1 << 12, 1 << 30])), tp_mode=int(rng.integers(0, 2)),
                                algo=int(rng.integers(0, 2)), bw=float(rng.uniform(0.3, 3)), lat=float(rng.uniform(0, 2))))
    sw = W.Sweep("hyb", tr, topos, W.points_array(pts))
    return sw


def large_points(seed):
    rng = np.random.Generator(np.random.PCG64(1300 + seed))
    tr = W.transformer_trace("tiny-gpt", 8, 64, 4, 256, 16, 100, 2, 11 + seed)
    topos = [W.ring(64, 50e9, 1e-6), W.star(64, 80e9, 1e-6), W.hierarchical(8, 8, 1.0, 0.125, 2.0),
             W.perturb_subset(W.hierarchical(32, 8, 1.0, 0.125, 4.0), 7 + seed)]
    P = W.make_point
    pts = [P(0, W.ST_DDP, dp=64, B=128, bucket=1 << 14, bw=2e9, lat=1e-6),
           P(1, W.ST_DDP, dp=48, B=96, bucket=0, bw=5e9, lat=2e-6, algo=W.ALG_TREE),
           P(1, W.ST_TP, tp=64, B=4, tp_mode=W.TPM_MEGATRON),
           P(1, W.ST_TP, tp=48, B=4, tp_mode=W.TPM_PAPER, algo=W.ALG_TREE),
           P(2, W.ST_HYBRID, dp=4, tp=8, pp=2, m=4, B=16, bucket=1 << 16, bw=100e9, lat=1e-6),
           P(2, W.ST_HYBRID, dp=8, tp=4, pp=2, m=2, B=16, bucket=0, bw=100e9, lat=2e-6, tp_mode=W.TPM_PAPER),
           P(3, W.ST_HYBRID, dp=8, tp=8, pp=4, m=4, B=32, bucket=1 << 18, bw=300e9, lat=1e-6),
           P(3, W.ST_HYBRID, dp=16, tp=4, pp=4, m=2, B=32, bucket=1 << 18, bw=300e9, lat=1e-6, algo=W.ALG_TREE),
           P(3, W.ST_PP, pp=8, m=4, B=8, bw=300e9, lat=1e-6)]
    sw = W.Sweep("large", tr, topos, W.points_array(pts))
    return sw


def random_photonic(seed):
    rng = np.random.Generator(np.random.PCG64(1700 + seed))
    tr = W.random_trace(rng, n_layers=int(rng.integers(3, 7)), max_ops_per_layer=4, b0=2)
    topos = []
    for g in (2, 3, 4, 8, 12, 16, 40):
        topos.append(W.photonic(g, ports=int(rng.integers(1, 5)), link_bw=float(rng.uniform(5e9, 80e9)),
                                setup=float(rng.choice([0.0, 1e-5, 2e-4])), lat=float(rng.choice([0.0, 1e-6])),
                                buf_slots=int(rng.integers(0, 3)),
                                ring_order=rng.permutation(g).astype(np.uint32)))
    topos += [W.ring(8, 40e9, 1e-6), W.mesh(2, 4, 60e9, 1e-6)]
    pts = []
    P = W.make_point
    for _ in range(300):
        ti = int(rng.integers(len(topos)))
        G = topos[ti].n_gpus
        st = int(rng.integers(0, 5))
        bw, lat = float(rng.uniform(0.3, 3.0)), float(rng.uniform(0.0, 2.0))
        algo = int(rng.integers(0, 2))
        if st in (W.ST_DP, W.ST_DDP):
            dp = int(rng.integers(1, G + 1))
            pts.append(P(ti, st, dp=dp, B=dp * int(rng.integers(1, 5)), algo=algo, bw=bw, lat=lat,
                         bucket=int(rng.choice([0, 1 << 12, 1 << 30]))))
        elif st == W.ST_TP:
            pts.append(P(ti, st, tp=int(rng.integers(1, G + 1)), B=int(rng.integers(1, 5)), algo=algo, bw=bw,
                         lat=lat, tp_mode=int(rng.integers(0, 2))))
        elif st == W.ST_PP:
            m = int(rng.integers(1, 5))
            pts.append(P(ti, st, pp=int(rng.integers(1, min(G, tr.n_layers) + 1)), m=m, B=m * int(rng.integers(1, 3)),
                         bw=bw, lat=lat))
        else:
            while True:
                dp, tpd, pp = int(rng.integers(1, 4)), int(rng.choice([1, 2, 4])), int(rng.integers(1, 4))
                if dp * tpd * pp <= G and pp <= tr.n_layers:
                    break
            m = int(rng.integers(1, 3))
            pts.append(P(ti, W.ST_HYBRID, dp=dp, tp=tpd, pp=pp, m=m, B=dp * m, algo=algo, bw=bw, lat=lat,
                         tp_mode=int(rng.integers(0, 2)), bucket=int(rng.choice([0, 1 << 30]))))
    sw = W.Sweep("phot", tr, topos, W.points_array(pts))
    return sw


def random_chunked(seed):
    """R25 pipelined rings: every ring-collective strategy with 0-8 chunks per step on uniform rings (the
    K3 ring fast-forward), random asymmetric topologies, a photonic net and 48-64-rank points (CTA kernel)."""
    rng = np.random.Generator(np.random.PCG64(2500 + seed))
    tr = W.random_trace(rng, n_layers=int(rng.integers(3, 6)), max_ops_per_layer=3, b0=2)
    topos = [W.ring(8, 50e9, 1e-6), W.ring(16, 100e9, 2e-6), W.star(8, 80e9, 1e-6),
             W.random_topology(rng, n_gpus=6, n_switch=1, p_edge=0.3), W.perturb(W.ring_graph(8, 90e9, 1e-6), seed),
             W.photonic(8, ports=2, link_bw=40e9, setup=1e-5, lat=1e-6, buf_slots=1),
             W.ring(64, 50e9, 1e-6)]
    pts = []
    P = W.make_point
    for _ in range(240):
        ti = int(rng.integers(len(topos)))
        G = topos[ti].n_gpus
        st = int(rng.choice([W.ST_DP, W.ST_DDP, W.ST_TP, W.ST_HYBRID]))
        c = int(rng.integers(0, 9))
        bw, lat = float(rng.uniform(0.3, 3.0)), float(rng.uniform(0.0, 2.0))
        algo = int(rng.integers(0, 2)) if rng.random() < 0.3 else W.ALG_RING
        full = G == 64 or rng.random() < 0.5   # (on the 64-ring a partial ring closes over > 8 hops: R3 limit)
        if st in (W.ST_DP, W.ST_DDP):
            dp = G if full else int(rng.integers(2, G + 1))
            pts.append(P(ti, st, dp=dp, B=dp * 2, algo=algo, bw=bw, lat=lat, chunks=c,
                         bucket=int(rng.choice([0, 1 << 12, 1 << 30]))))
        elif st == W.ST_TP:
            tpd = G if full else int(rng.integers(2, G + 1))
            pts.append(P(ti, st, tp=tpd, B=2, algo=algo, bw=bw, lat=lat, chunks=c, tp_mode=int(rng.integers(0, 2))))
        else:
            while True:
                dp, tpd, pp = int(rng.integers(1, 5)), int(rng.choice([1, 2, 4])), int(rng.integers(1, 3))
                if dp * tpd * pp <= G and pp <= tr.n_layers:
                    break
            m = int(rng.integers(1, 3))
            pts.append(P(ti, st, dp=dp, tp=tpd, pp=pp, m=m, B=dp * m * 2, algo=algo, bw=bw, lat=lat, chunks=c,
                         bucket=int(rng.choice([0, 1 << 12, 1 << 30])), tp_mode=int(rng.integers(0, 2))))
    pts.append(P(0, W.ST_DDP, dp=8, B=16, chunks=17))   # R25 limit -> BAD_CONFIG
    return W.Sweep("chunked", tr, topos, W.points_array(pts))


def random_redbcast(seed):
    """R26 AllReduce as ring Reduce + ring Broadcast (0-6 chunks) for DP / DDP / TP / HYBRID on uniform and
    asymmetric rings, a star, random graphs, a photonic net and 64-rank points (CTA kernel)."""
    return _random_algo(seed, W.ALG_REDBCAST, 2600, "redbcast")


def random_rsag(seed):
    """R29 AllReduce as ring ReduceScatter + ring AllGather (0-6 chunks), the same mix as random_redbcast."""
    return _random_algo(seed, W.ALG_RSAG, 3600, "rsag")


def random_dbtree(seed):
    """R27 double binary tree AllReduce (chunks ignored) on the GPU, the same mix as random_redbcast."""
    return _random_algo(seed, W.ALG_DBTREE, 4600, "dbtree")


def _random_algo(seed, algo, base, name):
    rng = np.random.Generator(np.random.PCG64(base + seed))
    tr = W.random_trace(rng, n_layers=int(rng.integers(3, 6)), max_ops_per_layer=3, b0=2)
    topos = [W.ring(8, 50e9, 1e-6), W.ring(16, 100e9, 2e-6), W.star(8, 80e9, 1e-6),
             W.random_topology(rng, n_gpus=6, n_switch=1, p_edge=0.3), W.perturb(W.ring_graph(8, 90e9, 1e-6), seed),
             W.photonic(8, ports=2, link_bw=40e9, setup=1e-5, lat=1e-6, buf_slots=1),
             W.ring(64, 50e9, 1e-6)]
    pts = []
    P = W.make_point
    for _ in range(200):
        ti = int(rng.integers(len(topos)))
        G = topos[ti].n_gpus
        st = int(rng.choice([W.ST_DP, W.ST_DDP, W.ST_TP, W.ST_HYBRID]))
        c = int(rng.integers(0, 7))
        bw, lat = float(rng.uniform(0.3, 3.0)), float(rng.uniform(0.0, 2.0))
        full = G == 64 or rng.random() < 0.5
        kw = dict(algo=algo, bw=bw, lat=lat, chunks=c)
        if st in (W.ST_DP, W.ST_DDP):
            dp = G if full else int(rng.integers(1, G + 1))
            pts.append(P(ti, st, dp=dp, B=dp * 2, bucket=int(rng.choice([0, 1 << 12, 1 << 30])), **kw))
        elif st == W.ST_TP:
            tpd = G if full else int(rng.integers(1, G + 1))
            pts.append(P(ti, st, tp=tpd, B=2, tp_mode=int(rng.integers(0, 2)), **kw))
        else:
            while True:
                dp, tpd, pp = int(rng.integers(1, 5)), int(rng.choice([1, 2, 4])), int(rng.integers(1, 3))
                if dp * tpd * pp <= G and pp <= tr.n_layers:
                    break
            m = int(rng.integers(1, 3))
            pts.append(P(ti, st, dp=dp, tp=tpd, pp=pp, m=m, B=dp * m * 2, bucket=int(rng.choice([0, 1 << 12, 1 << 30])),
                         tp_mode=int(rng.integers(0, 2)), **kw))
    pts.append(P(0, W.ST_DDP, dp=8, B=16, algo=7))   # unknown algorithm -> BAD_CONFIG
    return W.Sweep(name, tr, topos, W.points_array(pts))


def random_hop(seed):
    """R28 Hop points: both Fig. 16a graphs, 2-32 workers, backup workers / staleness / iteration gap, on
    topologies with dedicated links (ring-based, double ring), shared links (star, mesh, random) and the
    paper's 1-10x per-GPU slowdowns, mixed with DDP points so both kernels' segments share warps;
    the last point is invalid (odd worker count)."""
    rng = np.random.Generator(np.random.PCG64(2100 + seed))
    tr = W.random_trace(rng, n_layers=int(rng.integers(2, 6)), max_ops_per_layer=3, b0=2)
    if not (tr.ops["phase"] == W.PH_OPT).any():
        tr = W.random_trace(np.random.Generator(np.random.PCG64(1)), n_layers=3, max_ops_per_layer=3, b0=2)

    def ident(t):
        return W.Topology(t.name, t.n_nodes, t.n_gpus, t.links.copy(), np.arange(t.n_gpus, dtype=np.uint32))

    def slow(t, s):
        r = np.random.Generator(np.random.PCG64(s))
        u = r.uniform(1.0, 10.0, t.n_nodes)
        t = ident(t)
        t.links["bw_Bps"] = t.links["bw_Bps"] / u[t.links["src"]]
        return t
    topos = [ident(W.ring_graph(8, 25e9, 2e-6)), ident(W.double_ring(8, 25e9, 2e-6)),
             slow(W.ring_graph(8, 25e9, 2e-6), seed), slow(W.double_ring(8, 25e9, 2e-6), seed + 7),
             W.star(8, 40e9, 1e-6), W.mesh(2, 4, 30e9, 1e-6), ident(W.ring_graph(16, 30e9, 1e-6)),
             W.star(32, 60e9, 1e-6), W.random_topology(rng, n_gpus=4, n_switch=1, p_edge=0.4),
             slow(W.ring_graph(4, 20e9, 3e-6), seed + 3)]
    pts = []
    for _ in range(300):
        ti = int(rng.integers(len(topos)))
        G = topos[ti].n_gpus
        bw, lat = float(rng.uniform(0.3, 3.0)), float(rng.uniform(0.0, 2.0))
        if rng.random() < 0.15:
            dp = int(rng.integers(1, G + 1))
            pts.append(W.make_point(ti, W.ST_DDP, dp=dp, B=dp * 2, bw=bw, lat=lat))
            continue
        graph = int(rng.integers(0, 2))
        cand = [n for n in (2, 4, 8, 16, 32) if n <= G and (graph == 0 or n % 4 == 0)]
        n = int(rng.choice(cand))
        K = int(rng.integers(1, 6))
        hop = (int(rng.integers(0, 3)), int(rng.integers(0, 3)), int(rng.choice([0, 0, 1, 2])))
        pts.append(W.make_point(ti, W.ST_HOP, dp=n, m=K, B=n * int(rng.integers(1, 4)), tp_mode=graph, bw=bw,
                                lat=lat, hop=hop))
    pts.append(W.make_point(0, W.ST_HOP, dp=7, m=2, B=7))
    return W.Sweep("rand_hop", tr, topos, W.points_array(pts))
