"""GPU <-> oracle comparison rules:
bit-exact on status, counts, payload and the order hash; |gpu - ref| <= 1e-9 |ref| on times."""
import numpy as np

from paper_conf_isca_libwmvgjbj025_b200 import workloads as W

TIME_FIELDS = ("iter_time_s", "compute_busy_max_s", "comm_busy_s", "exposed_comm_s")
EXACT_FIELDS = ("status", "coll_payload_bytes", "n_compute", "n_flows", "n_collectives", "n_p2p", "n_instants",
                "n_wf_calls", "n_wf_rounds", "order_hash", "max_active_flows")
RTOL = 1e-9


def compare(got, ref, idx=None, allow_too_large=False):
    """Returns (list of mismatch strings, number of time fields that differ in the last bit)."""
    bad = []
    ulp = 0
    idx = range(len(ref)) if idx is None else idx
    for q, i in enumerate(idx):
        g, r = got[q], ref[q]
        if allow_too_large and g["status"] == W.PT_TOO_LARGE:
            continue
        for f in EXACT_FIELDS:
            if g[f] != r[f]:
                bad.append(f"point {i}: {f} gpu={g[f]} oracle={r[f]}")
        for f in TIME_FIELDS:
            a, b = float(g[f]), float(r[f])
            if abs(a - b) > RTOL * abs(b):
                bad.append(f"point {i}: {f} gpu={a!r} oracle={b!r}")
            elif a != b:
                ulp += 1
    return bad, ulp


def expected_too_large(sw):
    """Indices of the points the library documents as beyond its kernels (include/triosim.h
    TRIOSIM_PT_TOO_LARGE) that the oracle still simulates: tree / double-tree collectives over photonic
    links (for points that have a collective group) and double binary trees on HYBRID points with both a
    TP and a DP group."""
    P = sw.points
    phot = np.array([getattr(sw.topos[int(p["topo"])], "photonic", None) is not None if p["topo"] < len(sw.topos)
                     else False for p in P], bool)
    coll = np.where(P["strategy"] == W.ST_TP, P["tp"] > 1,
                    np.where(P["strategy"] == W.ST_HYBRID, (P["dp"] > 1) | (P["tp"] > 1),
                             np.where(P["strategy"] == W.ST_PP, False, P["dp"] > 1)))
    trees = (P["coll_algo"] == W.ALG_TREE) | (P["coll_algo"] == W.ALG_DBTREE)
    both = (P["strategy"] == W.ST_HYBRID) & (P["dp"] > 1) & (P["tp"] > 1) & (P["coll_algo"] == W.ALG_DBTREE)
    valid = P["strategy"] <= W.ST_HOP
    return np.flatnonzero(valid & ((phot & coll & trees) | both)).tolist()
