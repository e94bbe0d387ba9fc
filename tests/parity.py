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
