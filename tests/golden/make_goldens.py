"""Write the oracle's result records for whole sweeps (tests/golden/<name>.npz), the expected values of the
full-sweep GPU parity tests (tests/test_gpu_golden.py; every point of C1-C3, >= 10k of C4,
>= 100 of C5).  Calls only oracle/ (and the seeded input generators of workloads.py); nothing here comes
from the CUDA path.  Each file stores the sweep's point indices, the records and a SHA-256 of the sweep's
trace / topology / point bytes, so a test can prove it rebuilt the same inputs.

    python tests/golden/make_goldens.py [c1 c2 c3 c4 c5] [--procs N]
"""
from __future__ import annotations

import argparse
import hashlib
import multiprocessing as mp
import os
import sys
import time

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(os.path.dirname(HERE))
sys.path.insert(0, ROOT)

from paper_conf_isca_libwmvgjbj025_b200 import workloads as W  # noqa: E402

_SW = {}


def c5_sample():
    """>= 100 configs[4] points stratified by simulated GPU count N: per N, the
    heaviest structural classes by estimated work -- the largest dp x tp with the most micro-batches, on
    the perturbed (slow-link subset) topology at the highest oversubscription -- plus seeded random
    points; bandwidth / latency from the full axes."""
    return W.sweep_c5_parity()


SWEEPS = {"c1": W.sweep_c1, "c2": W.sweep_c2, "c3": W.sweep_c3, "c4": W.sweep_c4, "c5": c5_sample}


def sweep_digest(sw) -> str:
    h = hashlib.sha256()
    for a in (sw.trace.ops, sw.trace.tensors, sw.trace.io, sw.points):
        h.update(np.ascontiguousarray(a).tobytes())
    for t in sw.topos:
        h.update(np.ascontiguousarray(t.links).tobytes())
        h.update(np.ascontiguousarray(t.ring_order).tobytes())
        ph = getattr(t, "photonic", None)
        if ph is not None:
            h.update(np.asarray(ph).tobytes())
    for p in sw.plans or []:
        h.update(np.asarray(p, np.uint32).tobytes())
    return h.hexdigest()


def _work(args):
    name, idx = args
    import oracle
    if name not in _SW:
        _SW[name] = SWEEPS[name]()
    t0 = time.perf_counter()
    r = oracle.run_sweep(_SW[name], idx)
    return idx, r, time.perf_counter() - t0


def make(name, procs):
    import oracle
    oracle.build()
    sw = SWEEPS[name]()
    n = len(sw.points)
    # small chunks, heaviest-looking first (interleaved) so the pool stays busy to the end
    chunk = 1 if name == "c5" else 16
    chunks = [list(range(a, min(n, a + chunk))) for a in range(0, n, chunk)]
    rec = np.zeros(n, W.RESULT_DTYPE)
    secs = np.zeros(n)
    t0 = time.perf_counter()
    with mp.get_context("spawn").Pool(procs) as pool:
        for k, (idx, r, dt) in enumerate(pool.imap_unordered(_work, [(name, c) for c in chunks])):
            rec[idx] = r
            secs[idx] = dt / len(idx)
            if name == "c5":
                print(f"  {name} point {idx[0]}: {dt:.1f} s, {int(r['n_instants'][0])} instants", flush=True)
    out = os.path.join(HERE, f"{name}.npz")
    np.savez_compressed(out, records=rec.view(np.uint8), n=n, digest=sweep_digest(sw), oracle_s=secs)
    print(f"{name}: {n} points in {time.perf_counter() - t0:.1f} s -> {out} "
          f"({os.path.getsize(out)} B); statuses {np.bincount(rec['status'])}", flush=True)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("names", nargs="*", default=["c1", "c2", "c3", "c4"])
    ap.add_argument("--procs", type=int, default=os.cpu_count() or 1)
    a = ap.parse_args()
    for name in a.names:
        make(name, a.procs)


if __name__ == "__main__":
    main()
