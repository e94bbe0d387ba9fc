"""Write the oracle's result records for whole sweeps (tests/golden/<name>.npz), the expected values of the
full-sweep GPU parity tests (tests/test_gpu_golden.py; every point of C1-C3, >= 10k of C4,
>= 100 of C5).  Calls only oracle/ (and the seeded input generators of workloads.py); nothing here comes
from the CUDA path.  Each file stores the sweep's point indices, the records and a SHA-256 of the sweep's
trace / topology / point bytes, so a test can prove it rebuilt the same inputs.

    python tests/golden/make_goldens.py [c1 c2 c3 c4 c5] [--procs N]
    python tests/golden/make_goldens.py c5 --finalize-partial   (while a long run is still going)

--finalize-partial writes <name>.npz from the points the (still running) oracle has finished so far, with a
boolean `have` mask; the GPU test compares exactly those points and names the rest.  A finished run
overwrites the file with every record (no mask).
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
    ops = np.array(sw.trace.ops, copy=True)
    ops["kind"] = 0   # informational operator-name ids, numbered in first-use order per process
    for a in (ops, sw.trace.tensors, sw.trace.io, sw.points):
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
    # resumable: finished points are appended to <name>.partial (point bytes -> record), reused on a rerun
    part = os.path.join(HERE, f"{name}.partial.npz")
    cache = {}
    if os.path.exists(part):
        z = np.load(part)
        for pb, rb, sc in zip(z["points"], z["records"], z["secs"]):
            cache[pb.tobytes()] = (rb, float(sc))
    todo = []
    for c in chunks:
        hit = [cache.get(sw.points[i].tobytes()) for i in c]
        if all(h is not None for h in hit):
            for i, h in zip(c, hit):
                rec[i] = h[0].view(W.RESULT_DTYPE)[0]
                secs[i] = h[1]
        else:
            todo.append(c)
    if name == "c5":   # the heaviest-looking first, so the long points start at once
        todo.sort(key=lambda c: -float(sw.points[c[0]]["dp"]) * float(sw.points[c[0]]["tp"]) * float(sw.points[c[0]]["pp"]))

    def save_partial():
        done = [i for i in range(n) if secs[i] > 0 or rec[i]["status"] != 0 or rec[i]["n_instants"] > 0]
        np.savez(part, points=sw.points[done].view(np.uint8).reshape(len(done), -1),
                 records=rec[done].view(np.uint8).reshape(len(done), -1), secs=secs[done])
    t0 = time.perf_counter()
    with mp.get_context("spawn").Pool(procs) as pool:
        for k, (idx, r, dt) in enumerate(pool.imap_unordered(_work, [(name, c) for c in todo])):
            rec[idx] = r
            secs[idx] = max(dt / len(idx), 1e-9)
            if name == "c5":
                print(f"  {name} point {idx[0]}: {dt:.1f} s, {int(r['n_instants'][0])} instants", flush=True)
                save_partial()
    out = os.path.join(HERE, f"{name}.npz")
    np.savez_compressed(out, records=rec.view(np.uint8), n=n, digest=sweep_digest(sw), oracle_s=secs)
    if os.path.exists(part):
        os.remove(part)
    print(f"{name}: {n} points in {time.perf_counter() - t0:.1f} s -> {out} "
          f"({os.path.getsize(out)} B); statuses {np.bincount(rec['status'])}", flush=True)


def finalize_partial(name, where=HERE):
    """<name>.npz from <name>.partial.npz (both in `where`): the finished points' oracle records plus the
    `have` mask."""
    sw = SWEEPS[name]()
    n = len(sw.points)
    z = np.load(os.path.join(where, f"{name}.partial.npz"))
    cache = {pb.tobytes(): (rb, float(sc)) for pb, rb, sc in zip(z["points"], z["records"], z["secs"])}
    rec = np.zeros(n, W.RESULT_DTYPE)
    secs = np.zeros(n)
    have = np.zeros(n, bool)
    for i in range(n):
        h = cache.get(sw.points[i].tobytes())
        if h is not None:
            rec[i] = h[0].view(W.RESULT_DTYPE)[0]
            secs[i] = h[1]
            have[i] = True
    out = os.path.join(where, f"{name}.npz")
    np.savez_compressed(out, records=rec.view(np.uint8), n=n, digest=sweep_digest(sw), oracle_s=secs, have=have)
    return out
    print(f"{name}: {int(have.sum())} of {n} points finished by the oracle -> {out}; pending: "
          f"{np.flatnonzero(~have).tolist()}", flush=True)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("names", nargs="*", default=["c1", "c2", "c3", "c4"])
    ap.add_argument("--procs", type=int, default=os.cpu_count() or 1)
    ap.add_argument("--finalize-partial", action="store_true")
    a = ap.parse_args()
    for name in a.names:
        if a.finalize_partial:
            finalize_partial(name)
        else:
            make(name, a.procs)


if __name__ == "__main__":
    main()
