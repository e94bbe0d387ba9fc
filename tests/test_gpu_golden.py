"""Full-sweep GPU parity: EVERY point of configs[0..3] (C1 2, C2 10,000, C3 9,216,
C4 9,600) and the stratified configs[4] parity sample (100 points, 20 per N), simulated by the CUDA path
through the C ABI in the launch configuration bench.py times (one simulate_batch over the whole sweep /
N range), compared element by element with the oracle's records written by tests/golden/make_goldens.py
(which calls only oracle/).

Bit-exact on status, counts, payload and order hash; |gpu - oracle| <= 1e-9 |oracle| on times.  No
point may come back PT_TOO_LARGE (the oracle has no kernel limits; the expected list is empty).
"""
import os
import sys

import numpy as np
import pytest

from paper_conf_isca_libwmvgjbj025_b200 import workloads as W
from tests.parity import compare

HERE = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, os.path.join(HERE, "golden"))
import make_goldens as G  # noqa: E402

pytestmark = pytest.mark.gpu

EXPECTED_TOO_LARGE = {"c1": [], "c2": [], "c3": [], "c4": [], "c5": []}


@pytest.fixture(scope="module")
def ctx():
    import torch
    assert torch.cuda.is_available()
    from paper_conf_isca_libwmvgjbj025_b200 import triosim
    c = triosim.Context(0)
    yield c
    c.close()


def load(name):
    path = os.path.join(HERE, "golden", f"{name}.npz")
    if not os.path.exists(path):
        pytest.fail(f"missing golden file {path}: run tests/golden/make_goldens.py {name}")
    z = np.load(path)
    have = z["have"] if "have" in z.files else np.ones(int(z["n"]), bool)
    return z["records"].view(W.RESULT_DTYPE), str(z["digest"]), have


def _compare_full(ctx, name, select=None):
    ref, digest, have = load(name)
    sw = G.SWEEPS[name]()
    assert G.sweep_digest(sw) == digest, "the seeded generator no longer reproduces the golden sweep"
    assert len(ref) == len(sw.points)
    sel = np.ones(len(sw.points), bool) if select is None else np.asarray(select(sw.points), bool)
    pending = np.flatnonzero(sel & ~have).tolist()
    if pending:   # points the oracle had not finished when the file was written (make_goldens --finalize-partial)
        print(f"{name}: no oracle record yet for points {pending}; compared the other {int((sel & have).sum())}")
    idx = np.flatnonzero(sel & have)
    sub = W.Sweep(sw.name, sw.trace, sw.topos, sw.points[idx], sw.plans)
    got = ctx.run_sweep(sub)
    too_large = np.flatnonzero(got["status"] == W.PT_TOO_LARGE).tolist()
    assert too_large == EXPECTED_TOO_LARGE[name]
    bad, ulp = compare(got, ref[idx], idx)
    assert not bad, f"{len(bad)} mismatches, first: {bad[:5]}"
    print(f"{name}: {len(idx)} points bit-exact on counts/hash, {ulp} time fields differ in the last bits")


@pytest.mark.parametrize("name", ["c1", "c2", "c3", "c4"])
def test_full_sweep_matches_oracle(ctx, name):
    _compare_full(ctx, name)


def _n_of(P):
    return P["dp"].astype(np.int64) * P["tp"] * P["pp"]


def test_c5_sample_up_to_256_gpus(ctx):
    """The configs[4] sample's 60 points on 64-256 simulated GPUs, incl. the dp x tp = 64 heavy class
    (5.3M instants and up to 1.4e8 water-filling rounds per point); ~5 min on one B200."""
    _compare_full(ctx, "c5", lambda P: _n_of(P) <= 256)


@pytest.mark.skipif(os.environ.get("TS_C5_FULL") != "1",
                    reason="the 512/1024-GPU half of the C5 sample runs tens of minutes on one GPU: TS_C5_FULL=1 "
                           "(run for the record in profiles/r2_c5_golden_large.log)")
def test_c5_sample_512_and_1024_gpus(ctx):
    _compare_full(ctx, "c5", lambda P: _n_of(P) >= 512)
