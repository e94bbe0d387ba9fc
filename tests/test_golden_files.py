"""The stored oracle goldens (tests/golden/*.npz) on CPU: each file still matches the seeded generator's sweep
(SHA-256 of its inputs), has one record per point, and the C5 file is complete; plus the partial-run finaliser
of make_goldens (availability mask) on a synthetic partial file."""
import os
import sys

import numpy as np
import pytest

from paper_conf_isca_libwmvgjbj025_b200 import workloads as W

HERE = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, os.path.join(HERE, "golden"))
import make_goldens as G  # noqa: E402


@pytest.mark.parametrize("name", ["c1", "c2", "c3", "c4", "c5"])
def test_golden_file_matches_generator(name):
    z = np.load(os.path.join(HERE, "golden", f"{name}.npz"))
    sw = G.SWEEPS[name]()
    assert str(z["digest"]) == G.sweep_digest(sw)
    rec = z["records"].view(W.RESULT_DTYPE)
    assert len(rec) == len(sw.points) == int(z["n"])
    if "have" in z.files:
        assert z["have"].shape == (len(rec),)
    else:   # a complete run: every point simulated (the oracle has no kernel limits)
        assert (rec["status"] != W.PT_TOO_LARGE).all()
        assert (rec["n_instants"][rec["status"] == 0] > 0).all()


def test_finalize_partial_mask(tmp_path):
    sw = G.SWEEPS["c1"]()
    done = [1]
    fake = np.zeros(len(done), W.RESULT_DTYPE)
    fake["n_instants"] = 7
    np.savez(tmp_path / "c1.partial.npz", points=sw.points[done].view(np.uint8).reshape(len(done), -1),
             records=fake.view(np.uint8).reshape(len(done), -1), secs=np.ones(len(done)))
    out = G.finalize_partial("c1", str(tmp_path))
    z = np.load(out)
    assert z["have"].tolist() == [i in done for i in range(len(sw.points))]
    assert z["records"].view(W.RESULT_DTYPE)["n_instants"].tolist() == [7 if i in done else 0 for i in range(len(sw.points))]
