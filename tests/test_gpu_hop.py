"""GPU parity of the Hop decentralized-training path (NEXT 4, R28): the CUDA kernel
(K3's HOP mode, through the C ABI) against the oracle point by point -- results, order hash and counts --
plus the R23 timeline and R22 breakdown of a few points."""
import numpy as np
import pytest

import oracle
from paper_conf_isca_libwmvgjbj025_b200 import workloads as W
from tests import sweeps as S
from tests.parity import compare

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def ctx():
    import torch
    assert torch.cuda.is_available()
    from paper_conf_isca_libwmvgjbj025_b200 import triosim
    c = triosim.Context(0)
    yield c
    c.close()


@pytest.mark.parametrize("seed", range(4))
def test_random_hop_points(ctx, seed):
    sw = S.random_hop(seed)
    got = ctx.run_sweep(sw)
    ref = oracle.run_sweep(sw)
    assert got["status"][-1] == W.PT_BAD_DEGREES
    assert (got["status"][:-1] == 0).all(), np.unique(got["status"], return_counts=True)
    bad, ulp = compare(got, ref)
    assert not bad, bad[:5]


def test_fig16_vgg11_eight_workers(ctx):
    """The paper's setting: VGG-class training on 8 workers, ring-based and double-ring graphs, 8
    random 1-10x slowdown groups, with and without one backup worker."""
    sw = W.sweep_hop()
    got = ctx.run_sweep(sw)
    ref = oracle.run_sweep(sw)
    assert (got["status"] == 0).all()
    bad, _ = compare(got, ref)
    assert not bad, bad[:5]


def test_hop_timeline(ctx):
    from tests.test_gpu_timeline import _check
    sw = S.random_hop(1)
    idx = [i for i in range(len(sw.points) - 1) if sw.points[i]["strategy"] == W.ST_HOP][:12]
    assert _check(ctx, sw, idx) == len(idx)


def test_hop_breakdown(ctx):
    from tests.test_gpu_breakdown import _check
    _check(ctx, S.random_hop(2))
