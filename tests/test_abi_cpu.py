"""CPU-side checks of the boundary: the C-ABI library builds for sm_100a, loads, exports
every entry point include/triosim.h declares, and refuses to run without a B200 (no CPU
fallback).  No compute call is made here."""
import ctypes as C
import os
import re

import numpy as np
import pytest

from paper_conf_isca_libwmvgjbj025_b200 import build, triosim, workloads as W

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def declared():
    src = open(os.path.join(ROOT, "include", "triosim.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    src = re.sub(r"//[^\n]*", "", src)
    return sorted(set(re.findall(r"\b(triosim_[a-z_]+)\s*\(", src)) - {"triosim_status"})


@pytest.fixture(scope="module")
def lib():
    build.build()
    return triosim.load_library()


def test_exports_every_declared_symbol(lib):
    names = declared()
    assert len(names) >= 10
    for n in names:
        assert hasattr(lib, n), n
    assert set(triosim.EXPORTS) == set(names)


def test_record_sizes_match_header():
    src = open(os.path.join(ROOT, "include", "triosim.h")).read()
    sizes = dict(re.findall(r"sizeof\((triosim_\w+)\) == (\d+)", src))
    assert int(sizes["triosim_op"]) == W.OP_DTYPE.itemsize
    assert int(sizes["triosim_tensor"]) == W.TENSOR_DTYPE.itemsize
    assert int(sizes["triosim_link"]) == W.LINK_DTYPE.itemsize
    assert int(sizes["triosim_point"]) == W.POINT_DTYPE.itemsize
    assert int(sizes["triosim_result"]) == W.RESULT_DTYPE.itemsize


def test_no_gpu_means_loud_failure(lib):
    import torch
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    with pytest.raises(triosim.TrioSimError) as e:
        triosim.Context(0)
    assert e.value.status == -6  # TRIOSIM_EUNSUPPORTED


def test_sass_is_sm100a(lib):
    import subprocess
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", build.OUT], capture_output=True, text=True)
    assert "sm_100a" in out.stdout


def test_product_never_imports_oracle():
    pkg = os.path.join(ROOT, "paper_conf_isca_libwmvgjbj025_b200")
    for dp, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".h", ".cpp")):
                s = open(os.path.join(dp, f)).read()
                assert "import oracle" not in s and "from oracle" not in s and "triosim_oracle" not in s, f


# ---------------- the product's automatic stage plan (R8), host-only ----------------
def _brute_force_plan(tr, S):
    """Every composition of the layers into S contiguous non-empty stages; the smallest max stage cost
    (left fold of per-layer sums of trace times), ties -> the lexicographically smallest first layers."""
    import itertools
    L = int(tr.n_layers)
    lc = [0.0] * L
    for op in tr.ops:
        lc[int(op["layer"])] = lc[int(op["layer"])] + float(op["time_s"])
    best = None
    for cut in itertools.combinations(range(1, L), S - 1):
        b = (0,) + cut + (L,)
        worst = 0.0
        for k in range(S):
            c = 0.0
            for l in range(b[k], b[k + 1]):
                c = c + lc[l]
            worst = max(worst, c)
        key = (worst, b[:-1])
        if best is None or key < best:
            best = key
    return list(best[1])


@pytest.mark.parametrize("seed", range(12))
def test_stage_partition_matches_exhaustive_search(lib, seed):
    rng = np.random.Generator(np.random.PCG64(100 + seed))
    tr = W.random_trace(rng, n_layers=int(rng.integers(2, 10)))
    if seed % 3 == 0:   # ties: equal layer costs
        tr.ops["time_s"] = 2.0 ** -10
    for S in range(1, int(tr.n_layers) + 1):
        assert triosim.triosim_stage_partition(tr, S) == _brute_force_plan(tr, S), (seed, S)


def test_stage_partition_rejects_bad_arguments(lib):
    tr = W.mlp_trace()
    with pytest.raises(triosim.TrioSimError):
        triosim.triosim_stage_partition(tr, 0)
    with pytest.raises(triosim.TrioSimError):
        triosim.triosim_stage_partition(tr, int(tr.n_layers) + 1)
