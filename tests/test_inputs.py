"""The seeded generators produce identical bytes in their numpy and torch forms
(so GPU-side generation at full size feeds the oracle the same input), are
deterministic, block-independent, and have the shapes DESIGN.md's recipe states."""
import numpy as np
import pytest
import torch

import msort_inputs as mi

CASES = [("u32", d) for d in mi.DISTRIBUTIONS] + [("u64", "uniform"), ("f32", "uniform"), ("f64", "uniform")]


@pytest.mark.parametrize("kt,dist", CASES)
def test_numpy_equals_torch(kt, dist):
    n = 70001
    a = mi.np_generate(n, kt, dist, seed=3)
    b = mi.t_generate(n, kt, dist, seed=3).numpy()
    assert a.dtype == b.dtype and np.array_equal(a.view(np.uint8), b.view(np.uint8))
    # block-independence: a slice generated alone equals the slice of the whole
    s = mi.np_generate(n, kt, dist, seed=3, start=1234, count=999)
    assert np.array_equal(s.view(np.uint8), a[1234:2233].view(np.uint8))
    out = torch.empty(n, dtype=mi.torch_dtype(kt))
    mi.t_generate_into(out, n, kt, dist, seed=3, block=4096)
    assert np.array_equal(out.numpy().view(np.uint8), a.view(np.uint8))


def test_distribution_shapes():
    n = 1 << 16
    s = mi.np_generate(n, "u32", "sorted")
    assert np.all(s[:-1] <= s[1:]) and s[0] == 0
    r = mi.np_generate(n, "u32", "reverse")
    assert np.all(r[:-1] >= r[1:])
    ns = mi.np_generate(n, "u32", "nearly")
    frac = np.mean(ns != s)
    assert 0.005 < frac < 0.02
    z = mi.np_generate(n, "u32", "zipf_rank")
    assert np.mean(z == 1) > 0.1                # heavy hitter
    nm = mi.np_generate(n, "u32", "normal").astype(np.float64)
    assert abs(nm.mean() - 2 ** 31) < 2 ** 29 * 0.05 and abs(nm.std() - 2 ** 29) < 2 ** 29 * 0.05
    f = mi.np_generate(n, "f32", "uniform")
    fin = f[np.isfinite(f)]
    assert np.mean(np.abs(fin) <= 1000) > 0.98
    assert 0.003 < np.mean(~np.isfinite(f)) < 0.01
    assert np.any(np.signbit(f) & (f == 0)) and np.any(~np.signbit(f) & (f == 0))
