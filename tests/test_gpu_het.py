"""HET sort baseline (comparison leg of bench.py): GPU chunk sort + CPU
multiway merge must equal the oracle too."""
import numpy as np
import pytest
import torch

import msort_inputs as mi
from oracle import codec, sort

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("kt,chunks", [("u32", 8), ("f32", 4), ("u64", 3)])
def test_het_sort(kt, chunks):
    from baseline import het
    n = 300_007
    a = mi.np_generate(n, kt, "uniform", seed=4)
    h = torch.from_numpy(a.copy()).pin_memory()
    info = het.het_sort_host(h, kt, chunks=chunks)
    assert info["chunks"] == chunks
    assert np.array_equal(codec.bits_of(h.numpy(), kt), codec.bits_of(sort.oracle_sort(a, kt), kt))
