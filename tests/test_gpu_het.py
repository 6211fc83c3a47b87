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


@pytest.mark.parametrize("kt,n,chunk,devices", [("u32", 3_000_001, 1 << 18, [0]), ("f32", 1_000_003, 100_000, [0, 0]),
                                                 ("u64", 600_001, 1 << 16, [0, 0, 0]), ("u32", 5, 1 << 20, [0])])
def test_het_out_of_core(kt, n, chunk, devices):
    """NEXT-4: more keys than the sorter's device budget (two chunk buffers of `chunk`
    keys per GPU): chunk groups sorted one after another with the 2n pipeline, then one CPU multiway
    merge of every sorted chunk into a separate buffer - equal to the oracle."""
    from baseline import het
    a = mi.np_generate(n, kt, "uniform", seed=6)
    h = torch.from_numpy(a.copy()).pin_memory()
    out = torch.empty_like(h)
    info = het.het_ooc_sort(h, kt, chunk, devices, out)
    assert info["chunks"] == -(-n // chunk)
    assert info["chunk_groups"] == -(-info["chunks"] // len(devices))
    assert np.array_equal(codec.bits_of(out.numpy(), kt), codec.bits_of(sort.oracle_sort(a, kt), kt))
