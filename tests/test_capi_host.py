"""C-ABI library loads on a CPU-only host, exports every symbol include/msort.h
declares, and its host-only plan functions (Alg.2 schedule, reading Q6 swap
mapping) agree with the oracle's stage model.  No compute calls (no GPU)."""
import ctypes
import os
import re

import numpy as np
import pytest

from oracle import p2p

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _declared():
    with open(os.path.join(ROOT, "include", "msort.h")) as f:
        src = f.read()
    return sorted(set(re.findall(r"^\s*(?:int|uint64_t|const char\*)\s+(msort_\w+)\s*\(", src, re.M)))


def test_library_exports_every_declared_symbol():
    import paper_conf_sigmod_maltenbergeritr22_b200 as m
    lib = ctypes.CDLL(m.LIB_PATH)
    names = _declared()
    assert len(names) >= 20
    for nm in names:
        assert hasattr(lib, nm), nm
    assert sorted(m.EXPORTED) == names


def test_status_strings_and_errors_without_gpu():
    import paper_conf_sigmod_maltenbergeritr22_b200 as m
    assert m._lib.msort_status_string(0) == b"MSORT_OK"
    with pytest.raises(m.MsortError):
        m.msort_sort(1234, 10, "u32", 3)          # n_gpus not a power of two
    with pytest.raises(m.MsortError):
        m.msort_sort(1234, 10, 7, 1)              # bad key type
    m.msort_sort(0, 1, "u32", 1)                  # n <= 1: no-op


@pytest.mark.parametrize("g", [2, 4, 8])
def test_plan_matches_oracle_stage_model(g):
    import paper_conf_sigmod_maltenbergeritr22_b200 as m
    assert m.msort_plan_num_stages(g) == g - 1
    assert [m.msort_plan_stage(g, s) for s in range(g - 1)] == p2p.stage_labels(g)
    rng = np.random.default_rng(g)
    for trial in range(200):
        c = int(rng.integers(1, 6))
        data = rng.integers(0, 3 * g * c, g * c).astype(np.uint32)
        chunks = [np.sort(data[i * c:(i + 1) * c]) for i in range(g)]
        stages = p2p.run_stages(chunks)
        for s, st in enumerate(stages):
            partner, x, side = m.msort_plan_exchange(g, s, c, [op.p for op in st])
            for op in st:
                mid = op.lo + (op.hi - op.lo) // 2
                for d, xd in enumerate(op.xs):
                    L, R = mid - 1 - d, mid + d
                    assert partner[L] == R and partner[R] == L
                    assert x[L] == x[R] == xd
                    assert side[L] == 0 and side[R] == 1
