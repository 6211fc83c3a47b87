"""CPU oracle for the multi-GPU P2P sort hot path (Maltenberger et al., SIGMOD '22).

TEST INFRASTRUCTURE ONLY.  Only `tests/`, `__graft_entry__.smoke()` and the
`cpu_baseline` / `--impl reference` legs of `bench.py` may import anything in
this package.  The product (`paper_conf_sigmod_maltenbergeritr22_b200`) never
imports it, and this package never imports the product: the two share no code.
The only shared module is `msort_inputs` (seeded generators, no method
arithmetic).

Plain, slow, obviously-correct numpy / pure-Python code, each function citing
the PAPER.md passage it follows (`P:n` = line n of /root/reference/PAPER.md,
see DESIGN.md "Citations").  Pins against the paper and against mathematics
live in tests/test_oracle_*.py and tests/golden/.

Modules:
  codec   - key bit transform T / T^-1 (total order of floats; DESIGN reading Q1)
  sort    - the plain definition of the result: sorted multiset under T
  radix   - digit histograms and stable counting passes (LSD radix, §5.1)
  p2p     - Alg.1 pivot selection, swap, local merge, Alg.2 merge phase (§5.2)
  checks  - properties that hold at any size (sortedness, permutation,
            sampled order statistics) for full-size parity
"""
from . import codec, sort, radix, p2p, checks  # noqa: F401
