"""fp64 CPU oracle of the BTED hot path -- TEST INFRASTRUCTURE ONLY.

Only `tests/`, `__graft_entry__.smoke()` and `bench.py`'s `cpu_baseline` /
`--impl reference` legs may import, call, link or execute anything in this
package.  The product path (`paper_conf_date_sunbg021_b200/`) never does, and
shares no code with it: the two meet only through the seeded inputs of
`synth/` and through values compared in the tests.

Contents (each function cites the PAPER.md passage it follows):
  literal.py    numpy fp64 literal Algorithm 1 (TED) and Algorithm 2 (BTED)
  sampling.py   the counter-based batch sampler (Alg. 2 l.2), oracle side
  dense.py      ctypes loader for ted_dense.c (the same Algorithm 1 in plain
                C + OpenMP, fp64, for N up to the bench sizes)
  closed_form.py matrix-free fp64 evaluation of single scores after a given
                selected set (used to spot-check full-size runs)
"""
from .literal import gram_rbf, ted, bted, TedTrace  # noqa: F401
from .sampling import splitmix64, sample_batches  # noqa: F401
