"""Mutation check of the oracle pins, run as part of the CPU suite (VERDICT r1
"next" 1(c)).  Every mutant of tools/oracle_mutations.py -- one plausible
mistake in oracle/pf_oracle.c, built from a temporary copy -- must make at
least one of its pins fail; mutants listed as equivalent are skipped.  This
is what makes "the oracle is pinned" checkable: a pin set that a dropped
term, a wrong sign or index, or a wrong reading (A5 tau interpolation, A15
Dirichlet ghost, A16 inflow) survives is not a pin set."""
import concurrent.futures as cf
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, os.path.join(ROOT, "tools"))

import oracle_mutations as OM  # noqa: E402


def test_every_oracle_mutant_is_caught():
    idx = [i for i, m in enumerate(OM.MUTANTS) if m[2] is not None]
    with cf.ThreadPoolExecutor(min(8, os.cpu_count() or 1)) as ex:
        res = list(ex.map(OM.run_mutant, idx))
    missed = [OM.MUTANTS[i][1][:80] for i, caught, _ in res if not caught]
    assert not missed, missed
    assert len(res) >= 30
