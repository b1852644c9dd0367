"""Every plausible single-line mistake listed in scripts/mutate_oracle.py must fail at
least one CPU pin of the oracle.  Runs the mutants in parallel, one
pytest process each, against compiled copies of the oracle under /tmp."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, os.path.join(ROOT, "scripts"))


def test_every_mutant_fails_a_pin(tmp_path):
    import mutate_oracle
    ok, rows = mutate_oracle.run(str(tmp_path / "mut.md"), quiet=True)
    bad = [(r[0], r[2]) for r in rows if r[2] not in ("caught", "equivalent")]
    assert ok and not bad, bad
    assert sum(r[2] == "caught" for r in rows) >= 28
