"""The oracle's pins are strong enough: every plausible mistake in tools/mutate_oracle.py (swapped
index, dropped factor, missing quarantine, non-transitive happens-before, ...) applied to a private
copy of oracle/ makes tests/test_oracle_*.py fail.  Runs the mutants in parallel (~40 s on 16 cores)."""
import importlib.util
import os

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_every_oracle_mutant_is_killed(capsys):
    spec = importlib.util.spec_from_file_location("mutate_oracle", os.path.join(ROOT, "tools", "mutate_oracle.py"))
    m = importlib.util.module_from_spec(spec)
    spec.loader.exec_module(m)
    rc = m.main()
    out = capsys.readouterr().out
    assert rc == 0, out
    assert f"{len(m.MUTANTS)}/{len(m.MUTANTS)} mutants killed" in out
