"""The oracle's model pins bite: scripts/mutate_oracle.py applies 29
single-term mutations of the a4-a7 arithmetic (dropped terms, wrong
operands, swapped case conditions, extra rounding, f4 extensions) to a
temporary copy of oracle/oracle.c and requires each to fail at least one CPU
pin (tests/test_oracle_hand.py, tests/test_oracle_model.py).  ~1 min."""
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_every_model_mutant_is_killed():
    r = subprocess.run([sys.executable, os.path.join(ROOT, "scripts", "mutate_oracle.py")], cwd=ROOT,
                       capture_output=True, text=True, timeout=900)
    assert r.returncode == 0, r.stdout[-3000:] + r.stderr[-2000:]
    assert "29/29 mutants killed" in r.stdout
