"""compute-sanitizer over the CUDA path on small configs:
memcheck (out-of-bounds / misaligned accesses), racecheck (shared-memory
hazards in the scan kernels) and synccheck (barrier / warp-sync misuse),
each expected to report zero errors."""
import os
import shutil
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
SANITIZER = shutil.which("compute-sanitizer") or "/usr/local/cuda/bin/compute-sanitizer"

SCRIPT = r"""
import sys, numpy as np, torch
sys.path.insert(0, %r)
import gen
import paper_conf_ipps_chikinaat19_b200 as sel
for cfg, idx, flags in ((1, None, 0), (1, None, 2), (3, np.arange(0, 3000, 7), 0), (2, np.arange(0, 108, 9), 1)):
    b = gen.generate(cfg) if idx is None else gen.generate(cfg).select(idx)
    ev = sel.Evaluator((b.nests, b.accesses, b.launches, b.devices), len(b), flags)
    c = sel._as_bytes_tensor(b.cands, "candidate")
    r = ev.evaluate(c, want_counts=True, want_t_gpu=True)
    counts, status = sel.count_transactions(c, ev.tables, ev.workspace, flags)
    cyc, tg = sel.predict_gpu_cycles(c, ev.tables, counts, status)
    d = sel.select(c, tg, status)
    torch.cuda.synchronize()
    assert (d.cpu() == r["decision"].cpu()).all()
print("SANITIZER-RUN-OK")
""" % ROOT


@pytest.mark.parametrize("tool", ["memcheck", "racecheck", "synccheck"])
def test_compute_sanitizer(tool, tmp_path):
    import __graft_entry__
    __graft_entry__.build()
    if not os.path.exists(SANITIZER):
        pytest.skip("compute-sanitizer not found")
    script = tmp_path / "run.py"
    script.write_text(SCRIPT)
    p = subprocess.run([SANITIZER, "--tool", tool, "--error-exitcode", "9", sys.executable, str(script)],
                       capture_output=True, text=True, timeout=1200)
    out = p.stdout + p.stderr
    assert "SANITIZER-RUN-OK" in out, out[-3000:]
    assert p.returncode == 0, out[-3000:]
    ok = ("RACECHECK SUMMARY: 0 hazards" in out) if tool == "racecheck" else ("ERROR SUMMARY: 0 errors" in out)
    assert ok, out[-3000:]
