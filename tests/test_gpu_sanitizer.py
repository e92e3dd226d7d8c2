"""compute-sanitizer over the CUDA path on small configs:
memcheck (out-of-bounds / misaligned accesses), racecheck (shared-memory
hazards in the scan, sort and histogram kernels) and synccheck (barrier /
warp-sync misuse) on c1-c3 samples, a c5 slice and hand-written shapes that
reach every counting kernel (lane, queue with cp.async prefetch, big),
each expected to report zero errors.

compute-sanitizer is closed on the GPU pool this build runs on (runs under it
left GPUs needing a reset), so the sanitizer legs run only when
SEL_RUN_SANITIZER=1; by default the same script runs without it under
CUDA_LAUNCH_BLOCKING=1, where an out-of-bounds access surfaces as a launch
error at the failing kernel, and every result is cross-checked between the
fused and the split calls."""
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
# queue-kernel and lane-kernel shapes: element sizes 1/2 (handed to the warp kernel), depth 3,
# blocks that 32 does not divide (warp-rep classes), depth-2 residue histograms
launches = np.zeros(3, gen.LAUNCH_DTYPE)
launches[0], launches[1], launches[2] = (48, 65535, 0, 0), (200, 3, 0, 0), (128, 65535, 0, 0)
items = []
for e, d, cp in ((1, 1, 3), (2, 3, 6), (4, 2, 4), (8, 1, -8), (16, 2, 16), (4, 1, 100)):
    a = gen.make_access(base=(1 << 30) + 7 * e, c_par=(cp,), c_inner=[e * 3, 96 * e, 5 * e][:d], elem_bytes=e, depth=d)
    for li in range(3):
        items.append(dict(P0=97 + 11 * li, trip=[9, 5, 3][:d], depth=d, comp=[1.0] * (d + 1), accesses=[a, a], launch=li))
custom = gen.custom_batch(items, launches_=launches)
for cfg, idx, flags in ((1, None, 0), (1, None, 2), (3, np.arange(0, 3000, 7), 0), (2, np.arange(0, 108, 9), 1),
                        (5, None, 0), ("custom", None, 0), ("custom", None, 8)):
    if cfg == "custom":
        b = custom
    elif cfg == 5:
        b = gen.generate(5, 0, 768 * 3)
    else:
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


def test_shapes_blocking_launches(tmp_path):
    import __graft_entry__
    __graft_entry__.build()
    script = tmp_path / "run.py"
    script.write_text(SCRIPT)
    env = dict(os.environ, CUDA_LAUNCH_BLOCKING="1")
    p = subprocess.run([sys.executable, str(script)], capture_output=True, text=True, timeout=1200, env=env)
    out = p.stdout + p.stderr
    assert "SANITIZER-RUN-OK" in out and p.returncode == 0, out[-3000:]


@pytest.mark.parametrize("tool", ["memcheck", "racecheck", "synccheck"])
def test_compute_sanitizer(tool, tmp_path):
    import __graft_entry__
    if os.environ.get("SEL_RUN_SANITIZER") != "1":
        pytest.skip("compute-sanitizer is closed on this GPU pool; SEL_RUN_SANITIZER=1 runs it")
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
