mkdir -p gpurun_out
python __graft_entry__.py
cat > /tmp/r.py <<'PY'
import sys, numpy as np, torch
sys.path.insert(0, '.')
import gen
import paper_conf_ipps_chikinaat19_b200 as sel
b = gen.generate(1)
ev = sel.Evaluator((b.nests, b.accesses, b.launches, b.devices), len(b), 0)
c = sel._as_bytes_tensor(b.cands, "candidate")
r = ev.evaluate(c, want_counts=True, want_t_gpu=True)
torch.cuda.synchronize()
print("done")
PY
compute-sanitizer --tool racecheck --racecheck-report all python /tmp/r.py > gpurun_out/race.log 2>&1
tail -60 gpurun_out/race.log
