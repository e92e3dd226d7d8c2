"""torchrun worker for tests/test_gpu_split.py: config-4 partitioning
(dist.evaluate_split) on the reduced c4 batch; each rank writes its
all-reduced counts, cycles and decisions to $SPLIT_OUT/rank<r>.json."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_ipps_chikinaat19_b200 as sel  # noqa: E402
from paper_conf_ipps_chikinaat19_b200 import dist as D  # noqa: E402


def main():
    rank, world, _ = D.init()
    b = gen.generate(4)
    nests = b.nests.copy()
    nests["P0"] = 1 << 14
    ev = sel.Evaluator((nests, b.accesses, b.launches, b.devices), len(b))
    cands = sel._as_bytes_tensor(b.cands, "candidate")
    r = D.evaluate_split(cands, ev.tables, ev.workspace, rank, world)
    torch.cuda.synchronize()
    out = {"counts": r["counts"].cpu().tolist(), "cycles": r["cycles"].cpu().tolist(),
           "decision": r["decision"].cpu().tolist()}
    with open(os.path.join(os.environ["SPLIT_OUT"], f"rank{rank}.json"), "w") as f:
        json.dump(out, f)
    D.barrier(world)


if __name__ == "__main__":
    main()
