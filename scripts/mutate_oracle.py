#!/usr/bin/env python
"""Mutation check of the oracle's pins ("What's weak" #1).

Applies one plausible single-term mistake at a time to a temporary copy of
oracle/oracle.c -- a dropped term, a wrong operand, a swapped condition, an
extra rounding -- builds it, and runs the CPU pins of the model half
(tests/test_oracle_model.py, tests/test_oracle_hand.py) against it through
SEL_ORACLE_LIB.  Every mutant must fail at least one pin; the script exits
non-zero (and names the survivors) otherwise.

    python scripts/mutate_oracle.py [-k SUBSTRING] [-v]
"""
from __future__ import annotations

import argparse
import os
import subprocess
import sys
import tempfile
from concurrent.futures import ThreadPoolExecutor

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
SRC = os.path.join(ROOT, "oracle", "oracle.c")
PINS = ["tests/test_oracle_hand.py", "tests/test_oracle_model.py"]   # the fast hand pins first (-x)

# (name, passage it breaks, exact text in oracle.c, replacement)
MUTATIONS = [
    ("case 3 without Mem_L", "Fig. 4 case 3, P:L274",
     "E = r->MemL + r->Comp * N;", "E = r->Comp * N;"),
    ("case 2 without Comp/#Mem*(MWP-1)", "Fig. 4 case 2, P:L268",
     "E = (r->Mem * N) / r->MWP + Cp * (r->MWP - 1.0);", "E = (r->Mem * N) / r->MWP;"),
    ("case 1 without Comp/#Mem*(MWP-1)", "Fig. 4 case 1, P:L262",
     "E = (r->Mem + r->Comp) + Cp * (r->MWP - 1.0);", "E = r->Mem + r->Comp;"),
    ("case 2/3 condition swapped", "R1 (P:L265, L271)",
     "r->CWP >= r->MWP || r->Comp > r->Mem", "r->MWP >= r->CWP || r->Comp > r->Mem"),
    ("MWP_peak_BW without #Active_SMs", "Fig. 5, P:L288",
     "dev->mem_bw_Bps / (r->BWpw * (double)r->active_sms)", "dev->mem_bw_Bps / r->BWpw"),
    ("BW_per_warp without Freq", "Fig. 5, P:L284",
     "r->BWpw = (f_sm * LB) / r->MemL;", "r->BWpw = LB / r->MemL;"),
    ("Mem_L_uncoal with #Uncoal_per_mw instead of #Uncoal_per_mw - 1", "[H&K] Mem_L_uncoal",
     "r->MemL_u = Mem_LD + (upmw - 1.0) * dd_u;", "r->MemL_u = Mem_LD + upmw * dd_u;"),
    ("Departure_delay without #Uncoal_per_mw", "[H&K] Departure_delay",
     "r->Dep = (dd_u * upmw) * w_unc + dd_c * w_coal;", "r->Dep = dd_u * w_unc + dd_c * w_coal;"),
    ("Mem_cycles with the coalesced latency for uncoalesced accesses", "[H&K] Mem_cycles, P:L301",
     "r->Mem = r->MemL_u * n_unc + r->MemL_c * n_coal;", "r->Mem = r->MemL_c * n_unc + r->MemL_c * n_coal;"),
    ("Comp_cycles without the memory instructions", "R14",
     "r->Comp = issue * (comp + mem);", "r->Comp = issue * comp;"),
    ("CWP not capped at N", "Fig. 5, P:L296",
     "r->CWP = dmin((r->Mem + r->Comp) / r->Comp, N);", "r->CWP = (r->Mem + r->Comp) / r->Comp;"),
    ("#Uncoal_per_mw over all warp-accesses", "R12",
     "(W > C) ? (double)U / (double)(W - C) : 0.0", "(W > C) ? (double)U / (double)W : 0.0"),
    ("#Uncoal_Mem_insts per warp-access instead of per warp", "[H&K] #Uncoal_Mem_insts",
     "const double n_unc = (double)(W - C) / (double)WR;", "const double n_unc = (double)(W - C) / (double)W;"),
    ("Load_bytes_per_warp from lines", "R13",
     "const double LB = (32.0 * (double)S) / (double)W;", "const double LB = (128.0 * (double)S) / (double)W;"),
    ("ceil on #Rep", "R5",
     "const double Rep = (double)r->G / ((double)abps * (double)r->active_sms);",
     "const double Rep = ceil((double)r->G / ((double)abps * (double)r->active_sms));"),
    ("Exec without #OMP_Rep", "P:L225",
     "Exec = (E * Rep) * (double)r->R;", "Exec = E * Rep;"),
    ("R22 compute-only form without N", "R22",
     "Exec = (((issue * comp) * N) * Rep) * (double)r->R;", "Exec = ((issue * comp) * Rep) * (double)r->R;"),
    ("T_gpu without the launch overhead", "R20",
     "               + dev->launch_overhead_s;", "               + 0.0;"),
    ("T_gpu with the host-to-device bytes only", "R20, P:L57",
     "(double)(nest->bytes_h2d + nest->bytes_d2h) / dev->link_bw_Bps", "(double)nest->bytes_h2d / dev->link_bw_Bps"),
    ("T_cpu without the host clock", "P:L305",
     "r->t_cpu = cand->cpu_cycles / cand->cpu_hz;", "r->t_cpu = cand->cpu_cycles / 1e9;"),
    ("tie goes to the GPU", "R21",
     "r->decision = (r->t_gpu < r->t_cpu) ? 1 : 0;", "r->decision = (r->t_gpu <= r->t_cpu) ? 1 : 0;"),
    ("occupancy without the grid term", "R17",
     "abps = umin(abps, ceil_div(r->G, (uint64_t)dev->num_sms));", "abps = abps;"),
    ("#Active_SMs not capped by G", "R17",
     "r->active_sms = umin(r->G, (uint64_t)dev->num_sms);", "r->active_sms = (uint64_t)dev->num_sms;"),
    ("f4 sync term without #Active_blocks_per_SM", "F4a",
     "* (double)nest->n_sync) * (double)abps) * Rep)", "* (double)nest->n_sync)) * Rep)"),
    ("f4 register granularity: no warp rounding", "F4c",
     "warps = (warps / (uint64_t)dev->warp_alloc_gran) * (uint64_t)dev->warp_alloc_gran;", "warps = warps;"),
    ("f4 register granularity: per-thread registers not rounded", "F4c",
     "ceil_div((uint64_t)launch->regs_per_thread * 32, unit) * unit;", "(uint64_t)launch->regs_per_thread * 32;"),
    ("f4 shared-memory granularity ignored", "F4c",
     "smem_b = ceil_div(smem_b, (uint64_t)dev->smem_alloc_unit) * (uint64_t)dev->smem_alloc_unit;",
     "smem_b = smem_b;"),
    ("f4 sector transactions keep the line counts", "F4d",
     "const uint64_t U = dev->txn_sectors ? S : r->U;", "const uint64_t U = r->U;"),
    ("f4 sector transactions keep the coalesced class", "F4d",
     "const uint64_t C = dev->txn_sectors ? 0 : r->C;", "const uint64_t C = r->C;"),
]


def build(src_text: str, out_dir: str) -> str:
    c = os.path.join(out_dir, "oracle.c")
    with open(c, "w") as f:
        f.write(src_text)
    hdr = os.path.join(ROOT, "oracle", "oracle.h")
    os.symlink(hdr, os.path.join(out_dir, "oracle.h"))
    so = os.path.join(out_dir, "liboracle_mut.so")
    subprocess.check_call(["gcc", "-O2", "-std=c11", "-w", "-ffp-contract=off", "-fno-fast-math", "-fPIC",
                           "-shared", "-pthread", "-o", so, c, "-lm"])
    return so


def run_pins(so: str | None, verbose: bool) -> int:
    env = dict(os.environ)
    if so:
        env["SEL_ORACLE_LIB"] = so
    r = subprocess.run([sys.executable, "-m", "pytest", *PINS, "-x", "-q", "-m", "not gpu", "-p", "no:cacheprovider"],
                       cwd=ROOT, env=env, capture_output=True, text=True)
    if verbose:
        print(r.stdout[-800:])
    return r.returncode


def main() -> int:
    ap = argparse.ArgumentParser()
    ap.add_argument("-k", default="")
    ap.add_argument("-v", action="store_true")
    args = ap.parse_args()
    src = open(SRC).read()
    if run_pins(None, args.v) != 0:
        print("the pins fail on the unmutated oracle", file=sys.stderr)
        return 2
    survivors = []
    todo = [m for m in MUTATIONS if args.k in m[0]]

    def one(m):
        name, cite, old, new = m
        if src.count(old) != 1:
            return name, cite, None
        with tempfile.TemporaryDirectory() as d:
            so = build(src.replace(old, new), d)
            return name, cite, run_pins(so, args.v) != 0

    with ThreadPoolExecutor(max_workers=max(1, min(8, (os.cpu_count() or 2) // 2))) as ex:
        for name, cite, killed in ex.map(one, todo):
            if killed is None:
                print(f"MISSING  {name}: text not found exactly once in oracle.c", flush=True)
            else:
                print(f"{'killed ' if killed else 'SURVIVED'} {name}  ({cite})", flush=True)
            if not killed:
                survivors.append(name)
    print(f"{len(todo) - len(survivors)}/{len(todo)} mutants killed")
    return 1 if survivors else 0


if __name__ == "__main__":
    sys.exit(main())
