"""Hand-computed pins of the oracle's model half (a4-a7).

Every expected value below is worked out by hand in the comments from the
equations the paper prints (Figs. 4-5), the readings in
DESIGN.md (R1-R22, F4a-F4d) and the inputs of the test -- small numbers
chosen so that every intermediate is exact or obviously rounded -- and is
written in the test as plain arithmetic on literals, never by calling an
oracle routine.  The candidates are real loop nests evaluated end to end by
``oracle.evaluate`` (brute-force counts + model), so a wrong count, a dropped
term, a wrong sign or a swapped operand anywhere in a4-a7 changes a number
asserted here.  ``scripts/mutate_oracle.py`` checks that each of the model
mutations it applies to oracle.c fails at least one of these tests.

The hand device "D" (a made-up GPU with round numbers): 4 SMs, 64 warps /
2048 threads / 32 blocks per SM, 65536 registers, 65536 B shared memory,
Freq = 1 GHz, Mem_LD = 500 cycles, Departure_del_coal = 10,
Departure_del_uncoal = 20, 1 issue cycle per instruction, host link 1 GB/s,
launch overhead 5 us; the memory bandwidth varies per test.
"""
import numpy as np
import pytest

import gen
import oracle

BASE = 1 << 20          # 128-byte aligned array base


def device(mem_bw=1e12, **kw):
    d = np.zeros(1, gen.DEVICE_DTYPE)
    d[0] = (4, 64, 2048, 32, 65536, 65536, 1e9, mem_bw, 1e9, 5e-6, 500.0, 10.0, 20.0, 1.0, 0, 0, 0, 0)
    for k, v in kw.items():
        d[0][k] = v
    return d


def run(dev, P, B, access, trip=(), comp=(2.0,), gmax=65535, regs=0, smem=0, n_sync=0, h2d=0, d2h=0,
        cpu_cycles=1e6, cpu_hz=1e9):
    launches = np.zeros(1, gen.LAUNCH_DTYPE)
    launches[0] = (B, gmax, regs, smem)
    accesses = list(access) if isinstance(access, list) else [access]
    b = gen.custom_batch([dict(P0=P, trip=list(trip), comp=list(comp), accesses=accesses, device=0,
                               bytes_h2d=h2d, bytes_d2h=d2h, cpu_cycles=cpu_cycles, cpu_hz=cpu_hz)],
                         devices=dev, launches_=launches)
    b.nests["n_sync"] = n_sync
    r = oracle.evaluate(b)[0]
    assert r["status"] == 0
    return r


# stride 128 B (32 elements of 4 B): every lane of a warp touches its own line
STRIDED = gen.make_access(base=BASE, c_par=(128,), elem_bytes=4, depth=0)
# unit stride 4 B, aligned: one line, four sectors per full warp
UNIT = gen.make_access(base=BASE, c_par=(4,), elem_bytes=4, depth=0)


def test_case2_memory_bound_uncoalesced():
    """Fig. 4 case 2 (Mem >> Comp).  P = 4096, B = 128 (4 warps per block):
    G = 32 blocks, #OMP_Rep = 1; blocks per SM = min(32, 64/4, 2048/128,
    ceil(32/4)) = 8, so N = 32 warps, #Active_SMs = 4, #Rep = 32/(8*4) = 1.
    Counts: 128 warp-accesses, each 32 lines / 32 sectors, none coalesced:
    W = 128, L = S = U = 4096, C = 0, WR = 128.
    #Uncoal_per_mw = 4096/128 = 32; Mem_L_uncoal = 500 + (32 - 1) * 20 = 1120
    = Mem_L; Departure_delay = 20 * 32 = 640; MWP_Without_BW = 1120/640 =
    1.75.  Load_bytes = 32*4096/128 = 1024; BW_per_warp = 1e9*1024/1120;
    MWP_peak_BW = 1e12 / (BW_per_warp * 4) ~ 273 (not binding); MWP = 1.75.
    Comp = 1 * (2 + 1) = 3, Mem = 1120 * 1 = 1120, CWP = min(1123/3, 32) = 32.
    CWP >= MWP: case 2, Exec = Mem*N/MWP + Comp/#Mem*(MWP-1)
    = 1120*32/1.75 + 3/1*0.75 = 20480 + 2.25."""
    r = run(device(), 4096, 128, STRIDED)
    assert (r["W"], r["L"], r["S"], r["C"], r["U"], r["WR"]) == (128, 4096, 4096, 0, 4096, 128)
    assert (r["G"], r["R"], r["abps"], r["active_sms"], r["N"], r["Rep"]) == (32, 1, 8, 4, 32.0, 1.0)
    assert r["MemL"] == 1120.0 and r["Dep"] == 640.0 and r["MWP"] == 1.75 and r["CWP"] == 32.0
    assert r["hk_case"] == 2
    assert r["cycles"] == 20480.0 + 2.25


def test_case2_bandwidth_bound():
    """Fig. 5's bandwidth branch binds.  Same geometry as above
    (N = 32, #Active_SMs = 4, #Rep = 1), unit-stride coalesced access:
    W = 128, L = 128, S = 512, C = 128, U = 0.  #Uncoal_per_mw = 0 (R12),
    weights coal 1 / uncoal 0, so Mem_L = Mem_LD = 500, Departure_delay =
    Departure_del_coal = 10, MWP_Without_BW = min(500/10, 32) = 32.
    Load_bytes = 32*512/128 = 128 B; BW_per_warp = Freq * Load_bytes / Mem_L
    = 1e9 * 128 / 500 = 2.56e8 B/s; with Mem_Bandwidth = 3.072e9 B/s,
    MWP_peak_BW = 3.072e9 / (2.56e8 * 4) = 3, so MWP = 3.
    Comp = 3, Mem = 500 * 1 = 500, CWP = min(503/3, 32) = 32 >= MWP: case 2,
    Exec = 500*32/3 + 3/1*(3 - 1) = 16000/3 + 6."""
    r = run(device(mem_bw=3.072e9), 4096, 128, UNIT)
    assert (r["W"], r["L"], r["S"], r["C"], r["U"]) == (128, 128, 512, 128, 0)
    assert r["MemL"] == 500.0 and r["Dep"] == 10.0 and r["MWPnb"] == 32.0
    assert r["BWpw"] == 2.56e8 and r["MWPbw"] == 3.0 and r["MWP"] == 3.0
    assert r["hk_case"] == 2
    assert r["cycles"] == 16000.0 / 3.0 + 6.0


def test_case2_mixed_classes():
    """Coalesced and uncoalesced warp-accesses in one nest (H&K's weights,
    R12): the unit-stride and the 128-byte-strided access side by side, same
    geometry (N = 32, #Active_SMs = 4, #Rep = 1).  W = 256, C = 128, U = 4096,
    S = 512 + 4096 = 4608, WR = 128, #Mem_insts = 2.
    #Coal = #Uncoal = 128/128 = 1 per warp, weights 1/2 and 1/2,
    #Uncoal_per_mw = 4096/(256 - 128) = 32, Mem_L_uncoal = 1120,
    Mem_L = 1120/2 + 500/2 = 810, Departure_delay = 20*32/2 + 10/2 = 325,
    MWP_Without_BW = 810/325 (~2.49), Load_bytes = 32*4608/256 = 576,
    MWP_peak_BW = 1e12 / (1e9*576/810 * 4) ~ 352: MWP = 810/325.
    Comp = 1 * (2 + 2) = 4, Mem = 1120*1 + 500*1 = 1620,
    CWP = min(1624/4, 32) = 32: case 2,
    Exec = 1620*32/MWP + 4/2*(MWP - 1)."""
    r = run(device(), 4096, 128, [UNIT, STRIDED])
    assert (r["W"], r["C"], r["U"], r["S"], r["WR"], r["M_it"]) == (256, 128, 4096, 4608, 128, 2)
    assert r["MemL"] == 810.0 and r["Dep"] == 325.0 and r["Mem"] == 1620.0 and r["Comp"] == 4.0
    mwp = 810.0 / 325.0
    assert r["MWP"] == mwp and r["hk_case"] == 2
    assert r["cycles"] == 51840.0 / mwp + 2.0 * (mwp - 1.0)


def test_case3_compute_bound():
    """Fig. 4 case 3: Comp <= Mem with MWP > CWP.  Unit-stride
    access as above with ample bandwidth (MWP_peak_BW = 1e12 / (2.56e8*4)
    ~ 977), so MWP = min(32, 977, 32) = N = 32.  comp_insts = 499 gives
    Comp = 1 * (499 + 1) = 500 = Mem, so CWP = (500 + 500)/500 = 2 < N: not
    case 1; CWP >= MWP is false and Comp > Mem is false (equal): case 3,
    Exec = Mem_L + Comp * N = 500 + 500 * 32 = 16500."""
    r = run(device(), 4096, 128, UNIT, comp=(499.0,))
    assert r["MWP"] == 32.0 and r["CWP"] == 2.0 and r["Comp"] == 500.0 and r["Mem"] == 500.0
    assert r["hk_case"] == 3
    assert r["cycles"] == 500.0 + 500.0 * 32


def test_tgpu_exact():
    """R20 (transfers are part of the paper's measured time):
    T_gpu = Exec/Freq + (bytes_h2d + bytes_d2h)/link + launch overhead
    = 16500/1e9 + (1000 + 3000)/1e9 + 5e-6 for the case-3 candidate; with a
    host cost of 25600 cycles at 1 GHz (T_cpu = 2.56e-5 > 2.55e-5) the
    decision is GPU, and at 25400 cycles it is CPU."""
    r = run(device(), 4096, 128, UNIT, comp=(499.0,), h2d=1000, d2h=3000, cpu_cycles=25600.0)
    assert r["t_gpu"] == (16500.0 / 1e9 + 4000.0 / 1e9) + 5e-6
    assert r["t_cpu"] == 25600.0 / 1e9 and r["decision"] == 1
    r = run(device(), 4096, 128, UNIT, comp=(499.0,), h2d=1000, d2h=3000, cpu_cycles=25400.0)
    assert r["decision"] == 0


def test_non_integer_rep():
    """#Rep as a real ratio (R5): P = 1280, B = 128 gives G = 10 blocks;
    blocks per SM = min(32, 16, 16, ceil(10/4) = 3) = 3, N = 12 warps,
    #Active_SMs = 4, #Rep = 10/(3*4) = 5/6.  Unit-stride access: W = 40,
    S = 160, Load_bytes = 128, Mem_L = 500, MWP_Without_BW = min(50, 12) = 12,
    MWP_peak_BW ~ 977: MWP = N = 12; Comp = Mem = 500 -> CWP = 2: case 3,
    Exec_Cycles = 500 + 500 * 12 = 6500 per repetition set, x #Rep x #OMP_Rep
    = 6500 * (10/12) * 1."""
    r = run(device(), 1280, 128, UNIT, comp=(499.0,))
    assert (r["G"], r["abps"], r["N"]) == (10, 3, 12.0)
    assert r["Rep"] == 10.0 / 12.0
    assert r["hk_case"] == 3 and r["E"] == 6500.0
    assert r["cycles"] == (6500.0 * (10.0 / 12.0)) * 1.0


def test_single_warp_uncoalesced_serial():
    """Mem_L_uncoal on one lone warp (Fig. 4 case 1): P = 32,
    B = 32, G_max = 1: N = 1, #Rep = #OMP_Rep = 1.  The 128-byte-strided
    access inside an inner loop of 5 iterations (c_inner = 4 B) makes 5
    warp-accesses of 32 lines each: W = 5, U = 160, C = 0, WR = 1, M_it = 5.
    #Uncoal_per_mw = 160/5 = 32, Mem_L_uncoal = 500 + 31*20 = 1120; the warp
    runs serially: Mem = 1120 * 5/1 = 5600, comp = 1 + 2*5 = 11,
    Comp = 1 * (11 + 5) = 16; MWP = CWP = N = 1 (case 1):
    Exec = (Mem + Comp) + Comp/#Mem * (1 - 1) = 5616."""
    acc = gen.make_access(base=BASE, c_par=(128,), c_inner=(4,), elem_bytes=4, depth=1)
    r = run(device(), 32, 32, acc, trip=(5,), comp=(1.0, 2.0), gmax=1)
    assert (r["W"], r["U"], r["C"], r["WR"], r["M_it"]) == (5, 160, 0, 1, 5)
    assert r["N"] == 1.0 and r["hk_case"] == 1
    assert r["MemL_u"] == 1120.0 and r["Mem"] == 5600.0 and r["Comp"] == 16.0
    assert r["cycles"] == 5616.0


def test_omp_rep_multiplies():
    """#OMP_Rep: the case-2 candidate with G_max = 8 blocks runs
    ceil(4096 / (8*128)) = 4 repetitions; blocks per SM = min(8, ceil(8/4))
    = 2, N = 8, #Rep = 8/(2*4) = 1.  MWP = min(1.75, 8) = 1.75,
    CWP = min(1123/3, 8) = 8: case 2 with N = 8 per repetition:
    E = 1120*8/1.75 + 3*0.75 = 5120 + 2.25, Exec = E * 1 * 4."""
    r = run(device(), 4096, 128, STRIDED, gmax=8)
    assert (r["G"], r["R"], r["abps"], r["N"], r["Rep"]) == (8, 4, 2, 8.0, 1.0)
    assert r["hk_case"] == 2
    assert r["cycles"] == (5120.0 + 2.25) * 1.0 * 4


def test_f4_sync_term():
    """NEXT row f4 (readings F4a/F4b): with 2 barriers per parallel iteration
    the case-2 candidate adds Departure_delay * (MWP - 1) * #synch *
    #Active_blocks_per_SM * #Rep * #OMP_Rep = 640 * 0.75 * 2 * 8 * 1 * 1 =
    7680 cycles: 20482.25 + 7680."""
    r = run(device(), 4096, 128, STRIDED, n_sync=2)
    assert r["cycles"] == 20482.25 + 7680.0


def test_f4_register_granularity():
    """F4c: B = 96 (3 warps), 37 registers per thread.  Without granularity
    (R17) blocks per SM by registers = floor(65536 / (37 * 96)) = 18; with a
    256-register allocation unit and a warp granularity of 4: registers per
    warp = ceil(37*32/256)*256 = 5*256 = 1280, warps = floor(65536/1280) =
    51 -> 48, blocks = floor(48/3) = 16.  (Other limits: 32 blocks,
    floor(64/3) = 21, floor(2048/96) = 21; G = ceil(96000/96) = 1000,
    ceil(1000/4) = 250.)"""
    acc = gen.make_access(base=BASE, c_par=(4,), elem_bytes=4, depth=0)
    assert run(device(), 96000, 96, acc, regs=37)["abps"] == 18
    assert run(device(reg_alloc_unit=256, warp_alloc_gran=4), 96000, 96, acc, regs=37)["abps"] == 16
    assert run(device(reg_alloc_unit=256, warp_alloc_gran=1), 96000, 96, acc, regs=37)["abps"] == 17   # 51/3
    assert run(device(reg_alloc_unit=1, warp_alloc_gran=4), 96000, 96, acc, regs=37)["abps"] == 17     # 55 -> 52 warps, /3


def test_f4_smem_granularity():
    """F4c: B = 32 on an SM with 16384 B of shared memory and 300 B per
    block: floor(16384/300) = 54 blocks without granularity, but with a
    256 B allocation unit each block takes 512 B: floor(16384/512) = 32.
    (Other limits: 1000 blocks, 64 warps, 2048/32 = 64 threads.)"""
    acc = gen.make_access(base=BASE, c_par=(4,), elem_bytes=4, depth=0)
    dev = dict(max_blocks_per_sm=1000, smem_per_sm=16384)
    r0 = run(device(**dev), 32 * 1000 * 4, 32, acc, smem=300)
    r1 = run(device(smem_alloc_unit=256, **dev), 32 * 1000 * 4, 32, acc, smem=300)
    assert (r0["abps"], r1["abps"]) == (54, 32)


def test_f4_sector_transactions():
    """F4d: with 32 B-sector transactions every warp-access is one class whose
    transactions are its sectors (#Coal = 0, U = S).  The unit-stride
    candidate (W = 128, S = 512): #Uncoal_per_mw = 512/128 = 4,
    Mem_L = 500 + (4 - 1) * 20 = 560, Departure_delay = 20 * 4 = 80,
    MWP_Without_BW = 560/80 = 7; MWP_peak_BW ~ 1094: MWP = 7.  Comp = 3,
    Mem = 560 * 128/128 = 560, CWP = min(563/3, 32) = 32 >= 7: case 2,
    Exec = 560*32/7 + 3*(7 - 1) = 2560 + 18."""
    r = run(device(txn_sectors=1), 4096, 128, UNIT)
    assert r["MemL"] == 560.0 and r["Dep"] == 80.0 and r["MWP"] == 7.0
    assert r["hk_case"] == 2
    assert r["cycles"] == 2560.0 + 18.0
    # the line model on the same candidate: all coalesced, Mem_L = 500, MWP = 32 = N, CWP = 32: case 1,
    # Exec = (500 + 3) + 3 * 31
    r = run(device(), 4096, 128, UNIT)
    assert r["hk_case"] == 1 and r["cycles"] == (500.0 + 3.0) + 3.0 * 31


def test_no_memory_instruction():
    """R22: no memory instruction (W = 0): compute-bound with Mem_L = 0,
    Exec = issue * comp * N * #Rep * #OMP_Rep.  comp_insts = 7, P = 4096,
    B = 128 -> N = 32, #Rep = 1: 1 * 7 * 32 * 1 * 1 = 224."""
    launches = np.zeros(1, gen.LAUNCH_DTYPE)
    launches[0] = (128, 65535, 0, 0)
    b = gen.custom_batch([dict(P0=4096, trip=[], comp=[7.0], accesses=[], device=0)], devices=device(),
                         launches_=launches)
    r = oracle.evaluate(b)[0]
    assert r["status"] == 0 and r["W"] == 0 and r["hk_case"] == 0
    assert r["cycles"] == 224.0
