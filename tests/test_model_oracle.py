"""Pins for oracle/model_p.py (the paper's Eqs. 6-14) -- CPU only.

Eqs. (6)-(9) are integer arithmetic and pinned by hand-computed cases.
Eqs. (10)-(14) are parity UNPINNED against the paper (it prints no predicted
values and leaves Lat and f unspecified); they are checked here only for the
limits the prose fixes (f = 1 at full occupancy, f = n for a single warp,
Perf rising with BW and with Clock).
"""
import json
import os

import pytest

from oracle import model_p as mp

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")

GTX580 = mp.GPU(SM=16, BW=161e9, Smem=48 * 1024, Reg=32768, Blk_SM=8, Warp_SM=48, Lat=400, Clock=1.544e9)


def kern(TX=256, TY=1, RX=1, RY=8, r=1, s=4, regs=20, LX=512, LY=512):
    W, H = TX * RX, TY * RY
    return mp.Kernel(LX=LX, LY=LY, TX=TX, TY=TY, RX=RX, RY=RY, r=r, s=s,
                     K_R=regs * TX * TY, K_S=(W + 2 * r) * (H + 2 * r) * s, Ops=8 * r + 1)


def test_eq6_to_9_hand_case():
    k = kern()
    assert mp.blks(k) == 128                     # 512*512 / (256*8)
    # regs 20*256 = 5120 -> 6; smem (258*10*4 = 10320 B) -> 4; warps 48/8 = 6; Blk_SM 8
    assert mp.act_blks(GTX580, k) == 4
    assert mp.stages(GTX580, k) == 2             # ceil(128 / (16*4))
    assert mp.rem_blks(GTX580, k) == 4           # ceil((128 - 64) / 16)


def test_eq6_to_9_second_case():
    # (32, 4, 1, 4), r = 4 (Table IV best SP order 8 on GTX580)
    k = kern(TX=32, TY=4, RX=1, RY=4, r=4, regs=40)
    assert mp.blks(k) == 512 * 512 / (32 * 16)   # 512
    # regs 40*128 = 5120 -> 6; smem (40*24*4 = 3840) -> 12; warps 48/4 = 12; Blk_SM 8 -> 6
    assert mp.act_blks(GTX580, k) == 6
    assert mp.stages(GTX580, k) == 6             # ceil(512/96) = 6
    assert mp.rem_blks(GTX580, k) == 2           # ceil((512 - 5*96)/16) = ceil(32/16)


def test_f_limits():
    k = kern(TX=32, TY=1, RY=1)                  # one warp per block
    g = GTX580
    assert mp.f_hide(g, k, 1) == 1.0
    assert mp.f_hide(g, k, g.Warp_SM) == 1.0     # full occupancy: perfect hiding
    assert 1.0 <= mp.f_hide(g, k, 5) <= 5.0


def test_perf_monotone_in_bw_and_clock():
    k = kern()
    p0 = mp.perf(GTX580, k)
    faster_bw = mp.GPU(**{**GTX580.__dict__, "BW": 2 * GTX580.BW})
    faster_clk = mp.GPU(**{**GTX580.__dict__, "Clock": 2 * GTX580.Clock})
    assert mp.perf(faster_bw, k) > p0 > 0
    assert mp.perf(faster_clk, k) > p0


def test_literal_tc_is_slower_or_equal():
    k = kern()
    assert mp.perf(GTX580, k, literal_tc=True) <= mp.perf(GTX580, k)


@pytest.mark.parametrize("M,beta,N", [(400, 5, 20), (3, 5, 1), (101, 5, 6), (10, 100, 10)])
def test_top_n(M, beta, N):
    assert mp.top_n(M, beta) == N


def test_paper_tables_match_counting_formulas():
    with open(os.path.join(GOLDEN, "paper_tables.json")) as f:
        t = json.load(f)
    for order, extent, mem, flops in t["table1"]["rows"]:
        r = order // 2
        assert extent == 2 * r + 1 and mem == 6 * r + 2 and flops == 7 * r + 1
    for order, refs, fin, fnv in t["table2"]["rows"]:
        r = order // 2
        assert refs == 6 * r + 2 and fin == 8 * r + 1 and fnv == 7 * r + 1
