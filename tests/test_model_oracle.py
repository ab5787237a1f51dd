"""Pins for oracle/model_p.py (the paper's Eqs. 6-14) -- CPU only.

Eqs. (6)-(9) are integer arithmetic and pinned by hand-computed cases.
Eqs. (10)-(14): the paper prints no predicted values, so they are pinned by
hand derivations under the readings R12-R14 (tests/golden/model_p_hand.json,
two GTX580 cases that separate (Stages-1) from RemBlks, f(ActBlks) from
f(RemBlks) and BW from BW_SM), by a bandwidth-only closed form, and by the
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


# ---- Eqs. (10)-(14): hand-derived values (tests/golden/model_p_hand.json) ----------
def _hand_cases():
    with open(os.path.join(GOLDEN, "model_p_hand.json")) as f:
        d = json.load(f)
    g = {k: v for k, v in d["gpu"].items() if k != "name"}
    return mp.GPU(**g), d["cases"]


def _hand_kernel(c):
    k = c["kernel"]
    W, H = k["TX"] * k["RX"], k["TY"] * k["RY"]
    return mp.Kernel(LX=k["LX"], LY=k["LY"], TX=k["TX"], TY=k["TY"], RX=k["RX"], RY=k["RY"], r=k["r"], s=k["s"],
                     K_R=k["regs_per_thread"] * k["TX"] * k["TY"], K_S=(W + 2 * k["r"]) * (H + 2 * k["r"]) * k["s"],
                     Ops=k["Ops"])


@pytest.mark.parametrize("idx", [0, 1])
def test_eq10_to_14_hand_values(idx):
    """Each term of Eqs. (10)-(14) against the hand derivation, both R13 readings."""
    g, cases = _hand_cases()
    c = cases[idx]
    k = _hand_kernel(c)
    rel = 2e-9      # the golden values carry 10 significant digits
    it = c["integer"]
    assert (mp.blks(k), mp.act_blks(g, k), mp.stages(g, k), mp.rem_blks(g, k), mp.warp_blk(k)) == \
        (it["Blks"], it["ActBlks"], it["Stages"], it["RemBlks"], it["Warp_Blk"])
    assert mp.bytes_blk(k) == c["Bytes_Blk"]
    assert mp.f_hide(g, k, it["ActBlks"]) == pytest.approx(c["f_act"], rel=rel)
    assert mp.f_hide(g, k, it["RemBlks"]) == pytest.approx(c["f_rem"], rel=rel)
    assert mp.t_m(g, k) == pytest.approx(c["T_m"], rel=rel)
    assert mp.t_c(g, k) == pytest.approx(c["T_c"], rel=rel)
    assert mp.t_s(g, k) == pytest.approx(c["T_s"], rel=rel)
    assert mp.t_l(g, k) == pytest.approx(c["T_l"], rel=rel)
    assert mp.perf(g, k) == pytest.approx(c["Perf"], rel=rel)
    lit = c["literal"]
    assert mp.t_c(g, k, literal_tc=True) == pytest.approx(lit["T_c"], rel=rel)
    assert mp.t_s(g, k, literal_tc=True) == pytest.approx(lit["T_s"], rel=rel)
    assert mp.t_l(g, k, literal_tc=True) == pytest.approx(lit["T_l"], rel=rel)
    assert mp.perf(g, k, literal_tc=True) == pytest.approx(lit["Perf"], rel=rel)


def test_eq14_bandwidth_closed_form():
    """With Lat = 0, Ops = 0 and one block per SM (f = 1), Eqs. (10)-(14) reduce to every SM moving one
    block's bytes per stage at BW/SM: Perf = LX*LY*BW / (SM * Bytes_Blk * Stages) (Eq. 10)."""
    g = mp.GPU(SM=16, BW=161e9, Smem=48 * 1024, Reg=32768, Blk_SM=1, Warp_SM=48, Lat=0.0, Clock=1.544e9)
    k = mp.Kernel(LX=512, LY=512, TX=32, TY=4, RX=1, RY=4, r=4, s=4, K_R=40 * 128, K_S=3840, Ops=0)
    assert mp.act_blks(g, k) == 1 and mp.stages(g, k) == 32 and mp.rem_blks(g, k) == 1
    expect = 512 * 512 * 161e9 / (16 * 5888 * 32)
    assert mp.perf(g, k) == pytest.approx(expect, rel=1e-12)
