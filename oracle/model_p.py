"""The paper's analytic performance model, Eqs. (6)-(14) -- TEST INFRASTRUCTURE ONLY.

Written out literally from PAPER.md Sec. VI so the product's C++
implementation (``stencil_model_paper`` in the CUDA library) can be checked
against it.  Readings where the paper is silent or inconsistent are the ones
listed in DESIGN.md (R12-R15):

  R12  K_R, K_S are per *block* (registers/thread x threads; smem bytes/block),
       otherwise floor(Reg/K_R) in Eq. (7) is not a block count.
  R13  Eq. (11) multiplies by ActBlks although the prose calls T_c "the time
       required for a thread block" and Eq. (12) multiplies by
       ActBlks again.  ``literal_tc=False`` (default) drops ActBlks from
       Eq. (11); ``literal_tc=True`` keeps it.
  R14  f(n) is "linear", 1 at full occupancy and n for a single warp:
           f(n) = 1 + (n - 1) * (1 - (w - 1) / (Warp_SM - 1)),  w = n * Warp_Blk
       clamped to [1, n].  Bytes_Blk = s*[(TX*RX + 2r)(TY*RY + 2r) + TX*RX*TY*RY]
       (bytes read and written per plane).  Lat is in cycles.
  R15  N = max(1, ceil(beta * M / 100)).

The paper prints no predicted values and leaves Lat and f unspecified, so
Eqs. (10)-(14) are pinned by hand derivations under the readings above
(tests/golden/model_p_hand.json: every term of two GTX580 cases chosen so a
swapped (Stages-1)/RemBlks, f(ActBlks)/f(RemBlks) or BW/BW_SM fails), by a
bandwidth-only closed form and by the limits the prose fixes
(tests/test_model_oracle.py).  Eqs. (6)-(9) are pinned by hand-computed cases
in the same file.
"""
from __future__ import annotations

import math
from dataclasses import dataclass


@dataclass(frozen=True)
class GPU:
    """The parameter set of P:L331-333."""
    SM: int             # streaming multiprocessors
    BW: float           # off-chip bandwidth, bytes/s
    Smem: int           # per-SM shared-memory limit, bytes
    Reg: int            # per-SM register limit (32-bit registers)
    Blk_SM: int         # max resident blocks per SM
    Warp_SM: int        # max resident warps per SM
    Lat: float          # global-memory latency, cycles
    Clock: float        # SM clock, Hz


@dataclass(frozen=True)
class Kernel:
    LX: int
    LY: int
    TX: int
    TY: int
    RX: int
    RY: int
    r: int
    s: int              # bytes per element
    K_R: int            # registers per block
    K_S: int            # shared-memory bytes per block
    Ops: int            # flops per point (Table II: 8r+1 for in-plane)


def blks(k: Kernel) -> float:
    """Eq. (6): thread blocks per plane."""
    return (k.LX * k.LY) / ((k.TX * k.RX) * (k.TY * k.RY))


def warp_blk(k: Kernel) -> int:
    return math.ceil(k.TX * k.TY / 32)


def act_blks(g: GPU, k: Kernel) -> int:
    """Eq. (7)."""
    return min(g.Reg // k.K_R, g.Smem // k.K_S, g.Warp_SM // warp_blk(k), g.Blk_SM)


def stages(g: GPU, k: Kernel) -> int:
    """Eq. (8)."""
    return math.ceil(blks(k) / (g.SM * act_blks(g, k)))


def rem_blks(g: GPU, k: Kernel) -> int:
    """Eq. (9)."""
    return math.ceil((blks(k) - (stages(g, k) - 1) * act_blks(g, k) * g.SM) / g.SM)


def bytes_blk(k: Kernel) -> float:
    """Bytes read and written per block per plane (reading R14)."""
    W, H = k.TX * k.RX, k.TY * k.RY
    return k.s * ((W + 2 * k.r) * (H + 2 * k.r) + W * H)


def t_m(g: GPU, k: Kernel) -> float:
    """Eq. (10): T_m = Lat/Clock + Bytes_Blk/BW_SM with BW_SM = BW/SM."""
    return g.Lat / g.Clock + bytes_blk(k) / (g.BW / g.SM)


def t_c(g: GPU, k: Kernel, literal_tc: bool = False) -> float:
    """Eq. (11) (reading R13 unless literal_tc)."""
    per_block = k.Ops * k.RX * k.RY * warp_blk(k) / g.Clock
    return act_blks(g, k) * per_block if literal_tc else per_block


def f_hide(g: GPU, k: Kernel, n: int) -> float:
    """Latency-hiding factor f of Eqs. (12)-(13) (reading R14)."""
    if n <= 1:
        return 1.0
    w = n * warp_blk(k)
    if g.Warp_SM <= 1:
        return float(n)
    val = 1.0 + (n - 1) * (1.0 - (w - 1) / (g.Warp_SM - 1))
    return min(max(val, 1.0), float(n))


def t_s(g: GPU, k: Kernel, literal_tc: bool = False) -> float:
    """Eq. (12)."""
    a = act_blks(g, k)
    return f_hide(g, k, a) * t_m(g, k) + a * t_c(g, k, literal_tc)


def t_l(g: GPU, k: Kernel, literal_tc: bool = False) -> float:
    """Eq. (13)."""
    rb = rem_blks(g, k)
    return f_hide(g, k, rb) * t_m(g, k) + rb * t_c(g, k, literal_tc)


def perf(g: GPU, k: Kernel, literal_tc: bool = False) -> float:
    """Eq. (14): predicted points per second (LX*LY points per plane time)."""
    if act_blks(g, k) < 1:
        return 0.0
    return (k.LX * k.LY) / (t_s(g, k, literal_tc) * (stages(g, k) - 1) + t_l(g, k, literal_tc))


def top_n(M: int, beta: float) -> int:
    """N = beta/100 * M, reading R15."""
    return max(1, math.ceil(beta * M / 100.0))
