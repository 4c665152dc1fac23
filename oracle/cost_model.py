"""Paper-faithful cycle cost model of KAMI -- TEST INFRASTRUCTURE ONLY.

Follows PAPER.md Sec. 4.3-4.5 equation by equation, in the paper's notation
(Table 2):

  m, n, k   matrix sizes        p     number of warps
  s_e       bytes per element   L_sm  register->SMEM latency (cycles)
  B_sm      SMEM bytes / cycle  theta_r, theta_w  bank-conflict factors (1 = none)
  O_tc      ops / cycle / tensor core   n_tc  tensor cores per SM

Readings of garbled passages ("Readings"):
  R6  3D tiles: A_i m/cbrt(p) x k/cbrt(p)^2, B_i k/cbrt(p)^2 x n/cbrt(p)
      (the worked example T_all = 68 at PAPER.md L405 only holds this way).
  R7  Eq. (7) denominator is p^(3/2) (2mnk/(sqrt(p)^3 O_tc)), pinned by
      T_cp = 4 at PAPER.md L324; Eq. (11) denominator is p^(4/3).
  R8  T_all keeps p / n_tc without a ceiling (reproduces T_all = 60, L250).
  R21 V_cm is the per-stage volume of Eqs. (1)/(5)/(9).

Pinned by tests/test_cost_model.py against the three worked examples
(PAPER.md L246-250, L322-324, L405).
"""
from __future__ import annotations

from dataclasses import dataclass


@dataclass(frozen=True)
class PaperCost:
    V_cm: float
    T_cm: float
    T_cp: float
    T_all: float


def kami_1d(m, n, k, p, s_e, L_sm, B_sm, theta_r, theta_w, O_tc, n_tc) -> PaperCost:
    """Sec. 4.3, Eqs. (1)-(4)."""
    # Eq. (1): one warp writes B_z (k/p x n), p-1 warps read it.
    V_cm = 1 * (k / p * n) * s_e + (p - 1) * (k / p * n) * s_e
    # Eq. (2)
    T_cm = L_sm + (k * n * s_e) / (theta_w * p * B_sm) + ((p - 1) * k * n * s_e) / (theta_r * p * B_sm)
    # Eq. (3): flops(A_i[:, z-slice], B_z^Recv) / O_tc = 2 (m/p)(k/p) n / O_tc
    T_cp = 2 * (m / p) * (k / p) * n / O_tc
    # Eq. (4): p stages, each T_cm + (p / n_tc) T_cp
    T_all = p * (T_cm + (p / n_tc) * T_cp)
    return PaperCost(V_cm, T_cm, T_cp, T_all)


def kami_2d(m, n, k, p, s_e, L_sm, B_sm, theta_r, theta_w, O_tc, n_tc) -> PaperCost:
    """Sec. 4.4, Eqs. (5)-(8)."""
    q = p ** 0.5
    a_tile = (m / q) * (k / q)
    b_tile = (k / q) * (n / q)
    # Eq. (5): sqrt(p) writers and sqrt(p)(sqrt(p)-1) readers for each of A and B
    V_cm = (q * a_tile + q * (q - 1) * a_tile) * s_e + (q * b_tile + q * (q - 1) * b_tile) * s_e
    # Eq. (6)
    T_cm = L_sm + ((m * k + n * k) * s_e) / (theta_w * q * B_sm) + ((q - 1) * (m * k + n * k) * s_e) / (theta_r * q * B_sm)
    # Eq. (7) (reading R7): 2 (m/sqrt p)(k/sqrt p)(n/sqrt p) / O_tc
    T_cp = 2 * (m / q) * (k / q) * (n / q) / O_tc
    # Eq. (8)
    T_all = q * (T_cm + (p / n_tc) * T_cp)
    return PaperCost(V_cm, T_cm, T_cp, T_all)


def kami_3d(m, n, k, p, s_e, L_sm, B_sm, theta_r, theta_w, O_tc, n_tc) -> PaperCost:
    """Sec. 4.5, Eqs. (9)-(12) with reading R6 for the tile shapes."""
    c = round(p ** (1.0 / 3.0))
    assert c ** 3 == p, "3D needs a cubic warp count"
    a_tile = (m / c) * (k / (c * c))
    b_tile = (k / (c * c)) * (n / c)
    # Eq. (9), per layer: cbrt(p) writers, cbrt(p)(cbrt(p)-1) readers, times cbrt(p) layers
    V_cm = c * ((c * a_tile + c * (c - 1) * a_tile) * s_e + (c * b_tile + c * (c - 1) * b_tile) * s_e)
    # Eq. (10)
    T_cm = L_sm + ((m * k + n * k) * s_e) / (theta_w * c * B_sm) + ((c - 1) * (m * k + n * k) * s_e) / (theta_r * c * B_sm)
    # Eq. (11) (reading R7): 2 (m/c)(k/c^2)(n/c) / O_tc
    T_cp = 2 * (m / c) * (k / (c * c)) * (n / c) / O_tc
    # Eq. (12)
    T_all = c * (T_cm + (p / n_tc) * T_cp)
    return PaperCost(V_cm, T_cm, T_cp, T_all)


def paper_model(variant: str, m, n, k, p, s_e, L_sm, B_sm, theta_r, theta_w, O_tc, n_tc) -> PaperCost:
    fn = {"1d": kami_1d, "2d": kami_2d, "3d": kami_3d}[variant.lower()]
    return fn(m, n, k, p, s_e, L_sm, B_sm, theta_r, theta_w, O_tc, n_tc)


def register_estimate(m, n, k, regs_per_elem, threads) -> float:
    """Sec. 4.7: registers per thread to hold A, B and C of
    order m=n=k: (mk + kn + mn) * regs_per_elem / threads."""
    return (m * k + k * n + m * n) * regs_per_elem / threads
