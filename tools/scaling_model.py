#!/usr/bin/env python3
"""Modelled multi-GPU efficiency of the two Stage-1 partitions.

The band-pipeline recurrence of sw_api.cu (model_fill_time, the same model
choose_variant runs): with Q resident CTAs, nb bands, lag columns between
consecutive bands and cps columns per second per CTA,

    T(nb, Q, n) = (max((nb - 1) lag, floor((nb - 1) / Q) n + ((nb - 1) mod Q) lag) + n) / cps

Column stripes (one stripe of n / P columns per GPU): stripe g starts band 0
after g stripe sweeps, T_P = (P - 1) (n / P) / cps + T(nb, Q, n / P).
Band-cyclic (GPU g runs bands g, g + P, ...; one pipeline of P Q CTAs):
T_P = T(nb, P Q, n).  One GPU may add the tail launch: the
rows after the last full wave as 2048-row bands, one per SM.

Special rows (every k rows) that are not band bottoms slow the band that holds
them, and a slow band sets the pace of every band after it: the model
multiplies T by the measured factor (profiles/r02_spm3.txt): 1.049 when
they sit inside strips (the GEN kernel's staged rows, k not a multiple of
alpha), 1.099 at strip bottoms inside a band (k a multiple of alpha but not of
the band height).

Efficiency = T_1 / (P T_P), T_1 the best single-GPU time (tail included).
cps are the measured per-CTA column speeds (one B200; sw_api.cu kCands).
"""
import math

GEOMS = {  # variant: (alpha, band height, CTAs per SM, lag columns, cps_full, cps_solo)
    1: (16, 4096, 1, (2 * 8 + 2) * 64, 8.08e6, 7.74e6),
    8: (32, 4096, 2, (2 * 4 + 2) * 64, 4.25e6, 7.86e6),
    13: (30, 3840, 2, (2 * 4 + 2) * 64, 4.45e6, 8.17e6),
    10: (32, 8192, 1, (2 * 8 + 2) * 64, 4.49e6, 4.49e6),
    14: (34, 8704, 1, (2 * 8 + 2) * 64, 4.244e6, 4.244e6),
}
TAIL = (2048, (2 * 4 + 2) * 64, 12.0e6)  # alpha 16 x 4 warps, one CTA per SM (kTailCands)
NSM = 148
CONFIGS = {  # m, n, k (the bench / SURVEY special-row interval)
    "C3": (5_000_000, 5_000_000, 65_536),
    "C4": (10_000_000, 10_000_000, 131_072),
    "C5": (32_799_110, 46_944_323, 262_144),
}


def fill(nb, Q, n, lag, cps):
    b = nb - 1
    return (max(b * lag, (b // Q) * n + (b % Q) * lag) + n) / cps


def special_factor(g, m, k):
    al, bh = GEOMS[g][0], GEOMS[g][1]
    if k <= 0 or k >= m or k % bh == 0:
        return 1.0
    return 1.099 if k % al == 0 else 1.049 if k >= bh else 4.0


def t_stripes(m, n, k, P, g):
    al, bh, per, lag, cf, cs = GEOMS[g]
    nb = math.ceil(m / bh)
    Q = per * NSM
    cps = cs if nb <= NSM else cf
    w = n / P
    return ((P - 1) * w / cps + fill(nb, Q, w, lag, cps)) * special_factor(g, m, k)


def t_cyclic(m, n, k, P, g):
    al, bh, per, lag, cf, cs = GEOMS[g]
    nb = math.ceil(m / bh)
    Q = per * NSM * P
    cps = cs if nb <= NSM * P else cf
    return fill(nb, Q, n, lag, cps) * special_factor(g, m, k)


def t_one(m, n, k, g):
    """One GPU, with the tail launch when it helps (sw_api.cu choose_tail)."""
    al, bh, per, lag, cf, cs = GEOMS[g]
    t = t_cyclic(m, n, k, 1, g)
    Q = per * NSM
    nb = math.ceil(m / bh)
    nb1 = (nb // Q) * Q
    if per == 1 and Q < nb != nb1:
        tbh, tlag, tcps = TAIL
        nb2 = math.ceil((m - nb1 * bh) / tbh)
        if nb2 <= NSM:
            tt = (fill(nb1, Q, n, lag, cf) + (n + (nb2 - 1) * tlag) / tcps) * special_factor(g, m, k)
            t = min(t, tt)
    return t


def table():
    rows = []
    for name, (m, n, k) in CONFIGS.items():
        t1 = min(t_one(m, n, k, g) for g in GEOMS)
        for P in (1, 2, 4, 8):
            if P == 1:
                s = c = min((t_one(m, n, k, g), g) for g in GEOMS)
            else:
                s = min((t_stripes(m, n, k, P, g), g) for g in GEOMS)
                c = min((t_cyclic(m, n, k, P, g), g) for g in GEOMS)
            rows.append((name, P, t1 / (P * s[0]), s[1], t1 / (P * c[0]), c[1], m * n / c[0] / 1e9))
    return rows


if __name__ == "__main__":
    print(f"{'config':6} {'P':>2} {'stripes eff':>12} {'(var)':>5} {'cyclic eff':>11} {'(var)':>5} {'cyclic GCUPS':>13}")
    for name, P, es, gs, ec, gc, gcups in table():
        print(f"{name:6} {P:2d} {es:12.3f} {gs:5d} {ec:11.3f} {gc:5d} {gcups:13.0f}")
