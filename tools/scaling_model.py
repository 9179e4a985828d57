#!/usr/bin/env python3
"""Modelled multi-GPU efficiency of the two Stage-1 partitions.

The band-pipeline recurrence of sw_api.cu (model_fill_time, the same model
choose_variant runs): with Q resident CTAs, nb bands, lag columns between
consecutive bands and cps columns per second per CTA,

    T(nb, Q, n) = (max((nb - 1) lag, floor((nb - 1) / Q) n + ((nb - 1) mod Q) lag) + n) / cps

Column stripes (one stripe of n / P columns per GPU): stripe g starts band 0
after g stripe sweeps, T_P = (P - 1) (n / P) / cps + T(nb, Q, n / P).
Band-cyclic (GPU g runs bands g, g + P, ...; one pipeline of P Q CTAs):
T_P = T(nb, P Q, n).  Efficiency = T_1 / (P T_P), T_1 the best single-GPU
geometry.  cps are the measured per-CTA column speeds of sw_api.cu kCands
(one B200, profiles/r01_variants.txt).
"""
import math

GEOMS = {  # variant: (band height, CTAs per SM, lag columns, cps_full, cps_solo)
    1: (4096, 1, (2 * 8 + 2) * 64, 8.08e6, 7.74e6),
    8: (4096, 2, (2 * 4 + 2) * 64, 4.25e6, 7.86e6),
    13: (3840, 2, (2 * 4 + 2) * 64, 4.45e6, 8.17e6),
    10: (8192, 1, (2 * 8 + 2) * 64, 4.49e6, 4.49e6),
}
NSM = 148
CONFIGS = {"C3": (5_000_000, 5_000_000), "C4": (10_000_000, 10_000_000), "C5": (32_799_110, 46_944_323)}


def fill(nb, Q, n, lag, cps):
    b = nb - 1
    return (max(b * lag, (b // Q) * n + (b % Q) * lag) + n) / cps


def t_stripes(m, n, P, g):
    bh, per, lag, cf, cs = GEOMS[g]
    nb = math.ceil(m / bh)
    Q = per * NSM
    cps = cs if nb <= NSM else cf
    w = n / P
    return (P - 1) * w / cps + fill(nb, Q, w, lag, cps)


def t_cyclic(m, n, P, g):
    bh, per, lag, cf, cs = GEOMS[g]
    nb = math.ceil(m / bh)
    Q = per * NSM * P
    cps = cs if nb <= NSM * P else cf
    return fill(nb, Q, n, lag, cps)


def table():
    rows = []
    for name, (m, n) in CONFIGS.items():
        t1 = min(t_cyclic(m, n, 1, g) for g in GEOMS)
        for P in (1, 2, 4, 8):
            s = min((t_stripes(m, n, P, g), g) for g in GEOMS)
            c = min((t_cyclic(m, n, P, g), g) for g in GEOMS)
            rows.append((name, P, t1 / (P * s[0]), s[1], t1 / (P * c[0]), c[1], m * n / c[0] / 1e9))
    return rows


if __name__ == "__main__":
    print(f"{'config':6} {'P':>2} {'stripes eff':>12} {'(var)':>5} {'cyclic eff':>11} {'(var)':>5} {'cyclic GCUPS':>13}")
    for name, P, es, gs, ec, gc, gcups in table():
        print(f"{name:6} {P:2d} {es:12.3f} {gs:5d} {ec:11.3f} {gc:5d} {gcups:13.0f}")
