"""synth -- seeded synthetic DNA pairs shaped like the paper's workloads.

This is the ONE module both the CUDA path's tests/bench and the oracle's
tests use for inputs.  It holds none of the method's arithmetic: it only
draws bases.

Recipe
------
* Generator: ``numpy.random.Generator(PCG64(seed))``.  Background is i.i.d.
  uniform over ACGT.
* ``plant(src, s, g, mu, ins_frac)`` walks ``src`` base by base.  At each base,
  with probability ``g`` an indel of length ~ Geometric(mean ``mu``) starts:
  with probability ``ins_frac`` it is an insertion (that many random bases are
  emitted, then the current base is copied), otherwise a deletion (that many
  source bases, starting at the current one, are skipped).  Otherwise the base
  is copied, substituted with probability ``s`` by a uniformly chosen
  different base.  The result overwrites B from ``b0`` on, truncated at n.
* All random draws happen up front in a fixed order, so a config is a pure
  function of its seed.

Configs C1..C5 mirror BASELINE.json ``configs`` and the paper's Table II/III
shapes; see CONFIGS below.
"""
from __future__ import annotations

import hashlib
from dataclasses import dataclass, field

import numpy as np

ALPHABET = np.frombuffer(b"ACGT", dtype=np.uint8)


def _rng(seed: int) -> np.random.Generator:
    return np.random.Generator(np.random.PCG64(seed))


def random_codes(rng: np.random.Generator, n: int) -> np.ndarray:
    return rng.integers(0, 4, size=n, dtype=np.uint8)


def to_ascii(codes: np.ndarray) -> np.ndarray:
    return ALPHABET[codes]


def plant(rng: np.random.Generator, src: np.ndarray, s: float, g: float, mu: float, ins_frac: float) -> np.ndarray:
    """Mutated copy of ``src`` (codes 0..3); see module docstring."""
    L = len(src)
    u_ev = rng.random(L, dtype=np.float32) if L else np.zeros(0, np.float32)
    u_type = rng.random(L, dtype=np.float32)
    lens = rng.geometric(1.0 / mu, size=L) if (L and g > 0) else np.ones(L, np.int64)
    u_sub = rng.random(L, dtype=np.float32)
    offs = rng.integers(1, 4, size=L, dtype=np.uint8)
    subbed = src.copy()
    mask = u_sub < s
    subbed[mask] = (src[mask] + offs[mask]) % 4
    ev = np.flatnonzero(u_ev < g) if g > 0 else np.zeros(0, np.int64)
    n_ins = int(lens[ev][u_type[ev] < ins_frac].sum()) if len(ev) else 0
    ins_pool = random_codes(rng, n_ins)
    out = []
    pos = 0
    ip = 0
    for e in ev:
        if e < pos:
            continue  # inside a deletion
        out.append(subbed[pos:e])
        ln = int(lens[e])
        if u_type[e] < ins_frac:
            out.append(ins_pool[ip : ip + ln])
            ip += ln
            out.append(subbed[e : e + 1])
            pos = e + 1
        else:
            pos = e + ln
    if pos < L:
        out.append(subbed[pos:])
    return np.concatenate(out) if out else np.zeros(0, np.uint8)


def plant_gapless(rng: np.random.Generator, src: np.ndarray, n_sub: int) -> np.ndarray:
    """Copy of ``src`` with exactly ``n_sub`` substitutions at random distinct positions."""
    out = src.copy()
    pos = rng.choice(len(src), size=n_sub, replace=False)
    offs = rng.integers(1, 4, size=n_sub, dtype=np.uint8)
    out[pos] = (out[pos] + offs) % 4
    return out


@dataclass(frozen=True)
class Config:
    name: str
    m: int
    n: int
    seed: int
    k: int  # special_row_interval
    kind: str  # "plant", "gapless", "whole", "chromosome"
    params: dict = field(default_factory=dict)
    gpus: tuple = (1,)
    note: str = ""


# match +1, mismatch -3, first gap -5, extension -2: gap_open = 3, gap_ext = 2 (reading S2)
PAPER_SCORES = dict(match=1, mismatch=-3, gap_open=3, gap_ext=2)

CONFIGS = {
    "C1": Config("C1", 50_000, 50_000, 1, 1024, "plant",
                 dict(L=2000, a0=24_000, b0=10_000, s=0.05, g=0.002, mu=3.0, ins_frac=0.5),
                 note="BASELINE configs[0]: 50 KBP x 50 KBP, one planted 2 KBP region"),
    "C2": Config("C2", 542_868, 536_165, 2, 3840, "gapless",
                 dict(L=92, n_sub=11, a0=308_466, b0=455_042),
                 note="BASELINE configs[1]: Table II 543K x 536K sizes; Table III row 2 shape (P:392); "
                      "k = 3840, a multiple of every packed strip height (16, 30, 32)"),
    "C3": Config("C3", 5_000_000, 5_000_000, 3, 65_536, "whole",
                 dict(s=5e-5, g=3e-5, mu=10.0, ins_frac=0.5, b0=0),
                 gpus=(1, 2), note="BASELINE configs[2]: whole-length homology (B. anthracis shape, P:395)"),
    "C4": Config("C4", 10_000_000, 10_000_000, 4, 131_072, "plant",
                 dict(L=9107, a0=6_000_000, b0=5_000_000, s=0.005, g=5e-4, mu=2.0, ins_frac=0.5),
                 gpus=(1, 2, 4, 8), note="BASELINE configs[3]: Drosophila 2L/3L plant shape (P:397)"),
    "C5": Config("C5", 32_799_110, 46_944_323, 5, 262_144, "chromosome",
                 dict(b0=13_841_680, L=32_718_231, s=0.016, g=0.002, mu=20.7, ins_frac=0.63),
                 gpus=(8,), note="BASELINE configs[4]: chimp chr22 x human chr21 shape (Tables III, X)"),
}


def make_codes(cfg: Config | str):
    """(A_codes, B_codes) as uint8 arrays of 0..3 for a config."""
    if isinstance(cfg, str):
        cfg = CONFIGS[cfg]
    rng = _rng(cfg.seed)
    A = random_codes(rng, cfg.m)
    B = random_codes(rng, cfg.n)
    p = cfg.params
    if cfg.kind == "plant":
        seg = plant(rng, A[p["a0"] : p["a0"] + p["L"]], p["s"], p["g"], p["mu"], p["ins_frac"])
        b0 = p["b0"]
        seg = seg[: max(0, cfg.n - b0)]
        B[b0 : b0 + len(seg)] = seg
    elif cfg.kind == "gapless":
        seg = plant_gapless(rng, A[p["a0"] : p["a0"] + p["L"]], p["n_sub"])
        B[p["b0"] : p["b0"] + len(seg)] = seg[: max(0, cfg.n - p["b0"])]
    elif cfg.kind == "whole":
        seg = plant(rng, A, p["s"], p["g"], p["mu"], p["ins_frac"])
        b0 = p["b0"]
        seg = seg[: max(0, cfg.n - b0)]
        B[b0 : b0 + len(seg)] = seg
    elif cfg.kind == "chromosome":
        seg = plant(rng, A[: p["L"]], p["s"], p["g"], p["mu"], p["ins_frac"])
        b0 = p["b0"]
        seg = seg[: max(0, cfg.n - b0)]
        B[b0 : b0 + len(seg)] = seg
    else:
        raise ValueError(cfg.kind)
    return A, B


def make_pair(cfg: Config | str):
    """(A, B) as ASCII uint8 arrays (bytes 'A','C','G','T')."""
    A, B = make_codes(cfg)
    return to_ascii(A), to_ascii(B)


def random_pair(seed: int, m: int, n: int, lower_frac: float = 0.0, plant_len: int = 0,
                s: float = 0.05, g: float = 0.01, mu: float = 3.0, ins_frac: float = 0.5):
    """Small seeded pair for parity tests: random background, optionally one planted
    homologous segment (A[a0:a0+plant_len] mutated into B at b0), optionally a
    fraction of lower-case letters (the alphabet is case-insensitive)."""
    rng = _rng(seed)
    A = random_codes(rng, m)
    B = random_codes(rng, n)
    if plant_len and m > 0 and n > 0:
        L = min(plant_len, m)
        a0 = int(rng.integers(0, m - L + 1))
        seg = plant(rng, A[a0 : a0 + L], s, g, mu, ins_frac)
        b0 = int(rng.integers(0, max(1, n - min(len(seg), n) + 1)))
        seg = seg[: n - b0]
        B[b0 : b0 + len(seg)] = seg
    a, b = to_ascii(A), to_ascii(B)
    if lower_frac > 0:
        la = rng.random(m) < lower_frac
        lb = rng.random(n) < lower_frac
        a = a.copy(); b = b.copy()
        a[la] += 32
        b[lb] += 32
    return a, b


def sha256_pair(A: np.ndarray, B: np.ndarray) -> str:
    h = hashlib.sha256()
    h.update(np.ascontiguousarray(A).tobytes())
    h.update(b"|")
    h.update(np.ascontiguousarray(B).tobytes())
    return h.hexdigest()
