#!/usr/bin/env python3
"""Kernel-level timing of the Stage-1 fill (no reverse pass) for tuning:
python tools/fill_bench.py C3 [variants...] [--k K] [--reps R]."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import synth  # noqa: E402


def main():
    args = [a for a in sys.argv[1:] if not a.startswith("--")]
    opts = dict(a[2:].split("=") for a in sys.argv[1:] if a.startswith("--"))
    wl = args[0] if args else "C2"
    variants = [int(v) for v in args[1:]] or [int(os.environ.get("SWB_VARIANT", "1"))]
    reps = int(opts.get("reps", 2))
    cfg = synth.CONFIGS[wl]
    k = int(opts.get("k", cfg.k))
    A, B = synth.make_pair(cfg)
    dA = torch.from_numpy(A).cuda()
    dB = torch.from_numpy(B).cuda()
    from paper_conf_ipps_sandesm11_b200 import Context

    for v in variants:
        os.environ["SWB_VARIANT"] = str(v)
        ctx = Context(0)
        best = None
        for _ in range(reps):
            r, _ = ctx.align_stage1_dev(dA.data_ptr(), len(A), dB.data_ptr(), len(B), 1, -3, 3, 2, k=k,
                                        sink=(lambda *x: False) if k else None)
            st = ctx.stats()
            if best is None or st["fill_ms"] < best["fill_ms"]:
                best = st
        cells = len(A) * len(B)
        print(f"{wl} v{v} k={k} result={r.astuple()} fill_ms={best['fill_ms']:.2f} total_ms={best['total_ms']:.2f} "
              f"GCUPS(fill)={cells / best['fill_ms'] / 1e6:.1f} alpha={best['alpha']} warps={best['warps']} "
              f"grid={best['grid']} replays={best['replays']}", flush=True)
        ctx.close()


if __name__ == "__main__":
    main()
