"""Per-band timeline of the packed Stage-1 kernel on C2 (SWB_DEBUG_TIMES):
band start, the time its tile-0 border became available (io0: the band-start
wait of the wavefront), border-wait totals, band end."""
import os, sys, ctypes
sys.path.insert(0, '/root/repo')
os.environ['SWB_DEBUG_TIMES'] = '1'
import numpy as np, torch, synth
from paper_conf_ipps_sandesm11_b200 import Context
cfg = synth.CONFIGS['C2']; A, B = synth.make_pair(cfg)
dA = torch.from_numpy(A).cuda(); dB = torch.from_numpy(B).cuda()
os.environ['SWB_VARIANT'] = '8'
ctx = Context(0)
r, _ = ctx.align_stage1_dev(dA.data_ptr(), len(A), dB.data_ptr(), len(B), 1, -3, 3, 2, k=cfg.k, sink=lambda *x: False)
lib = ctx._lib; lib.swb_debug_times.restype = ctypes.c_int64
buf = (ctypes.c_uint64 * (80 * 40000))()
n = lib.swb_debug_times(ctx._h, buf, len(buf))
raw = np.frombuffer(buf, dtype=np.uint64, count=n).reshape(-1, 80).astype(np.float64)
t0 = raw[:, 0].min()
for b in [0, 1, 2, 3, 10, 66, 132]:
    print(b, "start", (raw[b, 0] - t0) / 1e3, "io0", (raw[b, 2] - t0) / 1e3 if raw[b, 2] else None, "prog", raw[b, 3], "spins0", raw[b, 4], "end", (raw[b, 15] - t0) / 1e3, "wait_us", raw[b, 5] / 1e3, "waits", raw[b, 7], "spins", raw[b, 6])
