"""SME launch timing probe: CUDA-event time of one sme_refine launch (1080p S64 4 RF) with the
SF planes L2-warm (back to back) vs after a 512 MiB write flush -- how much of SME is DRAM latency."""
import statistics
import sys
import torch
sys.path.insert(0, ".")
import paper_conf_icpp_ilicmrs14_b200 as F
from synth import gen_tex

W, H, S, NR = 1920, 1080, 64, 4
me = F.MotionEstimator(W, H, S, NR)
fr = [torch.from_numpy(gen_tex(W, H, t, 5)).cuda() for t in range(NR + 1)]
cf, rfs = fr[NR], [fr[NR - 1 - k] for k in range(NR)]
sfs = [me.interpolate(r) for r in rfs]
mvs, sads = me.estimate(cf, rfs)
out = None
flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
st = torch.cuda.current_stream()
for _ in range(3):
    out = me.refine(cf, sfs, mvs, sads, out=out)
torch.cuda.synchronize()
for mode in ("warm", "write-flushed"):
    ts = []
    for k in range(20):
        if mode != "warm":
            flush.fill_(k & 255)
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(st)
        out = me.refine(cf, sfs, mvs, sads, out=out)
        b.record(st)
        ts.append((a, b))
    torch.cuda.synchronize()
    v = [a.elapsed_time(b) * 1000 for a, b in ts]
    print("SME", mode, "median us", round(statistics.median(v), 2), "min", round(min(v), 2))
