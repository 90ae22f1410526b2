"""INT launch timing probe: CUDA-event time per launch, back to back (L2 warm) vs after
a 512 MiB read / write flush, to compare with ncu's gpu__time_duration."""
import statistics
import sys
import torch
sys.path.insert(0, ".")
import paper_conf_icpp_ilicmrs14_b200 as F
from synth import gen_tex

W, H, S = 1920, 1080, 64
me = F.MotionEstimator(W, H, S, 4)
f = torch.from_numpy(gen_tex(W, H, 0, 5)).cuda()
sf = me.new_sf()
flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
st = torch.cuda.current_stream()
for _ in range(5):
    me.interpolate(f, out=sf)
torch.cuda.synchronize()
for mode in ("warm", "read", "write"):
    ts = []
    for k in range(30):
        if mode == "read":
            flush.max()
        elif mode == "write":
            flush.fill_(k & 255)
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(st)
        me.interpolate(f, out=sf)
        b.record(st)
        ts.append((a, b))
    torch.cuda.synchronize()
    v = [a.elapsed_time(b) * 1000 for a, b in ts]
    print(mode, "median us", round(statistics.median(v), 2), "min", round(min(v), 2))
# 20 launches between one pair of events (back to back)
a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
a.record(st)
for _ in range(20):
    me.interpolate(f, out=sf)
b.record(st)
torch.cuda.synchronize()
print("20 back-to-back launches: us per launch", round(a.elapsed_time(b) * 1000 / 20, 2))
