"""INT timing probe (1080p S64 by default): int_interpolate alone, L2 flushed (read) before each,
for ME_OPT_INT_KERNEL 0 (per-thread global loads) and 1 (shared-memory tiled); outputs compared."""
import os
import statistics
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import __graft_entry__ as ge  # noqa: E402

ge.build()
import paper_conf_icpp_ilicmrs14_b200 as F  # noqa: E402
from synth import CONFIGS, make_workload  # noqa: E402

cfg = CONFIGS[sys.argv[1] if len(sys.argv) > 1 else "1080p_sa64_4rf"]
_, rfs = make_workload(cfg)
me = F.MotionEstimator(cfg.width, cfg.height, cfg.sa_range, cfg.n_rf)
rf = torch.from_numpy(rfs[0]).cuda()
flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
out = {}
for k in (0, 1, 0, 1):
    me.set_option(me.OPT_INT_KERNEL, k)
    sf = me.new_sf()
    ts = []
    for i in range(30):
        flush.max()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        me.interpolate(rf, out=sf)
        b.record()
        torch.cuda.synchronize()
        ts.append(a.elapsed_time(b))
    out[k] = sf
    print(f"int_kernel={k}: {statistics.median(ts) * 1e3:.1f} us (min {min(ts) * 1e3:.1f}), "
          f"equal: {torch.equal(out[0], sf)}")
