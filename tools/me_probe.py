"""ME timing probe: me_estimate alone (L2 flushed before each) on BASELINE configs, as a fraction of
the ALU px-absdiff roofline; build knobs via FEVES_NVCC_EXTRA (e.g. -DFEVES_ME_MINB=5).
python tools/me_probe.py [cfg ...]"""
import os
import statistics
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import __graft_entry__ as ge  # noqa: E402

ge.build()
import paper_conf_icpp_ilicmrs14_b200 as F  # noqa: E402
from synth import CONFIGS, make_workload  # noqa: E402

flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
for name in sys.argv[1:] or ["cif", "1080p_sa32", "1080p_sa64_4rf"]:
    cfg = CONFIGS[name]
    cf, rfs = make_workload(cfg)
    me = F.MotionEstimator(cfg.width, cfg.height, cfg.sa_range, cfg.n_rf)
    tcf, trfs = torch.from_numpy(cf).cuda(), [torch.from_numpy(r).cuda() for r in rfs]
    px = me.mb_rows * me.mb_cols * cfg.n_rf * cfg.sa_range ** 2 * 256
    for k in (0, 1):
        ts = []
        for i in range(20):
            flush.fill_(i)
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record()
            m, s = me.estimate(tcf, trfs)
            b.record()
            torch.cuda.synchronize()
            ts.append(a.elapsed_time(b))
        t = statistics.median(ts)
        print(f"{name} pass {k}: {t * 1e3:.1f} us (min {min(ts) * 1e3:.1f}), "
              f"{px / (t / 1e3) / 74.45e12:.3f} of the ALU roofline")
    me.close()
