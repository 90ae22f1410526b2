"""SME timing probe on the bench workload (1080p S64 4 RF): SME alone, L2 flushed before each
launch, for the global-load and the shared-memory staged kernel, + the staged kernel's
overflow count.  python tools/sme_probe.py [config]"""
import ctypes
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
cf, rfs = make_workload(cfg)
me = F.MotionEstimator(cfg.width, cfg.height, cfg.sa_range, cfg.n_rf)
tcf, trfs = torch.from_numpy(cf).cuda(), [torch.from_numpy(r).cuda() for r in rfs]
sfs = [me.interpolate(r) for r in trfs]
mvs, sads = me.estimate(tcf, trfs)
flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
F.lib().me_sme_overflow_count.argtypes = [ctypes.c_void_p]
ref = None
for k in (0, 1, 0, 1):
    me.set_option(me.OPT_SME_KERNEL, k)
    ts = []
    for i in range(20):
        flush.fill_(i)
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        q, qs = me.refine(tcf, sfs, mvs, sads)
        b.record()
        torch.cuda.synchronize()
        ts.append(a.elapsed_time(b))
    ovf = F.lib().me_sme_overflow_count(me._ctx) if k else -1
    if ref is None:
        ref = (q.clone(), qs.clone())
    same = torch.equal(ref[0], q) and torch.equal(ref[1], qs)
    print(f"sme_kernel={k}: {statistics.median(ts) * 1e3:.1f} us (min {min(ts) * 1e3:.1f}), overflow items {ovf} "
          f"of {cfg.n_rf * me.mb_rows * me.mb_cols}, equal to global kernel: {same}")
