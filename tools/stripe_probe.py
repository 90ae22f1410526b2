"""Per-rank stripe timing on ONE GPU: the step a rank of an N-way MB-row split runs (1080p, 4 RF,
SA 64), i.e. me_stream_push with me_set_rows(stripe) + halo-only copies, graph per frame, L2
flushed before each step, CUDA events.  The strong-scaling ceiling of the N-GPU run is
t(full frame) / (N * t(largest stripe)) before any exchange cost.
python tools/stripe_probe.py [N ...]"""
import os
import statistics
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import __graft_entry__ as ge  # noqa: E402

ge.build()
import paper_conf_icpp_ilicmrs14_b200 as F  # noqa: E402
from paper_conf_icpp_ilicmrs14_b200.shard import stripes  # noqa: E402
from synth import CONFIGS, ippp_sequence  # noqa: E402

cfg = CONFIGS["1080p_sa64_4rf"]
frames = [torch.from_numpy(f).cuda() for f in ippp_sequence(cfg.width, cfg.height, cfg.n_rf + 4, 1002)]
flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
full = None
RPC = [int(x) for x in os.environ.get("RPC", "1").split(",")]   # ME_OPT_RF_PER_CTA values to sweep
SPL = [int(x) for x in os.environ.get("SPLIT", "0").split(",")]  # ME_OPT_SME_SPLIT values to sweep
for n, rpc, spl in [(int(a), r, p) for a in (sys.argv[1:] or ["1", "2", "4", "8"]) for r in RPC for p in SPL]:
    me = F.MotionEstimator(cfg.width, cfg.height, cfg.sa_range, cfg.n_rf)
    me.set_option(me.OPT_RF_PER_CTA, rpc)
    me.set_option(me.OPT_SME_SPLIT, spl)
    if os.environ.get("PIPE"):
        me.set_option(me.OPT_PIPELINE_RF, int(os.environ["PIPE"]))
    r0, r1 = stripes(me.mb_rows, n)[0]                  # the largest stripe (first ranks get the extra row)
    me.set_rows(r0, r1)
    me.set_option(me.OPT_GRAPH, int(os.environ.get("GRAPH", "1")))
    if n > 1:
        me.set_option(me.OPT_HALO_ONLY, 1)
    out = (torch.empty(me.mv_shape() + (2,), dtype=torch.int16, device="cuda"),
           torch.empty(me.mv_shape(), dtype=torch.uint16, device="cuda"))
    me.stream_reset()
    for i in range(cfg.n_rf + 4):
        me.stream_push(frames[i % len(frames)], out=out)
    me.sync()
    ts = []
    for i in range(40):
        flush.fill_(i)
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        me.stream_push(frames[i % len(frames)], out=out)
        b.record()
        torch.cuda.synchronize()
        ts.append(a.elapsed_time(b))
    t = statistics.median(ts)
    me.set_timing(True)                                   # instrumented pass: per-module device times
    mods = []
    for i in range(10):
        flush.fill_(i)
        me.stream_push(frames[i % len(frames)], out=out)
        me.sync()
        mods.append(me.timings())
    me.set_timing(False)
    mi = [statistics.median(m[k] for m in mods) * 1e3 for k in range(3)]
    full = t if (n == 1 and full is None) else full
    eff = (full / (n * t)) if full else float("nan")
    print(f"N={n} rf/cta={rpc or cfg.n_rf} sme_split={spl}: stripe rows [{r0},{r1}) ({r1 - r0} rows): {t * 1e3:.1f} us per frame, "
          f"compute-only strong-scaling ceiling {eff:.3f}; INT {mi[0]:.1f} / ME {mi[1]:.1f} / SME {mi[2]:.1f} us")
    me.close()
