"""Small ME/INT/SME/stream cases for compute-sanitizer (no oracle, no asserts: the tool checks)."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import paper_conf_icpp_ilicmrs14_b200 as F
from synth import gen_tex

for (W, H, S, n) in [(64, 48, 16, 2), (37, 29, 8, 1), (96, 80, 64, 2), (48, 40, 128, 1), (160, 96, 32, 2), (70, 50, 18, 1)]:
    frames = [torch.from_numpy(gen_tex(W, H, t, 1)).cuda() for t in range(n + 2)]
    me = F.MotionEstimator(W, H, S, n)
    sfs = [me.new_sf() for _ in range(n)]
    me.encode_frame(frames[n], frames[:n], sfs, n_int=n, out_me=me.new_mvs())
    me.set_fused(True)
    me.encode_frame(frames[n], frames[:n], sfs, n_int=n, out_me=me.new_mvs())
    me.set_fused(False)
    for f in frames:
        me.stream_push(f)
    me.set_rows(0, 1)
    me.stream_reset()
    for f in frames:
        me.stream_push(f)
    torch.cuda.synchronize()
    me.close()
# G21 predicted-MV centre: predictors at and beyond the clamp, with the rate term (runtime-S ME, SME RD)
for (W, H, S, n, mp) in [(64, 48, 16, 2, 6), (37, 29, 8, 1, 5), (96, 64, 32, 2, 16)]:
    frames = [torch.from_numpy(gen_tex(W, H, t, 2)).cuda() for t in range(n + 2)]
    me = F.MotionEstimator(W, H, S, n, max_pmv=mp)
    rng = np.random.default_rng(S)
    pm = torch.from_numpy(rng.integers(-mp - 3, mp + 4, (me.mb_rows * me.mb_cols, n, 2)).astype(np.int16)).cuda()
    me.set_pmv(pm)
    me.set_lambda(5)
    sfs = [me.new_sf() for _ in range(n)]
    q, qs = me.encode_frame(frames[n], frames[:n], sfs, n_int=n, out_me=me.new_mvs())[1]
    me.mode_decision(q, qs)
    for f in frames:
        me.stream_push(f)
    torch.cuda.synchronize()
    me.close()
# round 2: both INT kernels, the staged SME (incl. the overflow list at S = 128), graph replay,
# host-buffer stream, flags
for (W, H, S, n) in [(200, 72, 64, 2), (854, 40, 32, 1), (200, 72, 128, 1), (33, 17, 16, 1)]:
    frames = [torch.from_numpy(gen_tex(W, H, t, 3)).cuda() for t in range(n + 8)]
    me = F.MotionEstimator(W, H, S, n)
    for ik in (0, 1):
        me.set_option(me.OPT_INT_KERNEL, ik)
        me.interpolate(frames[0])
    me.set_option(me.OPT_SME_KERNEL, 1)
    sfs = [me.new_sf() for _ in range(n)]
    me.encode_frame(frames[n], frames[:n], sfs, n_int=n, out_me=me.new_mvs())
    me.set_option(me.OPT_SME_KERNEL, 0)
    me.set_option(me.OPT_GRAPH, 1)
    out = me.new_mvs()
    for f in frames:
        me.stream_push(f, out=out)
    me.set_option(me.OPT_GRAPH, 0)
    me.stream_reset()
    ho = (torch.empty(me.mv_shape() + (2,), dtype=torch.int16).pin_memory(),
          torch.empty(me.mv_shape(), dtype=torch.uint16).pin_memory())
    for f in frames:
        me.stream_push(f.cpu().pin_memory(), out=ho)
    flags = torch.zeros(4, dtype=torch.int32, device="cuda")
    F.stream_write_value(torch.cuda.current_stream(), flags.data_ptr(), 1)
    me.stream_reset()
    for t, f in enumerate(frames):
        me.stream_push_flags(f.data_ptr(), out[0].data_ptr(), out[1].data_ptr(), wait_flag=flags.data_ptr(),
                             wait_value=1, signal_flag=flags.data_ptr() + 4, signal_value=t + 1)
    me.sync()
    torch.cuda.synchronize()
    me.close()
# session 3: every ME RF split and every SME work split (small frames: the auto split is 3)
for (W, H, S, n) in [(96, 80, 64, 3), (64, 48, 16, 2), (48, 40, 128, 3)]:
    frames = [torch.from_numpy(gen_tex(W, H, t, 4)).cuda() for t in range(n + 1)]
    me = F.MotionEstimator(W, H, S, n)
    sfs = [me.new_sf() for _ in range(n)]
    for rpc in (-1, 0, 1, 2):
        for split in (0, 1, 2, 3):
            me.set_option(me.OPT_RF_PER_CTA, rpc)
            me.set_option(me.OPT_SME_SPLIT, split)
            me.encode_frame(frames[n], frames[:n], sfs, n_int=n if rpc == -1 and split == 0 else 0,
                            out_me=me.new_mvs())
    torch.cuda.synchronize()
    me.close()
print("sanitize cases done")
