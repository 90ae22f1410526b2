import numpy as np, torch, sys
sys.path.insert(0, '.')
import __graft_entry__ as g; g.build()
import oracle, paper_conf_icpp_ilicmrs14_b200 as F
from synth import gen_noise
W,H,S=64,48,8
rf=gen_noise(W,H,0,W*H)
me=F.MotionEstimator(W,H,S,1)
sf=me.interpolate(torch.from_numpy(rf).cuda()).cpu().numpy()
pad,pitch,rows=oracle.sf_layout(W,H,S)
ref=oracle.int_planes(rf,pad,pitch,rows)
for ph in range(16):
    d=np.argwhere(sf[ph]!=ref[ph])
    print(ph, len(d), d[:4].tolist(), [(int(sf[ph][tuple(x)]), int(ref[ph][tuple(x)])) for x in d[:4]])
print('lib j row65:', sf[10][65][64:80].tolist())
print('orc j row65:', ref[10][65][64:80].tolist())
print('lib b row65:', sf[2][65][64:80].tolist())
