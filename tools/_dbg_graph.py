import os, sys, numpy as np, torch
sys.path.insert(0, os.getcwd())
import synth
from paper_conf_asplos_ji0x024_b200 import msm
from oracle.curves import CURVES
c = CURVES["bn254"]; n = 1024
e0, d = synth.point_seeds(c.r, 1)
pts = torch.empty((n, 16), dtype=torch.int32, device="cuda")
msm.gen_points("bn254", e0, d, n, pts)
ks = synth.scalars_range(c.r, 0, n, 3)
ctx = msm.Context("bn254", pts, n=n)
kd = torch.from_numpy(ks.view(np.int32)).cuda()
for i in range(4):
    print("run", i, ctx.run(kd)[0] % 1000, flush=True)
print(ctx.stats(), flush=True)
t = ctx.submit(ks); print("submit ok", flush=True); print(ctx.wait(t)[0] % 1000)
