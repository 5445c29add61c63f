"""Run the bench workload's step a few times for ncu (NVTX range 'profiled' around the last step).
usage: python tools/profile_step.py [--infer-only|--train-only] [--steps N]"""
import argparse, os, sys
sys.path.insert(0, os.path.join(os.path.dirname(os.path.abspath(__file__)), ".."))
import numpy as np, torch
from paper_conf_sigcomm_shubhas23_b200 import binding as B, specs as S, synth
ap = argparse.ArgumentParser()
ap.add_argument("--infer-only", action="store_true")
ap.add_argument("--train-only", action="store_true")
ap.add_argument("--steps", type=int, default=2)
ap.add_argument("--batch", type=int, default=256)
ap.add_argument("--k", type=int, default=1024)
ap.add_argument("--taus", type=str, default="0.3,0.5,0.7", help="exit thresholds (bench-calibrated: 0.43,0.23,0.26)")
a = ap.parse_args()
spec = S.resnet18_ee()
p = synth.init_params(spec, seed=1)
xb, y = synth.drifted_images(max(a.batch, a.k), 224, 224, 3, seed=1)
x = torch.from_numpy(xb.view(np.int16)).cuda().view(torch.bfloat16)
lab = torch.from_numpy(y).cuda()
m = B.Model(spec, max(a.batch, a.k), params=p)
app = B.App([m])
outs = B.alloc_outs(m, a.batch)
for i in range(a.steps):
    last = i == a.steps - 1
    if last:
        torch.cuda.synchronize()
        torch.cuda.nvtx.range_push("profiled")
    if not a.train_only:
        app.infer(x[:a.batch], [float(t) for t in a.taus.split(",")], [outs])
    if not a.infer_only:
        m.retrain_step(x[:a.k], lab[:a.k], lr=0.01)
    if last:
        torch.cuda.synchronize()
        torch.cuda.nvtx.range_pop()
torch.cuda.synchronize()
print("counts", outs["exit_counts"].cpu().numpy())
