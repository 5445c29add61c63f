"""Time the space-to-depth stem kernels at the retrain batch (ResNet-18 224x224) with the library's
per-class CUDA-event profiler."""
import os, sys
sys.path.insert(0, os.path.join(os.path.dirname(os.path.abspath(__file__)), ".."))
import torch
from paper_conf_sigcomm_shubhas23_b200 import binding as B
if os.environ.get("ADAINF_LIB"):  # A/B against another build
    B.LIB_PATH = os.environ["ADAINF_LIB"]
n = int(os.environ.get("N", "1024"))
reps = int(os.environ.get("REPS", "5"))
x = torch.randn(n, 224, 224, 3, device="cuda").to(torch.bfloat16)
w = (torch.randn(64, 7, 7, 3, device="cuda") * 0.08).to(torch.bfloat16)
b = torch.randn(64, device="cuda") * 0.1
dz = torch.randn(n, 112, 112, 64, device="cuda").to(torch.bfloat16)
for name, fn in [("fwd", lambda: B.dbg_stem_fwd(x, w, b)), ("wgrad", lambda: B.dbg_stem_wgrad(x, dz))]:
    fn(); torch.cuda.synchronize()
    B.prof_enable(True); B.prof_reset()
    for _ in range(reps): fn()
    torch.cuda.synchronize()
    q = B.prof_query(); B.prof_enable(False)
    print(name, {k: round(v[1] / reps * 1e3, 1) for k, v in q.items() if v[0]}, "us per call", flush=True)
