"""Role-wait analysis with the instrumented library: time the WS window kernel (layer1 fwd at B=1024) and
print per-role barrier wait cycles (avg per CTA): 0 producer<-wempty, 1 MMA<-tempty, 2 MMA<-wfull, 3 epi<-tfull."""
import ctypes, os, sys
import numpy as np, torch
sys.path.insert(0, os.path.join(os.path.dirname(os.path.abspath(__file__)), ".."))
from paper_conf_sigcomm_shubhas23_b200 import binding as B
B.LIB_PATH = os.path.join(os.path.dirname(os.path.abspath(__file__)), "timing_build", "libadainf.so")
L = B.lib()
L.adainf_dbg_wait_cycles.argtypes = [ctypes.c_void_p, ctypes.c_int]
n = int(os.environ.get("N", "1024"))
H, C = 56, 64
x = torch.randn(n, H, H, C, device="cuda").to(torch.bfloat16)
w = (torch.randn(C, 3, 3, C, device="cuda") * 0.05).to(torch.bfloat16)
b = torch.zeros(C, device="cuda")
res = torch.randn(n, H, H, C, device="cuda").to(torch.bfloat16)
buf = np.zeros((4096, 8), np.uint64)
for mode, kw in (("fwd", {}), ("fwd+res", {"res": res})):
    B.dbg_conv_fwd(x, w, b, 1, 1, act=1, **kw); torch.cuda.synchronize()
    L.adainf_dbg_wait_cycles(buf.ctypes.data, 1)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(); B.dbg_conv_fwd(x, w, b, 1, 1, act=1, **kw); e1.record(); torch.cuda.synchronize()
    L.adainf_dbg_wait_cycles(buf.ctypes.data, 1)
    ms = e0.elapsed_time(e1)
    per = buf[:148].astype(np.float64).mean(0)
    print(f"{mode}: {ms*1e3:.0f} us = {ms*1e-3*1.9e9:.0f} cycles; waits per CTA (warp-summed): prod<-wempty {per[0]/4:.0f} "
          f"mma<-tempty {per[1]:.0f} mma<-wfull {per[2]:.0f} epi<-tfull {per[3]/8:.0f} producer-issue {per[4]/4:.0f}")
