"""Determinism check of the stem weight gradient under the parity test's conditions."""
import sys, os
sys.path.insert(0, os.path.join(os.path.dirname(os.path.abspath(__file__)), ".."))
import torch
from paper_conf_sigcomm_shubhas23_b200 import binding as B
for case in [(2, 224, 224, 3), (3, 64, 48, 3)]:
    n, H, W, cin = case
    g = torch.Generator().manual_seed(4)
    x = torch.randn(n, H, W, cin, generator=g).to(torch.bfloat16).cuda()
    dz = torch.randn(n, H // 2, W // 2, 64, generator=g).to(torch.bfloat16).cuda()
    dz = dz * (torch.rand(n, H // 2, W // 2, 64, generator=g) < 0.25).to(torch.bfloat16).cuda()
    dw, db = B.dbg_stem_wgrad(x, dz)
    torch.cuda.synchronize()
    ref = torch.nn.grad.conv2d_weight(x.float().permute(0, 3, 1, 2), (64, cin, 7, 7), dz.float().permute(0, 3, 1, 2),
                                      stride=2, padding=3).permute(0, 2, 3, 1)
    for k in range(3):
        dw2, db2 = B.dbg_stem_wgrad(x, dz)
        torch.cuda.synchronize()
        d = (dw2 - dw).abs()
        nz = torch.nonzero(d)
        print(case, k, "maxdiff", float(d.max()), "ndiff", nz.shape[0], nz[:8, 1:].tolist(),
              "rel1 %.2e rel2 %.2e" % (float((dw - ref).norm() / ref.norm()), float((dw2 - ref).norm() / ref.norm())))
