"""Time adainf_select_retrain at BASELINE config 5 (131,072 x 512 candidates, PCA to 64, M = 1, k = 8,192) and
config 2 (16,384 x 64 -> 16, k = 1,024) with the library's per-class events; algorithmic bytes = X read once."""
import json
import os
import sys

sys.path.insert(0, os.path.join(os.path.dirname(os.path.abspath(__file__)), ".."))
import numpy as np
import torch
from paper_conf_sigcomm_shubhas23_b200 import binding as B
from paper_conf_sigcomm_shubhas23_b200 import synth

if os.environ.get("ADAINF_LIB"):
    B.LIB_PATH = os.environ["ADAINF_LIB"]
rows = []
for N, D, P, k in [(131072, 512, 64, 8192), (16384, 64, 16, 1024), (32768, 64, 16, 2048)]:
    Xb, Wb, ref = synth.embeddings(N, D, P, seed=5)
    X = torch.from_numpy(Xb.view(np.int16)).cuda().view(torch.bfloat16)
    W = torch.from_numpy(Wb.view(np.int16)).cuda().view(torch.bfloat16)
    R = torch.from_numpy(ref).cuda()
    run = lambda: B.select_retrain(X, W, R, k)
    run()
    torch.cuda.synchronize()
    B.prof_enable(True)
    B.prof_reset()
    reps = 10
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(reps):
        run()
    e1.record()
    torch.cuda.synchronize()
    q = B.prof_query()
    B.prof_enable(False)
    ms = e0.elapsed_time(e1) / reps
    rows.append({"N": N, "D": D, "P": P, "k": k, "ms_total": round(ms, 4),
                 "classes_us": {kk: round(v[1] / reps * 1e3, 1) for kk, v in q.items() if v[0]},
                 "floor_us": round(N * D * 2 / 6.5e12 * 1e6, 1)})
print(json.dumps(rows))
