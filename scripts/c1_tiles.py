"""C1 (Jacobi-2D 256^2, T=64) tile scan on one B200: CUDA-event time of stencil_run (min of 5) per tile."""
import itertools
import json
import math
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_ppopp_prajapatirradg17_b200 as hhc  # noqa: E402
from synth import field  # noqa: E402

dims, T = (256, 256), 64
a = field(1, dims)
d_in = torch.from_numpy(a).cuda()
d_out = torch.empty_like(d_in)
h = hhc.stencil_create(hhc.JACOBI2D_5PT, dims)
s = torch.cuda.current_stream()
res = []
for tT, tS1, tS2 in itertools.product((2, 4, 6, 8, 12, 16, 24, 32), (1, 2, 3, 4, 6, 8, 12), tuple(int(v) for v in os.environ.get("C1_S2", "32,64,128,256").split(","))):
    for thr in (0,):
        try:
            hhc.stencil_run(h, d_in, d_out, T, (tT, tS1, tS2, 0), thr, s)
            torch.cuda.synchronize()
        except Exception:
            continue
        best = math.inf
        for _ in range(5):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(s)
            hhc.stencil_run(h, d_in, d_out, T, (tT, tS1, tS2, 0), thr, s)
            e1.record(s)
            e1.synchronize()
            best = min(best, e0.elapsed_time(e1))
        res.append({"tile": [tT, tS1, tS2], "ms": best, "gups": 254 * 254 * T / best / 1e6})
res.sort(key=lambda r: r["ms"])
os.makedirs("gpurun_out/c1", exist_ok=True)
json.dump(res, open("gpurun_out/c1/c1_tiles.json", "w"), indent=0)
for r in res[:10]:
    print(r)
