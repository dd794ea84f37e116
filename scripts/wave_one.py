"""One wavefront-schedule run of W1 (for ncu): python scripts/wave_one.py tT tS"""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_ppopp_prajapatirradg17_b200 as hhc  # noqa: E402
from synth import field  # noqa: E402

tT, tS = int(sys.argv[1]), int(sys.argv[2])
n, T = (1 << 22) + 2, 1024
a = field(5, (n,))
d_in = torch.from_numpy(a).cuda()
d_out = torch.empty_like(d_in)
h = hhc.stencil_create(hhc.JACOBI1D_3PT, (n,))
for _ in range(2):
    hhc.stencil_run_wavefront(h, d_in, d_out, T, (tT, tS), torch.cuda.current_stream())
torch.cuda.synchronize()
print("ok")
