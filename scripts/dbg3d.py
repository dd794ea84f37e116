"""Debug: one small 3D case vs the oracle (env HHC_DBG / HHC_NO_TMA select variants)."""
import sys, numpy as np, torch
sys.path.insert(0, '.')
import oracle
import paper_conf_ppopp_prajapatirradg17_b200 as hhc
from synth import field
dims = tuple(int(x) for x in (sys.argv[1] if len(sys.argv) > 1 else "20,22,40").split(','))
tile = tuple(int(x) for x in (sys.argv[2] if len(sys.argv) > 2 else "4,2,3,32").split(','))
T = int(sys.argv[3]) if len(sys.argv) > 3 else 7
a = field(7, dims)
s = hhc.stencil_create(hhc.HEAT3D_7PT, dims, mode=hhc.FUSED)
d = torch.from_numpy(a).cuda(); o = torch.empty_like(d)
hhc.stencil_run(s, d, o, T, tile); torch.cuda.synchronize()
g = o.cpu().numpy(); e = oracle.run(hhc.HEAT3D_7PT, a, T, hhc.FUSED)
bad = np.argwhere(g.view(np.uint32) != e.view(np.uint32))
print("mismatches", len(bad), bad[:5].tolist())
