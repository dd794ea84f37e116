"""Experiment: does running two independent hexagons per SM (2 CTAs) beat one?"""
import sys, time, torch
sys.path.insert(0, '.')
import paper_conf_ppopp_prajapatirradg17_b200 as hhc
kind = int(sys.argv[1]) if len(sys.argv) > 1 else 2
S = int(sys.argv[2]) if len(sys.argv) > 2 else 16384
T = int(sys.argv[3]) if len(sys.argv) > 3 else 192
s = hhc.stencil_create(kind, (S, S))
a = torch.rand(S, S, device='cuda')
b = torch.empty_like(a)
st = torch.cuda.current_stream().cuda_stream
for spec in sys.argv[4:]:
    t, thr = spec.split(':')
    tile = tuple(int(x) for x in t.split(',')) + (0,)
    try:
        hhc.stencil_run(s, a.data_ptr(), b.data_ptr(), T, tile, int(thr), st)
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(3):
            hhc.stencil_run(s, a.data_ptr(), b.data_ptr(), T, tile, int(thr), st)
        e1.record(); torch.cuda.synchronize()
        ms = e0.elapsed_time(e1) / 3
        print(spec, f"{ms:.2f} ms", f"{(S-2)**2*T/ms/1e6:.1f} G/s", flush=True)
    except Exception as e:
        print(spec, 'ERR', e, flush=True)
