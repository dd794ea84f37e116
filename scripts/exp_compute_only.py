"""Experiment: normal vs compute-only (no global traffic) time of the HHC kernel."""
import sys, torch
sys.path.insert(0, '.')
import paper_conf_ppopp_prajapatirradg17_b200 as hhc
kind, S, T = int(sys.argv[1]), int(sys.argv[2]), int(sys.argv[3])
s = hhc.stencil_create(kind, (S, S))
a = torch.rand(S, S, device='cuda'); b = torch.empty_like(a)
st = torch.cuda.current_stream().cuda_stream
for spec in sys.argv[4:]:
    t, thr = spec.split(':')
    tile = tuple(int(x) for x in t.split(',')) + (0,)
    hhc.stencil_run(s, a.data_ptr(), b.data_ptr(), T, tile, int(thr), st); torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(3): hhc.stencil_run(s, a.data_ptr(), b.data_ptr(), T, tile, int(thr), st)
    e1.record(); torch.cuda.synchronize(); ms = e0.elapsed_time(e1) / 3
    v = hhc.stencil_microbench(3, kind, (S, S), T, tile, int(thr))
    hw = hhc.make_hw(n_sm=148, n_v=128, mtb_sm=32, r_sm=65536, m_sm_bytes=233472, m_block_bytes=232448, C_iter_s=1.0, L_s_per_word=0.0, tau_sync_s=0.0, T_sync_s=0.0, geometry=1, threads=int(thr))
    iters = hhc.model_predict(kind, (S, S), T, tile, hw)
    print(spec, f"normal {ms:.2f} ms  compute-only {v*iters*1e3:.2f} ms  ({(S-2)**2*T/ms/1e6:.0f} vs {(S-2)**2*T/(v*iters*1e3)/1e6:.0f} G/s)", flush=True)
