"""Experiment: normal vs compute-only (no global traffic) time of the HHC kernel.
usage: python scripts/exp_compute_only.py KIND S1xS2[xS3] T tile:threads ..."""
import sys, torch
sys.path.insert(0, '.')
import paper_conf_ppopp_prajapatirradg17_b200 as hhc
kind, dims, T = int(sys.argv[1]), tuple(int(x) for x in sys.argv[2].split('x')), int(sys.argv[3])
if len(dims) == 1: dims = (dims[0], dims[0])
s = hhc.stencil_create(kind, dims)
a = torch.rand(*dims, device='cuda'); b = torch.empty_like(a)
st = torch.cuda.current_stream().cuda_stream
n = hhc.updates(dims, T)
for spec in sys.argv[4:]:
    t, thr = spec.split(':')
    tile = tuple(int(x) for x in t.split(','))
    tile = tile + (0,) * (4 - len(tile))
    hhc.stencil_run(s, a.data_ptr(), b.data_ptr(), T, tile, int(thr), st); torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(3): hhc.stencil_run(s, a.data_ptr(), b.data_ptr(), T, tile, int(thr), st)
    e1.record(); torch.cuda.synchronize(); ms = e0.elapsed_time(e1) / 3
    v = hhc.stencil_microbench(3, kind, dims, T, tile, int(thr))
    hw = hhc.make_hw(n_sm=148, n_v=128, mtb_sm=32, r_sm=65536, m_sm_bytes=233472, m_block_bytes=232448, C_iter_s=1.0, L_s_per_word=0.0, tau_sync_s=0.0, T_sync_s=0.0, geometry=1, threads=int(thr))
    iters = hhc.model_predict(kind, dims, T, tile, hw)
    print(spec, f"normal {ms:.2f} ms  compute-only {v*iters*1e3:.2f} ms  ({n/ms/1e6:.0f} vs {n/(v*iters*1e3)/1e6:.0f} G/s)", flush=True)
