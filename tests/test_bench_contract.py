"""bench.py contract checks (the driver parses its one JSON line).

CPU: `--impl reference` (the tier's reference arm = the oracle on host cores)
prints one line with the contract keys.  GPU: the single-GPU line carries
roofline / cpu_baseline / e2e / clocks / gpu_launches, and the torchrun
(slab-decomposed) path runs end to end at world size 1 (the only GPU count
this environment has; N > 1 runs are the driver's)."""
import json
import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
KEYS = ["metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better", "scaling",
        "vs_baseline", "dtype", "data", "config"]


def _run(args, env=None, timeout=600):
    e = dict(os.environ)
    e.update(env or {})
    r = subprocess.run([sys.executable, *args], cwd=ROOT, capture_output=True, text=True, timeout=timeout, env=e)
    assert r.returncode == 0, r.stderr[-3000:]
    lines = [l for l in r.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1, r.stdout[-2000:]
    return json.loads(lines[0])


def test_reference_arm_line():
    d = _run(["bench.py", "--impl", "reference", "--config", "C1", "--steps", "1", "--warmup", "3"])
    for k in KEYS:
        assert k in d, k
    assert d["impl"] == "reference" and d["value"] > 0
    assert d["cpu_baseline"]["kind"] == "oracle" and d["cpu_baseline"]["cores"] >= 1
    assert d["e2e"]["h2d_bytes_per_step"] == 0 and d["e2e"]["d2h_bytes_per_step"] == 0


@pytest.mark.gpu
def test_single_gpu_line():
    d = _run(["bench.py", "--config", "C1", "--steps", "3", "--warmup", "3"])
    for k in KEYS + ["roofline", "cpu_baseline", "e2e", "clocks", "gpu_launches"]:
        assert k in d, k
    assert d["value"] > 0 and d["gpu_launches"] > 0
    r = d["roofline"]
    assert r["bound"] == "alu" and 0 < r["frac"] < 1 and abs(r["frac"] - r["achieved"] / r["peak"]) < 1e-3
    assert d["e2e"]["h2d_bytes_per_step"] == 256 * 256 * 4


@pytest.mark.gpu
def test_torchrun_slab_path_world1():
    d = _run(["-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "1", "--master-addr", "127.0.0.1",
              "--master-port", "29533", "bench.py", "--gpus", "2", "--config", "C1", "--steps", "2", "--warmup", "3"])
    for k in KEYS + ["roofline", "e2e", "clocks", "gpu_launches"]:
        assert k in d, k
    assert d["n_gpus"] == 1 and d["value"] > 0 and d["gpu_launches"] > 0


@pytest.mark.gpu
def test_torchrun_hexdist_path_world1():
    d = _run(["-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "1", "--master-addr", "127.0.0.1",
              "--master-port", "29534", "bench.py", "--gpus", "2", "--config", "C1", "--exchange", "hexdist",
              "--steps", "2", "--warmup", "3"])
    assert d["n_gpus"] == 1 and d["value"] > 0 and "f1" in d["config"]["parallelism"]


def test_bench_launch_configs_are_valid_tiles():
    """Every launch configuration bench.py can time -- the config tile/threads and
    the per-GPU-count tiles under torchrun -- passes the library's tile validation
    (host-only planner rules: smem, threads per kind, integrality)."""
    sys.path.insert(0, ROOT)
    import bench
    import paper_conf_ppopp_prajapatirradg17_b200 as hhc
    from paper_conf_ppopp_prajapatirradg17_b200 import dist
    for name, c in bench.CONFIGS.items():
        nd = len(c["dims"])
        tiles = {1: (tuple(c["tile"]), c["threads"])}
        for n in (2, 4, 8):
            t, thr, _ = dist.choose_tile(c, n) if nd > 1 else (tuple(c["tile"]), c["threads"], 0)
            tiles[n] = (t, thr)
        for n, (t, thr) in tiles.items():
            t = tuple(t) + (0,) * (4 - len(t))
            if c.get("schedule") == "wavefront":
                continue
            smem, block, _ = hhc.stencil_tile_resources(nd, t, thr, kind=c["kind"])
            assert block == thr and smem <= 227 * 1024, (name, n, t, thr)
