"""bench.py --gpus N without a torchrun environment re-launches itself as N ranks (one per GPU)
under torch.distributed.run.  Driven here on CPU: gloo, two ranks, the slab SpMV replaced by a torch
CSR product (--cpu-stub, a launcher hook that never produces a bench number)."""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_gpus_2_launches_two_ranks():
    env = {k: v for k, v in os.environ.items() if k not in ("RANK", "WORLD_SIZE", "LOCAL_RANK", "MASTER_ADDR",
                                                             "MASTER_PORT")}
    out = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--gpus", "2", "--cpu-stub",
                          "--scale", "2e-5", "--steps", "2", "--warmup", "0"],
                         capture_output=True, text=True, env=env, timeout=600, cwd=ROOT)
    assert out.returncode == 0, out.stderr[-2000:]
    lines = [ln for ln in out.stdout.splitlines() if ln.startswith("{")]
    assert len(lines) == 1, out.stdout            # rank 0 alone prints
    line = json.loads(lines[0])
    assert line["n_gpus"] == 2 and line["cpu_stub"] is True
    assert line["config"]["workload"] == "c5@2e-05"   # N > 1 defaults to configs[4] (C5)


def test_default_workload_per_gpu_count():
    sys.path.insert(0, ROOT)
    import bench
    assert bench.parse([]).config == "c3"                     # N = 1: configs[2], the headline
    assert bench.parse(["--gpus", "8"]).config == "c5"        # N > 1: configs[4]
    assert bench.parse(["--gpus", "4", "--config", "c2"]).config == "c2"
