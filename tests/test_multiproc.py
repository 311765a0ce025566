"""N>1 path on CPU: bench.py under torchrun with 2 ranks on gloo (replicas, no data-path
collective; only the barrier and the max/sum timing reductions cross ranks)."""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def run(nproc, steps=60):
    env = dict(os.environ, OMP_NUM_THREADS="1")
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={nproc}",
           "--master-addr", "127.0.0.1", "--master-port", str(29500 + nproc), os.path.join(ROOT, "bench.py"),
           "--simulate", "--gpus", str(nproc), "--steps", str(steps), "--warmup", "3"]
    out = subprocess.run(cmd, capture_output=True, text=True, timeout=240, env=env, cwd=ROOT)
    assert out.returncode == 0, out.stderr[-2000:]
    lines = [l for l in out.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1, out.stdout      # rank 0 alone prints
    return json.loads(lines[0])


def test_two_rank_replicas_weak_scaling():
    one = run(1)
    two = run(2)
    assert one["n_gpus"] == 1 and two["n_gpus"] == 2
    assert two["scaling"] == "weak"
    # two independent replicas with different seeds: aggregate throughput ~2x one replica
    assert 1.6 < two["value"] / one["value"] < 2.4
    assert two["lc_p99_ms"] <= 50.0 and one["lc_p99_ms"] <= 50.0
    assert "gloo" in two["config"]["parallelism"]


def test_replica_launcher_without_torchrun():
    """bench.py --gpus 2 (no torchrun) spawns two replica processes itself (CUDA_VISIBLE_DEVICES
    per replica on a GPU box), coordinating through files -- no process group, no NCCL."""
    env = dict(os.environ, OMP_NUM_THREADS="1")
    env.pop("WORLD_SIZE", None)
    res = []
    for n in (1, 2):
        out = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--simulate", "--gpus", str(n),
                              "--steps", "20", "--warmup", "3"], capture_output=True, text=True, timeout=240,
                             env=env, cwd=ROOT)
        assert out.returncode == 0, out.stderr[-2000:]
        lines = [l for l in out.stdout.splitlines() if l.startswith("{")]
        assert len(lines) == 1, out.stdout
        res.append(json.loads(lines[0]))
    one, two = res
    assert two["n_gpus"] == 2 and "files" in two["config"]["parallelism"]
    assert 1.6 < two["value"] / one["value"] < 2.4
