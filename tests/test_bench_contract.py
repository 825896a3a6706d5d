"""bench.py's reference arm (the CPU oracle, no GPU needed) prints the contract's JSON line:
one line, the native arm's metric / unit / config keys, exactly K timed steps after W warm-ups,
`impl`, `cpu_baseline` and a zero-byte `e2e`."""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_reference_arm_json_line():
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--impl", "reference", "--config", "c1",
                        "--steps", "2", "--warmup", "1", "--cpu-sample", "1"],
                       capture_output=True, text=True, timeout=600, cwd=ROOT)
    assert r.returncode == 0, r.stderr[-2000:]
    lines = [ln for ln in r.stdout.splitlines() if ln.strip()]
    assert len(lines) == 1
    d = json.loads(lines[0])
    assert d["impl"] == "reference"
    assert d["metric"] == "queries/s (CG-2Phase, all six kinds)" and d["unit"] == "queries/s"
    assert d["steps"] == 2 and d["warmup"] == 1 and d["higher_is_better"] is True
    assert d["value"] > 0 and d["ms_per_step"] > 0
    for k in ("workload", "n", "m_generated", "m_canonical", "kinds", "batch_per_kind_per_gpu", "K_hubs"):
        assert k in d["config"], k
    assert d["config"]["workload"] == "c1-rmat16" and d["config"]["m_canonical"] < d["config"]["m_generated"]
    cb = d["cpu_baseline"]
    assert cb["kind"] == "oracle" and cb["value"] == d["value"] and cb["cores"] >= 1 and cb["sample"]
    assert d["e2e"] == {"value": d["value"], "unit": "queries/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}


def test_reference_arm_other_ranks_exit_quietly():
    env = dict(os.environ, RANK="1", WORLD_SIZE="2")
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--impl", "reference", "--config", "c1",
                        "--steps", "1", "--warmup", "0"], capture_output=True, text=True, timeout=300, cwd=ROOT,
                       env=env)
    assert r.returncode == 0 and r.stdout.strip() == ""


def test_launch_plan_relaunch_and_mismatch():
    """`--gpus N` without a torchrun environment re-launches under torch.distributed.run with N
    ranks on 127.0.0.1; a torchrun environment whose WORLD_SIZE differs from --gpus is refused."""
    sys.path.insert(0, ROOT)
    import bench
    assert bench.launch_plan(1, {}) == "run"
    assert bench.launch_plan(8, {}) == "relaunch"
    assert bench.launch_plan(4, {"WORLD_SIZE": "4"}) == "run"
    msg = bench.launch_plan(4, {"WORLD_SIZE": "2"})
    assert msg not in ("run", "relaunch") and "WORLD_SIZE=2" in msg
    cmd = bench.torchrun_cmd(["--gpus", "8", "--steps", "3"], 8, 29511)
    assert cmd[1:4] == ["-m", "torch.distributed.run", "--nnodes=1"]
    assert "--nproc-per-node=8" in cmd and "--master-addr=127.0.0.1" in cmd and "--master-port=29511" in cmd
    assert cmd[-4:] == ["--gpus", "8", "--steps", "3"] and cmd[-5].endswith("bench.py")


def test_world_size_mismatch_exits_before_any_gpu_work():
    env = dict(os.environ, RANK="0", WORLD_SIZE="2", LOCAL_RANK="0")
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--gpus", "4", "--steps", "1"],
                       capture_output=True, text=True, timeout=300, cwd=ROOT, env=env)
    assert r.returncode == 2 and "WORLD_SIZE=2" in r.stderr and r.stdout.strip() == ""
