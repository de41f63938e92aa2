"""bench.py --impl reference (the oracle on the host's cores) runs without a GPU and prints
the contract's JSON line; the all-cores cpu_baseline helper reports the threads it used."""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_reference_arm_line():
    r = subprocess.run([sys.executable, "bench.py", "--impl", "reference", "--config", "tiny",
                        "--steps", "6", "--warmup", "2"], cwd=ROOT, capture_output=True,
                       text=True, timeout=300)
    assert r.returncode == 0, r.stderr[-2000:]
    lines = [ln for ln in r.stdout.splitlines() if ln.startswith("{")]
    assert len(lines) == 1
    d = json.loads(lines[0])
    assert d["impl"] == "reference" and d["value"] > 0 and d["unit"] == "seeds/s"
    assert d["steps"] == 6 and d["warmup"] == 2 and d["higher_is_better"] is True
    assert d["cpu_baseline"]["kind"] == "oracle" and d["cpu_baseline"]["cores"] >= 1
    assert d["e2e"]["h2d_bytes_per_step"] == 0 and d["e2e"]["value"] == d["value"]


def test_cpu_baseline_all_cores():
    sys.path.insert(0, ROOT)
    import bench
    import synth
    sh = synth.SHAPES["tiny"]
    g = synth.make_graph(sh)
    c = bench.cpu_baseline(g, sh, 0.5)
    assert c["kind"] == "oracle" and c["value"] > 0 and c["cores"] >= 1
    if c["cores"] > 1:
        assert c["single_thread"]["cores"] == 1


def test_bench_defaults_and_self_launch(monkeypatch):
    """The default workload is the headline (PA-shaped configs[3] at the paper's R% 0.22);
    `--gpus N` without a launcher re-executes bench.py under torch.distributed.run."""
    sys.path.insert(0, ROOT)
    import bench
    a = bench.parse([])
    assert a.config == "PA" and a.alpha == 0.22 and a.gpus == 1 and a.runs == 3
    assert bench.parse(["--config", "PR"]).alpha == 1.0
    assert bench.parse(["--config", "UK"]).alpha == 0.18
    calls = []

    def fake_call(cmd):
        calls.append(cmd)
        return 0

    monkeypatch.delenv("WORLD_SIZE", raising=False)
    monkeypatch.setattr(bench.subprocess, "call", fake_call)
    try:
        bench.main(["--gpus", "4", "--steps", "7"])
    except SystemExit as e:
        assert e.code == 0
    assert len(calls) == 1
    cmd = calls[0]
    assert "torch.distributed.run" in cmd and "--nproc-per-node=4" in cmd
    assert cmd[cmd.index("--master-addr") + 1] == "127.0.0.1"
    assert cmd[-4:] == ["--gpus", "4", "--steps", "7"]
