"""N>1 paths on the real GPU: two ranks sharing cuda:0 over gloo (NCCL needs one
GPU per rank; gpurun gives one).  DP: sharded PreSC + count all-reduce equals
the oracle's full counts bit for bit.  bench.py runs end to end under torchrun
in DP and factored modes."""
import json
import os
import socket
import subprocess
import sys

import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _dp_worker(rank, world, port, out):
    import torch.distributed as dist

    import paper_conf_eurosys_yangtswycyz22_b200 as glb
    import synth
    from paper_conf_eurosys_yangtswycyz22_b200 import parallel as par
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    g = synth.make_graph("tiny")
    sh = g.shape
    ctx = glb.Context(0)
    ctx.load_graph(g.indptr, g.indices, g.features)
    ctx.set_sampler("khop", fanouts=sh.fanouts, max_batch=sh.batch)
    ctx.set_train_set(g.train, sh.batch, g.seed)
    ctx.presample(2, rank, world)
    c = ctx.counts_tensor(glb.COUNT_PRESAMPLE).cpu()
    par.allreduce_counts(c)
    if rank == 0:
        np.save(out, c.numpy())
    dist.destroy_process_group()


def test_dp_presample_two_ranks_equals_oracle(tmp_path):
    import torch.multiprocessing as mp

    import oracle
    import synth
    out = str(tmp_path / "c.npy")
    mp.spawn(_dp_worker, args=(2, free_port(), out), nprocs=2, join=True)
    g = synth.make_graph("tiny")
    sh = g.shape
    full = oracle.GraphOracle(g.indptr, g.indices).presample("khop", g.train, sh.batch,
                                                            sh.fanouts, g.seed, 2)
    assert np.array_equal(np.load(out).view(np.uint32), full)


@pytest.mark.parametrize("mode,cache,handoff", [("dp", "replicated", "peer"),
                                                ("factored", "replicated", "peer"),
                                                ("factored", "replicated", "sendrecv"),
                                                ("dp", "sharded", "peer")])
def test_bench_two_ranks(mode, cache, handoff):
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node=2",
           "--master-addr", "127.0.0.1", "--master-port", str(free_port()), "bench.py",
           "--gpus", "2", "--steps", "16", "--warmup", "3", "--config", "tiny",
           "--backend", "gloo", "--mode", mode, "--no-sweep", "--no-cpu-baseline",
           "--cache", cache, "--alpha", "0.3" if cache == "sharded" else "1.0",
           "--handoff", handoff]
    r = subprocess.run(cmd, cwd=ROOT, capture_output=True, text=True, timeout=600)
    assert r.returncode == 0, r.stderr[-3000:]
    lines = [ln for ln in r.stdout.splitlines() if ln.startswith("{")]
    assert len(lines) == 1, r.stdout[-2000:]
    d = json.loads(lines[0])
    assert d["n_gpus"] == 2 and d["value"] > 0
    if mode == "factored":
        assert d["config"]["samplers"] + d["config"]["trainers"] == 2
        assert d["config"]["handoff"].startswith(handoff)
    if cache == "sharded":  # two shards of floor(0.3 V) rows: 60% of the vertices cached
        assert d["cache"]["layout"] == "sharded"
        assert d["cache"]["rows_cached"] == 2 * int(0.3 * 10000)
        assert d["cache"]["peer_hit_share"] > 0


def test_bench_self_launch_two_ranks():
    """`bench.py --gpus 2` without a launcher re-executes itself under torch.distributed.run
    (the driver's command line measures N ranks); local rank 0 generates the host inputs
    once and the other rank maps them (synth/shm.py)."""
    cmd = [sys.executable, "bench.py", "--gpus", "2", "--steps", "8", "--warmup", "3",
           "--runs", "2", "--config", "tiny", "--backend", "gloo", "--no-sweep",
           "--no-cpu-baseline", "--no-pr-alpha1"]
    env = {k: v for k, v in os.environ.items()
           if k not in ("WORLD_SIZE", "RANK", "LOCAL_RANK", "LOCAL_WORLD_SIZE")}
    r = subprocess.run(cmd, cwd=ROOT, capture_output=True, text=True, timeout=600, env=env)
    assert r.returncode == 0, r.stderr[-3000:]
    lines = [ln for ln in r.stdout.splitlines() if ln.startswith("{")]
    assert len(lines) == 1, r.stdout[-2000:]
    d = json.loads(lines[0])
    assert d["n_gpus"] == 2 and d["value"] > 0 and len(d["runs"]) == 2
    assert d["host_inputs"].startswith("node-shared")
    assert d["config"]["parallelism"] == "dp2"


def test_bench_ns_sweep_three_ranks():
    """Config 5's Ns sweep (Fig 15 analog): the adaptive factored split, then every
    Ns in 1..N-1 as its own N-rank run (3 ranks sharing cuda:0 over gloo + CUDA IPC)."""
    cmd = [sys.executable, "bench.py", "--gpus", "3", "--steps", "6", "--warmup", "3",
           "--config", "tiny", "--backend", "gloo", "--mode", "factored", "--ns-sweep",
           "--no-sweep", "--no-cpu-baseline", "--no-pr-alpha1", "--alpha", "1.0"]
    env = {k: v for k, v in os.environ.items()
           if k not in ("WORLD_SIZE", "RANK", "LOCAL_RANK", "LOCAL_WORLD_SIZE")}
    r = subprocess.run(cmd, cwd=ROOT, capture_output=True, text=True, timeout=900, env=env)
    assert r.returncode == 0, r.stderr[-3000:]
    lines = [ln for ln in r.stdout.splitlines() if ln.startswith("{")]
    assert len(lines) == 1, r.stdout[-2000:]
    d = json.loads(lines[0])
    assert d["n_gpus"] == 3 and d["config"]["mode"] == "factored"
    sw = d["ns_sweep"]
    assert [x["samplers"] for x in sw] == [1, 2] and all(x["value"] and x["value"] > 0 for x in sw)


def _shm_parity_worker(rank, world, port, out):
    import torch.distributed as dist

    import oracle
    import paper_conf_eurosys_yangtswycyz22_b200 as glb
    from synth import shm
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    store = dist.distributed_c10d._get_default_store()
    g = shm.make_graph_shared("tiny", rank, world, store).graph
    sh = g.shape
    ctx = glb.Context(0)
    ctx.load_graph(g.indptr, g.indices, g.features)  # every rank registers the SAME pages
    ctx.set_sampler("khop", fanouts=sh.fanouts, max_batch=sh.batch)
    ctx.set_train_set(g.train, sh.batch, g.seed)
    ctx.presample(1, rank, world)
    c = ctx.counts_tensor(glb.COUNT_PRESAMPLE).cpu()
    import paper_conf_eurosys_yangtswycyz22_b200.parallel as par
    par.allreduce_counts(c)
    ctx.counts_tensor(glb.COUNT_PRESAMPLE).copy_(c.cuda())
    ctx.build_cache(0.2)
    go = oracle.GraphOracle(g.indptr, g.indices, g.features)
    ob = oracle.epoch_batches(g.train, sh.batch, g.seed, 1)
    ok = True
    for b in range(rank, len(ob), world):  # DP: this rank's batches
        ctx.sample_batch(1, b)
        s = ctx.sample_result()
        o = torch.empty((s.sizes[-1], sh.D), dtype=torch.float32, device="cuda")
        ctx.extract_sample(o, stats=True)
        exp = go.sample_khop(ob[b], sh.fanouts, g.seed, 1, b)
        ok &= np.array_equal(s.uniq.cpu().numpy().view(np.uint32), exp.uniq)
        ok &= np.array_equal(o.cpu().numpy().view(np.uint32), go.extract(exp.uniq).view(np.uint32))
    with open(os.path.join(out, f"r{rank}"), "w") as f:
        f.write(str(int(ok)))
    ctx.close()
    dist.barrier()
    dist.destroy_process_group()


def test_node_shared_inputs_registered_by_every_rank(tmp_path):
    """Node-shared host inputs (synth/shm.py) under DP: both ranks register the same pinned
    pages for their GPU (here both cuda:0) and every batch's samples and extracted bytes
    equal the oracle's; the PreSC counts are summed over the ranks' shares."""
    import torch.multiprocessing as mp
    mp.spawn(_shm_parity_worker, args=(2, free_port(), str(tmp_path)), nprocs=2, join=True)
    assert open(tmp_path / "r0").read() == "1" and open(tmp_path / "r1").read() == "1"
