#!/usr/bin/env python
"""Benchmark: GNNLab sample+extract hot path on B200 (BASELINE.json metric).

One step = one mini-batch through the whole per-batch path: epoch shuffle
(a1, at epoch boundaries), sampling (a2 / a2'), dedup/relabel into blocks
(a3), mark (a4) and feature extract (a7) from the PreSC cache (a5/a6 run
once before the timed region, timed separately like Table 6, PAPER.md
L468-474).

Default workload (the headline): BASELINE.json configs[3], the largest
single-GPU configuration -- Papers100M-shaped synthetic graph (111 M vertices,
1.6 B edges, feat 128), PinSAGE random walks (3 layers x 4 walks of length 3,
top-5), batch 8000, PreSC#1, cache ratio alpha = 0.22 (the paper's R% for
PSG-PA, Table 5): 78 % of the vertices stay in pinned host memory, so the
extract is bound by the host link.  The line also carries
`pr_alpha1` (configs[1], Products-shaped, alpha = 1: every row an HBM hit).

  python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]

--gpus N without a launcher re-executes itself under torch.distributed.run
(one rank per GPU).  Under torchrun each rank owns one GPU; batches shard
round-robin (batch g = i*N + rank); the only collective is the all-reduce of
PreSC counts (and the max-over-ranks timing).  Host inputs are generated once
per node and mapped by every local rank (synth/shm.py).  Rank 0 prints ONE
JSON line.
"""
from __future__ import annotations

import argparse
import json
import math
import os
import socket
import statistics
import subprocess
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import synth  # noqa: E402

METRIC = "sample+extract seeds/sec at 1/2/4/8 B200; cache hit rate vs optimal (%)"
# cache ratio R% the paper ran each workload at (Table 5): GSG-PR 100 %,
# GCN-TW 25 %, PSG-PA 22 %, GSG-UK 18 %; the weighted variants follow their base graph
PAPER_ALPHA = {"tiny": 0.25, "PR": 1.0, "PRW": 1.0, "TW": 0.25, "TWW": 0.25, "PA": 0.22,
               "UK": 0.18}
PCIE_GEN5_X16_GBS = 64.0  # nominal per direction (context only)


def parse(argv=None):
    p = argparse.ArgumentParser()
    p.add_argument("--gpus", type=int, default=1)
    p.add_argument("--steps", type=int, default=20)
    p.add_argument("--warmup", type=int, default=5)
    p.add_argument("--impl", default="ours", choices=["ours", "reference"])
    p.add_argument("--config", default="PA", choices=list(synth.SHAPES))
    p.add_argument("--alpha", type=float, default=None,
                   help="cache ratio (default: the paper's R%% for the workload, PAPER_ALPHA)")
    p.add_argument("--runs", type=int, default=3,
                   help="timed regions of K steps each; value = their median (SURVEY §8(d))")
    p.add_argument("--sweep-steps", type=int, default=10)
    p.add_argument("--no-sweep", action="store_true")
    p.add_argument("--no-cpu-baseline", action="store_true")
    p.add_argument("--no-pr-alpha1", action="store_true",
                   help="skip the extra PR alpha=1 (all-HBM-hit) measurement")
    p.add_argument("--cpu-seconds", type=float, default=15.0)
    p.add_argument("--measure-epochs", type=int, default=10,
                   help="epochs whose accesses define H and the Optimal H* (L148 fn4)")
    p.add_argument("--k-sweep", default="1,2,3",
                   help="PreSC#K values for the Fig 11(a) analog (empty: skip)")
    p.add_argument("--mode", default="dp", choices=["dp", "factored"],
                   help="factored: Ns sampler + Nt trainer ranks (PAPER.md §5.2-5.3)")
    p.add_argument("--ns", type=int, default=0,
                   help="factored: force Ns sampler ranks (0: adaptive, Ns = ceil(N/(K+1)))")
    p.add_argument("--ns-sweep", action="store_true",
                   help="factored: also run every Ns in 1..N-1 (Fig 15 analog, L458-476)")
    p.add_argument("--handoff", default="peer", choices=["peer", "sendrecv"],
                   help="factored mode: peer = samples pushed into the trainer's HBM ring by one "
                        "copy kernel (glb_handoff_*, NVLink/IPC); sendrecv = torch.distributed "
                        "send/recv of a packed payload")
    p.add_argument("--handoff-slots", type=int, default=4)
    p.add_argument("--no-switching", action="store_true",
                   help="factored/peer: disable dynamic executor switching (PAPER.md L267-L277)")
    p.add_argument("--backend", default="nccl", choices=["nccl", "gloo"],
                   help="gloo: CPU-staged send/recv (lets N ranks share one GPU for testing)")
    p.add_argument("--relabel", default="auto", choices=["auto", "dense", "hash"],
                   help="relabel table (glb_set_relabel_mode)")
    p.add_argument("--host-alloc", default="register", choices=["register", "cuda", "thp"],
                   help="host feature memory: pageable + cudaHostRegister, or cudaHostAlloc")
    p.add_argument("--shared-inputs", default="auto", choices=["auto", "on", "off"],
                   help="one copy of the host inputs per node, mapped by every local rank")
    p.add_argument("--numa-replicas", default="auto", choices=["auto", "on", "off"],
                   help="with shared inputs: one feature-matrix replica per NUMA node, each "
                        "rank mapping the one on its GPU's node (auto = on with > 1 node)")
    p.add_argument("--cache", default="replicated", choices=["replicated", "sharded"],
                   help="sharded: each rank caches alpha*V distinct rows, peers read them over "
                        "NVLink (NEXT-3; glb_build_cache_sharded)")
    p.add_argument("--time-every", type=int, default=0,
                   help="CUDA events around every n-th extract launch of the timed region "
                        "(0: every launch when alpha < 1 -- ms-long, host-bound extracts -- else "
                        "every 8th: events between the launches of a 0.2-ms pipelined step cost "
                        "overlap; the first extract of a region, which starts with an empty "
                        "pipeline, is always among the timed ones)")
    p.add_argument("--host-gather", default="auto",
                   help="share of each batch's misses gathered by host threads "
                        "(glb_set_host_gather): a fraction, or 'auto' = 0.15 with the cold store "
                        "(0.25 without) when a feature row is <= 512 B and alpha < 1 (measured: "
                        "512-B zero-copy rows are bound by address translation, 1-KB rows are "
                        "not; DESIGN.md §7)")
    p.add_argument("--host-gather-threads", type=int, default=0,
                   help="host threads per rank (0: min(4, usable cores / local ranks - 1))")
    p.add_argument("--cold-store", default="auto", choices=["auto", "on", "off"],
                   help="misses read a rank-ordered pinned copy of the non-cached rows "
                        "(glb_set_cold_store); auto = on for <= 512-B rows at alpha < 1 with one "
                        "rank per node (the copy is per process)")
    p.add_argument("--clock-ms", type=float, default=2.0,
                   help="NVML clock / throttle-reason sampling period during the timed regions")
    p.add_argument("--pipeline", type=int, default=2, choices=[1, 2],
                   help="2: extract of batch b overlaps sampling of batch b+1 (two streams)")
    a = p.parse_args(argv)
    if a.alpha is None:
        a.alpha = PAPER_ALPHA.get(a.config, 1.0)
    return a


def dist_env():
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    local_world = int(os.environ.get("LOCAL_WORLD_SIZE", str(world)))
    return world, rank, local, local_world


def free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def launch_ranks(n, argv, capture=False):
    """Run this script under torch.distributed.run with n ranks on this node."""
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={n}",
           "--master-addr", "127.0.0.1", "--master-port", str(free_port()),
           os.path.abspath(__file__)] + list(argv)
    if capture:
        r = subprocess.run(cmd, capture_output=True, text=True)
        sys.stderr.write(r.stderr[-4000:])
        lines = [ln for ln in r.stdout.splitlines() if ln.startswith("{")]
        return r.returncode, (json.loads(lines[-1]) if lines else None)
    return subprocess.call(cmd), None


def workload_name(sh, alpha):
    samp = {"khop": f"k-hop {list(sh.fanouts)}",
            "weighted": f"weighted k-hop {list(sh.fanouts)} (edge weight = target year)",
            "rwalk": f"random walk {len(sh.fanouts)}x(4 walks, len 3, top-{sh.fanouts[0]})"}[sh.sampler]
    return (f"{sh.name}-shaped synthetic power-law graph (V={sh.V}, E={sh.E}, feat {sh.D}), "
            f"{samp}, batch {sh.batch}, PreSC#{sh.K}, alpha={alpha}")


def read_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


def host_info():
    """CPU model (lscpu), usable cores, NUMA nodes of this host (SURVEY §8(d) protocol)."""
    model = None
    try:
        out = subprocess.run(["lscpu"], capture_output=True, text=True, timeout=10).stdout
        for ln in out.splitlines():
            if ln.startswith("Model name:"):
                model = ln.split(":", 1)[1].strip()
    except Exception:
        pass
    if model is None:
        try:
            for ln in open("/proc/cpuinfo"):
                if ln.startswith("model name"):
                    model = ln.split(":", 1)[1].strip()
                    break
        except OSError:
            pass
    try:
        ncpu = len(os.sched_getaffinity(0))
    except AttributeError:
        ncpu = os.cpu_count() or 1
    import glob
    nodes = len(glob.glob("/sys/devices/system/node/node[0-9]*")) or 1
    return {"cpu_model": model, "nproc": ncpu, "numa_nodes": nodes}


def gpu_numa_node(index):
    """NUMA node of local CUDA device `index`: the sysfs numa_node of its PCI function (the
    address from the CUDA device properties, so CUDA's and NVML's device orders cannot be
    confused); 0 if unknown (a single-node host or a VM that hides it)."""
    try:
        import torch
        p = torch.cuda.get_device_properties(index)
        addr = f"{p.pci_domain_id:04x}:{p.pci_bus_id:02x}:{p.pci_device_id:02x}.0"
        return max(int(open(f"/sys/bus/pci/devices/{addr}/numa_node").read()), 0)
    except Exception:
        return 0


def gpu_info(index):
    """Driver, ECC, clocks, PCIe link and NUMA affinity of the GPU (nvidia-smi -q fields)."""
    try:
        import pynvml as nv
        nv.nvmlInit()
        vis = os.environ.get("CUDA_VISIBLE_DEVICES")
        phys = int(vis.split(",")[index]) if vis and vis.split(",")[0].isdigit() else index
        h = nv.nvmlDeviceGetHandleByIndex(phys)
        d = {"name": nv.nvmlDeviceGetName(h), "driver": nv.nvmlSystemGetDriverVersion()}
        try:
            v = nv.nvmlSystemGetCudaDriverVersion()
            d["driver_cuda"] = f"{v // 1000}.{v % 1000 // 10}"
        except Exception:
            pass
        try:
            import torch
            d["torch_cuda_runtime"] = torch.version.cuda
        except Exception:
            pass
        for k, f in (("ecc_mode", lambda: nv.nvmlDeviceGetCurrentEccMode(h)),
                     ("sm_max_mhz", lambda: nv.nvmlDeviceGetMaxClockInfo(h, nv.NVML_CLOCK_SM)),
                     ("mem_max_mhz", lambda: nv.nvmlDeviceGetMaxClockInfo(h, nv.NVML_CLOCK_MEM)),
                     ("pcie_gen", lambda: nv.nvmlDeviceGetCurrPcieLinkGeneration(h)),
                     ("pcie_width", lambda: nv.nvmlDeviceGetCurrPcieLinkWidth(h)),
                     ("numa_node", lambda: nv.nvmlDeviceGetNumaNodeId(h))):
            try:
                d[k] = f()
            except Exception:
                d[k] = None
        return d
    except Exception as e:  # noqa: BLE001
        return {"error": str(e)[:120]}


def hostlink_peak(dev):
    """Measured host->device link peak for the roofline, in this run: DMA of 1 GiB pinned
    host memory to HBM (copy engine), best of 5, CUDA events on the copying stream."""
    import torch
    n = 1 << 30
    h = torch.empty(n, dtype=torch.uint8, pin_memory=True)
    h[::4096] = 1
    d = torch.empty(n, dtype=torch.uint8, device=dev)
    s = torch.cuda.current_stream(dev)
    d.copy_(h, non_blocking=True)
    best = 0.0
    for _ in range(5):
        e0 = torch.cuda.Event(enable_timing=True)
        e1 = torch.cuda.Event(enable_timing=True)
        e0.record(s)
        d.copy_(h, non_blocking=True)
        e1.record(s)
        e1.synchronize()
        best = max(best, n / (e0.elapsed_time(e1) * 1e-3) / 1e9)
    del h, d
    torch.cuda.synchronize(dev)
    if hasattr(torch._C, "_host_emptyCache"):  # give the 1 GiB of pinned memory back
        torch._C._host_emptyCache()
    return best


class Clocks:
    """SM clock + throttle reasons sampled DURING the timed region (B200_PROFILING.md
    clocks line), via NVML from a background thread every ~2 ms (ctypes and CUDA
    syncs release the GIL).  Falls back to None when NVML is unavailable."""

    REASONS = {"hw_slowdown": "nvmlClocksEventReasonHwSlowdown",
               "hw_thermal_slowdown": "nvmlClocksEventReasonHwThermalSlowdown",
               "sw_thermal_slowdown": "nvmlClocksEventReasonSwThermalSlowdown",
               "sw_power_cap": "nvmlClocksEventReasonSwPowerCap",
               "hw_power_brake": "nvmlClocksEventReasonHwPowerBrakeSlowdown"}

    def __init__(self, index, interval_s=0.002):
        self.index = index
        self.interval = interval_s
        self.ok = False
        try:
            import pynvml
            pynvml.nvmlInit()
            vis = os.environ.get("CUDA_VISIBLE_DEVICES")
            phys = int(vis.split(",")[index]) if vis and vis.split(",")[0].isdigit() else index
            self.h = pynvml.nvmlDeviceGetHandleByIndex(phys)
            self.nv = pynvml
            self.max = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
            self.ok = True
        except Exception:
            pass

    def _run(self):
        nv = self.nv
        while not self.stop_flag:
            try:
                self.sm.append(nv.nvmlDeviceGetClockInfo(self.h, nv.NVML_CLOCK_SM))
                self.rs |= nv.nvmlDeviceGetCurrentClocksEventReasons(self.h)
            except Exception:
                pass
            time.sleep(self.interval)

    def _sample(self):
        try:
            self.sm.append(self.nv.nvmlDeviceGetClockInfo(self.h, self.nv.NVML_CLOCK_SM))
            self.rs |= self.nv.nvmlDeviceGetCurrentClocksEventReasons(self.h)
        except Exception:
            pass

    def start(self):
        if not self.ok:
            return
        import threading
        self.sm, self.rs, self.stop_flag = [], 0, False
        self._sample()
        self.th = None
        if self.interval > 0:  # <= 0: one sample at start and one at stop only
            self.th = threading.Thread(target=self._run, daemon=True)
            self.th.start()

    def stop(self):
        if not self.ok:
            return None
        self.stop_flag = True
        if self.th is not None:
            self.th.join()
        self._sample()
        if not self.sm:
            return None
        reasons = sorted(k for k, a in self.REASONS.items()
                         if hasattr(self.nv, a) and self.rs & getattr(self.nv, a))
        return {"sm_mhz": statistics.median(self.sm), "sm_max_mhz": self.max,
                "reasons": reasons, "samples": len(self.sm), "source": "nvml"}


# ------------------------------------------------------------------------------------------
def reference_arm(args):
    """--impl reference: the CPU oracle as it stands (test infrastructure; the one
    other place bench.py executes oracle/), on this arm's workload/metric, on the host's
    cores: the W warm-up and K timed mini-batches are spread over P threads (one
    GraphOracle scratch each; the oracle's C calls release the GIL), value = timed seeds /
    wall time of the timed batches."""
    world, rank, _, _ = dist_env()
    if rank != 0:
        return
    import concurrent.futures as cf

    import oracle
    sh = synth.SHAPES[args.config]
    g = synth.make_graph(sh)
    nb = math.ceil(sh.n_train / sh.batch)
    batches = {}

    def seeds_of(i):
        e, b = sh.K + i // nb, i % nb
        if e not in batches:
            batches[e] = oracle.epoch_batches(g.train, sh.batch, g.seed, e)
        return e, b, batches[e][b]

    jobs_w = [seeds_of(i) for i in range(args.warmup)]
    jobs_t = [seeds_of(i) for i in range(args.warmup, args.warmup + args.steps)]
    P = threads_for(sh, min(args.steps, 64))
    local = __import__("threading").local()

    def run(job):
        if not hasattr(local, "go"):
            local.go = oracle.GraphOracle(g.indptr, g.indices, g.features)
        e, b, sd = job
        s = local.go.sample(sh.sampler, sd, sh.fanouts, g.seed, e, b, g.weights)
        local.go.extract(s.uniq)
        return len(sd)

    with cf.ThreadPoolExecutor(P) as ex:
        list(ex.map(run, jobs_w))
        t0 = time.perf_counter()
        tot_s = sum(ex.map(run, jobs_t))
        tot_t = time.perf_counter() - t0
    v = tot_s / tot_t
    hi = host_info()
    line = {
        "impl": "reference", "metric": METRIC, "value": v, "unit": "seeds/s", "n_gpus": args.gpus,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * tot_t / args.steps,
        "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "u32",
        "data": "synthetic", "config": {"workload": workload_name(sh, args.alpha)},
        "cpu_baseline": {"value": v, "unit": "seeds/s", "cores": P, "kind": "oracle",
                         "cpu_model": hi["cpu_model"], "nproc": hi["nproc"],
                         "sample": f"{args.steps} full mini-batches (sample+relabel+extract) over "
                                   f"{P} threads, single-threaded C oracle per thread"},
        "e2e": {"value": v, "unit": "seeds/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


def threads_for(sh, cap):
    """Host threads for an oracle run: usable cores, capped by `cap` and by the memory one
    batch needs (lid scratch + buffers + extract output) against half the free host RAM."""
    try:
        ncpu = len(os.sched_getaffinity(0))
    except AttributeError:
        ncpu = os.cpu_count() or 1
    ub = sh.batch
    for k in sh.fanouts:
        ub = min(ub * (1 + k), sh.V)
    per_thread = 4 * sh.V + 6 * ub * 4 + ub * sh.D * 4
    try:
        import psutil
        avail = psutil.virtual_memory().available
    except Exception:
        avail = 8 << 30
    return max(1, min(ncpu, int(avail * 0.5 // max(per_thread, 1)), cap))


def cpu_baseline(g, sh, budget_s):
    """Oracle as it stands, timed on this host (rank 0, N=1), bounded sample."""
    import oracle
    go = oracle.GraphOracle(g.indptr, g.indices, g.features)
    bs = oracle.epoch_batches(g.train, sh.batch, g.seed, sh.K)
    t_tot, seeds, nb = 0.0, 0, 0
    while t_tot < budget_s and nb < len(bs):
        t0 = time.perf_counter()
        s = go.sample(sh.sampler, bs[nb], sh.fanouts, g.seed, sh.K, nb, g.weights)
        go.extract(s.uniq)
        t_tot += time.perf_counter() - t0
        seeds += len(bs[nb])
        nb += 1
    hi = host_info()
    single = {"value": seeds / t_tot, "unit": "seeds/s", "cores": 1, "kind": "oracle",
              "sample": f"{nb} mini-batches of epoch {sh.K} (sample+relabel+extract, "
                        f"{seeds} seeds, {t_tot:.1f} s), single-threaded C oracle"}
    par = cpu_baseline_parallel(go, g, sh, bs, max(2.0, budget_s * 2 / 3))
    if par is None:
        single.update({"cpu_model": hi["cpu_model"], "nproc": hi["nproc"]})
        return single
    par["single_thread"] = single
    par.update({"cpu_model": hi["cpu_model"], "nproc": hi["nproc"]})
    return par


def cpu_baseline_parallel(go, g, sh, bs, budget_s):
    """SURVEY §8(d) timing (ii): the same oracle on all usable host cores, over disjoint
    batches of epochs K, K+1, ... -- one thread per core, each with its own GraphOracle
    (lid scratch) over the shared graph; the oracle's sample and extract are C calls made
    through ctypes, which release the GIL, so the threads run in parallel.  The thread
    count is capped by the memory one batch needs (lid scratch + extract output) against
    half the available host RAM.  value = all seeds / the slowest thread's busy time."""
    import concurrent.futures as cf

    import oracle
    try:
        ncpu = len(os.sched_getaffinity(0))
    except AttributeError:
        ncpu = os.cpu_count() or 1
    P = threads_for(sh, 64)
    if P < 2:
        return None
    epochs = [bs] + [oracle.epoch_batches(g.train, sh.batch, g.seed, sh.K + i) for i in (1, 2, 3)]
    jobs = [(sh.K + i, b, s) for i, ep in enumerate(epochs) for b, s in enumerate(ep)]

    def run(p):
        o = oracle.GraphOracle(g.indptr, g.indices, g.features)
        t_tot, seeds, nb = 0.0, 0, 0
        for e, b, sd in jobs[p::P]:
            if nb and t_tot >= budget_s:
                break
            t0 = time.perf_counter()
            smp = o.sample(sh.sampler, sd, sh.fanouts, g.seed, e, b, g.weights)
            o.extract(smp.uniq)
            t_tot += time.perf_counter() - t0
            seeds += len(sd)
            nb += 1
        return seeds, t_tot, nb

    with cf.ThreadPoolExecutor(P) as ex:
        res = list(ex.map(run, range(P)))
    seeds = sum(r[0] for r in res)
    wall = max(r[1] for r in res)
    nb = sum(r[2] for r in res)
    return {"value": seeds / wall, "unit": "seeds/s", "cores": P, "kind": "oracle",
            "host_cpus": ncpu,
            "sample": f"{nb} mini-batches of epochs {sh.K}.. over {P} threads (disjoint batches, "
                      f"sample+relabel+extract, {seeds} seeds, slowest thread {wall:.1f} s), "
                      f"single-threaded C oracle per thread (ctypes releases the GIL)"}


# ------------------------------------------------------------------------------------------
def run_factored(args, ctx, g, sh, out, nb, world, rank, dev, stream, t_pre, t_cache, par, glb):
    """Factored mode (§5.2-5.3): profile Ts/Tt, split ranks into Ns samplers
    and Nt trainers (Ns = ceil(N/(K+1)), K = Tt/Ts, L262; or --ns), then samplers pull
    batches from the global scheduler and hand samples to trainers, which extract."""
    import torch
    import torch.distributed as dist
    cpu_comm = args.backend == "gloo"
    comm_dev = "cpu" if cpu_comm else dev
    # profile one sampler step and one trainer step (L260: "training an epoch in advance")
    ts_l, tt_l = [], []
    for i in range(max(args.warmup, 3)):
        e, b = par.dp_step_batch(i, rank, world, nb, sh.K)
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        ctx.sample_batch(e, b)
        s = ctx.sample_result()
        t1 = time.perf_counter()
        ctx.extract(s.uniq, out=out[:s.sizes[-1]])
        torch.cuda.synchronize()
        ts_l.append(t1 - t0)
        tt_l.append(time.perf_counter() - t1)
    prof = torch.tensor([statistics.median(ts_l), statistics.median(tt_l)], dtype=torch.float64)
    if world > 1:
        prof = prof.to(comm_dev)
        dist.all_reduce(prof)
        prof = prof.cpu() / world
    ns_adaptive = par.num_samplers(world, float(prof[0]), float(prof[1]))
    ns = min(max(args.ns, 1), world - 1) if (args.ns and world > 1) else ns_adaptive
    roles = par.Roles(ns, world)
    total = args.steps * world
    store = dist.distributed_c10d._get_default_store() if world > 1 else None
    tag = f"bench{ns}"
    seeds = {"n": 0}

    def sample_fn(gidx):
        e, b = sh.K + gidx // nb, gidx % nb
        ctx.sample_batch(e, b)
        blk = ctx.sample_result()
        return e, blk

    def extract_fn(gidx, epoch, sizes, nnz, payload):
        uniq = payload[0]
        if uniq.device.type != "cuda":
            uniq = uniq.to(dev, non_blocking=True)
        ctx.extract(uniq.contiguous(), out=out[:sizes[-1]])
        seeds["n"] += sizes[0]

    peer = args.handoff == "peer" and world > 1
    if peer:
        ho = par.PeerHandoff(ctx, roles, rank, slots=args.handoff_slots)
        ntrain = len(g.train)

        def sample_peer(gidx):  # asynchronous: no sizes read back on the sampler
            ctx.sample_batch(sh.K + gidx // nb, gidx % nb)

        def extract_peer(gidx):  # the pushed sample is the ctx's current one
            b = gidx % nb
            ctx.extract_sample(out)
            seeds["n"] += min(sh.batch, ntrain - b * sh.batch)

    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    if peer:
        if roles.is_sampler(rank):
            # dynamic switching: a sampler that would wait for a busy slot extracts the batch
            # itself (standby Trainer, same cache here: T_t' = T_t) when the profit is > 0
            par.run_sampler_peer(sample_peer, ho, total, store, tag,
                                 standby_fn=None if args.no_switching else extract_peer,
                                 t_train=float(prof[1]), t_standby=float(prof[1]))
        else:
            par.run_trainer_peer(extract_peer, ho, total, store, tag)
    elif world == 1:
        for gidx in range(total):
            e, blk = sample_fn(gidx)
            extract_fn(gidx, e, blk.sizes, blk.nnz, (blk.uniq,))
    elif roles.is_sampler(rank):
        if cpu_comm:
            orig = sample_fn

            def sample_fn(gidx):  # noqa: F811
                e, blk = orig(gidx)
                import types
                return e, types.SimpleNamespace(
                    sizes=blk.sizes, nnz=blk.nnz, uniq=blk.uniq.cpu(),
                    indptr=[x.cpu() for x in blk.indptr], indices=[x.cpu() for x in blk.indices],
                    weights=None if blk.weights is None else [x.cpu() for x in blk.weights])
        par.run_sampler(sample_fn, roles, rank, total, store, tag, comm_dev)
    else:
        par.run_trainer(extract_fn, roles, rank, total, store, tag, comm_dev)
    torch.cuda.synchronize()
    el = time.perf_counter() - t0
    red = torch.tensor([el, float(seeds["n"]), float(ho.standby if peer else 0)],
                       dtype=torch.float64)
    if world > 1:
        r2 = red.to(comm_dev)
        t_max = r2[:1].clone()
        dist.all_reduce(t_max, op=dist.ReduceOp.MAX)
        n_sum = r2[1:].clone()
        dist.all_reduce(n_sum)
        el, n_all, n_standby = float(t_max.cpu()), float(n_sum[0].cpu()), int(n_sum[1].cpu())
    else:
        n_all, n_standby = float(seeds["n"]), 0
    if rank == 0:
        line = {"metric": METRIC, "value": n_all / el, "unit": "seeds/s", "n_gpus": world,
                "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * el / args.steps,
                "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "u32",
                "data": "synthetic",
                "config": {"workload": workload_name(sh, args.alpha), "mode": "factored",
                           "samplers": ns, "trainers": world - ns, "ns_adaptive": ns_adaptive,
                           "ns_forced": bool(args.ns),
                           "Ts_ms": 1e3 * float(prof[0]), "Tt_ms": 1e3 * float(prof[1]),
                           "backend": args.backend, "parallelism": f"factored{ns}s{world - ns}t",
                           "handoff": (f"peer ({args.handoff_slots}-slot HBM ring per trainer, "
                                       "glb_handoff_*)") if peer else "sendrecv",
                           "standby_batches": n_standby,
                           "switching": peer and not args.no_switching},
                "timing": "host wall clock around the sampler/trainer loops (max over ranks)",
                "preprocess_s": {"presample": t_pre, "build_cache": t_cache}}
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()


# ------------------------------------------------------------------------------------------
def sampling_bytes(sh, sizes, nnz):
    """Algorithmic HBM bytes of sampling one batch: k-hop 32 B per frontier
    vertex (indptr pair) + 72 B per sampled edge (index sector, padded write, relabel probe,
    compaction); random walk 64 B per walk step (indptr + index sectors) + 40 B per kept
    edge (relabel probe, compaction)."""
    L = len(nnz)
    if sh.sampler == "rwalk":
        return sum(sizes[l] * synth.RW_WALKS * synth.RW_LEN * 64 + 40 * nnz[l] for l in range(L))
    return sum(32 * sizes[l] + 72 * nnz[l] for l in range(L))


def run_workload(args, sh, alpha, world, rank, local, local_world, dev, stream, full,
                 link_peak):
    """One workload through the DP path: inputs, load, PreSC, cache, `args.runs` timed
    regions of K steps, the untimed replay that counts each launch's units, the depth-1
    isolated extract replay, e2e through the public API, and (full) the hit-rate sweeps
    and the CPU oracle baseline.  Returns the fields of the JSON line."""
    import torch
    import torch.distributed as dist

    import paper_conf_eurosys_yangtswycyz22_b200 as glb
    from paper_conf_eurosys_yangtswycyz22_b200 import parallel as par

    def barrier():
        if world > 1:
            dist.barrier()

    t0 = time.perf_counter()
    shared, numa = None, None
    use_shared = world > 1 and local_world > 1 and args.shared_inputs != "off"
    if use_shared:
        from synth import shm
        store = dist.distributed_c10d._get_default_store()
        numa = None
        if args.numa_replicas == "on" or (args.numa_replicas == "auto"
                                          and host_info()["numa_nodes"] > 1):
            numa = gpu_numa_node(local)
        shared = shm.make_graph_shared(sh, local, local_world, store, numa_node=numa)
        g = shared.graph
    else:
        alloc = None
        if args.host_alloc == "cuda":
            def alloc(nbytes):  # cudaHostAlloc'ed (pinned, mapped under UVA) via torch
                return torch.empty(nbytes, dtype=torch.uint8, pin_memory=True).numpy()
        elif args.host_alloc == "thp":
            def alloc(nbytes):  # 2 MB transparent huge pages (madvise), registered by load_graph
                return synth.aligned_empty(nbytes, np.uint8, huge=True)
        g = synth.make_graph(sh, feature_alloc=alloc)
    barrier()
    t_gen = time.perf_counter() - t0

    ctx = glb.Context(local)
    ctx.set_stream(stream)
    t0 = time.perf_counter()
    ctx.load_graph(g.indptr, g.indices, g.features)
    t_load = time.perf_counter() - t0
    ctx.set_relabel_mode(args.relabel)
    if g.weights is not None:
        ctx.load_edge_weights(g.weights)
    if sh.sampler in ("khop", "weighted"):
        ctx.set_sampler(sh.sampler, fanouts=sh.fanouts, max_batch=sh.batch)
    else:
        ctx.set_sampler("rwalk", layers=len(sh.fanouts), walks=synth.RW_WALKS,
                        walk_len=synth.RW_LEN, topk=sh.fanouts[0], max_batch=sh.batch)
    ctx.set_train_set(g.train, sh.batch, g.seed)
    nb = ctx.num_batches

    # ---- preprocessing (Table 6 analog): PreSC#K and load_cache
    barrier()
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    ctx.presample(sh.K, rank, world)
    if world > 1:
        t_counts = ctx.counts_tensor(glb.COUNT_PRESAMPLE)
        if args.backend == "nccl":
            par.allreduce_counts(t_counts)  # u32 sums (< 2^31), NCCL over NVLink
        else:
            c = t_counts.cpu()
            par.allreduce_counts(c)
            t_counts.copy_(c)
    torch.cuda.synchronize()
    t_pre = time.perf_counter() - t0
    small_rows = 4 * sh.D <= 512 and alpha < 1.0
    cold = (small_rows and local_world == 1 and args.cache != "sharded"
            if args.cold_store == "auto" else args.cold_store == "on")
    ctx.set_cold_store(cold)
    t0 = time.perf_counter()
    if args.cache == "sharded":
        par.build_sharded_cache(ctx, alpha, rank, world)
    else:
        ctx.build_cache(alpha)
    torch.cuda.synchronize()
    t_cache = time.perf_counter() - t0
    hg = args.host_gather
    # the share the miss path measured best at (profiles/r02z, r02q2): smaller with the cold
    # store (fewer host regions left for the host threads to win); the store may have been
    # skipped (host memory), so ask the ctx whether it holds one
    cold_on = ctx.cold_store_rows > 0
    hg = ((0.15 if cold_on else 0.25) if small_rows else 0.0) if hg == "auto" else float(hg)
    if hg > 0:
        nt = args.host_gather_threads
        if nt <= 0:  # share the node's cores between the local ranks
            nt = min(4, max(2, host_info()["nproc"] // max(1, local_world) - 1))
        ctx.set_host_gather(hg, threads=nt)

    ctx_cache_rows = ctx.cache_size
    ub = sh.batch
    for k in sh.fanouts:
        ub = min(ub * (1 + k), sh.V)
    out = torch.empty((ub, sh.D), dtype=torch.float32, device=dev)

    def batch_of(i):
        return par.dp_step_batch(i, rank, world, nb, sh.K)

    def n_seeds(b):
        return min(sh.batch, sh.n_train - b * sh.batch)

    if args.mode == "factored":
        return run_factored(args, ctx, g, sh, out, nb, world, rank, dev, stream, t_pre, t_cache,
                            par, glb)

    ctx.set_pipeline(args.pipeline)
    xs = ctx.extract_stream() if args.pipeline == 2 else stream

    # ---- warmup
    for i in range(args.warmup):
        e, b = batch_of(i)
        ctx.sample_batch(e, b)
        ctx.extract_sample(out)
    ctx.sync()
    torch.cuda.synchronize()

    # ---- timed regions: device time, CUDA events on the launching streams (sampling on the
    # main stream, extract on the extract stream; the last kernel of a region is an extract).
    # Run r times steps [W + r*K, W + (r+1)*K): different batches, same protocol.
    K = args.steps
    te = args.time_every if args.time_every > 0 else (1 if alpha < 1.0 else 8)
    clocks = Clocks(local, args.clock_ms / 1e3)
    launches0 = ctx.launches
    ctx.set_timing(te)  # events around every te-th extract launch
    clocks.start()
    runs, run_ms, enq_ms, wall_ms = [], [], [], []
    for r in range(args.runs):
        steps = range(args.warmup + r * K, args.warmup + (r + 1) * K)
        barrier()
        torch.cuda.synchronize()
        t_start = torch.cuda.Event(enable_timing=True)
        t_end = torch.cuda.Event(enable_timing=True)
        t_start.record(stream)
        wall0 = time.perf_counter()
        seeds_done = 0
        for i in steps:
            e, b = batch_of(i)
            ctx.sample_batch(e, b)
            ctx.extract_sample(out)
            seeds_done += n_seeds(b)
        t_end.record(xs)
        enq_ms.append(1e3 * (time.perf_counter() - wall0))
        torch.cuda.synchronize()
        wall_ms.append(1e3 * (time.perf_counter() - wall0))
        barrier()
        el = torch.tensor([t_start.elapsed_time(t_end)], dtype=torch.float64, device=dev)
        tot = torch.tensor([float(seeds_done)], dtype=torch.float64, device=dev)
        if world > 1:
            if args.backend == "gloo":
                el, tot = el.cpu(), tot.cpu()
            dist.all_reduce(el, op=dist.ReduceOp.MAX)
            dist.all_reduce(tot)
        run_ms.append(float(el.item()))
        runs.append(float(tot.item()) / (float(el.item()) / 1e3))
    clk = clocks.stop()
    launches = (ctx.launches - launches0) / args.runs
    x_ms = ctx.extract_times()
    ctx.set_timing(False)
    med = sorted(range(args.runs), key=lambda j: runs[j])[args.runs // 2]
    value, elapsed_max = runs[med], run_ms[med]
    timed_steps = list(range(args.warmup, args.warmup + args.runs * K))

    # ---- replay (untimed) to count the units each timed launch processed
    nL, hits, misses, samp_b = [], [], [], []
    for i in timed_steps:
        e, b = batch_of(i)
        ctx.sample_batch(e, b)
        s = ctx.sample_result()
        st = ctx.extract_sample(out, stats=True)
        nL.append(s.sizes[-1])
        hits.append(st["hits"])
        misses.append(st["misses"])
        samp_b.append(sampling_bytes(sh, s.sizes, s.nnz))
    D = sh.D
    hbm_peak, hbm_src = read_peaks()
    # algorithmic HBM bytes of the extract launch: per row read (hit: cache row from HBM) +
    # write of the out row + the 8-byte (dst, src) work-list entry; host-link bytes: the
    # miss rows read over PCIe
    hbm_bytes = [h * (2 * 4 * D + 8) + m * (4 * D + 8) for h, m in zip(hits, misses)]
    link_bytes = [m * 4 * D for m in misses]
    sel = list(range(0, len(timed_steps), te))[: len(x_ms)]  # the timed launches
    ach_hbm = statistics.mean(hbm_bytes[j] / (t * 1e-3) for j, t in zip(sel, x_ms)) / 1e9
    ach_link = statistics.mean(link_bytes[j] / (t * 1e-3) for j, t in zip(sel, x_ms)) / 1e9
    x_mean = statistics.mean(x_ms)
    # the extract's binding roof: hits (HBM) and misses (host link) overlap in one launch
    bound_ms = statistics.mean(max(hbm_bytes[j] / hbm_peak, link_bytes[j] / link_peak) / 1e6
                               for j in sel)
    host_bound = statistics.mean(link_bytes) / link_peak > statistics.mean(hbm_bytes) / hbm_peak
    # ---- the same extract launches without the overlapping sampler (pipeline depth 1)
    iso = None
    if args.pipeline == 2:
        ctx.set_pipeline(1)
        iso_steps = timed_steps[: min(len(timed_steps), 100)]
        torch.cuda.synchronize()
        ctx.set_timing(True)
        i0 = torch.cuda.Event(enable_timing=True)
        i1 = torch.cuda.Event(enable_timing=True)
        i0.record(stream)
        sd = 0
        for i in iso_steps:
            e, b = batch_of(i)
            ctx.sample_batch(e, b)
            ctx.extract_sample(out)
            sd += n_seeds(b)
        i1.record(stream)
        torch.cuda.synchronize()
        xi = ctx.extract_times()
        ctx.set_timing(False)
        ctx.set_pipeline(2)
        ims = i0.elapsed_time(i1)
        # the sampling half alone (a1-a5 of the same batches, no extract)
        torch.cuda.synchronize()
        i0.record(stream)
        for i in iso_steps:
            e, b = batch_of(i)
            ctx.sample_batch(e, b)
        i1.record(stream)
        torch.cuda.synchronize()
        sms = i0.elapsed_time(i1) / len(iso_steps)
        a_hbm = statistics.mean(bb / (t * 1e-3) for bb, t in zip(hbm_bytes, xi)) / 1e9
        a_link = statistics.mean(bb / (t * 1e-3) for bb, t in zip(link_bytes, xi)) / 1e9
        iso = {"pipeline_depth": 1, "steps": len(iso_steps),
               "achieved": a_link if host_bound else a_hbm,
               "frac": (a_link / link_peak) if host_bound else (a_hbm / hbm_peak),
               "hbm_achieved": a_hbm, "hbm_frac": a_hbm / hbm_peak,
               "extract_ms_per_step": statistics.mean(xi),
               "ms_per_step": ims / len(iso_steps), "seeds_per_s": world * sd / (ims / 1e3),
               "sampling_ms_per_step": sms,
               "sampling_ms_per_step_is": "the same batches sampled alone (no extract), depth 1"}
    traffic = None
    tp = os.path.join(ROOT, "profiles", "traffic.json")
    if os.path.exists(tp):
        tj = json.load(open(tp))
        # the cold store changes the host-side layout the misses read: its own ncu entry
        traffic = ((ctx.cold_store_rows and tj.get(f"{sh.name}:{alpha}:cold"))
                   or tj.get(f"{sh.name}:{alpha}"))
    hbm_obj = {"achieved": ach_hbm, "peak": hbm_peak, "unit": "GB/s", "frac": ach_hbm / hbm_peak,
               "peak_source": hbm_src,
               "algorithmic_bytes_per_launch": statistics.mean(hbm_bytes[j] for j in sel)}
    link_obj = {"achieved": ach_link, "peak": link_peak, "unit": "GB/s",
                "frac": ach_link / link_peak,
                "peak_source": "DMA H2D of 1 GiB pinned host memory, best of 5, measured in "
                               f"this run (PCIe Gen5 x16 nominal {PCIE_GEN5_X16_GBS:.0f} GB/s)",
                "algorithmic_bytes_per_launch": statistics.mean(link_bytes[j] for j in sel)}
    # `traffic`: ncu bytes per launch on the binding roof (sysmem reads for the host link,
    # DRAM read + write for HBM), comparable with `algorithmic_bytes_per_launch`; the
    # other counters of the same capture in `traffic_detail`
    detail = traffic if isinstance(traffic, dict) else None
    if detail is not None:
        traffic = detail.get("sysmem_read_bytes") if host_bound else detail.get("dram_bytes")
    if host_bound:
        roof = {"kernel": "k_gather (extract a7)", "bound": "host-link", **link_obj,
                "traffic": traffic, "traffic_detail": detail, "hbm": hbm_obj}
    else:
        roof = {"kernel": "k_gather (extract a7)", "bound": "hbm", **hbm_obj, "traffic": traffic,
                "traffic_detail": detail,
                "host_link": link_obj}
    roof.update({
        "extract_ms_per_step": x_mean,
        "extract_share_of_step": x_mean / (elapsed_max / K),
        "kernel_bound_ms": bound_ms, "frac_of_binding_bound": bound_ms / x_mean,
        "timed_launches": f"every {te}th extract of the {args.runs} timed regions "
                          f"({len(x_ms)} launches)",
        "measured_with": f"pipeline depth {args.pipeline} (the timed region)",
        "isolated": iso})
    # the whole step's roof: sampling + extract HBM bytes against HBM, misses against the
    # host link, the two overlapping (SURVEY §8(d) "End-to-end bound per batch")
    step_bound = statistics.mean(max((samp_b[j] + hbm_bytes[j]) / hbm_peak,
                                     link_bytes[j] / link_peak) / 1e6
                                 for j in range(len(timed_steps)))
    path = {"bound_ms_per_step": step_bound, "measured_ms_per_step": elapsed_max / K,
            "frac": step_bound / (elapsed_max / K),
            "sampling_bytes_per_step": statistics.mean(samp_b),
            "extract_hbm_bytes_per_step": statistics.mean(hbm_bytes),
            "host_link_bytes_per_step": statistics.mean(link_bytes)}

    e2e = e2e_measure(args, ctx, g, sh, timed_steps, batch_of, n_seeds, out, xs, world, dev)
    import gc
    gc.collect()  # pinned host tensors used on the ctx's extract stream die before the ctx
    torch.cuda.synchronize()

    res = {"value": value, "ms_per_step": elapsed_max / K, "runs": runs,
           "runs_range": [min(runs), max(runs)], "runs_ms": run_ms,
           "roofline": roof, "path_roofline": path, "e2e": e2e, "gpu_launches": launches,
           "clocks": clk, "host_wall_ms_timed_region": wall_ms[med],
           "host_enqueue_ms_timed_region": enq_ms[med],
           "units": {"mean_n_L": statistics.mean(nL), "mean_hits": statistics.mean(hits),
                     "mean_misses": statistics.mean(misses)},
           "preprocess_s": {"generate_inputs": t_gen, "load_graph": t_load,
                            "presample": t_pre, "build_cache": t_cache},
           "cache": {"layout": args.cache, "rows_cached": ctx_cache_rows},
           "host_gather": ctx.host_gather,
           "cold_store_rows": ctx.cold_store_rows,
           "relabel_table": ctx.relabel_mode, "relabel_l2_window_bytes": ctx.relabel_l2_window,
           "host_inputs": (("node-shared memfd, generated once by local rank 0 and mapped by "
                            f"{local_world} ranks") + (f"; features replicated per NUMA node, this "
                                                       f"rank's GPU on node {numa}"
                                                       if numa is not None else "")
                           if shared else "private to this rank")}

    # ---- hit rate vs Optimal (accesses recorded over measured epochs, untimed)
    if args.cache == "sharded":
        k = ctx.last_extract_counts()
        res["cache"]["peer_hit_share"] = k["peer_hits"] / max(1, k["hits"] + k["misses"])
        barrier()  # peers may still read this rank's shard: nobody rebuilds before here
    if full and not args.no_sweep:
        res.update(hit_rate_sweeps(args, ctx, g, sh, alpha, world, rank, nb, out, stream, xs,
                                   batch_of, n_seeds, barrier))
    if full and rank == 0 and world == 1 and not args.no_cpu_baseline:
        res["cpu_baseline"] = cpu_baseline(g, sh, args.cpu_seconds)
    ctx.close()
    del out
    torch.cuda.empty_cache()
    return res


def e2e_measure(args, ctx, g, sh, timed_steps, batch_of, n_seeds, out, xs, world, dev):
    """e2e through the public API with host buffers: every step copies its seeds from
    pinned host memory (glb_sample_async, H2D on the ctx stream) and reads its result --
    the extract's (hits, misses, peer hits) -- back into pinned host memory (stream-ordered
    D2H); the host consumes the result of step j-D while step j runs (D = the pipeline
    depth).  Wall clock from the first call to the last result on the host."""
    import torch
    import torch.distributed as dist

    def barrier():
        if world > 1:
            dist.barrier()

    e2e_steps = timed_steps[: max(1, min(len(timed_steps), 200))]
    host_seeds = {}
    for i in e2e_steps:
        e, b = batch_of(i)
        if e not in host_seeds:
            ctx.shuffle(e)
            host_seeds[e] = ctx.permutation(sh.n_train)
    pinned = {}
    for i in e2e_steps:
        e, b = batch_of(i)
        pinned[i] = torch.from_numpy(host_seeds[e][b * sh.batch: b * sh.batch + n_seeds(b)]
                                     .view(np.int32).copy()).pin_memory()
    cnt_dev = ctx.extract_counts_tensor()
    cnt_host = torch.zeros((len(e2e_steps), 3), dtype=torch.int64).pin_memory()
    lag = max(1, args.pipeline)

    def e2e_run(sync_api):
        evs = []
        rows_seen = 0
        t0 = time.perf_counter()
        seeds_done = 0
        for j, i in enumerate(e2e_steps):
            e, b = batch_of(i)
            if sync_api:  # glb_sample (H2D seeds, D2H sizes, sync) + extract stats (sync)
                ctx.sample(pinned[i].numpy().view(np.uint32), seed=g.seed, epoch=e, batch=b)
                st = ctx.extract_sample(out, stats=True)
                rows_seen += st["hits"] + st["misses"]
            else:
                ctx.sample_async(pinned[i], seed=g.seed, epoch=e, batch=b)
                ctx.extract_sample(out)
                with torch.cuda.stream(xs):  # the stream the extract ran on
                    cnt_host[j].copy_(cnt_dev, non_blocking=True)
                    ev = torch.cuda.Event()
                    ev.record(xs)
                evs.append(ev)
                if j >= lag:
                    evs[j - lag].synchronize()
                    rows_seen += int(cnt_host[j - lag, 0] + cnt_host[j - lag, 1])
            seeds_done += n_seeds(b)
        for jj in range(max(0, len(evs) - lag), len(evs)):
            evs[jj].synchronize()
            rows_seen += int(cnt_host[jj, 0] + cnt_host[jj, 1])
        return time.perf_counter() - t0, seeds_done, rows_seen

    e2e_run(False)  # warm the pinned buffers / events
    barrier()
    torch.cuda.synchronize()
    e2e_secs, e2e_seeds, e2e_rows = e2e_run(False)
    sync_secs, sync_seeds, _ = e2e_run(True)
    e2e_t = torch.tensor([e2e_secs, sync_secs], dtype=torch.float64, device=dev)
    e2e_n = torch.tensor([float(e2e_seeds), float(sync_seeds)], dtype=torch.float64, device=dev)
    if world > 1:
        if args.backend == "gloo":
            e2e_t, e2e_n = e2e_t.cpu(), e2e_n.cpu()
        dist.all_reduce(e2e_t, op=dist.ReduceOp.MAX)
        dist.all_reduce(e2e_n)
    e2e_val = float(e2e_n[0].item()) / float(e2e_t[0].item())
    e2e_sync_val = float(e2e_n[1].item()) / float(e2e_t[1].item())
    h2d = 4 * statistics.mean(n_seeds(batch_of(i)[1]) for i in e2e_steps)
    d2h = 24  # the step's (hits, misses, peer hits) u64 result
    e2e = {"value": e2e_val, "unit": "seeds/s", "h2d_bytes_per_step": h2d,
           "d2h_bytes_per_step": d2h, "steps": len(e2e_steps),
           "api": "glb_sample_async(pinned host seeds) + glb_extract_sample + "
                  "D2H of the step's counts (host reads step j-D during step j, "
                  f"D = pipeline depth {lag})",
           "result_read_back": "the step's (hits, misses, peer hits) u64 counts; the gathered "
                               "features and blocks stay in HBM for the on-GPU consumer "
                               "(GNNLab's Trainer trains on the GPU, L252), so they do not "
                               "cross the host link",
           "rows_extracted": e2e_rows, "sync_api_value": e2e_sync_val,
           "sync_api": "glb_sample(host seeds; sizes D2H, sync) + glb_extract_sample "
                       "+ stats (sync) every step"}
    torch.cuda.synchronize()
    return e2e


def hit_rate_sweeps(args, ctx, g, sh, alpha, world, rank, nb, out, stream, xs, batch_of,
                    n_seeds, barrier):
    """alpha sweep (H, Optimal H*, Degree / Random policies, seeds/s), PreSC#K sweep and
    Table 2's footprint similarity over the measured epochs."""
    import torch

    import paper_conf_eurosys_yangtswycyz22_b200 as glb
    from paper_conf_eurosys_yangtswycyz22_b200 import parallel as par

    def reduce_counts(t):
        if world > 1:
            c = t if args.backend == "nccl" else t.cpu()
            par.allreduce_counts(c)
            if c is not t:
                t.copy_(c)
        return t

    per_epoch = []
    acc_sum = None
    # the sweeps rebuild the cache ~15 times: without the cold store (a host copy per build)
    ctx.set_cold_store(False)
    m0 = max([sh.K] + [int(x) for x in args.k_sweep.split(",") if x])
    for e in range(m0, m0 + args.measure_epochs):
        ctx.reset_counts(glb.COUNT_ACCESS)
        ctx.set_count_mode(glb.COUNT_ACCESS)
        for b in range(rank, nb, world):
            ctx.sample_batch(e, b)
        ctx.set_count_mode(glb.COUNT_NONE)
        ctx.sync()
        f = reduce_counts(ctx.counts_tensor(glb.COUNT_ACCESS))
        acc_sum = f.clone() if acc_sum is None else acc_sum.add_(f)
        if len(per_epoch) < 2:
            per_epoch.append(f.clone())
    ctx.counts_tensor(glb.COUNT_ACCESS).copy_(acc_sum)
    del acc_sum
    similarity = None
    if len(per_epoch) >= 2:
        v, num, den = ctx.footprint_similarity(per_epoch[0], per_epoch[1], 0.1)
        similarity = {"epochs": [m0, m0 + 1], "top_frac": 0.1, "value": v,
                      "numerator": num, "denominator": den, "source": "Table 2 (L329)"}
    def sweep_rate():
        """seeds/s of --sweep-steps pipelined steps with the cache as built (cold store off)"""
        torch.cuda.synchronize()
        s0 = torch.cuda.Event(enable_timing=True)
        s1 = torch.cuda.Event(enable_timing=True)
        s0.record(stream)
        sd = 0
        for i in range(args.sweep_steps):
            e, b = batch_of(i)
            ctx.sample_batch(e, b)
            ctx.extract_sample(out)
            sd += n_seeds(b)
        s1.record(xs)
        torch.cuda.synchronize()
        return sd * world / (s0.elapsed_time(s1) / 1e3)

    sweep, result_hit = [], None
    for a in sorted(set(sh.alphas) | {alpha}):
        policies = {}
        if 0.0 < a < 1.0:  # Fig 10 analog: Degree / Random vs PreSC vs Optimal
            for pol in ("degree", "random"):
                ctx.build_cache_policy(a, pol, seed=g.seed)
                hs = ctx.hit_stats()
                policies[pol] = hs["hits"] / hs["total"] if hs["total"] else 0.0
        ctx.build_cache(a)
        hs = ctx.hit_stats()
        H = hs["hits"] / hs["total"] if hs["total"] else 0.0
        Hs = hs["optimal_hits"] / hs["total"] if hs["total"] else 0.0
        sweep.append({"alpha": a, "cache_rows": hs["cache_rows"], "hit_rate": H,
                      "optimal_hit_rate": Hs,
                      "presc_vs_optimal_pct": (100.0 * H / Hs) if Hs > 0 else None,
                      "degree_hit_rate": policies.get("degree"),
                      "random_hit_rate": policies.get("random"),
                      "seeds_per_s": sweep_rate()})
        if a == alpha:
            result_hit = sweep[-1]
    k_sweep = []
    a_k = next((a for a in sh.alphas if 0.0 < a < 1.0), None)
    if args.k_sweep and a_k is not None:
        for K in [int(x) for x in args.k_sweep.split(",") if x]:
            ctx.reset_counts(glb.COUNT_PRESAMPLE)
            ctx.presample(K, rank, world)
            reduce_counts(ctx.counts_tensor(glb.COUNT_PRESAMPLE))
            ctx.build_cache(a_k)
            hs = ctx.hit_stats()
            H = hs["hits"] / hs["total"] if hs["total"] else 0.0
            Hs = hs["optimal_hits"] / hs["total"] if hs["total"] else 0.0
            k_sweep.append({"K": K, "alpha": a_k, "hit_rate": H, "optimal_hit_rate": Hs,
                            "presc_vs_optimal_pct": 100.0 * H / Hs if Hs else None})
    return {"hit_rate": result_hit, "alpha_sweep": sweep, "presc_k_sweep": k_sweep,
            "sweep_seeds_per_s_is": f"{args.sweep_steps} pipelined steps per point, cold store "
                                    "off (the sweeps rebuild the cache per point)",
            "measured_epochs": [m0, m0 + args.measure_epochs - 1],
            "footprint_similarity": similarity}


def main(argv=None):
    argv = sys.argv[1:] if argv is None else argv
    args = parse(argv)
    if args.impl == "reference":
        return reference_arm(args)
    if "WORLD_SIZE" not in os.environ and args.gpus > 1:
        # the driver's `bench.py --gpus N` without a launcher: one rank per GPU
        if args.ns_sweep and args.mode == "factored":
            return ns_sweep(args, argv)
        rc, _ = launch_ranks(args.gpus, argv)
        sys.exit(rc)
    import torch
    import torch.distributed as dist

    world, rank, local, local_world = dist_env()
    local = local % torch.cuda.device_count()
    if world > 1:
        torch.cuda.set_device(local)
        if args.backend == "nccl":
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
        else:
            dist.init_process_group("gloo")
    dev = torch.device("cuda", local)
    torch.cuda.set_device(dev)
    stream = torch.cuda.current_stream(dev)
    sh = synth.SHAPES[args.config]
    if world > 1:  # every rank measures its link while the others do (as in the run)
        dist.barrier()
    link_peak = hostlink_peak(dev)
    res = run_workload(args, sh, args.alpha, world, rank, local, local_world, dev, stream, True,
                       link_peak)
    if args.mode == "factored":
        return
    pr1 = None
    if not args.no_pr_alpha1 and args.config != "PR":
        r = run_workload(args, synth.SHAPES["PR"], 1.0, world, rank, local, local_world, dev,
                         stream, False, link_peak)
        pr1 = {"workload": workload_name(synth.SHAPES["PR"], 1.0), "value": r["value"],
               "unit": "seeds/s", "ms_per_step": r["ms_per_step"], "runs": r["runs"],
               "runs_range": r["runs_range"], "roofline": r["roofline"],
               "path_roofline": r["path_roofline"], "e2e_value": r["e2e"]["value"],
               "host_enqueue_ms_per_step": r["host_enqueue_ms_timed_region"] / args.steps,
               "gpu_launches": r["gpu_launches"], "clocks": r["clocks"]}
    if rank == 0:
        line = {
            "metric": METRIC, "value": res["value"], "unit": "seeds/s", "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": res["ms_per_step"],
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "u32",
            "data": "synthetic",
            "config": {"workload": workload_name(sh, args.alpha), "shape": sh.name,
                       "config_index": synth.CONFIG_INDEX.get(sh.name),
                       "V": sh.V, "E": sh.E, "feat_dim": sh.D, "batch": sh.batch,
                       "fanouts": list(sh.fanouts), "sampler": sh.sampler, "alpha": args.alpha,
                       "presample_K": sh.K, "parallelism": f"dp{world}",
                       "l2": "inputs larger than L2 (CSR %.2f GB, feature cache %.2f GB, host "
                             "matrix %.1f GB vs 126 MB L2)"
                             % ((8 * (sh.V + 1) + 4 * sh.E) / 1e9,
                                4 * sh.D * sh.V * args.alpha / 1e9, 4 * sh.D * sh.V / 1e9)},
            "runs": res["runs"], "runs_range": res["runs_range"],
            "value_is": f"median of {args.runs} timed regions of {args.steps} steps",
            "pipeline_depth": args.pipeline,
            "roofline": res["roofline"], "path_roofline": res["path_roofline"],
            "cpu_baseline": res.get("cpu_baseline"), "e2e": res["e2e"],
            "gpu_launches": res["gpu_launches"], "clocks": res["clocks"],
            "pr_alpha1": pr1,
            "host": host_info(), "gpu": gpu_info(local),
        }
        for k in ("cache", "host_gather", "cold_store_rows", "relabel_table", "relabel_l2_window_bytes", "host_inputs",
                  "host_wall_ms_timed_region", "host_enqueue_ms_timed_region", "hit_rate",
                  "alpha_sweep", "presc_k_sweep", "measured_epochs", "footprint_similarity",
                  "units", "preprocess_s"):
            if k in res:
                line[k] = res[k]
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()


def ns_sweep(args, argv):
    """Config 5's Ns sweep (Fig 15 analog): the adaptive split, then every
    Ns in 1..N-1, each a separate N-rank factored run; one line = the adaptive run plus the
    sweep."""
    base = [a for a in argv if a != "--ns-sweep"]
    rc, line = launch_ranks(args.gpus, base, capture=True)
    if rc != 0 or line is None:
        sys.exit(rc or 1)
    sweep = []
    for ns in range(1, args.gpus):
        r, ln = launch_ranks(args.gpus, base + ["--ns", str(ns)], capture=True)
        sweep.append({"samplers": ns, "trainers": args.gpus - ns,
                      "value": ln["value"] if ln else None, "rc": r})
    line["ns_sweep"] = sweep
    print(json.dumps(line), flush=True)


if __name__ == "__main__":
    main()
