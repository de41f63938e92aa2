"""NEXT-3 on one GPU: cost of the peer-sharded gather path (k_gather<SHARD>) against the
replicated cache, with the W shards emulated on cuda:0 (peers = other ctxs of this
process, so "peer" rows come from local HBM, not NVLink).  What this measures is the
kernel-side overhead of resolving a row's owner shard, and the hit rate a sharded
group reaches; NVLink bandwidth itself needs a multi-GPU box.

  python tools/shard_emulation.py [--config PR] [--world 8] [--alpha 0.125] [--steps 200]
"""
import argparse
import json
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_eurosys_yangtswycyz22_b200 as glb  # noqa: E402
import synth  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="PR")
ap.add_argument("--world", type=int, default=8)
ap.add_argument("--alpha", type=float, default=0.126)  # W*floor(alpha*V) >= V: no misses
ap.add_argument("--steps", type=int, default=200)
args = ap.parse_args()

g = synth.make_graph(args.config)
sh = g.shape


def make(rank, world, alpha, sharded):
    c = glb.Context(0)
    c.load_graph(g.indptr, g.indices, g.features)
    c.set_sampler(sh.sampler, fanouts=sh.fanouts, max_batch=sh.batch)
    c.set_train_set(g.train, sh.batch, g.seed)
    c.set_count_mode(glb.COUNT_PRESAMPLE)
    c.presample(sh.K)
    c.set_count_mode(glb.COUNT_NONE)
    if sharded:
        c.build_cache_sharded(alpha, rank, world)
    else:
        c.build_cache(alpha)
    return c


def run(c, label):
    nb = c.num_batches
    ub = sh.batch
    for k in sh.fanouts:
        ub = min(ub * (1 + k), sh.V)
    out = torch.empty((ub, sh.D), device="cuda:0")
    for i in range(5):
        c.sample_batch(sh.K, i % nb)
        c.extract_sample(out)
    c.sync()
    c.set_timing(True)
    t0, t1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    t0.record()
    seeds = 0
    for i in range(args.steps):
        e, b = sh.K + 1 + i // nb, i % nb
        c.sample_batch(e, b)
        c.extract_sample(out)
        seeds += min(sh.batch, len(g.train) - b * sh.batch)
    t1.record()
    torch.cuda.synchronize()
    xs = c.extract_times()
    c.set_timing(False)
    k = c.last_extract_counts()
    ms = t0.elapsed_time(t1)
    r = {"case": label, "seeds_per_s": seeds / (ms / 1e3), "ms_per_step": ms / args.steps,
         "extract_ms": sum(xs) / len(xs), "last_batch": k}
    print(json.dumps(r), flush=True)
    return r


res = []
full = make(0, 1, 1.0, False)
res.append(run(full, "replicated alpha=1.0"))
full.close()
group = [make(r, args.world, args.alpha, True) for r in range(args.world)]
for r, c in enumerate(group):
    for p, o in enumerate(group):
        if p != r:
            c.attach_peer_cache(p, dev_ptr=o.cache_device_ptr()[0])
res.append(run(group[0], f"sharded W={args.world} alpha={args.alpha} (emulated peers on cuda:0)"))
for c in group:
    c.close()
print(json.dumps({"config": args.config, "world": args.world, "alpha": args.alpha,
                  "results": res}))
