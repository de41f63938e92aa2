"""Sampling time per batch with and without the extract between batches (does the gather's
L2 streaming evict the relabel table / CSR offsets the sampler needs?)."""
import sys

import torch

sys.path.insert(0, ".")
import paper_conf_eurosys_yangtswycyz22_b200 as glb  # noqa: E402
import synth  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "PR"
g = synth.make_graph(cfg)
sh = g.shape
ctx = glb.Context(0)
ctx.load_graph(g.indptr, g.indices, g.features)
ctx.set_sampler(sh.sampler, fanouts=sh.fanouts, max_batch=sh.batch)
ctx.set_train_set(g.train, sh.batch, g.seed)
ctx.build_cache(1.0)
ub = sh.batch
for k in sh.fanouts:
    ub = min(ub * (1 + k), sh.V)
out = torch.empty((ub, sh.D), device="cuda")
nb = ctx.num_batches
E = lambda: torch.cuda.Event(enable_timing=True)  # noqa: E731
for mode in ["sample only", "sample+extract", "sample+l2flush"]:
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    for i in range(5):
        ctx.sample_batch(2, i % nb)
    torch.cuda.synchronize()
    ts = []
    for i in range(60):
        a, z = E(), E()
        a.record()
        ctx.sample_batch(3, i % nb)
        z.record()
        if mode == "sample+extract":
            ctx.extract_sample(out)
        elif mode == "sample+l2flush":
            flush.add_(1)
        ts.append((a, z))
    torch.cuda.synchronize()
    ms = sorted(a.elapsed_time(z) for a, z in ts)
    print(f"{cfg} {mode:16s} sampling median {ms[len(ms)//2]*1e3:7.1f} us  min {ms[0]*1e3:7.1f}")
