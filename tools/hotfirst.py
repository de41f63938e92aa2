"""Experiment for DESIGN §12.1: does a hot-first vertex numbering make the large graphs'
relabel tables L2-pinnable?  Build a config's graph, renumber it by the generator's degree
rank (rank 0 = heaviest vertex; features left in place -- timing only), and time the
pipelined sample+extract step (CUDA events, 200 steps) on the original graph, on the
renumbered one, and on the renumbered one with its table's first GLB_L2_PIN_PREFIX_MB
pinned (set in the environment of the third run by the caller).
usage: python tools/hotfirst.py TW [orig|hot]"""
import json
import sys
import time

import numpy as np
import torch

sys.path.insert(0, ".")
import paper_conf_eurosys_yangtswycyz22_b200 as glb  # noqa: E402
import synth  # noqa: E402

cfg, which = sys.argv[1], sys.argv[2]
g = synth.make_graph(cfg)
sh = g.shape
indptr, indices, train = g.indptr, g.indices, g.train
if which == "hot":
    t0 = time.time()
    order = synth.rank_order(sh.V, g.seed)            # new id r -> old vertex order[r]
    inv = np.empty(sh.V, np.uint32)
    inv[order] = np.arange(sh.V, dtype=np.uint32)     # old vertex -> new id
    deg = np.diff(indptr).astype(np.int64)
    ndeg = deg[order]
    nindptr = np.zeros(sh.V + 1, np.uint64)
    np.cumsum(ndeg, out=nindptr[1:])
    shift = indptr[:-1][order].astype(np.int64) - nindptr[:-1].astype(np.int64)
    pos = np.repeat(shift, ndeg)
    pos += np.arange(sh.E, dtype=np.int64)
    nindices = inv[indices[pos]]
    del pos
    indptr, indices, train = nindptr, nindices, np.sort(inv[train])
    print(f"renumbered in {time.time() - t0:.1f} s", file=sys.stderr)
ctx = glb.Context(0)
ctx.load_graph(indptr, indices, g.features)
ctx.set_sampler(sh.sampler, fanouts=sh.fanouts, max_batch=sh.batch)
ctx.set_train_set(train, sh.batch, g.seed)
ctx.build_cache(1.0)
ctx.set_pipeline(2)
ub = sh.batch
for k in sh.fanouts:
    ub = min(ub * (1 + k), sh.V)
out = torch.empty((ub, sh.D), device="cuda")
nb = ctx.num_batches
main = torch.cuda.current_stream()


def run(n, first):
    for i in range(first, first + n):
        ctx.sample_batch(1 + i // nb, i % nb)
        ctx.extract_sample(out)


run(10, 0)
torch.cuda.synchronize()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record(main)
run(200, 10)
xs = ctx.extract_stream()
main.wait_stream(xs)
e1.record(main)
torch.cuda.synchronize()
ms = e0.elapsed_time(e1) / 200
print(json.dumps({"config": cfg, "graph": which, "us_per_step": 1e3 * ms,
                  "l2_window_bytes": ctx.relabel_l2_window}))
