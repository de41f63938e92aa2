"""Steps right after a load_cache rebuild: PA-shaped, PreSC#1; build at alpha=1, then at 0.22 (host
misses, host-assisted 0.15), then time 3 windows of 10 pipelined steps each; repeat with a
PreSC#K re-run in between, as bench.py's K sweep does.  Prints ms per step per window."""
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import paper_conf_eurosys_yangtswycyz22_b200 as glb  # noqa: E402
import synth  # noqa: E402

sh = synth.SHAPES["PA"]
g = synth.make_graph(sh)
dev = torch.device("cuda", 0)
ctx = glb.Context(0)
ctx.load_graph(g.indptr, g.indices, g.features)
ctx.set_sampler("rwalk", layers=len(sh.fanouts), walks=synth.RW_WALKS, walk_len=synth.RW_LEN,
                topk=sh.fanouts[0], max_batch=sh.batch)
ctx.set_train_set(g.train, sh.batch, g.seed)
ctx.set_pipeline(2)
ctx.set_host_gather(0.15, threads=4)
ctx.presample(1)
out = torch.empty((sh.batch * 216 + 64, sh.D), device=dev)


def window(tag, first_batch):
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    for i in range(10):
        ctx.sample_batch(2, first_batch + i)
        ctx.extract_sample(out)
    ctx.sync()
    torch.cuda.synchronize()
    print(json.dumps({"window": tag, "ms_per_step": (time.perf_counter() - t0) * 100}), flush=True)


for rep in range(2):
    ctx.build_cache(1.0)
    window(f"rep{rep} alpha=1", 0)
    if rep == 1:
        ctx.presample(1)
    t0 = time.perf_counter()
    ctx.build_cache(0.22)
    print(json.dumps({"build_cache_s": time.perf_counter() - t0}), flush=True)
    for w in range(3):
        window(f"rep{rep} alpha=0.22 w{w}", 10 + 10 * w)
