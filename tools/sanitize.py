"""Small end-to-end run (tiny config, both relabel modes, k-hop + random walk, PreSC,
cache, extract with hits and misses, pipeline depth 2) for compute-sanitizer, under each
library variant (environment knobs read at glb_create): default, warp / block-staged
relabel pre-dedup, host-assisted misses, one miss bin per row (device scan), the
warp-independent gather, a capped miss-block count, the cold store (with and without
host-assisted misses)."""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, ".")
import oracle  # noqa: E402
import paper_conf_eurosys_yangtswycyz22_b200 as glb  # noqa: E402
import synth  # noqa: E402

g = synth.make_graph("tiny")
sh = g.shape
go = oracle.GraphOracle(g.indptr, g.indices, g.features)
VARIANTS = [{}, {"GLB_RELABEL_DEDUP": "1"}, {"GLB_RELABEL_DEDUP": "2"},
            {"GLB_HOST_GATHER": "400", "GLB_HOST_GATHER_THREADS": "2"},
            {"GLB_MISS_BIN_LOG2": "7", "GLB_GATHER_WARP": "1"}, {"GLB_MISS_BLOCKS": "3"},
            {"GLB_GATHER_LIDORDER": "0", "GLB_HOST_GATHER": "400", "GLB_HOST_GATHER_THREADS": "2"},
            {"GLB_COLD_STORE": "1", "GLB_HOST_GATHER": "150", "GLB_HOST_GATHER_THREADS": "2"},
            {"GLB_COLD_STORE": "1"}]
KEYS = {k for v in VARIANTS for k in v}
for var, mode in [(v, m) for v in VARIANTS for m in ["dense", "hash"]]:
    for k in KEYS:
        os.environ.pop(k, None)
    os.environ.update(var)
    ctx = glb.Context(0)
    ctx.load_graph(g.indptr, g.indices, g.features)
    ctx.set_relabel_mode(mode)
    ctx.set_sampler("khop", fanouts=sh.fanouts, max_batch=sh.batch)
    ctx.set_train_set(g.train, sh.batch, g.seed)
    ctx.presample(1)
    ctx.build_cache(0.3)
    out = torch.empty((sh.batch * 66, g.D), device="cuda")
    for depth in [1, 2]:
        ctx.set_pipeline(depth)
        for b in range(4):
            ctx.sample_batch(1, b)
            ctx.extract_sample(out)
        ctx.sync()
    ctx.set_pipeline(1)
    ctx.sample_batch(1, 5)
    s = ctx.sample_result()
    ctx.extract_sample(out)
    ctx.sync()
    exp = go.sample_khop(oracle.epoch_batches(g.train, sh.batch, g.seed, 1)[5], sh.fanouts, g.seed, 1, 5)
    assert np.array_equal(s.uniq.cpu().numpy().view(np.uint32), exp.uniq)
    ids = torch.from_numpy(exp.uniq.view(np.int32)).cuda()
    o2 = ctx.extract(ids)
    assert np.array_equal(o2.cpu().numpy().view(np.uint32), go.extract(exp.uniq).view(np.uint32))
    if var.get("GLB_COLD_STORE") == "1":
        assert ctx.cold_store_rows > 0
    ctx.set_sampler("rwalk", layers=2, max_batch=sh.batch)
    ctx.sample_batch(1, 2)
    ctx.sample_result()
    ctx.close()
print("sanitize run ok")
