"""Small run of this round's new device paths for compute-sanitizer: the a8 handoff (push
kernel, trainer-side mark of a received sample, extract of it; pipeline depths 1 and 2) and
the TMA bulk-copy gathers (hits and host misses, GLB_GATHER_BULK / GLB_MISS_BULK)."""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, ".")
os.environ["GLB_GATHER_BULK"] = "1"
os.environ["GLB_MISS_BULK"] = "1"
import oracle  # noqa: E402
import paper_conf_eurosys_yangtswycyz22_b200 as glb  # noqa: E402
import synth  # noqa: E402

g = synth.make_graph("tiny")
sh = g.shape
go = oracle.GraphOracle(g.indptr, g.indices, g.features)


def make(alpha):
    c = glb.Context(0)
    c.load_graph(g.indptr, g.indices, g.features)
    c.set_sampler("khop", fanouts=sh.fanouts, max_batch=sh.batch)
    c.set_train_set(g.train, sh.batch, g.seed)
    if alpha is not None:
        c.presample(1)
        c.build_cache(alpha)
    return c


out = torch.empty((sh.batch * 66, g.D), device="cuda")
for depth in [1, 2]:
    t, s = make(0.3), make(None)
    t.set_pipeline(depth)
    s.set_pipeline(depth)
    t.handoff_connect(0, s.handoff_attach(1, t.handoff_create(2)))
    batches = oracle.epoch_batches(g.train, sh.batch, g.seed, 1)
    for i, b in enumerate([0, 1, 2, 15]):
        s.sample_batch(1, b)
        s.handoff_send(1, i % 2, b)
        t.handoff_recv(0, i % 2)
        t.extract_sample(out)
        t.handoff_release(i % 2)
        t.sync()
        n = t.sample_result if False else None
        exp = go.sample_khop(batches[b], sh.fanouts, g.seed, 1, b)
        assert np.array_equal(out[: len(exp.uniq)].cpu().numpy().view(np.uint32),
                              go.extract(exp.uniq).view(np.uint32))
    s.close()
    t.close()
print("sanitize handoff/bulk run ok")
