"""a8 push-kernel cost on one GPU: two ctxs on cuda:0 (sampler: topology only; trainer:
ring of 2 slots), PR batches; CUDA events around glb_handoff_send on the sampler's stream
time k_push alone.  Bytes = the sample's header + uniq + every block's indptr/indices
(what the kernel moves, read + write); on one GPU both sides are HBM, on an NVSwitch box
the writes cross NVLink."""
import json
import sys

import torch

sys.path.insert(0, ".")
import paper_conf_eurosys_yangtswycyz22_b200 as glb  # noqa: E402
import synth  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "PR"
g = synth.make_graph(cfg)
sh = g.shape


def make(features):
    c = glb.Context(0)
    c.load_graph(g.indptr, g.indices, g.features if features else None)
    c.set_sampler("khop", fanouts=sh.fanouts, max_batch=sh.batch)
    c.set_train_set(g.train, sh.batch, g.seed)
    return c


trainer, sampler = make(True), make(False)
trainer.build_cache(1.0)
trainer.handoff_connect(0, sampler.handoff_attach(1, trainer.handoff_create(2)))
main = torch.cuda.current_stream()
ts, nbytes = [], []
for i in range(24):
    b = i % trainer.num_batches
    sampler.sample_batch(1, b)
    s = sampler.sample_result()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(main)
    sampler.handoff_send(1, i % 2, b)
    e1.record(main)
    trainer.handoff_recv(0, i % 2)
    trainer.handoff_release(i % 2)
    torch.cuda.synchronize()
    if i >= 4:
        ts.append(e0.elapsed_time(e1) * 1e3)
        words = s.sizes[-1] + sum(s.sizes[l] + 1 for l in range(len(s.nnz))) + sum(s.nnz)
        nbytes.append(2 * 4 * words)  # read + write
ts.sort()
med = ts[len(ts) // 2]
mb = sum(nbytes) / len(nbytes)
print(json.dumps({"config": cfg, "push_us_median": med, "bytes_per_push_rw": mb,
                  "achieved_GBps": mb / (med * 1e-6) / 1e9, "n": len(ts)}))
