"""Per-step timeline of sampling (main stream) vs extract (extract stream)."""
import sys

import torch

sys.path.insert(0, ".")
import paper_conf_eurosys_yangtswycyz22_b200 as glb  # noqa: E402
import synth  # noqa: E402

depth = int(sys.argv[1]) if len(sys.argv) > 1 else 2
g = synth.make_graph("PR")
sh = g.shape
ctx = glb.Context(0)
ctx.load_graph(g.indptr, g.indices, g.features)
ctx.set_sampler("khop", fanouts=sh.fanouts, max_batch=sh.batch)
ctx.set_train_set(g.train, sh.batch, g.seed)
ctx.build_cache(1.0)
ctx.set_pipeline(depth)
xs = ctx.extract_stream()
main = torch.cuda.current_stream()
out = torch.empty((sh.batch * 26 * 11, sh.D), device="cuda")
for b in range(5):
    ctx.sample_batch(1, b)
    ctx.extract_sample(out)
ctx.sync()
E = lambda: torch.cuda.Event(enable_timing=True)  # noqa: E731
t0 = E()
t0.record(main)
ev = []
for b in range(5, 15):
    a, z, x0, x1 = E(), E(), E(), E()
    a.record(main)
    ctx.sample_batch(1, b)
    z.record(main)
    x0.record(xs)
    ctx.extract_sample(out)
    x1.record(xs)
    ev.append((a, z, x0, x1))
torch.cuda.synchronize()
for i, (a, z, x0, x1) in enumerate(ev):
    print(f"step {i}: sample {t0.elapsed_time(a)*1e3:8.1f} -> {t0.elapsed_time(z)*1e3:8.1f} us   "
          f"extract {t0.elapsed_time(x0)*1e3:8.1f} -> {t0.elapsed_time(x1)*1e3:8.1f} us")
