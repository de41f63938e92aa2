"""Host-side enqueue cost per API call (is the bench host-bound?)."""
import sys
import time

import torch

sys.path.insert(0, ".")
import paper_conf_eurosys_yangtswycyz22_b200 as glb  # noqa: E402
import synth  # noqa: E402

g = synth.make_graph("PR")
sh = g.shape
ctx = glb.Context(0)
ctx.load_graph(g.indptr, g.indices, g.features)
ctx.set_sampler("khop", fanouts=sh.fanouts, max_batch=sh.batch)
ctx.set_train_set(g.train, sh.batch, g.seed)
ctx.build_cache(1.0)
out = torch.empty((sh.batch * 26 * 11, sh.D), device="cuda")
x = torch.zeros(1, device="cuda")
for _ in range(3):
    ctx.sample_batch(1, 0)
    ctx.extract_sample(out)
torch.cuda.synchronize()
N = 200
t = time.perf_counter()
for i in range(N):
    x.add_(1)
print("torch add_ launch: %.1f us" % ((time.perf_counter() - t) / N * 1e6))
torch.cuda.synchronize()
t = time.perf_counter()
for i in range(N):
    ctx.sample_batch(1, i % 24)
te = time.perf_counter()
torch.cuda.synchronize()
print("sample_batch enqueue: %.1f us/call, drain %.1f us/call" % ((te - t) / N * 1e6, (time.perf_counter() - t) / N * 1e6))
t = time.perf_counter()
for i in range(N):
    ctx.extract_sample(out)
te = time.perf_counter()
torch.cuda.synchronize()
print("extract_sample enqueue: %.1f us/call, drain %.1f us/call" % ((te - t) / N * 1e6, (time.perf_counter() - t) / N * 1e6))
ctx.set_timing(True)
t = time.perf_counter()
for i in range(N):
    ctx.extract_sample(out)
te = time.perf_counter()
torch.cuda.synchronize()
print("extract_sample+timing enqueue: %.1f us/call" % ((te - t) / N * 1e6))
import ctypes  # noqa: E402
L = glb.lib()
t = time.perf_counter()
for i in range(N):
    L.glb_kernel_launches(ctx._h)
print("ctypes trivial call: %.2f us" % ((time.perf_counter() - t) / N * 1e6))
