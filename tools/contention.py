"""Why does the sampler slow down ~2x when the gather of the previous batch runs beside it
(pipeline depth 2)?  Time k-hop sampling of PR batches (CUDA events, main stream) alone and
next to a DRAM hog on a side stream: (a) copy-engine D2D memcpy (no SM resources),
(b) an SM copy kernel (torch copy_, many threads), (c) the library's own extract
(k_gather) of an earlier batch.  Also reports each hog's bandwidth alone."""
import sys

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
main = torch.cuda.current_stream()
side = torch.cuda.Stream(priority=0)
N = 20
big_a = torch.empty(1 << 30, dtype=torch.uint8, device="cuda")
big_b = torch.empty_like(big_a)
out = torch.empty((sh.batch * 26 * 11, sh.D), device="cuda")
E = lambda: torch.cuda.Event(enable_timing=True)  # noqa: E731


def sample_time(hog=None):
    for b in range(3):
        ctx.sample_batch(1, b)
    torch.cuda.synchronize()
    ts = []
    for b in range(3, 3 + N):
        if hog is not None:
            with torch.cuda.stream(side):
                hog()
        s, e = E(), E()
        s.record(main)
        ctx.sample_batch(1, b)
        e.record(main)
        torch.cuda.synchronize()
        ts.append(s.elapsed_time(e) * 1e3)
    ts.sort()
    return ts[len(ts) // 2]


def hog_bw(hog, nbytes):
    torch.cuda.synchronize()
    s, e = E(), E()
    with torch.cuda.stream(side):
        s.record(side)
        hog()
        e.record(side)
    torch.cuda.synchronize()
    return nbytes / (s.elapsed_time(e) * 1e-3) / 1e9, s.elapsed_time(e) * 1e3


import ctypes  # noqa: E402
_rt = ctypes.CDLL("libcudart.so.12")
_rt.cudaMemcpyAsync.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_size_t, ctypes.c_int,
                                ctypes.c_void_p]
fa, fb = big_a.view(torch.float32), big_b.view(torch.float32)


def ce_copy():  # cudaMemcpyAsync D2D (copy engine)
    assert _rt.cudaMemcpyAsync(big_b.data_ptr(), big_a.data_ptr(), big_a.numel(), 3,
                               side.cuda_stream) == 0


def sm_copy():  # elementwise SM kernel, many threads
    torch.add(fa, 1.0, out=fb)


# the previous batch's uniq for the extract hog
ctx.sample_batch(1, 0)
prev = ctx.sample_result()
uniq = prev.uniq.clone()


def gather():
    ctx.extract(uniq, out=out[: uniq.numel()])


print("sampling alone                 %.1f us" % sample_time())
for name, hog, nb in [("copy-engine D2D 1 GB", ce_copy, 2 << 30), ("SM copy_ 1 GB", sm_copy, 2 << 30)]:
    bw, t = hog_bw(hog, nb)
    print("%-22s alone %.0f GB/s (%.0f us); sampling beside it %.1f us" % (name, bw, t, sample_time(hog)))
n = uniq.numel()
bw, t = hog_bw(gather, n * sh.D * 4 * 2)
print("%-22s alone %.0f GB/s (%.0f us); sampling beside it %.1f us" %
      ("library extract (LSU)", bw, t, sample_time(lambda: [gather() for _ in range(3)])))
