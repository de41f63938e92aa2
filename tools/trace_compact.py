"""Timeline of compaction tiles (needs a GLB_TRACE=1 build).  Debug tool."""
import ctypes
import sys

import numpy as np
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
for b in range(5):
    ctx.sample_batch(1, b)
ctx.sync()
buf = np.zeros((8, 4096, 8), np.uint64)
glb.lib().glb_trace_dump(buf.ctypes.data, buf.nbytes)
for hop in range(2):
    t = buf[hop].astype(np.int64)
    n = int((t[:, 0] > 0).sum())
    t = t[:n]
    t0 = t[:, 0].min()
    rel = (t - t0) / 1e3  # %globaltimer ns -> us since the first tile claim of this hop
    print(f"hop {hop}: {n} tiles; span {rel[:, 5].max():.1f} us")
    names = ["claim", "loaded", "lookback", "scanned", "done", "end"]
    for ev in range(6):
        print(f"  {names[ev]:9s} min {rel[:, ev].min():7.1f} med {np.median(rel[:, ev]):7.1f} max {rel[:, ev].max():7.1f}")
    for i in list(range(0, n, max(1, n // 12))):
        print("   tile", i, " ".join(f"{x:7.1f}" for x in rel[i, :6]))

# sampler kernel spans next to the compaction tiles (one batch; needs GLB_TRACE=1)
L = glb.lib()
L.glb_trace_reset()
ctx.sample_batch(1, 7)
ctx.sync()
buf = np.zeros((8, 4096, 8), np.uint64)
L.glb_trace_dump(buf.ctypes.data, buf.nbytes)
kt = np.zeros((8, 2), np.uint64)
L.glb_ktrace_dump(kt.ctypes.data)
T0 = int(kt[0, 0])
for hop in range(2):
    t = buf[hop].astype(np.int64)
    n = int((t[:, 0] > 0).sum())
    t = t[:n]
    print(f"hop {hop}: k_khop {(int(kt[hop,0])-T0)/1e3:7.1f} -> {(int(kt[hop,1])-T0)/1e3:7.1f} us; "
          f"compact tiles claim {(t[:,0].min()-T0)/1e3:7.1f} .. {(t[:,0].max()-T0)/1e3:7.1f}, "
          f"loaded med {(np.median(t[:,1])-T0)/1e3:7.1f}, lookback done max {(t[:,2].max()-T0)/1e3:7.1f}, "
          f"end max {(t[:,5].max()-T0)/1e3:7.1f} us ({n} tiles)")
