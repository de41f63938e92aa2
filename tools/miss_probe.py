"""Probe the library's zero-copy miss gather on a Papers100M-sized feature matrix.

Loads a features-only graph (V x D f32 in registered host memory, no edges) with an
empty cache (alpha = 0: every row is a miss) and times glb_extract on id lists of
`--n` ids drawn uniformly from the first `span` rows, for several spans (the region
the misses fall in) and miss orderings (GLB_MISS_BIN_LOG2).  CUDA events on the ctx
stream around each extract (mark + miss ordering + gather).

  python tools/miss_probe.py --V 111059956 --D 128 --n 442000
"""
from __future__ import annotations

import argparse
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import synth  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--V", type=int, default=111_059_956)
    ap.add_argument("--D", type=int, default=128)
    ap.add_argument("--n", type=int, default=442_000)
    ap.add_argument("--spans", default="1.0,0.5,0.25,0.05")
    ap.add_argument("--bins", default="21,0")
    ap.add_argument("--reps", type=int, default=5)
    ap.add_argument("--region-fracs", default="",
                    help="also draw the ids from a random subset (this fraction) of the 2 MB regions "
                         "of the whole matrix: same span, fewer distinct regions per extract")
    args = ap.parse_args()
    import paper_conf_eurosys_yangtswycyz22_b200 as glb
    t0 = time.perf_counter()
    feats = synth.gen_features(args.V, args.D, 1234)
    indptr = np.zeros(args.V + 1, np.uint64)
    indices = np.zeros(0, np.uint32)
    print(json.dumps({"features_gb": feats.nbytes / 1e9, "gen_s": time.perf_counter() - t0}),
          flush=True)
    rng = np.random.default_rng(7)
    for b in [int(x) for x in args.bins.split(",")]:
        os.environ["GLB_MISS_BIN_LOG2"] = str(b)
        ctx = glb.Context(0)
        ctx.load_graph(indptr, indices, feats)
        ctx.build_cache(0.0)
        out = torch.empty((args.n, args.D), dtype=torch.float32, device="cuda")
        s = torch.cuda.current_stream()
        for span in [float(x) for x in args.spans.split(",")]:
            hi = max(1, int(args.V * span))
            ids = rng.choice(hi, size=min(args.n, hi), replace=False).astype(np.int32)
            for order in ("random", "sorted"):
                v = np.sort(ids) if order == "sorted" else ids
                dv = torch.from_numpy(v).cuda()
                ctx.extract(dv, out=out[:v.size])
                ts = []
                for _ in range(args.reps):
                    e0 = torch.cuda.Event(enable_timing=True)
                    e1 = torch.cuda.Event(enable_timing=True)
                    e0.record(s)
                    ctx.extract(dv, out=out[:v.size])
                    e1.record(s)
                    torch.cuda.synchronize()
                    ts.append(e0.elapsed_time(e1))
                ms = min(ts)
                print(json.dumps({"miss_bin_log2": b, "span_rows": hi,
                                  "span_gb": hi * args.D * 4 / 1e9, "input_order": order,
                                  "n": int(v.size), "row_bytes": 4 * args.D, "ms": ms,
                                  "gbs": v.size * 4 * args.D / (ms * 1e-3) / 1e9}), flush=True)
        rows_per_region = (2 << 20) // (args.D * 4)
        nreg = (args.V + rows_per_region - 1) // rows_per_region
        for rf in [float(x) for x in args.region_fracs.split(",") if x]:
            regs = rng.choice(nreg, size=max(1, int(nreg * rf)), replace=False)
            cand = (regs[:, None] * rows_per_region + np.arange(rows_per_region)[None, :]).ravel()
            cand = cand[cand < args.V]
            ids = rng.choice(cand, size=args.n, replace=False).astype(np.int32)
            dv = torch.from_numpy(np.sort(ids)).cuda()
            ctx.extract(dv, out=out)
            ts = []
            for _ in range(args.reps):
                e0 = torch.cuda.Event(enable_timing=True)
                e1 = torch.cuda.Event(enable_timing=True)
                e0.record(s)
                ctx.extract(dv, out=out)
                e1.record(s)
                torch.cuda.synchronize()
                ts.append(e0.elapsed_time(e1))
            ms = min(ts)
            print(json.dumps({"miss_bin_log2": b, "region_frac": rf, "regions": int(len(regs)),
                              "n": args.n, "ms": ms, "gbs": args.n * 4 * args.D / (ms * 1e-3) / 1e9}),
                  flush=True)
        ctx.close()
        del out
        torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
