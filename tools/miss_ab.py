"""A/B of the host-miss ordering in the extract (a7 misses over PCIe).

For each GLB_MISS_BIN_LOG2 value (0 = misses in relabel order, k = ordered by
2^k-byte bins of the host matrix; 21 = 2 MB pages), one library context on the
same generated graph: PreSC#K, load_cache(alpha), then `--steps` pipelined
steps (depth 2) and the same at depth 1, CUDA events around every extract.
Prints one JSON line per (setting, depth): extract ms, misses per step, host
GB/s = miss bytes / extract time, ms per step.

  python tools/miss_ab.py --config PA --alpha 0.22 --bins 21,0,16,12,9
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import synth  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="PA")
    ap.add_argument("--alpha", type=float, default=0.22)
    ap.add_argument("--bins", default="21,0,16,12,9")
    ap.add_argument("--steps", type=int, default=30)
    ap.add_argument("--env", default="", help="extra env k=v,k=v applied before each ctx")
    ap.add_argument("--hg", default="0", help="host-gather fractions in permille (glb_set_host_gather)")
    ap.add_argument("--hg-threads", type=int, default=0)
    args = ap.parse_args()
    import paper_conf_eurosys_yangtswycyz22_b200 as glb
    from paper_conf_eurosys_yangtswycyz22_b200 import parallel as par
    sh = synth.SHAPES[args.config]
    t0 = time.perf_counter()
    g = synth.make_graph(sh)
    print(json.dumps({"generate_s": time.perf_counter() - t0}), flush=True)
    for kv in filter(None, args.env.split(",")):
        k, v = kv.split("=")
        os.environ[k] = v
    for b, hg in [(int(x), int(y)) for x in args.bins.split(",") for y in args.hg.split(",")]:
        os.environ["GLB_MISS_BIN_LOG2"] = str(b)
        ctx = glb.Context(0)
        ctx.load_graph(g.indptr, g.indices, g.features)
        if g.weights is not None:
            ctx.load_edge_weights(g.weights)
        if sh.sampler in ("khop", "weighted"):
            ctx.set_sampler(sh.sampler, fanouts=sh.fanouts, max_batch=sh.batch)
        else:
            ctx.set_sampler("rwalk", layers=len(sh.fanouts), walks=synth.RW_WALKS,
                            walk_len=synth.RW_LEN, topk=sh.fanouts[0], max_batch=sh.batch)
        ctx.set_train_set(g.train, sh.batch, g.seed)
        nb = ctx.num_batches
        ctx.presample(sh.K)
        ctx.build_cache(args.alpha)
        if hg:
            ctx.set_host_gather(hg / 1000.0, threads=args.hg_threads)
        ub = sh.batch
        for k in sh.fanouts:
            ub = min(ub * (1 + k), sh.V)
        out = torch.empty((ub, sh.D), dtype=torch.float32, device="cuda")
        stream = torch.cuda.current_stream()
        for depth in (2, 1):
            ctx.set_pipeline(depth)
            xs = ctx.extract_stream() if depth == 2 else stream
            for i in range(5):
                e, bb = par.dp_step_batch(i, 0, 1, nb, sh.K)
                ctx.sample_batch(e, bb)
                ctx.extract_sample(out)
            ctx.sync()
            ctx.set_timing(1)
            s0 = torch.cuda.Event(enable_timing=True)
            s1 = torch.cuda.Event(enable_timing=True)
            s0.record(stream)
            for i in range(5, 5 + args.steps):
                e, bb = par.dp_step_batch(i, 0, 1, nb, sh.K)
                ctx.sample_batch(e, bb)
                ctx.extract_sample(out)
            s1.record(xs)
            torch.cuda.synchronize()
            xms = ctx.extract_times()
            ctx.set_timing(0)
            misses = []
            for i in range(5, 5 + args.steps):
                e, bb = par.dp_step_batch(i, 0, 1, nb, sh.K)
                ctx.sample_batch(e, bb)
                st = ctx.extract_sample(out, stats=True)
                misses.append(st["misses"])
            mb = [m * 4 * sh.D for m in misses]
            gbs = statistics.mean(b_ / (t * 1e-3) for b_, t in zip(mb, xms)) / 1e9
            print(json.dumps({"config": sh.name, "alpha": args.alpha, "miss_bin_log2": b,
                              "depth": depth, "ms_per_step": s0.elapsed_time(s1) / args.steps,
                              "extract_ms": statistics.mean(xms),
                              "misses_per_step": statistics.mean(misses),
                              "host_gbs": gbs, "env": args.env, "host_gather": ctx.host_gather}),
                  flush=True)
        ctx.close()
        del out
        torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
