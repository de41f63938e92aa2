"""A/B of library environment knobs on one generated graph (one process, one graph).

Each variant is a set of environment variables applied before a fresh library context is
created (the library reads its GLB_* knobs at glb_create): PreSC#K, load_cache(alpha),
then `--steps` pipelined steps (depth 2) timed with CUDA events, every extract timed.
Prints one JSON line per variant: ms per step, extract ms, misses, host GB/s.

  python tools/ab_env.py --config TW --alpha 1.0 \
      --variants "base:;dedup:GLB_RELABEL_DEDUP=1"
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
    ap.add_argument("--config", default="PR")
    ap.add_argument("--alpha", type=float, default=1.0)
    ap.add_argument("--variants", required=True, help="name:K=V,K=V;name2:...")
    ap.add_argument("--steps", type=int, default=60)
    ap.add_argument("--repeat", type=int, default=2, help="rounds over all variants")
    ap.add_argument("--host-gather", type=float, default=0.0)
    ap.add_argument("--relabel", default="auto")
    ap.add_argument("--depths", default="2", help="pipeline depths to time, e.g. 2,1")
    args = ap.parse_args()
    import paper_conf_eurosys_yangtswycyz22_b200 as glb
    from paper_conf_eurosys_yangtswycyz22_b200 import parallel as par
    sh = synth.SHAPES[args.config]
    t0 = time.perf_counter()
    g = synth.make_graph(sh)
    print(json.dumps({"generate_s": time.perf_counter() - t0}), flush=True)
    variants = []
    for v in filter(None, args.variants.split(";")):
        name, _, kv = v.partition(":")
        variants.append((name, dict(x.split("=") for x in filter(None, kv.split(",")))))
    keys = {k for _, env in variants for k in env}
    for rnd in range(args.repeat):
        for name, env in variants:
            for k in keys:
                os.environ.pop(k, None)
            os.environ.update(env)
            ctx = glb.Context(0)
            ctx.load_graph(g.indptr, g.indices, g.features)
            ctx.set_relabel_mode(args.relabel)
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
            if args.host_gather:
                ctx.set_host_gather(args.host_gather)
            ub = sh.batch
            for k in sh.fanouts:
                ub = min(ub * (1 + k), sh.V)
            out = torch.empty((ub, sh.D), dtype=torch.float32, device="cuda")
            stream = torch.cuda.current_stream()
            for depth in [int(x) for x in args.depths.split(",")]:
                ctx.set_pipeline(depth)
                xs = ctx.extract_stream() if depth == 2 else stream
                for i in range(5):
                    e, b = par.dp_step_batch(i, 0, 1, nb, sh.K)
                    ctx.sample_batch(e, b)
                    ctx.extract_sample(out)
                ctx.sync()
                ctx.set_timing(1)
                s0 = torch.cuda.Event(enable_timing=True)
                s1 = torch.cuda.Event(enable_timing=True)
                s0.record(stream)
                for i in range(5, 5 + args.steps):
                    e, b = par.dp_step_batch(i, 0, 1, nb, sh.K)
                    ctx.sample_batch(e, b)
                    ctx.extract_sample(out)
                s1.record(xs)
                torch.cuda.synchronize()
                xms = ctx.extract_times()
                ctx.set_timing(0)
                misses = []
                for i in range(5, 5 + min(args.steps, 10)):
                    e, b = par.dp_step_batch(i, 0, 1, nb, sh.K)
                    ctx.sample_batch(e, b)
                    misses.append(ctx.extract_sample(out, stats=True)["misses"])
                m = statistics.mean(misses)
                print(json.dumps({"config": sh.name, "alpha": args.alpha, "variant": name, "env": env,
                                  "round": rnd, "depth": depth, "ms_per_step": s0.elapsed_time(s1) / args.steps,
                                  "extract_ms": statistics.mean(xms), "misses_per_step": m,
                                  "host_gbs": m * 4 * sh.D / (statistics.mean(xms) * 1e-3) / 1e9}),
                      flush=True)
            ctx.close()
            del out
            torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
