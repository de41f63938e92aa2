"""How many distinct 2 MB regions of the host feature matrix does one batch's miss set touch,
with rows stored by gid (as generated) vs. by PreSC rank (cold rows in hotness order)?

  python tools/region_count.py --config PA --alpha 0.22 --batches 5
"""
from __future__ import annotations

import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

import synth  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="PA")
    ap.add_argument("--alpha", type=float, default=0.22)
    ap.add_argument("--batches", type=int, default=5)
    args = ap.parse_args()
    import paper_conf_eurosys_yangtswycyz22_b200 as glb
    sh = synth.SHAPES[args.config]
    g = synth.make_graph(sh, features=False)
    ctx = glb.Context(0)
    ctx.load_graph(g.indptr, g.indices, None)
    if sh.sampler in ("khop", "weighted"):
        ctx.set_sampler(sh.sampler, fanouts=sh.fanouts, max_batch=sh.batch)
    else:
        ctx.set_sampler("rwalk", layers=len(sh.fanouts), walks=synth.RW_WALKS,
                        walk_len=synth.RW_LEN, topk=sh.fanouts[0], max_batch=sh.batch)
    ctx.set_train_set(g.train, sh.batch, g.seed)
    ctx.presample(sh.K)
    counts = ctx.get_counts(glb.COUNT_PRESAMPLE)
    V = g.V
    order = np.lexsort((np.arange(V), -counts.astype(np.int64)))  # (count desc, gid asc)
    rank = np.empty(V, np.int64)
    rank[order] = np.arange(V)
    C = int(np.floor(args.alpha * V))
    rows_per_region = (2 << 20) // (4 * sh.D)
    for b in range(args.batches):
        ctx.sample_batch(sh.K, b)
        s = ctx.sample_result()
        u = s.uniq.cpu().numpy().view(np.uint32).astype(np.int64)
        miss = u[rank[u] >= C]
        by_gid = np.unique(miss // rows_per_region).size
        by_rank = np.unique((rank[miss] - C) // rows_per_region).size
        print(json.dumps({"batch": b, "misses": int(miss.size), "regions_gid_order": by_gid,
                          "regions_rank_order": by_rank,
                          "regions_total_cold": int((V - C + rows_per_region - 1) // rows_per_region)}),
              flush=True)


if __name__ == "__main__":
    main()
