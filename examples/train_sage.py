"""A plain PyTorch GraphSAGE consumer of the sample+extract path (the Train stage is an
unmodified torch consumer outside the hot path, BASELINE.json north_star).

Per mini-batch: glb_sample_batch -> per-hop blocks (CSR over local ids), glb_extract_sample ->
input features of every sampled vertex, then a 2-layer mean-aggregator GraphSAGE
(L353: "GraphSAGE ... 2 layers") forward + backward + SGD step in torch.

  python examples/train_sage.py [--config PR] [--steps 50]
"""
import argparse
import os
import sys
import time

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_eurosys_yangtswycyz22_b200 as glb  # noqa: E402
import synth  # noqa: E402


class SageLayer(torch.nn.Module):
    def __init__(self, d_in, d_out):
        super().__init__()
        self.self_w = torch.nn.Linear(d_in, d_out)
        self.neigh_w = torch.nn.Linear(d_in, d_out, bias=False)

    def forward(self, h_src, indptr, indices, n_dst):
        # mean over each dst vertex's sampled in-neighbours (block CSR: dst -> src lids)
        deg = (indptr[1:] - indptr[:-1]).clamp(min=1).unsqueeze(1).to(h_src.dtype)
        dst = torch.repeat_interleave(torch.arange(n_dst, device=h_src.device),
                                      indptr[1:] - indptr[:-1])
        agg = torch.zeros((n_dst, h_src.shape[1]), device=h_src.device, dtype=h_src.dtype)
        agg.index_add_(0, dst, h_src[indices.long()])
        return self.self_w(h_src[:n_dst]) + self.neigh_w(agg / deg)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="PR")
    ap.add_argument("--steps", type=int, default=50)
    ap.add_argument("--hidden", type=int, default=256)
    ap.add_argument("--classes", type=int, default=47)
    args = ap.parse_args()
    g = synth.make_graph(args.config)
    sh = g.shape
    assert sh.sampler == "khop", "this example uses k-hop blocks"
    ctx = glb.Context(0)
    ctx.load_graph(g.indptr, g.indices, g.features)
    ctx.set_sampler("khop", fanouts=sh.fanouts, max_batch=sh.batch)
    ctx.set_train_set(g.train, sh.batch, g.seed)
    ctx.set_count_mode(glb.COUNT_PRESAMPLE)
    ctx.presample(1)                      # PreSC#1
    ctx.set_count_mode(glb.COUNT_NONE)
    ctx.build_cache(0.25)
    L = len(sh.fanouts)
    dims = [sh.D] + [args.hidden] * (L - 1) + [args.classes]
    layers = torch.nn.ModuleList(SageLayer(dims[i], dims[i + 1]) for i in range(L)).cuda()
    opt = torch.optim.SGD(layers.parameters(), lr=0.01)
    labels = torch.randint(0, args.classes, (sh.V,), device="cuda")  # synthetic labels
    nb = ctx.num_batches
    t0 = time.perf_counter()
    for step in range(args.steps):
        e, b = 1 + step // nb, step % nb
        ctx.sample_batch(e, b)
        blk = ctx.sample_result()
        h = torch.empty((blk.sizes[-1], sh.D), device="cuda")
        ctx.extract_sample(h)
        # the deepest block first: block l maps frontier l+1 (src) onto frontier l (dst)
        for l in reversed(range(L)):
            h = layers[L - 1 - l](h[: blk.sizes[l + 1]], blk.indptr[l].long(), blk.indices[l],
                                  blk.sizes[l])
            if l:
                h = torch.relu(h)
        loss = torch.nn.functional.cross_entropy(h, labels[blk.uniq[: blk.sizes[0]].long()])
        opt.zero_grad()
        loss.backward()
        opt.step()
        if step % 10 == 0:
            print(f"step {step}: loss {loss.item():.4f}")
    torch.cuda.synchronize()
    print(f"{args.steps} steps in {time.perf_counter() - t0:.2f} s")


if __name__ == "__main__":
    main()
