"""A plain PyTorch GraphSAGE consumer of the sample+extract path (the Train stage is an
unmodified torch consumer outside the hot path, BASELINE.json north_star).

Per mini-batch: glb_sample_batch -> per-hop blocks (CSR over local ids), glb_extract_sample ->
input features of every sampled vertex, then a 2-layer mean-aggregator GraphSAGE
(L353: "GraphSAGE ... 2 layers") forward + backward + SGD step in torch.

  python examples/train_sage.py [--config PR] [--steps 50] [--pipeline]

--pipeline: the Trainer's Extract/Train pipelining ("a pipelining mechanism
... to overlap the Extract and Train stages"): the library runs at depth 2
on its own stream, so batch b+1 is sampled and its features extracted (extract stream)
while torch trains on batch b; the sample slots are double-buffered (batch b's blocks stay
valid until batch b+2 is sampled) and so are the feature buffers.
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


def train(config="PR", steps=50, hidden=256, classes=47, pipeline=False, alpha=0.25, seed=0,
          log=print):
    """Train `steps` mini-batches; returns the per-step losses (floats) and the seconds."""
    g = synth.make_graph(config)
    sh = g.shape
    assert sh.sampler == "khop", "this example uses k-hop blocks"
    ctx = glb.Context(0)
    ctx.load_graph(g.indptr, g.indices, g.features)
    ctx.set_sampler("khop", fanouts=sh.fanouts, max_batch=sh.batch)
    ctx.set_train_set(g.train, sh.batch, g.seed)
    ctx.set_count_mode(glb.COUNT_PRESAMPLE)
    ctx.presample(1)                      # PreSC#1
    ctx.set_count_mode(glb.COUNT_NONE)
    ctx.build_cache(alpha)
    L = len(sh.fanouts)
    dims = [sh.D] + [hidden] * (L - 1) + [classes]
    torch.manual_seed(seed)
    layers = torch.nn.ModuleList(SageLayer(dims[i], dims[i + 1]) for i in range(L)).cuda()
    opt = torch.optim.SGD(layers.parameters(), lr=0.01)
    labels = torch.randint(0, classes, (sh.V,), device="cuda")  # synthetic labels
    nb = ctx.num_batches
    ub = sh.batch
    for k in sh.fanouts:
        ub = min(ub * (1 + k), sh.V)
    train_stream = torch.cuda.current_stream()
    if pipeline:
        ctx.set_pipeline(2)
        side = torch.cuda.Stream()
        ctx.set_stream(side)  # sample_result syncs this stream only, never the training
        xs = ctx.extract_stream()
    feats = [torch.empty((ub, sh.D), device="cuda") for _ in range(2)]

    def fetch(step):
        """Sample + extract mini-batch `step` (asynchronous extract at depth 2)."""
        e, b = 1 + step // nb, step % nb
        if pipeline:  # the sample slot and feature buffer of step-2 are free once the
            side.wait_stream(train_stream)  # training enqueued so far has run
        ctx.sample_batch(e, b)
        blk = ctx.sample_result()  # sizes (syncs the sampler's stream)
        h = feats[step % 2]
        ctx.extract_sample(h)
        ev = None
        if pipeline:
            ev = torch.cuda.Event()
            ev.record(xs)
        return blk, h, ev

    losses = []
    t0 = time.perf_counter()
    nxt = fetch(0)
    for step in range(steps):
        blk, h, ev = nxt
        if pipeline and step + 1 < steps:
            nxt = fetch(step + 1)  # overlaps the training of `step` below
        if ev is not None:
            train_stream.wait_event(ev)
        h = h[: blk.sizes[-1]]
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
        losses.append(loss.detach())
        if not pipeline and step + 1 < steps:
            nxt = fetch(step + 1)
        if log and step % 10 == 0:
            log(f"step {step}: loss {loss.item():.4f}")
    torch.cuda.synchronize()
    secs = time.perf_counter() - t0
    ctx.close()
    return [float(x) for x in losses], secs


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="PR")
    ap.add_argument("--steps", type=int, default=50)
    ap.add_argument("--hidden", type=int, default=256)
    ap.add_argument("--classes", type=int, default=47)
    ap.add_argument("--pipeline", action="store_true")
    args = ap.parse_args()
    _, secs = train(args.config, args.steps, args.hidden, args.classes, args.pipeline)
    print(f"{args.steps} steps in {secs:.2f} s (pipeline={args.pipeline})")


if __name__ == "__main__":
    main()
