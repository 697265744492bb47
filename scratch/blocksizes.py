"""Print per-hop block sizes of the products-shape workload (scratch; not a test)."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch, aptgen, oracle
import paper_conf_ppopp_mal0c0wlc25_b200.apt as A
cfg = aptgen.CONFIGS[sys.argv[1] if len(sys.argv) > 1 else "products"]
g = aptgen.make_graph(cfg)
train = aptgen.train_nodes(g, cfg)
torch.cuda.set_device(0)
ctx = A.Ctx(0, 1, 0)
gr = ctx.graph_load(g.indptr, g.indices)
perm = oracle.epoch_perm(train, cfg.sample_seed, 0)
for step in range(3):
    seeds = torch.as_tensor(perm[step * cfg.batch:(step + 1) * cfg.batch]).cuda()
    b = ctx.sample(gr, seeds, len(seeds), cfg.fanouts, cfg.sample_seed, step)
    for h in range(len(cfg.fanouts)):
        v = b.block(h)
        print(f"step {step} hop {h}: n_dst {v.n_dst} n_src {v.n_src} n_edges {v.n_edges}")
    b.close()
