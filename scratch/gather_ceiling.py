import sys, numpy as np, torch
sys.path.insert(0, '/root/repo')
import aptgen, paper_conf_ppopp_mal0c0wlc25_b200.apt as A
cfg = aptgen.CONFIGS['products']
g = aptgen.make_graph(cfg)
ctx = A.Ctx(0, 1, 0)
gr = ctx.graph_load(g.indptr, g.indices)
fs = ctx.fstore_create(gr, A.GDP, A.BF16, cfg.dim, None, cfg.feat_seed)
rng = np.random.default_rng(0)
for n, uniq in ((482000, False), (217000, True), (482000, True)):
    if uniq:
        ids = rng.choice(g.n, size=n, replace=False).astype(np.int32)
    else:
        ids = rng.integers(0, g.n, size=n).astype(np.int32)
    idd = torch.as_tensor(ids).cuda()
    out = torch.empty(n * 104 * 2, dtype=torch.uint8, device='cuda')
    flush = torch.empty(256 << 20, dtype=torch.uint8, device='cuda')
    ts = []
    for it in range(8):
        flush.zero_(); torch.cuda.synchronize()
        e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
        e0.record(); ctx.gather(fs, idd, n, out); e1.record(); torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1))
    t = min(ts[2:]) * 1e-3
    print(f"gather n={n} uniq={uniq}: {t*1e6:.1f} us, {n*208/t/1e9:.0f} GB/s of rows read (+ same written)")
