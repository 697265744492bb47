"""Debug: GAT layer-1 gradients, bf16 vs f32 GPU vs oracle (scratch)."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tests"))
import numpy as np, torch, aptgen, oracle
from oracle import gat
import test_gpu_gat as T
import paper_conf_ppopp_mal0c0wlc25_b200.apt as A
cfg = aptgen.CONFIGS["tiny"]; g = aptgen.make_graph(cfg); train = aptgen.train_nodes(g, cfg)
torch.cuda.set_device(0)
res = {}
for dtype in ["f32", "bf16"]:
    ctx, part, tr, params, labels, dims, att = T._setup(A, cfg, g, train, "GDP", 1, dtype)
    tr.layer_fwd(0)
    perm = oracle.epoch_perm(train, cfg.sample_seed, 0)
    seeds = perm[:cfg.batch]
    blocks, blk, x, c, h_cmp, (a_s, a_d) = T._layer1_oracle(cfg, g, seeds, params, att, dims, True, dtype)
    rng = np.random.default_rng(1)
    n1, d1 = c["h"].shape
    dh = rng.normal(size=(n1, d1)).astype(np.float32)
    tr.layer_bwd([torch.as_tensor(dh).cuda()], d1)
    gpre = dh.astype(np.float64) * (c["pre"] > 0)
    gW, ga_s, ga_d, gb_ = gat.backward(blk.indptr, blk.indices, x, blk.n_dst, params[0][0], a_s, a_d, c, gpre, T.HEADS)
    res[dtype] = dict(dW=tr.read("dW", 1), db=tr.read("db", 1)[0], dA=tr.read("dA", 1)[0], G=tr.read("G", 1))
    print(dtype, "oracle |dW| max", np.abs(gW).max(), "gpu-oracle dW max", np.abs(res[dtype]["dW"] - gW).max(),
          "rel fro", np.linalg.norm(res[dtype]["dW"] - gW) / np.linalg.norm(gW))
    print(dtype, "db diff", np.abs(res[dtype]["db"] - gb_).max(), "da_src diff", np.abs(res[dtype]["dA"][:d1] - ga_s.reshape(-1)).max(),
          "|da_src|", np.abs(ga_s).max(), "da_dst diff", np.abs(res[dtype]["dA"][d1:] - ga_d.reshape(-1)).max())
    print(dtype, "G vs gpre", np.abs(res[dtype]["G"] - gpre).max())
    # split dW: projection part only (a = 0 contribution)  -- rows per head
    F = d1 // T.HEADS
    err = np.abs(res[dtype]["dW"] - gW)
    print(dtype, "per-head max err", [float(err[h*F:(h+1)*F].max()) for h in range(T.HEADS)])
print("bf16 vs f32 GPU dW max", np.abs(res["bf16"]["dW"] - res["f32"]["dW"]).max())
