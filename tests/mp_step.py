"""One process per rank, all on one B200 (CUDA IPC within the device stands in for
NVLink): a training step of every strategy through the multi-process path
(peer-mapped buffers, device barriers, peer all-reduce) against the oracle.
Launched by tests/test_gpu_multiprocess.py under torchrun; rank 0 prints RESULT."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402
import torch.distributed as dist  # noqa: E402

import aptgen  # noqa: E402
import oracle  # noqa: E402
from oracle import model  # noqa: E402
from oracle import strategy as S  # noqa: E402
import paper_conf_ppopp_mal0c0wlc25_b200.apt as A  # noqa: E402

sys.path.insert(0, os.path.join(ROOT, "tests"))
from parity_util import assert_close, reconcile, sum_bounds  # noqa: E402


def check(errors, tag, *args):
    try:
        assert_close(*args)
    except AssertionError as e:
        errors.append(f"{tag}: {str(e)[:300]}")


def main():
    rank, world = int(os.environ["RANK"]), int(os.environ["WORLD_SIZE"])
    dev = int(os.environ.get("APT_TEST_DEVICE", os.environ.get("LOCAL_RANK", 0)))
    dist.init_process_group("gloo")
    torch.cuda.set_device(dev)
    fanout_sets = [tuple(int(x) for x in f.split(",")) for f in (sys.argv[3] if len(sys.argv) > 3 else "5,5").split(";")]
    g = aptgen.make_graph(aptgen.CONFIGS["tiny"])
    train = aptgen.train_nodes(g, aptgen.CONFIGS["tiny"])
    labels = aptgen.labels(aptgen.CONFIGS["tiny"], g.n)
    part = aptgen.partition(g.n, world)
    errors = []
    for fanouts, dtype, strategy in [(f, d, s) for f in fanout_sets for d in sys.argv[1].split(",")
                                     for s in sys.argv[2].split(",")]:
        cfg = aptgen.CONFIGS["tiny"].replace(fanouts=fanouts)
        params = aptgen.weights(cfg)
        p64 = [(W.astype(np.float64), b.astype(np.float64)) for W, b in params]
        perm = oracle.epoch_perm(train, cfg.sample_seed, 0)
        if True:
            ctx = A.Ctx(rank, world, dev)
            ctx.set_exchange(dist)
            gr = ctx.graph_load(g.indptr, g.indices, part)
            dt = A.DTYPE[dtype]
            fs = ctx.fstore_create(gr, A.NFP if strategy == "NFP" else A.GDP, dt, cfg.dim, None, cfg.feat_seed)
            if strategy != "NFP":   # every row through this rank's view of the sharded store (peer shards via IPC)
                ids = np.arange(0, g.n, 7, dtype=np.int32)
                esz = 2 if dtype == "bf16" else 4
                pitch = (cfg.dim + 7) // 8 * 8 if dtype == "bf16" else (cfg.dim + 3) // 4 * 4
                buf = torch.zeros(len(ids) * pitch * esz, dtype=torch.uint8, device="cuda")
                torch.cuda.synchronize()            # torch's zero-fill runs on another stream than the library's
                ctx.gather(fs, torch.as_tensor(ids.astype(np.int64)).cuda(), len(ids), buf)
                torch.cuda.synchronize()
                raw = buf.cpu().numpy()
                if dtype == "bf16":
                    got = (raw.view(np.uint16).astype(np.uint32) << 16).view(np.float32).reshape(len(ids), pitch)
                else:
                    got = raw.view(np.float32).reshape(len(ids), pitch)
                ref = oracle.features(cfg.feat_seed, ids.astype(np.int64), cfg.dim)
                bad = ~(got[:, :cfg.dim] == ref).all(1)
                if bad.any():
                    errors.append(f"{strategy}/{dtype}/rank{rank}: store rows wrong: {int(bad.sum())} of {len(ids)}, "
                                  f"owners {np.bincount(part[ids[bad]], minlength=world).tolist()}")
            dims = [cfg.dim] + [d for _, d in cfg.dims()]
            tr = A.Trainer(ctx, gr, fs, dims, cfg.fanouts, cfg.batch, dt, 0.1, cfg.sample_seed, cfg.feat_seed,
                           A.STRATEGY[strategy], labels)
            tr.set_params(params)
            tr.set_epoch(train, 0)
            tr.use_graph(True)
            steps = min(2, tr.steps_per_epoch())
            for step in range(steps):
                tr.step(step, update=False)
                try:
                    ctx.sync()                      # device error word: a barrier timeout would show here
                except Exception as e:
                    errors.append(f"{strategy}/{dtype}/step{step}/rank{rank}: {e}")
                gb = oracle.global_batch(perm, step, world, cfg.batch)
                seeds = S.assign_seeds(strategy, gb, part, world, cfg.batch)
                K = len(cfg.fanouts)
                blocks = [oracle.sample_blocks(g, seeds[r], cfg.fanouts, cfg.sample_seed, step) for r in range(world)]
                refs = [model.train_step(blocks[r], cfg.feat_seed, cfg.dim, p64, labels[seeds[r]], len(gb), dtype,
                                         snp=(part, world) if strategy == "SNP" else None) for r in range(world)]
                # every rank's hidden activations (its ReLU mask bits, reading T3) to every process
                Hs = [None] * world
                dist.all_gather_object(Hs, [tr.read("H", l, rank=rank) for l in range(1, K)])
                bds = []
                for r in range(world):
                    refs[r], bd = reconcile(blocks[r], p64, refs[r], dtype, len(gb), Hs[r])
                    bds.append(bd)
                sb = sum_bounds(bds)
                tag = f"{strategy}/{dtype}/K{K}/step{step}/rank{rank}"
                if not np.array_equal(tr.read("seeds", rank=rank)[:, 0], seeds[rank]):
                    errors.append(f"{tag}: seeds")
                for l in range(1, K + 1):
                    check(errors, tag, tr.read("H", l, rank=rank), refs[rank]["cache"]["h"][l - 1], dtype, f"H{l}",
                          bds[rank]["H"][l - 1])
                for l in range(1, K + 1):
                    if strategy == "NFP" and l == 1:
                        continue   # column-owned: checked on the assembled slices below
                    check(errors, tag, tr.read("dW", l, rank=rank), sum(x["grads"][l - 1][0] for x in refs), dtype,
                          f"dW{l}", sb["dW"][l - 1])
                    check(errors, tag, tr.read("db", l, rank=rank)[0], sum(x["grads"][l - 1][1] for x in refs),
                          dtype, f"db{l}", sb["db"][l - 1])
                if strategy == "NFP":
                    lo, hi = S.col_range(rank, world, cfg.dim)
                    check(errors, tag, tr.read("dW", 1, rank=rank)[:, lo:hi],
                          sum(x["grads"][0][0] for x in refs)[:, lo:hi], dtype, "dW1 slice", sb["dW"][0][:, lo:hi])
            for h in (tr, fs, gr):
                h.close()
            ctx.close()
    allerr = [None] * world
    dist.all_gather_object(allerr, errors)
    if rank == 0:
        flat = [e for x in allerr for e in x]
        print("RESULT", "OK" if not flat else "FAIL " + "; ".join(flat[:20]), flush=True)
    dist.destroy_process_group()


if __name__ == "__main__":
    main()
