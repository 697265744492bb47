"""bench.py -- seeds/s of APT's per-mini-batch sampled-subgraph step on B200.

Contract (task statement + SURVEY.md §8(d)):
  python bench.py --gpus N --steps K --warmup W [--impl apt|reference]
One step = one pass of the whole hot path over one global batch: seed selection
(S1), 3-hop Philox sampling + compaction (S2/S3), the layer-1 strategy forward
(S4-S9: fused gather + mean, tcgen05 projection), upper layers + CE loss (S10),
backward (S10/S11), gradient all-reduce + SGD.  All of it runs in libapt.so's
sm_100a kernels, replayed as one CUDA graph per step.

Workload (BASELINE.json configs[1]): synthetic ogbn-products shape, R-MAT
2.4M nodes / 62M undirected edges, d=100 (bf16 rows padded to 104), GraphSAGE
100->256->256->47, fanout [10,10,10], B=1024 seeds per GPU.

value      = seeds/s of the whole job (C*B seeds per step / max-over-ranks step time)
e2e        = the same through apt_trainer_step_host (host batch in, host loss out)
roofline   = the dominant kernel (layer-1 fused gather + mean, HBM bound)
cpu_baseline = the oracle (oracle/, single thread) on the first steps of the
               same epoch, rank 0 at N=1 only.
--impl reference: the oracle itself, timed on the host cores (this tier has no
installable reference implementation; its reference arm is the oracle).
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

import aptgen  # noqa: E402

METRIC = "seeds/s"
STRATS = ("GDP", "NFP", "SNP", "DNP")


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=100)
    ap.add_argument("--warmup", type=int, default=20)
    ap.add_argument("--impl", default="apt", choices=["apt", "reference"])
    ap.add_argument("--config", default="products", choices=sorted(aptgen.CONFIGS))
    ap.add_argument("--strategy", default="GDP", choices=list(STRATS))
    ap.add_argument("--dtype", default="bf16", choices=["bf16", "f32"])
    ap.add_argument("--no-graph", action="store_true", help="eager launches instead of CUDA-graph replay")
    ap.add_argument("--no-pipeline", action="store_true",
                    help="sample each step inside it instead of overlapping the next step's sampling (A/B)")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--cpu-steps", type=int, default=3, help="oracle steps for cpu_baseline")
    ap.add_argument("--e2e-steps", type=int, default=50)
    ap.add_argument("--no-planner", action="store_true")
    ap.add_argument("--flush", default="write+read", choices=["write", "write+read"],
                    help="L2 flush between timed steps: a 256 MB write, then (default) a 256 MB read so the "
                         "write's dirty lines reach DRAM before the step (both outside the events)")
    ap.add_argument("--dryrun-steps", type=int, default=0, help="dry-run steps (0: one full epoch, P:142)")
    ap.add_argument("--emulate-max-c", type=int, default=4,
                    help="also time every strategy with C ranks emulated on the GPU, for C up to this")
    ap.add_argument("--verbose", action="store_true")
    ap.add_argument("--gat-heads", type=int, default=0,
                    help="layer 1 as a GAT layer with this many heads (BASELINE config 5; 0: GraphSAGE-mean)")
    ap.add_argument("--feat-dim", type=int, default=0, help="override the config's input dim d (sweeps)")
    ap.add_argument("--hidden", type=int, default=0, help="override the config's hidden dim d' (sweeps)")
    ap.add_argument("--fanouts", default="", help="override the fanouts, e.g. 15,10 (layer 1 first; NEXT #4 sweep)")
    ap.add_argument("--partition", default="range", choices=["range", "random", "ldg"],
                    help="edge-cut partition for SNP/DNP and the store's row sharding (apt_partition; NEXT #3)")
    return ap.parse_args()


def dist_env():
    return int(os.environ.get("RANK", 0)), int(os.environ.get("WORLD_SIZE", 1)), int(os.environ.get("LOCAL_RANK", 0))


GAT_HEADS = 0   # set from --gat-heads
PARTITION = "range"   # set from --partition
_PART_CACHE = {}


def partition(A, g, C):
    """The job's edge-cut partition into C parts (apt_partition, the library's host
    partitioner; "range" is the generator's planted partition)."""
    return _partition(A, g, C)[0]


def _partition(A, g, C):
    key = (id(g), C, PARTITION)
    if key not in _PART_CACHE:
        _PART_CACHE[key] = A.partition(g.indptr, g.indices, C, PARTITION, seed=7) if C > 1 else \
            (np.zeros(g.n, np.int32), 0)
    return _PART_CACHE[key]


def workload_config(cfg):
    dims = "->".join(str(d) for d in [cfg.dim] + [o for _, o in cfg.dims()])
    return {"workload": f"synthetic ogbn-{cfg.name} shape (R-MAT {cfg.n} nodes / {cfg.m} undirected edges)"
            if cfg.name != "tiny" else f"tiny R-MAT {cfg.n} nodes / {cfg.m} edges",
            "model": (f"GAT layer 1 ({GAT_HEADS} heads) + GraphSAGE-mean upper layers " + dims) if GAT_HEADS
            else "GraphSAGE-mean " + dims,
            "fanouts": list(cfg.fanouts), "batch_per_gpu": cfg.batch, "feat_dim": cfg.dim}


# --------------------------------------------------------------------- clocks
class ClockSampler:
    """nvidia-smi clocks + throttle reasons sampled during the timed region."""
    Q = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.hw_slowdown,"
         "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
         "clocks_event_reasons.sw_power_cap")

    def __init__(self, index):
        self.index, self.rows, self.stop_ev = index, [], threading.Event()

    def _run(self):
        while not self.stop_ev.is_set():
            try:
                out = subprocess.run(["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.Q}",
                                      "--format=csv,noheader,nounits"], capture_output=True, text=True,
                                     timeout=5).stdout.strip()
                if out:
                    self.rows.append([x.strip() for x in out.split(",")])
            except Exception:
                pass
            self.stop_ev.wait(0.1)

    def __enter__(self):
        self.th = threading.Thread(target=self._run, daemon=True)
        self.th.start()
        return self

    def __exit__(self, *a):
        self.stop_ev.set()
        self.th.join(timeout=10)

    def summary(self):
        if not self.rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"], "samples": 0}
        sm = [float(r[0]) for r in self.rows if r[0].replace(".", "").isdigit()]
        mx = [float(r[1]) for r in self.rows if r[1].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for r in self.rows for i in range(4) if len(r) > 3 + i and r[3 + i] == "Active"})
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": reasons, "samples": len(self.rows)}


# --------------------------------------------------------------------- oracle legs
def oracle_steps(cfg, g, train, labels, n_steps, world=1):
    """Time the oracle (test infrastructure, single thread) on the first n_steps
    global steps of epoch 0: sampling + compaction + fp64 SAGE fwd/bwd."""
    from threadpoolctl import threadpool_limits

    import oracle
    from oracle import model
    params = [(W.astype(np.float64), b.astype(np.float64)) for W, b in aptgen.weights(cfg)]
    perm = oracle.epoch_perm(train, cfg.sample_seed, 0)
    B = world * cfg.batch
    times, seeds_done = [], 0
    with threadpool_limits(limits=1):
        for t in range(n_steps):
            seeds = perm[t * B:(t + 1) * B]
            t0 = time.perf_counter()
            blocks = oracle.sample_blocks(g, seeds, cfg.fanouts, cfg.sample_seed, t)
            if GAT_HEADS:
                gat_oracle_step(cfg, blocks, params, labels[seeds], len(seeds))
            else:
                model.train_step(blocks, cfg.feat_seed, cfg.dim, params, labels[seeds], len(seeds), "bf16")
            times.append(time.perf_counter() - t0)
            seeds_done += len(seeds)
    return times, seeds_done


def host_cpu():
    """The box's host CPU model and core count (the oracle baseline's machine)."""
    model = "unknown"
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                model = line.split(":", 1)[1].strip()
                break
    except OSError:
        pass
    return {"model": model, "nproc": os.cpu_count()}


def gat_oracle_step(cfg, blocks, params, labels_s, n_global):
    """The oracle's step with a GAT first layer (oracle/gat.py, fp64) and SAGE-mean upper
    layers: forward, CE loss, backward of every layer (test infrastructure timed as a baseline)."""
    import oracle
    from oracle import gat, model
    K = len(blocks)
    blk = blocks[K - 1]
    x = oracle.features(cfg.feat_seed, blk.src, cfg.dim)
    W1, b1 = params[0]
    F = W1.shape[0] // GAT_HEADS
    rng = np.random.default_rng(cfg.weight_seed + 100)
    a_s = (rng.normal(size=W1.shape[0]) * 0.3).reshape(GAT_HEADS, F)
    a_d = (rng.normal(size=W1.shape[0]) * 0.3).reshape(GAT_HEADS, F)
    c = gat.forward(blk.indptr, blk.indices, x, blk.n_dst, W1, a_s, a_d, b1, GAT_HEADS, relu=K > 1)
    Hs, pres = [c["h"]], [c["pre"]]
    for l in range(2, K + 1):
        b2 = blocks[K - l]
        W, b = params[l - 1]
        pre = oracle.aggregate(b2.indptr, b2.indices, Hs[-1]) @ W.T + b
        pres.append(pre)
        Hs.append(np.maximum(pre, 0.0) if l < K else pre)
    _, gl = model.ce_loss_grad(Hs[-1], labels_s, n_global)
    for l in range(K, 1, -1):
        b2 = blocks[K - l]
        W, _ = params[l - 1]
        dH = oracle.aggregate_bwd(b2.indptr, b2.indices, gl @ W, b2.n_src)
        gl = dH * (pres[l - 2] > 0)
    gat.backward(blk.indptr, blk.indices, x, blk.n_dst, W1, a_s, a_d, c, gl, GAT_HEADS)


def run_reference(args, cfg):
    rank, world, _ = dist_env()
    if rank != 0:
        return 0
    g = aptgen.make_graph(cfg)
    train = aptgen.train_nodes(g, cfg)
    labels = aptgen.labels(cfg, g.n)
    n = args.warmup + args.steps
    times, _ = oracle_steps(cfg, g, train, labels, n, args.gpus)
    timed = times[args.warmup:]
    B = args.gpus * cfg.batch
    ms = 1e3 * sum(timed) / len(timed)
    value = B / (ms / 1e3)
    sample = (f"{args.steps} timed global steps of epoch 0 after {args.warmup} warm-up, {B} seeds each, "
              f"full fanout {list(cfg.fanouts)} sampling + fp64 SAGE fwd/bwd, one host thread")
    line = {"impl": "reference", "metric": METRIC, "value": value, "unit": "seeds/s", "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": workload_config(cfg),
            "cpu_baseline": {"value": value, "unit": "seeds/s", "cores": 1, "kind": "oracle", "sample": sample,
                             "host": host_cpu()},
            "e2e": {"value": value, "unit": "seeds/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)
    return 0


# --------------------------------------------------------------------- product leg
def run_apt(args, cfg):
    import torch
    import torch.distributed as dist

    import paper_conf_ppopp_mal0c0wlc25_b200.apt as A

    rank, world, local = dist_env()
    if world != args.gpus:
        raise SystemExit(f"--gpus {args.gpus} but WORLD_SIZE={world}")
    # APT_DEVICE_OVERRIDE: plumbing test with several ranks on one GPU (numbers then meaningless)
    local = int(os.environ.get("APT_DEVICE_OVERRIDE", local))
    torch.cuda.set_device(local)
    if world > 1:
        if "APT_DEVICE_OVERRIDE" in os.environ:   # NCCL refuses two ranks on one GPU
            dist.init_process_group("gloo")
        else:
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    # one non-default stream shared by torch (events, L2 flush) and the library
    # high priority: the library's sampling stream (next step's batch) runs at default
    # priority and fills the gaps the compute chain leaves
    stream = torch.cuda.Stream(priority=-1)
    torch.cuda.set_stream(stream)
    A.lib()   # fails loudly if libapt.so is missing: there is no CPU path

    g = aptgen.make_graph(cfg)
    train = aptgen.train_nodes(g, cfg)
    labels = aptgen.labels(cfg, g.n)
    part = partition(A, g, world)
    dt = A.DTYPE[args.dtype]
    ctx = A.Ctx(rank if world > 1 else 0, world, local, stream.cuda_stream)
    if world > 1:
        ctx.set_exchange(dist)   # CUDA-IPC peer mappings + device barrier (bootstrap only)
    gr = ctx.graph_load(g.indptr, g.indices, part)
    strat = A.STRATEGY[args.strategy]
    fs = ctx.fstore_create(gr, strat if strat == A.NFP else A.GDP, dt, cfg.dim, None, cfg.feat_seed)
    tr = make_trainer(A, ctx, gr, fs, cfg, dt, strat, labels)
    tr.set_params(aptgen.weights(cfg))
    tr.set_epoch(train, 0)
    tr.use_graph(not args.no_graph)
    if args.no_pipeline:
        tr.set_pipeline(False)
    spe = tr.steps_per_epoch()

    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")   # 256 MB > 126 MB L2
    # the read pass evicts the zeroed (dirty) lines, so the step starts on a cold L2 of clean
    # foreign lines instead of paying the flush's own write-backs (~126 MB) inside its timed region
    flush_rd = torch.ones(64 << 20, dtype=torch.int32, device="cuda") if args.flush == "write+read" else None
    flush_out = torch.empty((), dtype=torch.int32, device="cuda")
    for i in range(args.warmup):
        tr.step(i % spe)
    torch.cuda.synchronize()

    K = args.steps
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(K)]
    agg_ms, phases, step_ids, agg_bytes, step_bytes = [], [], [], [], []
    bf = 2 if args.dtype == "bf16" else 4
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    l0 = ctx.launches()
    with ClockSampler(local) as clk:
        for i in range(K):
            s = (args.warmup + i) % spe
            flush.zero_()                      # L2 flushed between timed steps (outside the events)
            if flush_rd is not None:
                torch.amax(flush_rd, dim=0, out=flush_out)
            ev[i][0].record(stream)
            tr.step(s)
            ev[i][1].record(stream)
            ph = tr.phase_ms()                 # syncs; device time inside the step comes from events
            phases.append(ph)
            agg_ms.append(ph[5])
            step_ids.append(s)
            agg_bytes.append(layer1_bytes(ctx, gr, tr, cfg, rank, s, bf))   # outside the events
            if i < 5 and not GAT_HEADS:
                step_bytes.append(step_phase_bytes(ctx, gr, g, tr, cfg, rank, s, bf))
        torch.cuda.synchronize()
    launches = ctx.launches() - l0
    if world > 1:
        dist.barrier()
    step_ms = [a.elapsed_time(b) for a, b in ev]
    ms_local = sum(step_ms) / K
    ms = ms_local
    if world > 1:
        tt = torch.tensor([ms_local], device="cuda")
        dist.all_reduce(tt, op=dist.ReduceOp.MAX)
        ms = float(tt.item())
    value = world * cfg.batch / (ms / 1e3)
    pct = {f"p{q}": float(np.percentile(step_ms, q)) for q in (10, 50, 90)}

    # ---- one full epoch, timed as a whole (validates epoch = steps x step time);
    # all steps of epoch 0 back to back through the pipelined graph, no L2 flush in between
    epoch_measured = None
    if spe <= 4096:
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()
        ee0, ee1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        ee0.record(stream)
        for s_ in range(spe):
            tr.step(s_)
        ee1.record(stream)
        torch.cuda.synchronize()
        epoch_measured = ee0.elapsed_time(ee1) / 1e3
        if world > 1:
            tt = torch.tensor([epoch_measured], device="cuda")
            dist.all_reduce(tt, op=dist.ReduceOp.MAX)
            epoch_measured = float(tt.item())

    # ---- e2e: host global batches in (pinned), host losses out, through the public
    # pipelined call apt_trainer_step_host_pipelined (submit batch t+1, run batch t): each
    # timed call copies one batch in, runs one step, copies one loss out
    rng = np.random.default_rng(1234)
    host_perm = rng.permutation(train)
    B = world * cfg.batch
    e2e_times, h2d = [], 0
    tr.use_graph(not args.no_graph)
    n_calls = args.warmup + args.e2e_steps + 1
    batches = [torch.as_tensor(host_perm[(i * B) % (len(host_perm) - B):][:B].copy()).pin_memory()
               for i in range(n_calls)]
    # apt_trainer_step_host_async: each call writes the next batch, launches its step
    # (H2D of the batch, the step, D2H of the loss) and returns the previous step's loss, so
    # the device always has a step queued; the timed region is the wall clock of the timed
    # calls (every one copies a batch in and a loss out), closed by apt_trainer_loss
    for i in range(args.warmup + 1):
        tr.step_host_async(batches[i], i % spe)
    if world > 1:
        dist.barrier()
    tr.loss()                                 # drains the warm-up calls
    t0 = time.perf_counter()
    for i in range(args.warmup + 1, n_calls):
        tr.step_host_async(batches[i], i % spe)
    tr.loss()                                 # the last launched step's loss (syncs)
    t1 = time.perf_counter()
    e2e_times = [(t1 - t0) / max(1, n_calls - args.warmup - 1)]
    h2d = 4 * (1 + B)                         # pinned staging [n, ids] as int32 (ids converted on the host)
    e2e_s = sum(e2e_times) / len(e2e_times)
    if world > 1:
        tt = torch.tensor([e2e_s], device="cuda")
        dist.all_reduce(tt, op=dist.ReduceOp.MAX)
        e2e_s = float(tt.item())

    peaks = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json"))) if os.path.exists(
        os.path.join(ROOT, "MEASURED_PEAKS.json")) else None
    hbm_peak = peaks["hbm_gbs"] if peaks else 6650.0
    # with the pipeline (GDP, SAGE) the layer-1 gather+mean timed inside step i belongs to
    # the NEXT batch (the sampling branch aggregates it, trainer z_prefetch): pair its time
    # with the bytes of step i+1 (consecutive steps only)
    if not args.no_pipeline and not GAT_HEADS and args.strategy == "GDP" and os.environ.get("APT_Z_PREFETCH", "0") != "0":
        pairs = [(agg_ms[i], agg_bytes[i + 1]) for i in range(len(agg_ms) - 1) if step_ids[i + 1] == step_ids[i] + 1]
        agg_ms, agg_bytes = [p_[0] for p_ in pairs], [p_[1] for p_ in pairs]
    achieved = sum(agg_bytes) / (sum(agg_ms) * 1e-3) / 1e9
    # DRAM traffic of the same kernel from one committed `ncu --set full` capture of this
    # workload (dram__bytes_read + dram__bytes_write per launch), next to the algorithmic bytes
    traffic, traffic_src = None, None
    tpath = os.path.join(ROOT, "profiles", "r02_ncu_agg_l1_traffic.json")
    if not GAT_HEADS and args.dtype == "bf16" and cfg.name == "products" and cfg.fanouts == (10, 10, 10) \
            and os.path.exists(tpath):
        tj = json.load(open(tpath))
        traffic, traffic_src = tj["traffic_bytes_per_launch"], tj["source"]
    mean_agg = sum(agg_ms) / len(agg_ms)
    phase_mean = [sum(p[j] for p in phases) / len(phases) for j in range(6)]

    out = {
        "metric": METRIC, "value": value, "unit": "seeds/s", "n_gpus": world, "steps": K, "warmup": args.warmup,
        "ms_per_step": ms, "higher_is_better": True, "scaling": "weak", "vs_baseline": None,
        "dtype": args.dtype, "data": "synthetic",
        "epoch_s": spe * ms / 1e3, "steps_per_epoch": spe, "epoch_s_measured": epoch_measured,
        "ms_per_step_pct": pct,
        "config": dict(workload_config(cfg), strategy=args.strategy, parallelism=f"{args.strategy.lower()}{world}",
                       global_batch=B, l2=("flushed between timed steps (256 MB write, then a 256 MB read that "
                                           "writes the flush's dirty lines back; outside the events); inputs also > L2"
                                           if args.flush == "write+read" else
                                           "flushed between timed steps (256 MB write); inputs also > L2"),
                       cuda_graph=not args.no_graph, pipelined_sampling=not args.no_pipeline),
        "e2e": {"value": B / e2e_s, "unit": "seeds/s", "h2d_bytes_per_step": h2d, "d2h_bytes_per_step": 4,
                "timing": "host wall clock over the timed apt_trainer_step_host_async calls (each: next batch H2D, one "
                          "step, its loss D2H; the previous step's loss returned) closed by a syncing loss read, "
                          "max over ranks"},
        "gpu_launches": int(launches),
        "roofline": {"bound": "hbm", "achieved": achieved, "peak": hbm_peak, "unit": "GB/s",
                     "frac": (achieved / hbm_peak) if achieved else None, "traffic": traffic,
                     "traffic_source": traffic_src, "algorithmic_bytes_per_launch": sum(agg_bytes) / len(agg_bytes),
                     "kernel": "gat_fwd_kernel (layer-1 fused gather+attention+weighted sums)" if GAT_HEADS
                     else "agg_l1_flat_kernel (layer-1 fused gather+mean)",
                     "peak_source": "MEASURED_PEAKS.json hbm_gbs" if peaks else "fallback 6.65 TB/s",
                     "share_of_step": mean_agg / ms_local,
                     # context, not the peak: random 208-B row reads measured alone on one B200
                     # (tools/micro/gather_ceiling.cu, steady state over a 10x table)
                     "random_row_ceiling": {"gbs": RANDOM_ROW_CEILING_GBS, "frac": achieved / RANDOM_ROW_CEILING_GBS,
                                            "source": "profiles/r02_gather_ceiling.txt"}
                     if not GAT_HEADS and achieved else None},
        "step_roofline": step_roofline(step_bytes, hbm_peak, ms) if step_bytes else None,
        "phases_ms": {"sample": phase_mean[0], "layer1_fwd": phase_mean[1], "upper_fwd_loss": phase_mean[2],
                      "backward": phase_mean[3], "allreduce_sgd": phase_mean[4], "agg_kernel": phase_mean[5]},
        "clocks": clk.summary(),
    }
    if rank == 0 and world == 1 and not args.no_planner:
        out["planner"] = planner_report(A, g, cfg, train, labels, args, stream, ms_local)
        # the workload's access skew next to the paper's Table 3 (reading R12)
        n_acc = spe   # one whole epoch (the paper ranks nodes over training; a prefix undercounts the tail)
        counts0 = tr.access_counts(n_acc)
        # "the top-1% nodes of two epochs overlap by 94.77%": the same statistic here
        tr.set_epoch(train, 1)
        counts1 = tr.access_counts(n_acc)
        tr.set_epoch(train, 0)
        k1 = max(1, g.n // 100)
        top0 = np.argsort(-counts0.astype(np.int64), kind="stable")[:k1]
        top1 = np.argsort(-counts1.astype(np.int64), kind="stable")[:k1]
        out["planner"]["epoch_top1pct_overlap"] = len(np.intersect1d(top0, top1)) / k1
        out["planner"]["dryrun_vs_epoch"] = {
            f"C{C}": {"dryrun_wall_s": out["planner"][f"C{C}"]["dryrun_wall_s"], "epoch_s_measured_C1": epoch_measured,
                      "note": "paper P:279: 25 s dry-run vs 449 s of GDP training (T4s)"} for C in (2, 4, 8)}
        out["access_skew"] = {"steps": n_acc, "buckets": ["<1%", "1-5%", "5-10%", "10-20%", "20-50%", "50-100%"],
                              "table": skew_table(counts0),
                              "paper_table3": {"PS": [0.501, 0.348, 0.088, 0.047, 0.017, 0.0],
                                               "FS": [0.177, 0.294, 0.191, 0.188, 0.135, 0.016]}}
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        times, nseeds = oracle_steps(cfg, g, train, labels, args.cpu_steps, 1)
        out["cpu_baseline"] = {"value": nseeds / sum(times), "unit": "seeds/s", "cores": 1, "kind": "oracle",
                               "host": host_cpu(),
                               "sample": f"first {args.cpu_steps} steps of epoch 0 ({cfg.batch} seeds each, "
                                         f"full step: sampling + fp64 {'GAT layer 1 + ' if GAT_HEADS else ''}SAGE "
                                         f"fwd/bwd), one host thread"}
    if rank == 0:
        print(json.dumps(out), flush=True)
    if world > 1:
        dist.destroy_process_group()
    return 0


def planner_report(A, g, cfg, train, labels, args, stream, gdp_ms):
    """APT's Planner on this workload: link trials, then for C = 2, 4, 8 a dry-run
    of every strategy over the first steps of the epoch (all C ranks' blocks counted on this
    GPU: sampling is a pure function of (seed, node, hop, step)) and Eq. 2's prediction per
    strategy + the pick.  Predictions only for C > 1: this run has one GPU, so no C > 1 step
    is measured; at C = 1 every strategy is the measured GDP step."""
    dt = A.DTYPE[args.dtype]
    rep = {"note": "pred = T_build + T_load + T_shuffle per step (max over ranks), common T_train excluded; "
                   "NVLink betas are the pool's measured references (no peer GPU in this run)"}
    for C in (2, 4, 8):
        ctx = A.Ctx(-1, C, 0, stream.cuda_stream)
        gr = ctx.graph_load(g.indptr, g.indices, partition(A, g, C))
        fs = ctx.fstore_create(gr, A.GDP, dt, cfg.dim, None, cfg.feat_seed)
        tr = make_trainer(A, ctx, gr, fs, cfg, dt, A.GDP, labels)
        tr.set_epoch(train, 0)
        st = tr.dryrun(args.dryrun_steps or tr.steps_per_epoch())
        bw = ctx.profile_links()
        pick, pred = A.select_strategy(st, bw)
        steps = max(1, st.steps)
        rep[f"C{C}"] = {"dryrun_steps": st.steps, "dryrun_wall_s": st.t_dryrun_s,
                        "steps_per_epoch": tr.steps_per_epoch(),
                        "t_build_ms_per_step": {s: 1e3 * max(st.t_build_s[i][r] for r in range(C)) / steps
                                                for i, s in enumerate(STRATS)},
                        "t_resample_ms_per_step": {s: 1e3 * max(st.t_resample_s[i][r] for r in range(C)) / steps
                                                   for i, s in enumerate(STRATS)},
                        "pred_ms_per_step": {s: 1e3 * p / steps for s, p in zip(STRATS, pred)},
                        "partition": PARTITION, "edge_cut_frac": _partition(A, g, C)[1] / max(1, g.nnz),
                        "pick": STRATS[pick],
                        "n_vs_per_step": sum(st.n_vs[r] for r in range(C)) / steps,
                        "n_vd_per_step": sum(st.n_vd[r] for r in range(C)) / steps}
        if C <= args.emulate_max_c:
            em = emulated_strategy_times(A, g, cfg, train, labels, C, dt, stream)
            fastest = min(em, key=em.get)
            rep[f"C{C}"]["emulated_ms_per_step"] = em
            rep[f"C{C}"]["emulated_fastest"] = fastest
            # the pick's slowdown vs the measured fastest, on the emulated job (target <= 1.10)
            rep[f"C{C}"]["pick_slowdown_vs_fastest_emulated"] = em[STRATS[pick]] / em[fastest]
        if C == 2:
            rep["bw_profile"] = {"local_gather_GBps": bw.beta_Bps[0] / 1e9, "local_gather_alpha_us": bw.alpha_s[0] * 1e6,
                                 "host_read_GBps": bw.beta_Bps[7] / 1e9, "measured": list(bw.measured)}
        for h in (tr, fs, gr):
            h.close()
        ctx.close()
    # C = 1: every strategy through its own driver (identity exchanges), timed
    em1 = emulated_strategy_times(A, g, cfg, train, labels, 1, dt, stream)
    rep["C1"] = {"measured_ms_per_step": em1, "bench_gdp_ms_per_step": gdp_ms, "pick": "GDP",
                 "fastest": min(em1, key=em1.get),
                 "note": "at C = 1 every strategy degenerates to GDP's arithmetic; each ran through its own "
                         "driver (5 steps, CUDA graph, no L2 flush); GDP is also the timed bench step"}
    return rep


def emulated_strategy_times(A, g, cfg, train, labels, C, dt, stream, steps=5):
    """Every strategy's full step with all C ranks emulated on this one GPU (rank = -1: the
    same kernels, "peer" buffers local): evidence that all four strategies run on device at
    this scale.  The C ranks time-share one GPU and no byte crosses NVLink, so these are not
    C-GPU step times (the Planner's predictions above are)."""
    import torch
    out = {}
    for s in STRATS:
        ctx = A.Ctx(-1, C, 0, stream.cuda_stream) if C > 1 else A.Ctx(0, 1, 0, stream.cuda_stream)
        gr = ctx.graph_load(g.indptr, g.indices, partition(A, g, C))
        fs = ctx.fstore_create(gr, A.NFP if s == "NFP" else A.GDP, dt, cfg.dim, None, cfg.feat_seed)
        tr = make_trainer(A, ctx, gr, fs, cfg, dt, A.STRATEGY[s], labels)
        tr.set_params(aptgen.weights(cfg))
        tr.set_epoch(train, 0)
        tr.use_graph(True)
        for i in range(3):
            tr.step(i)
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        for i in range(3, 3 + steps):
            tr.step(i)
        e1.record(stream)
        torch.cuda.synchronize()
        out[s] = e0.elapsed_time(e1) / steps
        for h in (tr, fs, gr):
            h.close()
        ctx.close()
    return out


def layer1_bytes(ctx, gr, tr, cfg, rank, step, bf):
    """Algorithmic bytes of the layer-1 fused gather+mean launch of `step`:
    cnt N_d*4 + neighbour ids E_1*4 + unique source rows U*d*b_f + Z write N_d*d*b_z, with
    N_d, E_1, U from apt_sample on the same seeds and step (bit-identical blocks by O2/O3)."""
    import torch
    seeds = torch.as_tensor(tr.read("seeds", rank=rank)[:, 0].astype(np.int64)).cuda()
    b = ctx.sample(gr, seeds, len(seeds), cfg.fanouts, cfg.sample_seed, step)
    v = b.block(len(cfg.fanouts) - 1)
    n = v.n_dst * 4 + v.n_edges * 4 + v.n_src * cfg.dim * bf + v.n_dst * cfg.dim * bf
    if GAT_HEADS:   # GAT: per-head Z rows and the per-edge scores kept for the backward
        n += v.n_dst * cfg.dim * bf * (GAT_HEADS - 1) + v.n_edges * GAT_HEADS * 4
    b.close()
    return n


def skew_table(counts, edges=(0.01, 0.05, 0.10, 0.20, 0.50, 1.0)):
    """Table 3's layout: nodes ranked by access count, share of all accesses
    per rank bucket."""
    c = np.sort(np.asarray(counts, np.int64))[::-1]
    total = max(1, int(c.sum()))
    out, lo = [], 0
    for e in edges:
        hi = int(round(e * len(c)))
        out.append(float(c[lo:hi].sum()) / total)
        lo = hi
    return out


def step_phase_bytes(ctx, gr, g, tr, cfg, rank, step, bf):
    """Algorithmic HBM bytes of one whole GDP step at C = 1, per phase (SURVEY §8(d)'s
    per-phase table), every tensor counted at the width the path stores
    it: bf16 mode keeps Z, the hidden activations (R11), the backward's G (R4) and
    dZ / deg (R13) and the weights' copies in bf16, the logits and their gradient in
    fp32; fp32 mode keeps everything in fp32.  Phases: sampling (indptr sector +
    neighbour sectors + writes), compaction (+ the block transposes of the upper hops),
    the layer-1 gather of unique rows + mean, every projection, the upper layers'
    means, loss, backward (dZ = G W, the mean's backward reading the mask and writing
    G, every dW = G^T Z) and SGD.  Block sizes come from apt_sample on the same seeds
    and step."""
    seeds_h = tr.read("seeds", rank=rank)[:, 0].astype(np.int64)
    import torch
    seeds = torch.as_tensor(seeds_h).cuda()
    K = len(cfg.fanouts)
    b = ctx.sample(gr, seeds, len(seeds), cfg.fanouts, cfg.sample_seed, step)
    dims = [cfg.dim] + [o for _, o in cfg.dims()]
    half = bf == 2
    b_z = b_w = 2 if half else 4      # Z, bf16 weight copies (tensor-core operands)
    b_h = 2 if half else 4            # hidden activations as stored (R11)
    b_g = 2 if half else 4            # G read by the contractions / written by the pull (R4)
    b_dz = 2 if half else 4           # dZ / deg rows (R13)
    ph = {"sampling": 0, "compaction": 0, "layer1_gather_mean": 0, "projections": 0, "upper_means": 0,
          "loss": 0, "backward": 0, "sgd": 0}
    for h in range(K):
        dst, src, indptr, _ = b.block_host(h)
        k = cfg.fanouts[K - 1 - h]
        deg = (g.indptr[dst.astype(np.int64) + 1] - g.indptr[dst.astype(np.int64)]).astype(np.int64)
        nb = np.where(deg <= k, (4 * deg + 31) // 32 * 32, k * 32)
        E = int(indptr[-1]) if len(indptr) else 0
        N, U = len(dst), len(src)
        layer = K - h
        din, dout = dims[layer - 1], dims[layer]
        ph["sampling"] += N * 32 + int(nb.sum()) + N * k * 8
        ph["compaction"] += E * 12 + U * 8 + (E * 12 if layer > 1 else 0)     # + block transpose
        if layer == 1:
            ph["layer1_gather_mean"] += U * din * bf + E * 4 + (N + 1) * 4 + N * din * b_z
            ph["backward"] += N * (dout * b_g + din * b_z)                      # dW1 = G^T Z
        else:
            ph["upper_means"] += U * din * b_h + E * 4 + (N + 1) * 4 + N * din * b_z
            ph["backward"] += (N * dout * b_g + din * dout * b_w + N * din * b_dz   # dZ = (G W) / deg
                               + N * din * b_dz + E * 8 + U * din * b_h            # pull: dZ, (v, deg), mask
                               + U * din * b_g                                     # ... writes G_{l-1}
                               + N * (dout * b_g + din * b_z))                      # dW = G^T Z
        b_out = 4 if layer == K else b_h                                            # logits fp32
        ph["projections"] += N * din * b_z + N * dout * b_out + din * dout * b_w
        if layer == K:
            ph["loss"] += N * dout * 4 + N * dout * (4 + (2 if half else 0))        # logits -> G (+ bf16 copy)
    nparam = sum(dims[i] * dims[i + 1] + dims[i + 1] for i in range(K))
    ph["sgd"] = nparam * (4 + 4 + 4 + b_w)
    b.close()
    return ph


RANDOM_ROW_CEILING_GBS = 3505.0   # x10 uniq_sorted / uniq_random, unroll 8, bpsm 4 (profiles/r02_gather_ceiling.txt)


def step_roofline(step_bytes, peak_gbs, ms):
    """T_roof / T_meas of the whole step: T_roof = the step's algorithmic
    HBM bytes / the measured HBM peak (every phase HBM-bound at C = 1, no NVLink)."""
    keys = step_bytes[0].keys()
    mean = {k: sum(s[k] for s in step_bytes) / len(step_bytes) for k in keys}
    total = sum(mean.values())
    t_roof_ms = total / (peak_gbs * 1e9) * 1e3
    return {"bound": "hbm", "bytes_per_step": total, "bytes_by_phase": mean, "peak_gbs": peak_gbs,
            "t_roof_ms": t_roof_ms, "t_meas_ms": ms, "frac": t_roof_ms / ms,
            "note": "T_roof = algorithmic bytes (SURVEY 8(d) table, sector-granular random reads, "
                    "unique rows once) / measured HBM peak; mean over the first timed steps"}


def make_trainer(A, ctx, gr, fs, cfg, dt, strat, labels, lr=0.05):
    """The product's trainer for this workload (GAT layer 1 when --gat-heads > 0)."""
    dims = [cfg.dim] + [d for _, d in cfg.dims()]
    tr = A.Trainer(ctx, gr, fs, dims, cfg.fanouts, cfg.batch, dt, lr, cfg.sample_seed, cfg.feat_seed, strat, labels,
                   gat_heads=GAT_HEADS)
    if GAT_HEADS:
        rng = np.random.default_rng(cfg.weight_seed + 100)
        tr.set_attention((rng.normal(size=dims[1]) * 0.3).astype(np.float32),
                         (rng.normal(size=dims[1]) * 0.3).astype(np.float32))
    return tr


def main():
    global GAT_HEADS
    args = parse()
    cfg = aptgen.CONFIGS[args.config]
    GAT_HEADS = args.gat_heads
    global PARTITION
    PARTITION = args.partition
    over = {}
    if args.feat_dim:
        over["dim"] = args.feat_dim
    if args.hidden:
        over["hidden"] = args.hidden
    if args.fanouts:
        over["fanouts"] = tuple(int(x) for x in args.fanouts.split(","))
    if over:
        cfg = cfg.replace(**over)
    if args.impl == "reference":
        return run_reference(args, cfg)
    return run_apt(args, cfg)


if __name__ == "__main__":
    sys.exit(main())
