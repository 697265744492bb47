"""One process per rank (all on one B200 here: CUDA IPC within the device stands in
for NVLink): apt_profile_links times every peer operator over the peers' mapped
tables (S13) instead of falling back to the pool's references.
Launched by tests/test_gpu_multiprocess.py under torchrun; rank 0 prints RESULT."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402
import torch.distributed as dist  # noqa: E402

import paper_conf_ppopp_mal0c0wlc25_b200.apt as A  # noqa: E402


def main():
    rank, world = int(os.environ["RANK"]), int(os.environ["WORLD_SIZE"])
    dev = int(os.environ.get("APT_TEST_DEVICE", os.environ.get("LOCAL_RANK", 0)))
    dist.init_process_group("gloo")
    torch.cuda.set_device(dev)
    errors = []
    ctx = A.Ctx(rank, world, dev)
    ctx.set_exchange(dist)
    bw = ctx.profile_links()
    for op in range(8):
        if bw.measured[op] != 1:
            errors.append(f"rank{rank}: op {op} not measured")
        if not (bw.beta_Bps[op] > 1e8 and bw.alpha_s[op] >= 0.0):
            errors.append(f"rank{rank}: op {op} alpha {bw.alpha_s[op]} beta {bw.beta_Bps[op]}")
    ctx.sync()
    ctx.close()
    allerr = [None] * world
    dist.all_gather_object(allerr, errors)
    if rank == 0:
        flat = [e for x in allerr for e in x]
        print("RESULT", "OK" if not flat else "FAIL " + "; ".join(flat[:20]), flush=True)
        print("BETAS_GBPS", [round(b / 1e9, 1) for b in bw.beta_Bps], "ALPHAS_US", [round(a * 1e6, 2) for a in bw.alpha_s])
    dist.destroy_process_group()


if __name__ == "__main__":
    main()
