#!/bin/bash
# NVLink evidence for the fused peer-memory collectives (GDP/DNP peer-row gathers, the
# Reshuffle's peer-store / peer-reduce epilogue, the work-list pushes, the gradient
# all-reduce) on a node with >= 2 NVLink-connected B200s.  ncu profiles ONE rank (rank 0)
# of a 2-rank job (the other rank runs unprofiled); per kernel launch it records the
# NVLink bytes received / transmitted (user data, 32-B granularity) next to the duration,
# so that achieved NVLink GB/s = (nvlrx + nvltx user bytes) / duration can be set against
# the 770 GB/s per-direction peer-copy reference (900 GB/s nominal).
#   tools/ncu_nvlink.sh <STRATEGY> [bench args...]        e.g. tools/ncu_nvlink.sh DNP
set -u
S=${1:-DNP}; shift || true
mkdir -p gpurun_out
cat > /tmp/apt_ncu_rank0.sh <<'INNER'
#!/bin/bash
if [ "${RANK:-0}" = "0" ]; then
  exec ncu --metrics gpu__time_duration.sum,nvlrx__bytes_data_user.sum,nvltx__bytes_data_user.sum \
       --clock-control none -k regex:'agg_l1|agg_kernel|rowtile|permute|gather_g|allreduce|resample' \
       --launch-skip 200 -c 60 --csv --log-file gpurun_out/nvlink_rank0.csv python "$@"
else
  exec python "$@"
fi
INNER
chmod +x /tmp/apt_ncu_rank0.sh
timeout 1200 python -m torch.distributed.run --nnodes=1 --nproc-per-node=2 --master-addr 127.0.0.1 \
  --master-port 29561 --no-python /tmp/apt_ncu_rank0.sh bench.py --gpus 2 --strategy "$S" --steps 5 --warmup 3 \
  --no-planner --no-cpu-baseline "$@" > gpurun_out/nvlink_job.log 2>&1
echo "rank-0 launch list with NVLink bytes: gpurun_out/nvlink_rank0.csv"
