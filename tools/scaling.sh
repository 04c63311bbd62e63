#!/bin/bash
# Multi-GPU runs on one node (needs N GPUs): the default bench c3 (256 frames
# split over the ranks, strong), c2 (weak replicas) and c4 (row stripes,
# strong; the line times both the in-kernel peer halos and the NCCL exchange).
# Usage: bash tools/scaling.sh [max_gpus]
mkdir -p gpurun_out
MAX=${1:-8}
for n in 1 2 4 8; do
  [ $n -gt $MAX ] && break
  for wl in c3 c2 c4; do
    if [ $n -eq 1 ]; then
      timeout 900 python bench.py --workload $wl --steps 20 --warmup 3 --no-cpu-baseline > gpurun_out/scale_${wl}_n$n.json 2> gpurun_out/scale_${wl}_n$n.err
    else
      timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node $n --master-addr 127.0.0.1 \
        --master-port $((29600 + n)) bench.py --gpus $n --workload $wl --steps 20 --warmup 3 \
        > gpurun_out/scale_${wl}_n$n.json 2> gpurun_out/scale_${wl}_n$n.err
    fi
    echo "$wl n=$n rc=$? $(python -c "import json; d=json.load(open('gpurun_out/scale_${wl}_n$n.json')); print(round(d['value']), d['scaling'], round(d['ms_per_step'], 4))" 2>/dev/null)"
  done
done
