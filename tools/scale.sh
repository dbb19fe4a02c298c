#!/bin/bash
# Scaling runs of BASELINE.json configs 3 and 4 and the Table-2 analog
# (overlap of the halo exchange with the interior mu tiles on / off,
# P:L1519-1544) on one node with N GPUs (one process per GPU, NCCL over
# NVLink).  Each line of gpurun_out/scale/ is the bench JSON of one run; the
# driver's own SCALE run uses `bench.py --gpus N` (config 3 weak scaling).
#   bash tools/scale.sh [max_gpus=8]
MAX=${1:-8}
OUT=gpurun_out/scale
mkdir -p $OUT
run() {  # n, tag, extra env, extra args
  local n=$1 tag=$2 envs=$3; shift 3
  if [ "$n" == 1 ]; then
    env $envs timeout 1200 python bench.py --gpus 1 "$@" > $OUT/${tag}_n1.json 2> $OUT/${tag}_n1.err
  else
    env $envs timeout 1200 python -m torch.distributed.run --nnodes=1 --nproc-per-node $n --master-addr 127.0.0.1 \
      --master-port $((29500 + n)) bench.py --gpus $n "$@" > $OUT/${tag}_n$n.json 2> $OUT/${tag}_n$n.err
  fi
}
for n in 1 2 4 8; do
  [ $n -le $MAX ] || continue
  # config 3: 256^3 block per GPU, weak scaling (blocks tile x-y, growth axis unsplit)
  run $n weak "" --steps 200 --warmup 10 --no-cpu-baseline
  # config 4: fixed 512 x 512 x 1024 periodic domain in z-slabs, strong scaling
  run $n strong "" --config strong --steps 20 --warmup 3 --no-cpu-baseline --autotune 1
  # Table-2 analog: the halo exchange serialised with the sweeps
  [ $n -gt 1 ] && run $n weak_nooverlap "PF_OVERLAP=0" --steps 200 --warmup 10 --no-cpu-baseline --no-e2e --autotune 0
done
echo done > $OUT/DONE
