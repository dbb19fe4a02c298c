#!/bin/bash
# A/B of explicit pf_tuning settings on the config-2 bench (no auto-tuning).
# usage: bash tools/gpu_ab_tuning.sh TAG '{json}' '{json}' ...
TAG=${1:-abt}
OUT=gpurun_out/$TAG
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
shift
i=0
for t in "$@"; do
  i=$((i+1))
  echo "$i: $t" >> $OUT/configs.txt
  timeout 300 python bench.py --steps 100 --warmup 5 --no-cpu-baseline --no-e2e --autotune 0 --tuning "$t" > $OUT/bench_$i.json 2>> $OUT/bench.err
done
echo done > $OUT/DONE
