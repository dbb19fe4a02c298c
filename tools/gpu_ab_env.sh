#!/bin/bash
# A/B of environment settings on the config-2 bench (default tuning, no auto-tuning)
# usage: bash tools/gpu_ab_env.sh TAG 'ENV=..' 'ENV=..' ...   ('-' = no extra environment)
TAG=${1:-abe}
OUT=gpurun_out/$TAG
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
shift
i=0
for e in "$@"; do
  i=$((i+1))
  echo "$i: $e" >> $OUT/configs.txt
  if [ "$e" == "-" ]; then e=""; fi
  env $e timeout 300 python bench.py --steps 100 --warmup 5 --no-cpu-baseline --no-e2e --autotune 0 --tuning '{}' > $OUT/bench_$i.json 2>> $OUT/bench.err
done
echo done > $OUT/DONE
