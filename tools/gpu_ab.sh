#!/bin/bash
# A/B of tuning knobs (env) on the bench
TAG=${1:-ab}
OUT=gpurun_out/$TAG
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
shift
i=0
for cfg in "$@"; do
  i=$((i+1))
  env $cfg timeout 300 python bench.py --steps 100 --warmup 5 --no-cpu-baseline --no-e2e > $OUT/bench_$i.json 2>> $OUT/bench.err
  echo "$i: $cfg" >> $OUT/configs.txt
done
echo done > $OUT/DONE
