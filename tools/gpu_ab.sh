#!/bin/bash
# A/B of tuning knobs: bench lines for each PF_MU_TY
TAG=${1:-ab}
OUT=gpurun_out/$TAG
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
for t in 2 4 8; do
  PF_MU_TY=$t timeout 300 python bench.py --steps 100 --warmup 5 --no-cpu-baseline --no-e2e > $OUT/bench_muty$t.json 2>> $OUT/bench.err
done
echo done > $OUT/DONE
