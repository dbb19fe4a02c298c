#!/bin/bash
# A/B of the committed tree (ab_head/, extracted by git archive) against the
# working tree on the same box: config-2 bench, default tuning, no auto-tuning.
# usage: bash tools/gpu_ab_tree.sh TAG [ENV=..]   (ENV applies to the working tree)
TAG=${1:-abtree}
OUT=$PWD/gpurun_out/$TAG
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
(cd ab_head && python -c "import __graft_entry__ as g; g.build()" > $OUT/build_head.log 2>&1)
for i in 1 2 3; do
  (cd ab_head && timeout 300 python bench.py --steps 100 --warmup 5 --no-cpu-baseline --no-e2e --autotune 0 > $OUT/head_$i.json 2>> $OUT/bench.err)
  env $2 timeout 300 python bench.py --steps 100 --warmup 5 --no-cpu-baseline --no-e2e --autotune 0 > $OUT/work_$i.json 2>> $OUT/bench.err
done
echo done > $OUT/DONE
