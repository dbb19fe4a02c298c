#!/bin/bash
# A/B of tuning knobs (env) on the bench; optional parity tests per config (AB_TESTS=1)
TAG=${1:-ab}
OUT=gpurun_out/$TAG
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
shift
i=0
for cfg in "$@"; do
  i=$((i+1))
  echo "$i: $cfg" >> $OUT/configs.txt
  if [ -n "$AB_TESTS" ]; then
    env $cfg timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -x -q > $OUT/pytest_$i.log 2>&1
    echo "exit $?" >> $OUT/pytest_$i.log
  fi
  env $cfg timeout 300 python bench.py --steps 100 --warmup 5 --no-cpu-baseline --no-e2e > $OUT/bench_$i.json 2>> $OUT/bench.err
done
echo done > $OUT/DONE
