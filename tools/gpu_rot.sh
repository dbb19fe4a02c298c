#!/bin/bash
# A/B of the mu-sweep row rotation (mu_rot) at 256^3 + its GPU tests
TAG=${1:-rot}
OUT=gpurun_out/$TAG
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
i=0
for t in '{}' '{"mu_rot": 1}' '{}' '{"mu_rot": 1}'; do
  i=$((i+1))
  echo "$i: $t" >> $OUT/configs.txt
  timeout 300 python bench.py --steps 100 --warmup 5 --no-cpu-baseline --no-e2e --autotune 0 --tuning "$t" > $OUT/bench_$i.json 2>> $OUT/bench.err
done
timeout 600 python -m pytest tests/test_gpu_autotune.py -x -q -k "corners" > $OUT/pytest.log 2>&1; echo "pytest exit $?" >> $OUT/pytest.log
echo done > $OUT/DONE
