#!/bin/bash
# cluster-mode mu-sweep: GPU tests of the knob + A/B timing at 256^3
TAG=${1:-cly}
OUT=gpurun_out/$TAG
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
timeout 600 python -m pytest tests/test_gpu_autotune.py -x -q -k "cluster or corners" > $OUT/pytest.log 2>&1; echo "pytest exit $?" >> $OUT/pytest.log
i=0
for t in '{}' '{"mu_cly": 2}' '{"mu_cly": 4}' '{}' '{"mu_cly": 2}' '{"mu_cly": 4}'; do
  i=$((i+1))
  echo "$i: $t" >> $OUT/configs.txt
  timeout 300 python bench.py --steps 100 --warmup 5 --no-cpu-baseline --no-e2e --autotune 0 --tuning "$t" > $OUT/bench_$i.json 2>> $OUT/bench.err
done
echo done > $OUT/DONE
