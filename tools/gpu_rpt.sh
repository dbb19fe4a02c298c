#!/bin/bash
# mu_rpt = 2 (two tile rows per thread): GPU tests + A/B timing at 256^3
TAG=${1:-rpt}
OUT=gpurun_out/$TAG
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
i=0
for t in '{}' '{"mu_rpt": 2, "mu_ty": 8, "mu_minb": 2}' '{"mu_rpt": 2, "mu_ty": 6, "mu_minb": 3}' '{"mu_rpt": 2, "mu_ty": 8, "mu_minb": 2, "mu_rpf": 0}' '{}' '{"mu_rpt": 2, "mu_ty": 8, "mu_minb": 2}'; do
  i=$((i+1))
  echo "$i: $t" >> $OUT/configs.txt
  timeout 300 python bench.py --steps 100 --warmup 5 --no-cpu-baseline --no-e2e --autotune 0 --tuning "$t" > $OUT/bench_$i.json 2>> $OUT/bench.err
done
timeout 600 python -m pytest tests/test_gpu_autotune.py -x -q -k "corners or layouts" > $OUT/pytest.log 2>&1; echo "pytest exit $?" >> $OUT/pytest.log
echo done > $OUT/DONE
