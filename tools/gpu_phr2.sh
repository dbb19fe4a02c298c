#!/bin/bash
# phi_rpt = 2 (two tile rows per thread in the phi-sweep): GPU tests + A/B timing at 256^3
TAG=${1:-phr2}
OUT=gpurun_out/$TAG
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
i=0
for t in '{}' '{"phi_rpt": 2, "phi_ty": 8, "phi_minb": 3}' '{"phi_rpt": 2, "phi_ty": 4, "phi_minb": 6}' '{"phi_rpt": 2, "phi_ty": 8, "phi_minb": 4}' '{"phi_rpt": 2, "phi_ty": 4, "phi_minb": 5}' '{}' '{"phi_rpt": 2, "phi_ty": 8, "phi_minb": 3}'; do
  i=$((i+1))
  echo "$i: $t" >> $OUT/configs.txt
  timeout 300 python bench.py --steps 100 --warmup 5 --no-cpu-baseline --no-e2e --autotune 0 --tuning "$(python -c "import json,sys; d=json.loads(sys.argv[1]); d['mu_pfd']=3; print(json.dumps(d))" "$t")" > $OUT/bench_$i.json 2>> $OUT/bench.err
done
timeout 600 python -m pytest tests/test_gpu_autotune.py -x -q -k "corners" > $OUT/pytest.log 2>&1; echo "pytest exit $?" >> $OUT/pytest.log
echo done > $OUT/DONE
