#!/bin/bash
# session s24: phi x-ghost columns written by the phi-sweep (phi_xghost) A/B;
# bench with the stress set auto-tuned
OUT=gpurun_out/${1:-r02s24}
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
for i in 1 2; do
  for t in '{"phi_xghost": 0}' '{"phi_xghost": 1}'; do
    echo "$t" >> $OUT/ab.jsonl
    timeout 300 python bench.py --steps 100 --warmup 5 --no-cpu-baseline --no-e2e --no-stress --no-p2 --autotune 0 --tuning "$t" >> $OUT/ab.jsonl 2>> $OUT/bench.err
  done
done
timeout 900 python bench.py --steps 100 --warmup 5 --no-cpu-baseline --no-e2e --no-p2 > $OUT/bench_stress.json 2>> $OUT/bench.err
echo done > $OUT/DONE
