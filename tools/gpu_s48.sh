#!/bin/bash
# session s48: why is the mu-sweep 656 us in the ncu launch list but 820 us in the bench?
OUT=gpurun_out/${1:-r02s48}
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
export PF_BENCH_ALLOW_SHORT=1
TUNE=$(cat profiles/r02_tuning.json)
for st in 10 50 200; do
  timeout 300 python bench.py --steps $st --warmup 3 --no-cpu-baseline --no-e2e --no-stress --no-p2 --autotune 0 --tuning "$TUNE" > $OUT/b_$st.json 2>> $OUT/bench.err
  python -c "import json; r=json.loads(open('$OUT/b_$st.json').read().strip().splitlines()[-1]); print('steps $st', round(r['value']), round(r['ms_per_step'],4), 'mu', round(r['kernels']['mu_sweep_ms'],4), 'phi', round(r['kernels']['phi_sweep_ms'],4), r['clocks'])" >> $OUT/summary.txt
done
timeout 600 ncu --metrics gpu__time_duration.sum,sm__cycles_elapsed.avg.per_second --clock-control none --csv --log-file $OUT/launches_nocache.csv --cache-control none \
   python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-e2e --no-stress --no-p2 --autotune 0 --tuning "$TUNE" > $OUT/ncu1.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum,sm__cycles_elapsed.avg.per_second --clock-control none --csv --log-file $OUT/launches_cache.csv \
   python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-e2e --no-stress --no-p2 --autotune 0 --tuning "$TUNE" > $OUT/ncu2.log 2>&1
echo done > $OUT/DONE
