#!/bin/bash
# quick GPU iteration: tests, bench (tuned + naive), optional ncu of the tuned kernels
TAG=${1:-quick}
OUT=gpurun_out/$TAG
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
timeout 900 python -m pytest tests -m gpu -x -q > $OUT/pytest_gpu.log 2>&1; echo "pytest exit $?" >> $OUT/pytest_gpu.log
timeout 300 python bench.py --steps 100 --warmup 5 --no-cpu-baseline --no-e2e --autotune 0 > $OUT/bench.json 2> $OUT/bench.err
timeout 300 python bench.py --steps 50 --warmup 5 --no-cpu-baseline --no-e2e --variant tuned > $OUT/bench_tuned.json 2>> $OUT/bench.err
if [ "$2" == "ncu" ]; then
timeout 900 ncu --set full --clock-control none --import-source on -k regex:pf_jit_mu -s 3 -c 1 -o $OUT/prof_mu \
   python bench.py --steps 4 --warmup 3 --no-cpu-baseline --no-e2e --autotune 0 > $OUT/ncu_mu.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:pf_jit_phi -s 3 -c 1 -o $OUT/prof_phi \
   python bench.py --steps 4 --warmup 3 --no-cpu-baseline --no-e2e --autotune 0 > $OUT/ncu_phi.log 2>&1
fi

if [ "$3" == "launches" ]; then
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches.csv \
   python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-e2e --autotune 0 > $OUT/ncu_launch.log 2>&1
fi
echo done > $OUT/DONE
