#!/bin/bash
# session s54: final round-2 evidence (with the p2.ds bench sub-line) -- GPU suite, smoke, bench (config 2 with all lines; config 4),
# ncu launch list, ncu --set full of the P1 sweeps and of the specialised P2 sweeps
TAG=${1:-r02s54}
OUT=gpurun_out/$TAG
mkdir -p $OUT
nvidia-smi > $OUT/nvidia-smi.txt 2>&1
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
timeout 2400 python -m pytest tests -m gpu -q > $OUT/pytest_gpu.log 2>&1; echo "pytest exit $?" >> $OUT/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke.log 2>&1
timeout 900 python bench.py --steps 200 --warmup 10 > $OUT/bench.json 2> $OUT/bench.err
timeout 900 python bench.py --config strong --steps 20 --warmup 3 --no-cpu-baseline --autotune 1 > $OUT/bench_strong.json 2>> $OUT/bench.err
TUNE=$(python -c "import json; print(json.dumps(json.load(open('$OUT/bench.json'))['config']['tuning']))" 2>/dev/null || echo '{}')
echo "$TUNE" > $OUT/tuning.json
export PF_BENCH_ALLOW_SHORT=1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches.csv \
   python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-e2e --no-stress --no-p2 --autotune 0 --tuning "$TUNE" > $OUT/ncu_launch.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:pf_jit_mu -s 3 -c 1 -o $OUT/prof_mu \
   python bench.py --steps 4 --warmup 3 --no-cpu-baseline --no-e2e --no-stress --no-p2 --autotune 0 --tuning "$TUNE" > $OUT/ncu_mu.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:pf_jit_phi -s 3 -c 1 -o $OUT/prof_phi \
   python bench.py --steps 4 --warmup 3 --no-cpu-baseline --no-e2e --no-stress --no-p2 --autotune 0 --tuning "$TUNE" > $OUT/ncu_phi.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:pf_p2_jit -s 2 -c 2 -o $OUT/prof_p2jit \
   python tools/p2_run.py 256 4 > $OUT/ncu_p2jit.log 2>&1
echo done > $OUT/DONE
