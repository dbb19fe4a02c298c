#!/bin/bash
# Auto-tuning session (NEXT-2): GPU tests, then bench with pf_autotune on the
# config-2 block and on the config-4 domain.  usage: bash tools/gpu_tune.sh [tag]
TAG=${1:-tune}
OUT=gpurun_out/$TAG
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_autotune.py tests/test_gpu_parity.py -m gpu -x -q > $OUT/pytest_gpu.log 2>&1; echo "pytest exit $?" >> $OUT/pytest_gpu.log
timeout 600 python bench.py --steps 100 --warmup 5 --no-cpu-baseline --no-e2e > $OUT/bench_default.json 2> $OUT/bench.err
timeout 900 python bench.py --steps 100 --warmup 5 --no-cpu-baseline --no-e2e --autotune 2 > $OUT/bench_autotune.json 2>> $OUT/bench.err
timeout 900 python bench.py --config strong --steps 10 --warmup 3 --no-cpu-baseline --autotune 1 > $OUT/bench_strong_autotune.json 2>> $OUT/bench.err
echo done > $OUT/DONE
