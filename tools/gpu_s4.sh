#!/bin/bash
# session r02 s4: GPU suite (multi-block, aux, sanitizer), fp64 micro with clocks, bench (growing DS), DS tuning
OUT=gpurun_out/r02s4
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
timeout 2400 python -m pytest tests -m gpu -q > $OUT/pytest_gpu.log 2>&1; echo "exit $?" >> $OUT/pytest_gpu.log
nvidia-smi --query-gpu=index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active --format=csv -lms 100 > $OUT/fp64_clocks.csv &
SMI=$!
timeout 120 tools/build/fp64_micro > $OUT/fp64_micro.json 2>&1
kill $SMI
timeout 900 python bench.py --steps 200 --warmup 10 > $OUT/bench.json 2> $OUT/bench.err
timeout 1200 python tools/ds_tune.py --steps 20000 --check 2000 --vs 0.02,0.03 --Gs 0.02 --zf 0.49 > $OUT/ds_tune.jsonl 2> $OUT/ds_tune.err
echo done > $OUT/DONE
