#!/bin/bash
# session s30 (round 2 re-entry): GPU suite, smoke, default bench line
OUT=gpurun_out/${1:-r02s30}
mkdir -p $OUT
nvidia-smi > $OUT/nvidia-smi.txt 2>&1
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
timeout 2400 python -m pytest tests -m gpu -q > $OUT/pytest_gpu.log 2>&1; echo "pytest exit $?" >> $OUT/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke.log 2>&1
timeout 900 python bench.py --steps 200 --warmup 10 > $OUT/bench.json 2> $OUT/bench.err
echo done > $OUT/DONE
