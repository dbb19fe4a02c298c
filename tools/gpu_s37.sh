#!/bin/bash
# session s37: mu_hasync default -- P1 GPU parity / autotune / fullsize / multiblock suites, bench
OUT=gpurun_out/${1:-r02s37}
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
timeout 2000 python -m pytest tests/test_gpu_parity.py tests/test_gpu_autotune.py tests/test_gpu_fullsize.py tests/test_gpu_multiblock.py tests/test_gpu_aux.py -m gpu -q > $OUT/pytest.log 2>&1; echo "exit $?" >> $OUT/pytest.log
timeout 900 python bench.py --steps 200 --warmup 10 --no-cpu-baseline --no-p2 > $OUT/bench.json 2> $OUT/bench.err
echo done > $OUT/DONE
