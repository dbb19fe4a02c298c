#!/bin/bash
# session s31: P2 run-time specialisation -- P2 GPU tests, P2 bench line (jit vs generic), ncu of the P2 jit sweeps
OUT=gpurun_out/${1:-r02s31}
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
timeout 1500 python -m pytest tests/test_gpu_p2.py tests/test_gpu_aux.py -m gpu -q -x > $OUT/pytest.log 2>&1; echo "exit $?" >> $OUT/pytest.log
timeout 900 python bench.py --steps 40 --warmup 5 --no-cpu-baseline --no-e2e --no-stress > $OUT/bench.json 2>> $OUT/bench.err
timeout 600 ncu --set full --clock-control none --import-source on -k regex:pf_p2_jit -s 2 -c 2 -o $OUT/prof_p2jit \
   python tools/p2_run.py 256 4 > $OUT/ncu_p2jit.log 2>&1
echo done > $OUT/DONE
