#!/bin/bash
# session s21: P2 defaults (phi 8x2, mu 4x4) -- parity, bench line, ncu of both side kernels
OUT=gpurun_out/${1:-r02s21}
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
timeout 1200 python -m pytest tests/test_gpu_p2.py -m gpu -q -x > $OUT/pytest_p2.log 2>&1; echo "exit $?" >> $OUT/pytest_p2.log
timeout 600 python bench.py --steps 40 --warmup 5 --no-cpu-baseline --no-e2e --no-stress --autotune 0 > $OUT/bench.json 2>> $OUT/bench.err
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_phi_side -s 2 -c 1 -o $OUT/prof_p2phi \
   python tools/p2_run.py 256 4 > $OUT/ncu_p2phi.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_mu_side -s 2 -c 1 -o $OUT/prof_p2mu \
   python tools/p2_run.py 256 4 > $OUT/ncu_p2mu.log 2>&1
echo done > $OUT/DONE
