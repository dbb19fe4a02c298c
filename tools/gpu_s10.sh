#!/bin/bash
# session r02 s10: P2 bench + ncu of the P2 march kernels
OUT=gpurun_out/r02s10
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
timeout 600 python bench.py --steps 40 --warmup 5 --no-cpu-baseline --no-e2e --no-stress --autotune 0 > $OUT/bench.json 2> $OUT/bench.err
export PF_BENCH_ALLOW_SHORT=1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_phi_march -s 1 -c 1 -o $OUT/prof_p2phi \
   python bench.py --steps 4 --warmup 3 --no-cpu-baseline --no-e2e --no-stress --autotune 0 > $OUT/ncu_p2phi.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_mu_march -s 1 -c 1 -o $OUT/prof_p2mu \
   python bench.py --steps 4 --warmup 3 --no-cpu-baseline --no-e2e --no-stress --autotune 0 > $OUT/ncu_p2mu.log 2>&1
echo done > $OUT/DONE
