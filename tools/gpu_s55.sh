#!/bin/bash
# session s55: ncu --set full of the P1 mu / phi sweeps with their generated source imported (PF_JIT_DUMP)
OUT=gpurun_out/${1:-r02s55}
mkdir -p $OUT/jitsrc
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
export PF_BENCH_ALLOW_SHORT=1 PF_JIT_DUMP=$PWD/$OUT/jitsrc
TUNE=$(cat profiles/r02_tuning.json)
timeout 900 ncu --set full --clock-control none --import-source on -k regex:pf_jit_mu -s 3 -c 1 -o $OUT/prof_mu_src \
   python bench.py --steps 4 --warmup 3 --no-cpu-baseline --no-e2e --no-stress --no-p2 --autotune 0 --tuning "$TUNE" > $OUT/ncu_mu.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:pf_jit_phi -s 3 -c 1 -o $OUT/prof_phi_src \
   python bench.py --steps 4 --warmup 3 --no-cpu-baseline --no-e2e --no-stress --no-p2 --autotune 0 --tuning "$TUNE" > $OUT/ncu_phi.log 2>&1
echo done > $OUT/DONE
