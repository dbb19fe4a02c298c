#!/bin/bash
# ncu --set full of the specialised sweeps only
TAG=${1:-prof}
OUT=gpurun_out/$TAG
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:pf_jit_mu -s 3 -c 1 -o $OUT/prof_mu \
   python bench.py --steps 4 --warmup 3 --no-cpu-baseline --no-e2e --autotune 0 > $OUT/ncu_mu.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:pf_jit_phi -s 3 -c 1 -o $OUT/prof_phi \
   python bench.py --steps 4 --warmup 3 --no-cpu-baseline --no-e2e --autotune 0 > $OUT/ncu_phi.log 2>&1
echo done > $OUT/DONE
