#!/bin/bash
# session s38: ncu --set full of the mu-sweep with the halo ring staged by cp.async (default tuning), TMA box check
OUT=gpurun_out/${1:-r02s38}
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
export PF_BENCH_ALLOW_SHORT=1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:pf_jit_mu -s 3 -c 1 -o $OUT/prof_mu \
   python bench.py --steps 4 --warmup 3 --no-cpu-baseline --no-e2e --no-stress --no-p2 --autotune 0 > $OUT/ncu_mu.log 2>&1
timeout 300 ncu --metrics gpu__time_duration.sum --csv python tools/tma_box_check.py > $OUT/tma_box.csv 2>&1
echo done > $OUT/DONE
