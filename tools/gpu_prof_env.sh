#!/bin/bash
# ncu --set full of the specialised mu-sweep (and phi-sweep) for env configs: bash tools/gpu_prof_env.sh TAG "CFG1" "CFG2" ...
TAG=${1:-profenv}
OUT=gpurun_out/$TAG
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
shift
i=0
for cfg in "$@"; do
  i=$((i+1))
  echo "$i: $cfg" >> $OUT/configs.txt
  env $cfg timeout 900 ncu --set full --clock-control none --import-source on -k regex:pf_jit_mu -s 3 -c 1 -o $OUT/prof_mu_$i \
     python bench.py --steps 4 --warmup 3 --no-cpu-baseline --no-e2e > $OUT/ncu_mu_$i.log 2>&1
done
echo done > $OUT/DONE
