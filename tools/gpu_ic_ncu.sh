#!/bin/bash
# D.8 follow-up: per-IC ncu captures of both sweeps (IC-R vs IC-L) and the
# step-rate check with nvidia-smi power / clock samples during it.
OUT=gpurun_out/${1:-ic}
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
(nvidia-smi --query-gpu=timestamp,clocks.sm,power.draw,clocks_throttle_reasons.active --format=csv -lms 200 > $OUT/smi.csv) &
SMI=$!
timeout 600 python tools/ic_independence.py > $OUT/ic.json 2> $OUT/ic.err
kill $SMI
for ic in R L; do
  for k in mu phi; do
    timeout 600 ncu --set full --clock-control none -k regex:pf_jit_$k -s 8 -c 1 -o $OUT/prof_${k}_$ic \
      python tools/ic_probe.py $ic > $OUT/ncu_${k}_$ic.log 2>&1
  done
done
echo done > $OUT/DONE
