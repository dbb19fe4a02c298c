#!/bin/bash
# session r02 s6: slab schedule parity + A/B + DRAM bytes per step (ncu), TMA probe variants
OUT=gpurun_out/r02s6
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
for m in entry direct; do for t in 0 1 2; do timeout 60 tools/build/tma_probe2 $m $t >> $OUT/tma_probe2.jsonl 2>&1; done; done
timeout 1200 python -m pytest tests/test_gpu_autotune.py tests/test_gpu_aux.py -m gpu -q > $OUT/pytest.log 2>&1; echo "exit $?" >> $OUT/pytest.log
bash tools/gpu_ab_env.sh r02s6/ab - "PF_SCHED=1 PF_SLAB=1" "PF_SCHED=1 PF_SLAB=2" "PF_SCHED=1 PF_SLAB=4" - "PF_SCHED=1 PF_SLAB=1"
for cfg in "PF_SCHED=0" "PF_SCHED=1 PF_SLAB=1" "PF_SCHED=1 PF_SLAB=2"; do
  tag=$(echo $cfg | tr ' =' '__')
  env $cfg PF_BENCH_ALLOW_SHORT=1 timeout 600 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_sector_hit_rate.pct \
     --clock-control none --csv --log-file $OUT/ncu_$tag.csv \
     python bench.py --steps 3 --warmup 3 --no-cpu-baseline --no-e2e --no-stress --autotune 0 > $OUT/ncu_$tag.log 2>&1
done
echo done > $OUT/DONE
