#!/bin/bash
# session s46: sched 2 with one mu CTA per SM (PF_MU_SMEM_PAD) so phi CTAs can share the SMs
OUT=gpurun_out/${1:-r02s46}
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
for pad in 0 90; do
  for t in '{}' '{"sched": 2, "slab": 4}' '{"sched": 2, "slab": 2}' '{"sched": 2, "slab": 1}'; do
    PF_MU_SMEM_PAD=$pad timeout 300 python bench.py --steps 100 --warmup 5 --no-cpu-baseline --no-e2e --no-stress --no-p2 --autotune 0 --tuning "$t" > $OUT/b.json 2>> $OUT/bench.err
    python -c "import json,sys; r=json.loads(open('$OUT/b.json').read().strip().splitlines()[-1]); print('pad $pad', '$t', round(r['value']), round(r['ms_per_step'],4), round(r['kernels']['mu_sweep_ms'],4))" >> $OUT/summary.txt
  done
done
echo done > $OUT/DONE
