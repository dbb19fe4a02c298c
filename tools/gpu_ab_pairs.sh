#!/bin/bash
# Same-box A/B of pf_tuning settings on the config-2 bench (mu / phi / step
# times; no auto-tuning), every setting run ROUNDS times in alternation.
# usage: bash tools/gpu_ab_pairs.sh TAG ROUNDS '{json}' '{json}' ...
TAG=${1:-abp}
ROUNDS=${2:-2}
OUT=gpurun_out/$TAG
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
shift 2
for r in $(seq 1 $ROUNDS); do
  i=0
  for t in "$@"; do
    i=$((i+1))
    echo "$r $i: $t" >> $OUT/configs.txt
    timeout 300 python bench.py --steps 100 --warmup 5 --no-cpu-baseline --no-e2e --no-stress --no-p2 --autotune 0 \
      --tuning "$t" > $OUT/bench_${r}_$i.json 2>> $OUT/bench.err
  done
done
python - "$OUT" <<'PY' > $OUT/summary.txt
import glob, json, os, sys
d = sys.argv[1]
for f in sorted(glob.glob(os.path.join(d, "bench_*.json"))):
    try:
        r = json.loads(open(f).read().strip().splitlines()[-1])
        k = r["kernels"]
        print(os.path.basename(f), round(r["value"]), "mu", round(k["mu_sweep_ms"], 4), "phi", round(k["phi_sweep_ms"], 4), "step", round(r["ms_per_step"], 4))
    except Exception as e:
        print(f, "ERR", e)
PY
echo done > $OUT/DONE
