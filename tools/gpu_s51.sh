#!/bin/bash
# session s51: phi-sweep knob combinations the coordinate search does not visit
OUT=gpurun_out/${1:-r02s51}
mkdir -p $OUT
bash tools/gpu_ab_pairs.sh r02s51ab 2 '{}' '{"phi_minb": 4}' '{"phi_minb": 4, "phi_prefetch": 2, "phi_pfd": 2}' '{"phi_minb": 4, "phi_prefetch": 1, "phi_pfd": 3}' '{"phi_prefetch": 2, "phi_pfd": 3}' '{"phi_zc": 16, "phi_minb": 4}' '{"phi_ty": 8, "phi_minb": 2}'
echo done > $OUT/DONE
