#!/bin/bash
# session s61: taller two-rows tiles at one CTA per SM, now with the staged halo ring
OUT=gpurun_out/${1:-r02s61}
mkdir -p $OUT
bash tools/gpu_ab_pairs.sh r02s61ab 2 '{}' '{"mu_ty": 16, "mu_minb": 1}' '{"mu_ty": 12, "mu_minb": 1}' '{"mu_ty": 16, "mu_minb": 1, "mu_zc": 32}'
echo done > $OUT/DONE
