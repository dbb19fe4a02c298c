#!/bin/bash
# session s62: 32x16 two-rows tiles at one CTA per SM -- z-chunk / prefetch distance
OUT=gpurun_out/${1:-r02s62}
mkdir -p $OUT
bash tools/gpu_ab_pairs.sh r02s62ab 1 '{}' '{"mu_ty": 16, "mu_minb": 1, "mu_zc": 40}' '{"mu_ty": 16, "mu_minb": 1, "mu_zc": 48}' '{"mu_ty": 16, "mu_minb": 1, "mu_zc": 64}' '{"mu_ty": 16, "mu_minb": 1, "mu_zc": 32, "mu_pfd": 6}' '{"mu_ty": 16, "mu_minb": 1, "mu_zc": 37}' '{"mu_ty": 16, "mu_minb": 1, "mu_zc": 26}'
echo done > $OUT/DONE
