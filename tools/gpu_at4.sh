OUT=gpurun_out/at4; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
timeout 900 python bench.py --steps 200 --warmup 10 --no-cpu-baseline --no-e2e --autotune 4 > $OUT/bench_at4.json 2> $OUT/bench.err
timeout 900 python bench.py --steps 200 --warmup 10 --no-cpu-baseline --no-e2e --autotune 2 --tuning '{"mu_zc": 16, "phi_zc": 16}' > $OUT/bench_zc16.json 2>> $OUT/bench.err
echo done > $OUT/DONE
