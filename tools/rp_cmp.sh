export BENCH_ARGS="--config 5 --steps 3 --warmup 3"
bash tools/variant_cmp.sh default rph path rphpath
for v in default rph path rphpath; do mv gpurun_out/var_$v.json gpurun_out/var5_$v.json; done
export BENCH_ARGS="--layout 1 --steps 3 --warmup 3"
bash tools/variant_cmp.sh default rph path rphpath
