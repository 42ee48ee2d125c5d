# Compare liblt.so builds (tools/variants/liblt_<tag>.so; "default" = the in-tree build) on the
# headline workload. Usage: bash tools/variant_cmp.sh tag1 tag2 ...  (bench lines -> gpurun_out/var_<tag>.json)
for v in "$@"; do
  if [ "$v" = default ]; then unset LT_LIBRARY; else export LT_LIBRARY=tools/variants/liblt_$v.so; fi
  python bench.py --no-cpu-baseline --no-e2e $BENCH_ARGS > gpurun_out/var_$v.json 2> gpurun_out/var_$v.err
done
