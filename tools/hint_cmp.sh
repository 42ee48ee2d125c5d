python -m pytest tests/test_gpu_pagerank.py -x -q > gpurun_out/pr_tests.log 2>&1; echo rc=$? >> gpurun_out/pr_tests.log
for v in default nohint pathonly visonly; do
  if [ $v = default ]; then unset LT_LIBRARY; else export LT_LIBRARY=tools/variants/liblt_$v.so; fi
  python bench.py --app pagerank --no-cpu-baseline --no-e2e > gpurun_out/hint_pr_$v.json 2>&1
  python bench.py --no-cpu-baseline --no-e2e > gpurun_out/hint_dw_$v.json 2>&1
done
