python -m pytest tests/test_gpu_out_of_core.py -x -q -p no:cacheprovider > gpurun_out/p_ooc_tests.log 2>&1; tail -2 gpurun_out/p_ooc_tests.log
B="python bench.py --no-cpu-baseline --no-e2e --steps 2 --warmup 1 --partitions 64 --graph-pool-gb 8"
$B --ooc-prefetch 0 > gpurun_out/p_g8_pf0.json 2>gpurun_out/p_err.txt
$B --ooc-prefetch 1 > gpurun_out/p_g8_pf1.json 2>>gpurun_out/p_err.txt
$B --ooc-prefetch 1 --zero-copy 0 > gpurun_out/p_g8_pf1_zc0.json 2>>gpurun_out/p_err.txt
$B --ooc-prefetch 0 --zero-copy 0 > gpurun_out/p_g8_pf0_zc0.json 2>>gpurun_out/p_err.txt
for f in gpurun_out/p_g8_*.json; do python - "$f" <<'PY'
import json, sys
d = json.loads(open(sys.argv[1]).read().strip().splitlines()[-1])
h = d["host_link"]
print(sys.argv[1], round(d["value"] / 1e9, 3), "G steps/s", round(h["achieved_gbs"], 1), "GB/s", round(h["frac"], 3),
      "copies", h["explicit_copies"], "pf", h.get("prefetches"), "zc", h["zero_copy_launches"], "hits", h["pool_hits"], "it", h["iterations"])
PY
done
