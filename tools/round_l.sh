# L2 persisting set-aside (lt_config.l2_persist) against the evict_last-tagged lines: PageRank visit
# counters (cfg 4) and the CSR row_ptr gathers of cfg 5 (LT_RP_HINT=1 build).
B="python bench.py --no-cpu-baseline --no-e2e --steps 3 --warmup 3"
$B --app pagerank --l2-persist 0 > gpurun_out/l_pr_p0.json 2>/dev/null
$B --app pagerank --l2-persist 1 > gpurun_out/l_pr_p1.json 2>/dev/null
$B --l2-persist 1 > gpurun_out/l_dw_p1.json 2>/dev/null
$B --config 5 --layout 1 --l2-persist 0 > gpurun_out/l_c5_p0.json 2>/dev/null
LT_LIBRARY=tools/variants/liblt_rphint.so $B --config 5 --layout 1 --l2-persist 1 > gpurun_out/l_c5_rp_p1.json 2>/dev/null
LT_LIBRARY=tools/variants/liblt_rphint.so $B --config 5 --layout 1 --l2-persist 0 > gpurun_out/l_c5_rp_p0.json 2>/dev/null
for f in gpurun_out/l_*.json; do python - "$f" <<'PY'
import json, sys
try:
    d = json.loads(open(sys.argv[1]).read().strip().splitlines()[-1])
    print(sys.argv[1], round(d["value"] / 1e9, 2), "G steps/s", round(d["roofline"]["avg_launch_ms"], 2), "ms/launch")
except Exception as e:
    print(sys.argv[1], "failed", e)
PY
done
python -c "
import torch; p=torch.cuda.get_device_properties(0); print('L2', p.L2_cache_size)"
