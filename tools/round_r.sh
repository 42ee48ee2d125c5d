# Prefetching lane refill (lt_config.refill = 3, k_update_pf): parity suite, then P sweep against the
# batch kernel (refill auto/off) and the plain refill kernel; MINB 4 (default build) vs MINB 3 variant.
python -m pytest tests -m gpu -x -q -p no:cacheprovider > gpurun_out/r_gputests.log 2>&1; tail -3 gpurun_out/r_gputests.log
B="python bench.py --steps 3 --warmup 3 --no-cpu-baseline --no-e2e"
for p in 1 4 16 64; do for rf in 0 2 3; do
  $B --partitions $p --refill $rf > gpurun_out/r_p${p}_rf$rf.json 2>/dev/null
done
LT_LIBRARY=tools/variants/liblt_pf3.so $B --partitions $p --refill 3 > gpurun_out/r_p${p}_rf3_minb3.json 2>/dev/null
done
for f in gpurun_out/r_p*.json; do python -c "
import json,sys; d=json.load(open('$f')); s=d['per_step']; print('$f', round(d['value']/1e9,2), round(s['update_ms'],1), s['sweeps'], s['update_launches'])"; done
