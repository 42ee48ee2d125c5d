# A/B on one box: chunk install-ahead (current) vs on-demand install (prev), P = 4 and 16.
B="python bench.py --steps 3 --warmup 3 --no-cpu-baseline --no-e2e"
for i in 1 2; do for p in 4 16; do for v in default prev; do
  if [ $v = default ]; then unset LT_LIBRARY; else export LT_LIBRARY=tools/variants/liblt_$v.so; fi
  $B --partitions $p > gpurun_out/x_p${p}_rf0_${v}_$i.json 2>/dev/null
  $B --partitions $p --refill 2 > gpurun_out/x_p${p}_rf2_${v}_$i.json 2>/dev/null
done; done; done
unset LT_LIBRARY
for f in gpurun_out/x_p*.json; do python -c "
import json,sys; d=json.load(open('$f')); s=d['per_step']; print('$f', round(d['value']/1e9,2), round(s['update_ms'],1))"; done
