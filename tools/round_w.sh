# P > 1 L2 policy probe: visit-start row_ptr loads evict_last (vh), record stores streaming (stcs), both.
B="python bench.py --steps 3 --warmup 3 --no-cpu-baseline --no-e2e"
for p in 4 16; do for v in default vh stcs vhstcs; do
  if [ $v = default ]; then unset LT_LIBRARY; else export LT_LIBRARY=tools/variants/liblt_$v.so; fi
  $B --partitions $p > gpurun_out/w_p${p}_$v.json 2>/dev/null
  $B --partitions $p --refill 2 > gpurun_out/w_p${p}_rf2_$v.json 2>/dev/null
done; done
unset LT_LIBRARY
for f in gpurun_out/w_p*.json; do python -c "
import json,sys; d=json.load(open('$f')); s=d['per_step']; print('$f', round(d['value']/1e9,2), round(s['update_ms'],1))"; done
