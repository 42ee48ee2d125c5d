# P > 1: lane refill with an idle-lane threshold (th8/16/24 builds) and the batch kernel at ILP 2/4.
B="python bench.py --steps 3 --warmup 3 --no-cpu-baseline --no-e2e"
for p in 4 16; do
  $B --partitions $p > gpurun_out/y_p${p}_batch.json 2>/dev/null
  for ilp in 2 4; do $B --partitions $p --ilp $ilp > gpurun_out/y_p${p}_ilp$ilp.json 2>/dev/null; done
  $B --partitions $p --refill 2 > gpurun_out/y_p${p}_rf.json 2>/dev/null
  for t in 8 16 24; do LT_LIBRARY=tools/variants/liblt_th$t.so $B --partitions $p --refill 2 > gpurun_out/y_p${p}_rf_th$t.json 2>/dev/null; done
done
LT_LIBRARY=tools/variants/liblt_th8.so $B > gpurun_out/y_p1_th8.json 2>/dev/null
LT_LIBRARY=tools/variants/liblt_th8.so $B --config 3 > gpurun_out/y_c3_th8.json 2>/dev/null
for f in gpurun_out/y_*.json; do python -c "
import json,sys; d=json.load(open('$f')); s=d['per_step']; print('$f', round(d['value']/1e9,2), round(s['update_ms'],1))"; done
