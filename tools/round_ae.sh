# batch update kernel at P > 1 with more resident blocks per SM (register budget 51 / 42), plus the
# headline bench with the single-thread oracle figure
B="python bench.py --steps 3 --warmup 3 --no-cpu-baseline --no-e2e"
for p in 4 16; do for v in default ub5 ub6; do
  if [ $v = default ]; then unset LT_LIBRARY; else export LT_LIBRARY=tools/variants/liblt_$v.so; fi
  $B --partitions $p > gpurun_out/ae_p${p}_$v.json 2>/dev/null
done; done
unset LT_LIBRARY
for f in gpurun_out/ae_p*.json; do python -c "
import json,sys; d=json.load(open('$f')); s=d['per_step']; print('$f', round(d['value']/1e9,2), round(s['update_ms'],1))"; done
python bench.py > gpurun_out/ae_bench.json 2> gpurun_out/ae_bench.err; python -c "
import json; d=json.load(open('gpurun_out/ae_bench.json')); print(d['value'], d['cpu_baseline'])"
