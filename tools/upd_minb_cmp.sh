# k_update (P > 1 batch kernel) register budget: LT_UPD_MINB 4 (shipped) vs 3, cfg 4 DeepWalk at P = 4, 16.
out=gpurun_out/upd_minb_cmp.jsonl; : > $out
for i in 1 2; do
for P in 4 16; do
  for v in upd3 default; do
    if [ $v = default ]; then unset LT_LIBRARY; else export LT_LIBRARY=tools/variants/liblt_$v.so; fi
    r=$(timeout 240 python bench.py --config 4 --partitions $P --steps 3 --warmup 3 --no-cpu-baseline --no-e2e 2>/dev/null | tail -1)
    python -c "import json,sys; d=json.loads(sys.argv[1]); print(json.dumps({'variant':'$v','P':$P,'value':d['value'],'ms':d['ms_per_step']}))" "$r" >> $out
  done
done
done
unset LT_LIBRARY
