# k_update_rf register budget: LT_RF_MINB override (4: 64 regs; 3 / 2: no spills) vs the shipped per-app bound, P = 1 workloads.
out=gpurun_out/rf_minb_cmp.jsonl
for cfg in "--config 4" "--config 3" "--config 4 --app pagerank"; do
  for v in ${VARIANTS:-default rf3 rf2}; do
    if [ $v = default ]; then unset LT_LIBRARY; else export LT_LIBRARY=tools/variants/liblt_$v.so; fi
    r=$(timeout 240 python bench.py $cfg --steps 5 --warmup 3 --no-cpu-baseline --no-e2e 2>/dev/null | tail -1)
    python -c "import json,sys; d=json.loads(sys.argv[1]); print(json.dumps({'variant':'$v','args':'$cfg','value':d['value'],'ms':d['ms_per_step'],'frac':d['roofline']['frac'],'parity':(d.get('parity_sample') or {}).get('mismatched_walks')}))" "$r" >> $out
  done
done
unset LT_LIBRARY
cat $out
