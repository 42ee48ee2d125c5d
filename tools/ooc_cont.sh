# Out-of-core (cfg 4 graph in pinned host memory): continuation into resident partitions (f4) on/off.
for cfg in "64 4" "64 8" "16 4"; do
  set -- $cfg
  for c in 0 1; do
    python bench.py --partitions $1 --graph-pool-gb $2 --continue-resident $c --steps 3 --warmup 3 --no-cpu-baseline --no-e2e \
      > gpurun_out/ooc_P$1_G$2_c$c.json 2> gpurun_out/ooc_P$1_G$2_c$c.err
  done
done
