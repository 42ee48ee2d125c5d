# BASELINE configs[4]: UK-Union-shaped Kronecker scale 28 (5.5B tuples), |V| DeepWalk walks l=80.
python bench.py --config 5 --steps 3 --warmup 3 --cpu-seconds 10 > gpurun_out/bench_cfg5_resident.json 2> gpurun_out/bench_cfg5_resident.err
python bench.py --config 5 --partitions 64 --graph-pool-gb 11 --steps 2 --warmup 3 --no-cpu-baseline --no-e2e \
  > gpurun_out/bench_cfg5_ooc.json 2> gpurun_out/bench_cfg5_ooc.err
