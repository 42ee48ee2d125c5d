# PageRank + PPR (cfg 3) measurements and ncu captures for profiles/.
python bench.py --config 3 --cpu-seconds 10 > gpurun_out/bench_cfg3.json 2> gpurun_out/bench_cfg3.err
python bench.py --app pagerank --cpu-seconds 10 > gpurun_out/bench_cfg4_pagerank.json 2> gpurun_out/bench_cfg4_pagerank.err
ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches_pagerank.csv \
  python bench.py --app pagerank --steps 2 --warmup 1 --no-cpu-baseline --no-e2e > /dev/null 2>&1
ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches_cfg3.csv \
  python bench.py --config 3 --steps 2 --warmup 1 --no-cpu-baseline --no-e2e > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:k_update -s 2 -c 1 -f -o gpurun_out/pagerank_full \
  python tools/profile_run.py --app pagerank --steps 3 > gpurun_out/pagerank_full.log 2>&1
