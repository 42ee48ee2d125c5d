# fused peer-exchange superstep: ownership tests, whole GPU suite, superstep loop timing (threaded ranks)
timeout 900 python -m pytest tests/test_gpu_ownership.py -x -q -p no:cacheprovider > gpurun_out/af_own.log 2>&1; tail -3 gpurun_out/af_own.log
for w in 2 4 8; do
  python tools/own_overhead.py --world $w --p2p >> gpurun_out/af_own.jsonl 2>>gpurun_out/af_own.err
  python tools/own_overhead.py --world $w --fused >> gpurun_out/af_own.jsonl 2>>gpurun_out/af_own.err
done
cat gpurun_out/af_own.jsonl
timeout 1500 python -m pytest tests -m gpu -x -q -p no:cacheprovider > gpurun_out/af_gputests.log 2>&1; tail -3 gpurun_out/af_gputests.log
