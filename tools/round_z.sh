# new parity cases: partition bounds beyond shared memory (P >= 8192), Lemire rejection chain at d = 2^31+1
python -m pytest tests/test_gpu_parity.py -x -q -p no:cacheprovider -k "beyond_shared or rejection_chain" > gpurun_out/z_new.log 2>&1; tail -5 gpurun_out/z_new.log
python -m pytest tests -m gpu -x -q -p no:cacheprovider > gpurun_out/z_gputests.log 2>&1; tail -3 gpurun_out/z_gputests.log
