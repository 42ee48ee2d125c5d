# peer exchange: ownership tests (threads + two processes over CUDA IPC), then the whole GPU suite
timeout 900 python -m pytest tests/test_gpu_ownership.py -x -q -p no:cacheprovider > gpurun_out/aa_own.log 2>&1; tail -15 gpurun_out/aa_own.log
timeout 1200 python -m pytest tests -m gpu -x -q -p no:cacheprovider > gpurun_out/aa_gputests.log 2>&1; tail -3 gpurun_out/aa_gputests.log
