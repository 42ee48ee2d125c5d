# Multi-rank launch of bench.py on a 1-GPU box (all ranks share cuda:0; gloo for the collectives).
# Checks the driver's torchrun path end to end at small size; the numbers are not measurements.
# Round 2: --gpus N defaults to the ownership mode (peer exchange, paths on rank 0, replicas bound), and
# `bench.py --gpus 2` without torchrun launches its own ranks.
export LT_BENCH_SHARE_DEVICE=1
out=${1:-gpurun_out}
for n in 2 4; do
  python -m torch.distributed.run --nnodes=1 --nproc-per-node $n --master-addr 127.0.0.1 --master-port 29511 \
    bench.py --gpus $n --steps 3 --warmup 3 --config 2 --no-cpu-baseline > $out/multirank_own_n$n.json 2> $out/multirank_own_n$n.err
  echo "own (default) n=$n rc=$?"
  python -m torch.distributed.run --nnodes=1 --nproc-per-node $n --master-addr 127.0.0.1 --master-port 29512 \
    bench.py --impl reference --gpus $n --steps 2 --warmup 3 --config 2 > $out/multirank_ref_n$n.json 2> $out/multirank_ref_n$n.err
  echo "ref n=$n rc=$?"
done
python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29513 \
  bench.py --gpus 2 --steps 3 --warmup 3 --config 2 --no-cpu-baseline --mode replicas \
  > $out/multirank_replicas_n2.json 2> $out/multirank_replicas_n2.err
echo "replicas n=2 rc=$?"
python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29514 \
  bench.py --gpus 2 --steps 3 --warmup 3 --config 2 --no-cpu-baseline --no-e2e --exchange nccl \
  > $out/multirank_own_nccl_n2.json 2> $out/multirank_own_nccl_n2.err
echo "own all-to-all n=2 rc=$?"
# --gpus 2 without torchrun: bench.py launches the ranks itself
python bench.py --gpus 2 --steps 2 --warmup 3 --config 2 --no-cpu-baseline > $out/multirank_selflaunch_n2.json 2> $out/multirank_selflaunch_n2.err
echo "self-launched n=2 rc=$?"
