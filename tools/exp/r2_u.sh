# round 2: the distributed path with the real GPU build (two gloo ranks on cuda:0) and the torchrun/NCCL bench
# arm at N = 1 (process group, barrier, max-over-ranks timing on hardware)
cd ${GRAFT_REPO_ROOT:-.}
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_dist.py -q -s > gpurun_out/r2u_dist.log 2>&1; tail -n 2 gpurun_out/r2u_dist.log
timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 1 --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 1 --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/r2u_torchrun.log 2>&1; echo "torchrun rc=$?"; tail -c 400 gpurun_out/r2u_torchrun.log
