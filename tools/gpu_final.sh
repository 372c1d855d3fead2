# final round measurements: the standard round script + the driver's torchrun launch form at N=1
bash tools/gpu_round.sh
timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 1 --master-addr 127.0.0.1 --master-port 29511 \
  bench.py --gpus 1 --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/bench_torchrun.json 2> gpurun_out/bench_torchrun.err
tail -c 600 gpurun_out/bench_torchrun.json
