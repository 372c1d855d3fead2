# Validation + A/B of the two tensor-core tile geometries on one box (run under gpurun):
# the GPU parity suite, smoke, then full searches of C5 / C2 / C3-512 with each geometry forced.
# usage: bash tools/gpu_check.sh <tag>
T=${1:-r02}
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.limit --format=csv
timeout 1500 python -m pytest tests -m gpu -q -x --durations=10 2>&1 | tail -16 > gpurun_out/${T}_pytest_gpu.log; tail -3 gpurun_out/${T}_pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -3
for t in 128 224; do
  timeout 300 python tools/run_search.py --config C2 --tile $t --repeat 2 2>&1 | tail -1
  timeout 300 python tools/run_search.py --config C3 --n-snps 512 --tile $t 2>&1 | tail -1
  timeout 300 python tools/run_search.py --config C5 --tile $t 2>&1 | tail -1
done 2>&1 | tee gpurun_out/${T}_geom_ab.log
