# Diagnostics: G128 variants on C2 / C3-512, and the kernel time against the number of SMs used (is the C2 kernel
# bound per SM or by a chip-wide L2 -> SM limit?).  usage: bash tools/exp_grid.sh <tag> <lib> [<lib> ...]
T=$1; shift
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.limit --format=csv
{
for L in "$@"; do
  export EPI4_LIB=$PWD/paper_conf_icpp_nobreiss22_b200/$L
  echo "=== $L"
  timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "C1 or ragged or ties" 2>&1 | tail -1
  for r in 1 2; do timeout 300 python tools/run_search.py --config C2 --tile 128 2>&1 | tail -1; done
  timeout 300 python tools/run_search.py --config C3 --n-snps 512 --tile 128 2>&1 | tail -1
done
export EPI4_LIB=$PWD/paper_conf_icpp_nobreiss22_b200/libepi4.so
for g in 148 112 74 38; do echo "grid $g"; timeout 300 python tools/run_search.py --config C2 --grid $g 2>&1 | tail -1; done
for g in 148 74; do echo "grid $g C5-512"; timeout 300 python tools/run_search.py --config C5 --n-snps 512 --grid $g 2>&1 | tail -1; done
} 2>&1 | tee gpurun_out/${T}_grid.log
