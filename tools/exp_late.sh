# Diagnostics: producer load order (LATE) and per-geometry register split, per library variant: quick parity,
# C5 sub-window + full C5 (N = 224) and C2 (N = 128).   usage: bash tools/exp_late.sh <tag> <lib> [<lib> ...]
T=$1; shift
mkdir -p gpurun_out
{
for L in "$@"; do
  export EPI4_LIB=$PWD/paper_conf_icpp_nobreiss22_b200/$L
  echo "=== $L"
  timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "C1 or ragged or subwindow" 2>&1 | tail -1
  timeout 300 python tools/run_search.py --config C2 --repeat 2 2>&1 | tail -1
  timeout 300 python tools/run_search.py --config C5 --n-snps 512 --repeat 2 2>&1 | tail -1
  timeout 300 python tools/run_search.py --config C5 2>&1 | tail -1
done
} 2>&1 | tee gpurun_out/${T}_late.log
