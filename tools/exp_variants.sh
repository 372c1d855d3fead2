# Kernel-variant A/B on one box (diagnostics): for each library variant (EPI4_LIB), the GPU parity suite without the
# long C3 cases, then search timings on C2, C5-512 and C3-512 (tools/run_search.py, library CUDA events).
# usage: bash tools/exp_variants.sh <tag> <lib> [<lib> ...]   (libs relative to paper_conf_icpp_nobreiss22_b200/)
T=$1; shift
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.limit --format=csv
for L in "$@"; do
  export EPI4_LIB=$PWD/paper_conf_icpp_nobreiss22_b200/$L
  echo "=== $L"
  timeout 900 python -m pytest tests -m gpu -q -x -k "not C3 and not C4_windowed" 2>&1 | tail -3
  for r in 1 2; do
    timeout 300 python tools/run_search.py --config C2 2>&1 | tail -1
  done
  timeout 300 python tools/run_search.py --config C5 --n-snps 512 2>&1 | tail -1
  timeout 300 python tools/run_search.py --config C3 --n-snps 512 2>&1 | tail -1
done 2>&1 | tee gpurun_out/${T}_variants.log
