# Diagnostics: top-k list (per-warp registers vs locked CTA list) x K2 filter (FFMA2 pairs vs scalar) on C2 and a
# C5 sub-window, both geometries' defaults; plus a compute-sanitizer smoke run printed to stdout.
# usage: bash tools/exp_topk.sh <tag> <lib> [<lib> ...]
T=$1; shift
mkdir -p gpurun_out
{
for L in "$@"; do
  export EPI4_LIB=$PWD/paper_conf_icpp_nobreiss22_b200/$L
  echo "=== $L"
  timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "C1 or ties or ragged" 2>&1 | tail -1
  for r in 1 2; do timeout 300 python tools/run_search.py --config C2 2>&1 | tail -1; done
  timeout 300 python tools/run_search.py --config C5 --n-snps 512 2>&1 | tail -1
done
unset EPI4_LIB
which compute-sanitizer; ls /usr/local/cuda/bin/compute-sanitizer
timeout 600 compute-sanitizer --tool memcheck python tools/run_search.py --config C1 --tile 128 2>&1 | tail -15
} 2>&1 | tee gpurun_out/${T}_topk.log
