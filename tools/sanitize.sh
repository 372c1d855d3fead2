# compute-sanitizer on a C1 search: both pipes, both tensor-core tile geometries, top-16 (the
# race-free per-warp register lists) and top-64 (the CTA list under a shared-memory spin lock, which racecheck
# cannot model); logs under gpurun_out/
mkdir -p gpurun_out
run() {   # tool tag args...
  local tool=$1 tag=$2; shift 2
  timeout 900 compute-sanitizer --tool $tool --print-limit 20 python tools/run_search.py --config C1 "$@" \
    > gpurun_out/sanitize_${tool}_${tag}.log 2>&1
  echo "$tool $tag rc=$? $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY|Error|error' gpurun_out/sanitize_${tool}_${tag}.log | tail -2 | tr '\n' ' ')"
}
for tool in memcheck racecheck synccheck initcheck; do
  run $tool tc128 --pipe tc --tile 128
  run $tool tc224 --pipe tc --tile 224
  run $tool lop3 --pipe lop3
done
run racecheck tc128_top64 --pipe tc --tile 128 --top-k 64
