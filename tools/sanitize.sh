# compute-sanitizer on a C1 search, both pipes; logs under gpurun_out/
mkdir -p gpurun_out
for tool in memcheck racecheck synccheck initcheck; do
  for pipe in tc lop3; do
    timeout 900 compute-sanitizer --tool $tool --print-limit 20 python tools/run_search.py --config C1 --pipe $pipe \
      > gpurun_out/sanitize_${tool}_${pipe}.log 2>&1
    echo "$tool $pipe rc=$? $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY|Error|error' gpurun_out/sanitize_${tool}_${pipe}.log | tail -2 | tr '\n' ' ')"
  done
done
