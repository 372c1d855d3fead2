for r in 1 2; do
  timeout 120 python tools/run_search.py --units 300 2>&1 | tail -1 | cut -c60-90 | sed "s/^/tree /"
  EPI4_STAGES=42 timeout 120 python tools/run_search.py --units 300 2>&1 | tail -1 | cut -c60-90 | sed "s/^/tree42 /"
  for v in "$@"; do (cd variants/$v && timeout 120 python tools/run_search.py --units 300 2>&1 | tail -1 | cut -c60-90 | sed "s/^/$v /"); done
done
