# A/B timing of variants/<name> against the working tree on the first 300 C2 units, alternated
for r in 1 2; do
  timeout 120 python tools/run_search.py --units 300 2>&1 | tail -1 | sed "s/best.*quad \([0-9.]*\) ms.*/quad \1 ms/;s/^/tree /"
  for v in "$@"; do (cd variants/$v && timeout 120 python tools/run_search.py --units 300 2>&1 | tail -1 | sed "s/best.*quad \([0-9.]*\) ms.*/quad \1 ms/;s/^/$v /"); done
done
timeout 120 python tools/run_search.py 2>&1 | tail -1 | sed "s/best.*quad \([0-9.]*\) ms.*/quad \1 ms/;s/^/tree full /"
for v in "$@"; do (cd variants/$v && timeout 120 python tools/run_search.py 2>&1 | tail -1 | sed "s/best.*quad \([0-9.]*\) ms.*/quad \1 ms/;s/^/$v full /"); done
