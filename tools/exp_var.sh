# timing of variants built by tools/mk_variant.sh under variants/<name> (300 units of C2)
for v in "$@"; do
  for dbg in 0 2; do (cd variants/$v && EPI4_VERBOSE=1 timeout 120 python tools/run_search.py --units 300 --debug $dbg 2>&1 | tail -1 | sed "s/^/$v /"); done
done
