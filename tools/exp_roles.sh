# role isolation on C2 (first 300 plan units): debug bits 1 skip producers, 2 skip scoring, 4 skip MMA
for dbg in 0 1 2 3 4 6; do EPI4_VERBOSE=1 timeout 120 python tools/run_search.py --units 300 --debug $dbg 2>&1 | tail -1; done
if [ -d variants/prof ]; then
  for dbg in 0 2; do (cd variants/prof && timeout 120 python tools/run_search.py --units 300 --debug $dbg 2>&1 | tail -1 | sed "s/^/prof /"); done
fi
