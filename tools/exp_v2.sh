# packed epilogue + split A/B rings: parity, then timings on the first 300 C2 units
timeout 900 python -m pytest tests -m gpu -q -x 2>&1 | tail -3
for st in 44 42; do EPI4_STAGES=$st EPI4_VERBOSE=1 timeout 120 python tools/run_search.py --units 300 2>&1 | tail -2; done
for dbg in 1 2 3 6; do timeout 120 python tools/run_search.py --units 300 --debug $dbg 2>&1 | tail -1; done
for v in as1; do (cd variants/$v && timeout 120 python tools/run_search.py --units 300 2>&1 | tail -1 | sed "s/^/$v /"); done
(cd variants/prof && timeout 120 python tools/run_search.py --units 300 2>&1 | tail -1 | sed "s/^/prof /")
timeout 300 python tools/run_search.py --repeat 2 2>&1 | tail -1
