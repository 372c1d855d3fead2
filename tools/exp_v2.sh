timeout 900 python -m pytest tests -m gpu -q -x 2>&1 | tail -3
for st in 44 42; do EPI4_STAGES=$st EPI4_VERBOSE=1 timeout 120 python tools/run_search.py --units 300 2>&1 | tail -2 | cut -c1-120; done
for dbg in 2 3 131 135; do timeout 120 python tools/run_search.py --units 300 --debug $dbg 2>&1 | tail -1 | cut -c1-100; done
(cd variants/prof && timeout 120 python tools/run_search.py --units 300 2>&1 | tail -1 | sed "s/^/prof /")
(cd variants/prof && timeout 120 python tools/run_search.py --units 300 --debug 64 > ../../gpurun_out/trace0.log 2>&1)
timeout 300 python tools/run_search.py --repeat 2 2>&1 | tail -1
