# quick GPU check: parity tests + timing of the quad kernel on C2 (300 units and full) with debug variants
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q -x 2>&1 | tail -2
for dbg in 0 2; do EPI4_VERBOSE=1 timeout 120 python tools/run_search.py --units 300 --debug $dbg 2>&1 | tail -2; done
timeout 300 python tools/run_search.py --repeat 2 2>&1 | tail -1
