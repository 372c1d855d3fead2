# per-role wait counters (instrumented build) on the first 300 C2 units: full, no scoring, no build+scoring
cd variants/prof
for dbg in 0 2 3; do timeout 120 python tools/run_search.py --units 300 --debug $dbg 2>&1 | tail -1 | sed 's/.*quad /quad /'; done
timeout 120 python tools/run_search.py --units 300 --debug 64 > ../../gpurun_out/trace0.log 2>&1
