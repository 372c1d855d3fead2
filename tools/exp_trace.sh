mkdir -p gpurun_out
cd scratch/prof
for dbg in 0 2 1 4 5 7 16; do timeout 120 python tools/run_search.py --units 300 --debug $dbg 2>&1 | tail -1; done
timeout 120 python tools/run_search.py --units 300 --debug 64 > ../../gpurun_out/trace.log 2>&1
tail -1 ../../gpurun_out/trace.log
