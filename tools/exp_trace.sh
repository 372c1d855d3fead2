mkdir -p gpurun_out
cd variants/prof
timeout 120 python tools/run_search.py --units 300 --debug 64 > ../../gpurun_out/trace0.log 2>&1
timeout 120 python tools/run_search.py --units 300 --debug 66 > ../../gpurun_out/trace2.log 2>&1
tail -1 ../../gpurun_out/trace0.log
