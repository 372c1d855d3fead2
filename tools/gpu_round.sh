# Round measurement set (run under gpurun): parity tests, smoke, bench (ours + reference arm), ncu launch list of
# the bench command, full ncu captures of the hot kernel in both tile geometries (N = 224 on a C5 slice, N = 128 on
# a C2 slice), summarised on the box (tools/ncu_summary.py) so that gpurun_out/ stays under the copy-back limit.
# (compute-sanitizer is closed on this GPU pool; tools/sanitize.sh is kept for boxes where it runs.)
# usage: bash tools/gpu_round.sh <tag>
set -x
T=${1:-r02}
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.limit --format=csv
timeout 1500 python -m pytest tests -m gpu -q -x --durations=15 2>&1 | tail -30 > gpurun_out/${T}_pytest_gpu.log; tail -5 gpurun_out/${T}_pytest_gpu.log
grep -q " failed\| error" gpurun_out/${T}_pytest_gpu.log && { echo "GPU tests failed: stopping"; exit 1; }
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -3 | tee gpurun_out/${T}_smoke.log
timeout 1500 python bench.py --steps 5 --warmup 3 > gpurun_out/${T}_bench.json 2> gpurun_out/${T}_bench.err; tail -c 1500 gpurun_out/${T}_bench.json; tail -5 gpurun_out/${T}_bench.err
timeout 900 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/${T}_bench_ref.json 2>&1; tail -c 800 gpurun_out/${T}_bench_ref.json
timeout 1200 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${T}_launches.csv python bench.py --also none --steps 2 --warmup 3 --no-cpu-baseline > gpurun_out/${T}_ncu_launches_bench.log 2>&1; tail -2 gpurun_out/${T}_ncu_launches_bench.log
python tools/ncu_summary.py launches gpurun_out/${T}_launches.csv "${T}: ncu launch list of python bench.py --also none --steps 2 --warmup 3 (C5, 1 B200)" > gpurun_out/${T}_ncu_launches_summary.txt 2>&1; cat gpurun_out/${T}_ncu_launches_summary.txt
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:k_quad_tc --launch-skip 1 -c 1 -o /tmp/${T}_full_C5slice -f python tools/run_search.py --config C5 --units 12 > gpurun_out/${T}_ncu_full_c5.log 2>&1; tail -2 gpurun_out/${T}_ncu_full_c5.log
python tools/ncu_summary.py full /tmp/${T}_full_C5slice.ncu-rep "${T}: k_quad_tc, C5 first 12 plan units (N = 224 geometry), --set full" > gpurun_out/${T}_ncu_full_k_quad_tc_C5slice.txt 2>&1; cat gpurun_out/${T}_ncu_full_k_quad_tc_C5slice.txt
python tools/ncu_summary.py stalls /tmp/${T}_full_C5slice.ncu-rep > gpurun_out/${T}_ncu_stalls_C5slice.txt 2>&1; head -30 gpurun_out/${T}_ncu_stalls_C5slice.txt
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_quad_tc --launch-skip 1 -c 1 -o /tmp/${T}_full_C2slice -f python tools/run_search.py --config C2 --units 300 > gpurun_out/${T}_ncu_full_c2.log 2>&1; tail -2 gpurun_out/${T}_ncu_full_c2.log
python tools/ncu_summary.py full /tmp/${T}_full_C2slice.ncu-rep "${T}: k_quad_tc, C2 first 300 plan units (N = 128 geometry), --set full" > gpurun_out/${T}_ncu_full_k_quad_tc_C2slice.txt 2>&1; cat gpurun_out/${T}_ncu_full_k_quad_tc_C2slice.txt
rm -f gpurun_out/*.ncu-rep
du -sh gpurun_out
