# Round measurement set (run under gpurun): parity tests, smoke, bench (ours + reference arm),
# ncu launch list of the bench command, one full ncu capture of the hot kernel.
set -x
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.limit --format=csv
timeout 900 python -m pytest tests -m gpu -q -x 2>&1 | tail -15 > gpurun_out/pytest_gpu.log; cat gpurun_out/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -3
timeout 600 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; tail -c 4000 gpurun_out/bench.json; tail -5 gpurun_out/bench.err
timeout 600 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/bench_ref.json 2>&1; tail -c 1500 gpurun_out/bench_ref.json
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline > gpurun_out/ncu_launches_bench.log 2>&1; tail -2 gpurun_out/ncu_launches_bench.log
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_quad_tc --launch-skip 1 -c 1 -o gpurun_out/prof_quad_full python tools/run_search.py --units 300 > gpurun_out/ncu_full.log 2>&1; tail -2 gpurun_out/ncu_full.log
