# Round-level GPU job: smoke, GPU tests, bench (both arms), compute-sanitizer logs,
# ncu launch list + full capture of the headline kernel.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
timeout 2400 python -m pytest tests -m gpu -q --timeout 1200 --timeout-method thread > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 900 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$?" >> gpurun_out/bench.err
timeout 600 python bench.py --steps 8 --no-rows --no-cpu --no-e2e --rebalance --count-exchange board > gpurun_out/bench_board.json 2> gpurun_out/bench_board.err
timeout 600 python bench.py --impl reference > gpurun_out/bench_ref.json 2> gpurun_out/bench_ref.err
# (compute-sanitizer is refused on the GPU pool since round r02f; the last
#  clean runs are profiles/sanitizer_r02d.log)
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv python bench.py --steps 2 --warmup 3 --no-rows --no-e2e --no-cpu > gpurun_out/ncu_list.log 2>&1
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:irregular_kernel -s 3 -c 1 -o gpurun_out/prof_headline -f python bench.py --steps 1 --warmup 3 --no-rows --no-e2e --no-cpu > gpurun_out/ncu_full.log 2>&1
tail -n 3 gpurun_out/smoke.log gpurun_out/pytest_gpu.log gpurun_out/bench.err; tail -n 2 gpurun_out/ncu_full.log
