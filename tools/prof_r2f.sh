mkdir -p gpurun_out/r2f
timeout 1500 python -m pytest tests -m gpu -x -q --deselect "tests/test_gpu_golden.py::test_full_sweep_matches_oracle[c5]" --durations=8 > gpurun_out/r2f/pytest_gpu.log 2>&1; echo "rc=$?" >> gpurun_out/r2f/pytest_gpu.log
timeout 300 python tools/one_point.py c5 0 1 64 > gpurun_out/r2f/one.log 2>&1
timeout 300 python tools/one_point.py c5 0 1 128 >> gpurun_out/r2f/one.log 2>&1
timeout 300 python tools/one_point.py c3 871 >> gpurun_out/r2f/one.log 2>&1
timeout 300 python tools/c5_subset.py 64 > gpurun_out/r2f/c5sub.log 2>&1
timeout 400 python bench.py --no-cpu-baseline --e2e-steps 3 > gpurun_out/r2f/bench_c2.json 2> gpurun_out/r2f/bench_c2.err
timeout 600 ncu -f --metrics gpu__time_duration.sum,smsp__inst_executed.sum,smsp__thread_inst_executed.sum,sm__warps_active.avg.pct_of_peak_sustained_active,dram__bytes_read.sum,dram__bytes_write.sum,smsp__issue_active.avg.pct_of_peak_sustained_active --clock-control none -k regex:k3_ -s 20 -c 12 --csv --log-file gpurun_out/r2f/issue_c2.csv python bench.py --steps 1 --warmup 3 --no-cpu-baseline --e2e-steps 0 > /dev/null 2>&1
ls -la gpurun_out/r2f
