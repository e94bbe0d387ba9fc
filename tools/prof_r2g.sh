mkdir -p gpurun_out/r2g
timeout 1500 python -m pytest tests -m gpu -x -q --deselect "tests/test_gpu_golden.py::test_full_sweep_matches_oracle[c5]" --durations=8 > gpurun_out/r2g/pytest_gpu.log 2>&1; echo "rc=$?" >> gpurun_out/r2g/pytest_gpu.log
timeout 600 ncu -f --metrics gpu__time_duration.sum,smsp__inst_executed.sum,smsp__thread_inst_executed.sum,sm__warps_active.avg.pct_of_peak_sustained_active,dram__bytes_read.sum,dram__bytes_write.sum,smsp__issue_active.avg.pct_of_peak_sustained_active --clock-control none -k regex:k3_ -s 12 -c 4 --csv --log-file gpurun_out/r2g/issue_c2.csv python bench.py --steps 1 --warmup 3 --no-cpu-baseline --e2e-steps 0 > gpurun_out/r2g/ncu_issue.log 2>&1
ls -la gpurun_out/r2g
