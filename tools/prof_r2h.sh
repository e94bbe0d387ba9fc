mkdir -p gpurun_out/r2h
timeout 1500 python -m pytest tests -m gpu -x -q --deselect "tests/test_gpu_golden.py::test_full_sweep_matches_oracle[c5]" --durations=8 > gpurun_out/r2h/pytest_gpu.log 2>&1; echo "rc=$?" >> gpurun_out/r2h/pytest_gpu.log
timeout 900 ncu -f --set full --clock-control none --import-source on -k regex:k3_ -s 1 -c 1 -o /tmp/one_c5b python tools/one_point.py c5 0 1 64 > gpurun_out/r2h/ncu_c5.log 2>&1
ncu -i /tmp/one_c5b.ncu-rep --page raw --csv > gpurun_out/r2h/one_c5_raw.csv 2>&1
ncu -i /tmp/one_c5b.ncu-rep --page source --csv --print-source sass 2>/dev/null | gzip > gpurun_out/r2h/one_c5_src.csv.gz
ls -la gpurun_out/r2h
