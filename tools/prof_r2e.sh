mkdir -p gpurun_out/r2e
timeout 1500 python -m pytest tests -m gpu -x -q --deselect "tests/test_gpu_golden.py::test_full_sweep_matches_oracle[c5]" --durations=12 > gpurun_out/r2e/pytest_gpu.log 2>&1; echo "rc=$?" >> gpurun_out/r2e/pytest_gpu.log
timeout 600 ncu -f --set full --clock-control none --import-source on -k regex:k3_ -s 1 -c 1 -o /tmp/one_c5 python tools/one_point.py c5 0 1 64 > gpurun_out/r2e/ncu_c5.log 2>&1
ncu -i /tmp/one_c5.ncu-rep --page raw --csv > gpurun_out/r2e/one_c5_raw.csv 2>&1
ncu -i /tmp/one_c5.ncu-rep --page source --csv --print-source sass 2>/dev/null | gzip > gpurun_out/r2e/one_c5_src.csv.gz
for n in 64 128 256 512 1024; do timeout 900 python tools/c5_subset.py $n >> gpurun_out/r2e/c5sub.log 2>&1; echo "N=$n rc=$?" >> gpurun_out/r2e/c5sub.log; done
mkdir -p gpurun_out/r2e/c5sub && mv gpurun_out/c5sub_N*.npy gpurun_out/r2e/c5sub/ 2>/dev/null
ls -la gpurun_out/r2e
