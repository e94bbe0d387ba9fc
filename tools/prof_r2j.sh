mkdir -p gpurun_out/r2j
timeout 1500 python -m pytest tests -m gpu -x -q --deselect "tests/test_gpu_golden.py::test_full_sweep_matches_oracle[c5]" --durations=8 > gpurun_out/r2j/pytest_gpu.log 2>&1; echo "rc=$?" >> gpurun_out/r2j/pytest_gpu.log
timeout 300 python bench.py --no-cpu-baseline --e2e-steps 2 > gpurun_out/r2j/bench_c2.json 2> gpurun_out/r2j/bench_c2.err
TS_WIDEN_FROM=8 timeout 300 python bench.py --no-cpu-baseline --e2e-steps 2 > gpurun_out/r2j/bench_c2_w8.json 2> gpurun_out/r2j/bench_c2_w8.err
timeout 1200 python tools/c5_subset.py 256 > gpurun_out/r2j/c5sub.log 2>&1; echo "rc=$?" >> gpurun_out/r2j/c5sub.log
timeout 1500 python tools/c5_subset.py 1024 >> gpurun_out/r2j/c5sub.log 2>&1; echo "rc=$?" >> gpurun_out/r2j/c5sub.log
ls -la gpurun_out/r2j
