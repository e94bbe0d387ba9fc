mkdir -p gpurun_out/r2i
timeout 1500 python -m pytest tests -m gpu -x -q --deselect "tests/test_gpu_golden.py::test_full_sweep_matches_oracle[c5]" --durations=8 > gpurun_out/r2i/pytest_gpu.log 2>&1; echo "rc=$?" >> gpurun_out/r2i/pytest_gpu.log
timeout 300 python tools/one_point.py c5 0 1 64 > gpurun_out/r2i/one.log 2>&1
timeout 300 python tools/one_point.py c5 0 1 128 >> gpurun_out/r2i/one.log 2>&1
timeout 400 python tools/c5_subset.py 64 > gpurun_out/r2i/c5sub.log 2>&1
ls -la gpurun_out/r2i
