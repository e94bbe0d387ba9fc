# after: FF hash split over twin lanes, distinct-rate rounds (K3), owner-maintained shares (K3h)
mkdir -p gpurun_out/r2d
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/r2d/pytest_gpu.log 2>&1; echo "rc=$?" >> gpurun_out/r2d/pytest_gpu.log
timeout 400 python bench.py --no-cpu-baseline --e2e-steps 3 > gpurun_out/r2d/bench_c2.json 2> gpurun_out/r2d/bench_c2.err
python tools/one_point.py c3 871 >> gpurun_out/r2d/one.log 2>&1
python tools/one_point.py c4 1116 >> gpurun_out/r2d/one.log 2>&1
for n in 64 128 256; do timeout 300 python tools/one_point.py c5 0 1 $n >> gpurun_out/r2d/one.log 2>&1; done
for n in 512 1024; do timeout 600 python tools/one_point.py c5 0 1 $n >> gpurun_out/r2d/one.log 2>&1; echo "N=$n rc=$?" >> gpurun_out/r2d/one.log; done
timeout 300 python bench.py --config c3 --no-cpu-baseline --e2e-steps 1 > gpurun_out/r2d/bench_c3.json 2> gpurun_out/r2d/bench_c3.err
timeout 300 python bench.py --config c4 --no-cpu-baseline --e2e-steps 1 > gpurun_out/r2d/bench_c4.json 2> gpurun_out/r2d/bench_c4.err
ls -la gpurun_out/r2d
