# GPU tests + bench lines for every config (one gpurun call); outputs under gpurun_out/
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -x -q --durations=15 > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 200 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1
timeout 400 python bench.py > gpurun_out/bench_c2.json 2> gpurun_out/bench_c2.err
timeout 300 python bench.py --impl reference > gpurun_out/ref_c2.json 2> gpurun_out/ref_c2.err
timeout 300 python bench.py --config wafer --no-cpu-baseline > gpurun_out/bench_wafer.json 2> gpurun_out/bench_wafer.err
timeout 300 python bench.py --config c3 --no-cpu-baseline > gpurun_out/bench_c3.json 2> gpurun_out/bench_c3.err
timeout 300 python bench.py --config c4 --no-cpu-baseline > gpurun_out/bench_c4.json 2> gpurun_out/bench_c4.err
timeout 600 python bench.py --config c5 --no-cpu-baseline --steps 2 --e2e-steps 1 > gpurun_out/bench_c5.json 2> gpurun_out/bench_c5.err
tail -3 gpurun_out/pytest_gpu.log; for f in gpurun_out/bench_*.json gpurun_out/ref_c2.json; do echo $f; head -c 300 $f; echo; done
