# Round-2 evidence: full GPU suite (incl. the C5 goldens), smoke, bench lines, reference arm, ncu launch list and
# a full capture of the dominant C2 kernel (exported to CSV on the box)
mkdir -p gpurun_out/final
timeout 2400 python -m pytest tests -m gpu -q --durations=15 > gpurun_out/final/pytest_gpu.log 2>&1; echo "rc=$?" >> gpurun_out/final/pytest_gpu.log
timeout 200 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/final/smoke.log 2>&1
timeout 500 python bench.py > gpurun_out/final/bench_c2.json 2> gpurun_out/final/bench_c2.err
timeout 300 python bench.py --impl reference > gpurun_out/final/ref_c2.json 2> gpurun_out/final/ref_c2.err
for c in c3 c4 hop wafer; do timeout 400 python bench.py --config $c --no-cpu-baseline --e2e-steps 2 > gpurun_out/final/bench_$c.json 2> gpurun_out/final/bench_$c.err; done
timeout 400 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/final/launches_c2.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --e2e-steps 0 > /dev/null 2>&1
timeout 600 ncu -f --set full --clock-control none --import-source on -k regex:k3_timeline -s 12 -c 4 -o /tmp/final_k3 python bench.py --steps 1 --warmup 3 --no-cpu-baseline --e2e-steps 0 > gpurun_out/final/ncu_full.log 2>&1
ncu -i /tmp/final_k3.ncu-rep --page raw --csv > gpurun_out/final/c2_k3_raw.csv 2>&1
ncu -i /tmp/final_k3.ncu-rep --page source --csv --print-source sass 2>/dev/null | gzip > gpurun_out/final/c2_k3_src.csv.gz
ls -la gpurun_out/final
