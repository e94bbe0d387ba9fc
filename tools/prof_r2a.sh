# Round 2 evidence: GPU suite after the R19 hash change, C3/C4 per-class latency, C3 tail, C5 per-instant
# latency, ncu full captures of the C3/C4 K3 launches (exported to CSV on the box; the .ncu-rep stay there)
mkdir -p gpurun_out/r2a
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/r2a/pytest_gpu.log 2>&1; echo "rc=$?" >> gpurun_out/r2a/pytest_gpu.log
timeout 300 python tools/c34_probe.py c3 c4 > gpurun_out/r2a/c34.log 2>&1
timeout 200 python tools/c3_tail.py > gpurun_out/r2a/c3_tail.log 2>&1
for n in 64 128 256; do timeout 120 python tools/c5_one.py $n 1 >> gpurun_out/r2a/c5_one.log 2>&1; echo "N=$n rc=$?" >> gpurun_out/r2a/c5_one.log; done
for c in c3 c4; do
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:k3_ -s 0 -c 4 -o /tmp/${c}_k3 python bench.py --config $c --steps 1 --warmup 3 --no-cpu-baseline --e2e-steps 0 > gpurun_out/r2a/ncu_$c.log 2>&1
  ncu -i /tmp/${c}_k3.ncu-rep --page raw --csv > gpurun_out/r2a/${c}_k3_raw.csv 2>&1
  ncu -i /tmp/${c}_k3.ncu-rep --page source --csv --print-source sass > gpurun_out/r2a/${c}_k3_src.csv 2>/dev/null
  gzip -f gpurun_out/r2a/${c}_k3_src.csv
done
ls -la gpurun_out/r2a
