# single-point ncu of the heaviest C3 / C4 points (by index), C5 per-instant latency across N; golden parity
mkdir -p gpurun_out/r2c
timeout 900 python -m pytest tests/test_gpu_golden.py -x -q -k "not c5" > gpurun_out/r2c/golden.log 2>&1; echo "rc=$?" >> gpurun_out/r2c/golden.log
for spec in "c3 871" "c4 1116"; do
  set -- $spec
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:k3_ -s 1 -c 1 -o /tmp/one_$1 python tools/one_point.py $1 $2 1 > gpurun_out/r2c/ncu_one_$1.log 2>&1
  ncu -i /tmp/one_$1.ncu-rep --page raw --csv > gpurun_out/r2c/one_$1_raw.csv 2>&1
  ncu -i /tmp/one_$1.ncu-rep --page source --csv --print-source sass 2>/dev/null | gzip > gpurun_out/r2c/one_$1_src.csv.gz
done
for n in 128 256 512 1024; do timeout 300 python tools/one_point.py c5 0 1 $n >> gpurun_out/r2c/c5_n.log 2>&1; echo "N=$n rc=$?" >> gpurun_out/r2c/c5_n.log; done
ls -la gpurun_out/r2c
