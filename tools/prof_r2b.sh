# single-point latency + ncu of the heaviest C3 / C4 points and a C5 N=64 point; bench smoke of the new bench.py
mkdir -p gpurun_out/r2b
python tools/one_point.py c3 heaviest > gpurun_out/r2b/one.log 2>&1
python tools/one_point.py c4 heaviest >> gpurun_out/r2b/one.log 2>&1
timeout 120 python tools/one_point.py c5 0 1 64 >> gpurun_out/r2b/one.log 2>&1
for c in c3 c4; do
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:k3_ -s 1 -c 1 -o /tmp/one_$c python tools/one_point.py $c heaviest 1 > gpurun_out/r2b/ncu_one_$c.log 2>&1
  ncu -i /tmp/one_$c.ncu-rep --page raw --csv > gpurun_out/r2b/one_${c}_raw.csv 2>&1
  ncu -i /tmp/one_$c.ncu-rep --page source --csv --print-source sass 2>/dev/null | gzip > gpurun_out/r2b/one_${c}_src.csv.gz
done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k3_ -s 0 -c 1 -o /tmp/one_c5 python tools/one_point.py c5 0 0 64 > gpurun_out/r2b/ncu_one_c5.log 2>&1
ncu -i /tmp/one_c5.ncu-rep --page raw --csv > gpurun_out/r2b/one_c5_raw.csv 2>&1
ncu -i /tmp/one_c5.ncu-rep --page source --csv --print-source sass 2>/dev/null | gzip > gpurun_out/r2b/one_c5_src.csv.gz
timeout 400 python bench.py --no-cpu-baseline --e2e-steps 3 > gpurun_out/r2b/bench_c2.json 2> gpurun_out/r2b/bench_c2.err
TS_SHARE_GPU=1 TS_DIST_BACKEND=gloo timeout 400 python bench.py --gpus 2 --steps 3 --e2e-steps 1 --no-cpu-baseline --dump-records /tmp/rec2.bin > gpurun_out/r2b/bench_g2.json 2> gpurun_out/r2b/bench_g2.err
timeout 400 python bench.py --sweep-scale 2 --steps 3 --e2e-steps 1 --no-cpu-baseline --dump-records /tmp/rec1.bin > gpurun_out/r2b/bench_s2.json 2> gpurun_out/r2b/bench_s2.err
cmp /tmp/rec1.bin /tmp/rec2.bin > gpurun_out/r2b/cmp.log 2>&1; echo "cmp rc=$?" >> gpurun_out/r2b/cmp.log; ls -la /tmp/rec*.bin >> gpurun_out/r2b/cmp.log
ls -la gpurun_out/r2b
