# Round-2 final evidence on the final kernels: GPU suite (incl. C5 goldens <= 256 GPUs), smoke, bench lines C2 (driver
# default) / C3 / C4 / Hop / wafer, reference arm, ncu launch list, full ncu of K3 on C2/C3/C4 (+ C2 source page),
# the C5 subset bench line (its records are compared with tests/golden/c5.npz afterwards)
O=gpurun_out/final
mkdir -p $O
timeout 1800 python -m pytest tests -m gpu -q --durations=10 > $O/pytest_gpu.log 2>&1; echo "rc=$?" >> $O/pytest_gpu.log
timeout 200 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "rc=$?" >> $O/smoke.log
timeout 500 python bench.py > $O/bench_c2.json 2> $O/bench_c2.err
timeout 300 python bench.py --impl reference > $O/ref_c2.json 2> $O/ref_c2.err
for c in c3 c4 hop wafer; do timeout 400 python bench.py --config $c --no-cpu-baseline --e2e-steps 2 > $O/bench_$c.json 2> $O/bench_$c.err; done
timeout 400 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_c2.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --e2e-steps 0 > /dev/null 2>&1
for c in c2 c3 c4; do
  timeout 900 ncu -f --set full --clock-control none --import-source on -k regex:k3_ -o /tmp/full_$c python tools/ncu_one.py $c > $O/ncu_full_$c.log 2>&1
  ncu -i /tmp/full_$c.ncu-rep --page raw --csv > $O/full_${c}_raw.csv 2>&1
done
ncu -i /tmp/full_c2.ncu-rep --page source --csv --print-source sass 2>/dev/null | gzip > $O/src_c2.csv.gz
timeout 2400 python tools/c5_bench.py > $O/bench_c5_subset.json 2> $O/bench_c5_subset.err
ls -la $O
