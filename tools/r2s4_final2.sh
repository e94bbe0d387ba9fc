# Refresh the evidence touched by the last kernel changes: C2 bench line (driver default) + reference arm, wafer,
# Hop, ncu launch list and full capture of C2's K3 (issue evidence bench.py prints), smoke
O=gpurun_out/final2
mkdir -p $O
timeout 200 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "rc=$?" >> $O/smoke.log
timeout 500 python bench.py > $O/bench_c2.json 2> $O/bench_c2.err
timeout 300 python bench.py --impl reference > $O/ref_c2.json 2> $O/ref_c2.err
for c in wafer hop c3 c4; do timeout 400 python bench.py --config $c --no-cpu-baseline --e2e-steps 2 > $O/bench_$c.json 2> $O/bench_$c.err; done
timeout 400 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_c2.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --e2e-steps 0 > /dev/null 2>&1
timeout 900 ncu -f --set full --clock-control none --import-source on -k regex:k3_ -o /tmp/full_c2 python tools/ncu_one.py c2 > $O/ncu_full_c2.log 2>&1
ncu -i /tmp/full_c2.ncu-rep --page raw --csv > $O/full_c2_raw.csv 2>&1
ls -la $O
