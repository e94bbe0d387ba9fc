# A/B on C4 (and C3): current (shuffle distinct-rate count) vs previous build, 3 repetitions each, interleaved
O=gpurun_out/s4i
mkdir -p $O
for rep in 1 2 3; do
  for cfg in c4 c3; do
    for lib in paper_conf_isca_libwmvgjbj025_b200/libtriosim.so paper_conf_isca_libwmvgjbj025_b200/libtriosim_prev.so; do
      TRIOSIM_LIB=$lib timeout 300 python bench.py --config $cfg --no-cpu-baseline --e2e-steps 1 2>>$O/ab.err | python -c "import json,sys; d=json.load(sys.stdin); print('$cfg', '$lib'[-12:], d['value'], d['ms_per_step'], d['roofline']['k3_ms'], d['clocks']['sm_mhz'], d['clocks']['samples'])" >> $O/ab.txt
    done
  done
done
cat $O/ab.txt
