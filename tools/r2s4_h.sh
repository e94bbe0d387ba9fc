# shuffle distinct-rate count (K3 W <= 16), blocked-send cache (K3 PIPE), serial minima for <= 4 warps (K3h): parity + A/B
O=gpurun_out/s4h
mkdir -p $O
timeout 1500 python -m pytest tests -m gpu -q -x -k "not c5_sample" > $O/pytest_gpu.log 2>&1; echo "rc=$?" >> $O/pytest_gpu.log
for cfg in c3 c4 c2; do
  for lib in paper_conf_isca_libwmvgjbj025_b200/libtriosim.so paper_conf_isca_libwmvgjbj025_b200/libtriosim_prev.so; do
    for rep in 1 2; do
      TRIOSIM_LIB=$lib timeout 300 python bench.py --config $cfg --no-cpu-baseline --e2e-steps 1 2>>$O/ab.err | python -c "import json,sys; d=json.load(sys.stdin); print('$cfg', '$lib'[-12:], d['value'], d['ms_per_step'], d['roofline']['k3_ms'], d['clocks']['sm_mhz'], d['clocks']['samples'])" >> $O/ab.txt
    done
  done
done
cat $O/ab.txt
